"""Multi-process plumbing for the one-process-per-GPU mode (torchrun).

torch.distributed carries only control data here: the barrier, the max over
ranks of a timing, and the 64-byte CUDA IPC handles that let a rank open a
peer GPU's buffer and pull from it over NVLink with the library's copy kernel
(clEnqueueCopyBuffer on a b2clCreateBufferFromIpcHandle object).  Nothing on
the data path is a collective: the hot path partitions into independent
images / row bands, and the one real exchange -- migrating
a band to a neighbour -- is point-to-point.
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def env():
    """(rank, world_size, local_rank) from the torchrun environment (1-process defaults)."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def ring_neighbors(rank: int, world: int):
    """(left, right) ranks of the migration ring: rank d pulls from d-1 and is pulled by d+1."""
    return (rank - 1) % world, (rank + 1) % world


def row_bands(height: int, world: int):
    """Contiguous row bands [r0, r1) of an image of `height` rows over `world` ranks
    (shard d owns rows [d*H/G, (d+1)*H/G))."""
    return [(d * height // world, (d + 1) * height // world) for d in range(world)]


def linear_halo(r0: int, r1: int, height: int, wrap: bool):
    """Texel rows a unit-scale, row-aligned LINEAR read of output rows [r0, r1)
    needs beyond its own band: one row on each side, wrapped for REPEAT /
    MIRRORED_REPEAT, dropped at the image edge otherwise."""
    rows = []
    for r in (r0 - 1, r1):
        if 0 <= r < height:
            rows.append(r)
        elif wrap:
            rows.append(r % height)
    return rows


def exchange_bytes(payload: bytes) -> list[bytes]:
    """All ranks' payloads (e.g. IPC handles), in rank order."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return [payload]
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, payload)
    return out


def max_over_ranks(value: float, device=None) -> float:
    """Max of a per-rank timing (the bench reports the slowest rank)."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64,
                     device=device if device is not None else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def min_over_ranks(value: float, device=None) -> float:
    return -max_over_ranks(-float(value), device)
