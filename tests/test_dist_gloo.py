"""World-size-2 tests of the multi-process plumbing on CPU (gloo, 127.0.0.1):
ring neighbours, IPC-handle exchange, max-over-ranks timing, and that the
row-band partition of an output grid, computed band by band on two ranks
(oracle) and gathered, equals the single-process result bit for bit
(sharding must not change any value)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_sc_kimdjjl15_b200 import dist as bdist
from paper_conf_sc_kimdjjl15_b200 import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    import torch.distributed as dist

    import oracle as orc
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        r, w, lr = bdist.env()
        assert (r, w, lr) == (rank, world, rank)
        # handles: every rank sees every rank's 64 bytes, in rank order
        handles = bdist.exchange_bytes(bytes([rank]) * 64)
        assert handles == [bytes([k]) * 64 for k in range(world)]
        left, right = bdist.ring_neighbors(rank, world)
        assert handles[left][0] == (rank - 1) % world
        # timing: the bench reports the slowest rank
        assert bdist.max_over_ranks(1.0 + rank) == float(world)
        assert bdist.min_over_ranks(1.0 + rank) == 1.0
        # sharded sampling of a row band == the same rows of the full grid
        W, H = 40, 37
        codes = synth.image_codes(synth.rng(60), orc.RGBA, orc.FLOAT, W, H)
        img = orc.Image(codes, W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
        A = synth.affine_translate_2d(W, H)
        r0, r1 = bdist.row_bands(H, world)[rank]
        band = orc.read_grid(img, True, orc.ADDRESS_REPEAT, orc.FILTER_LINEAR, orc.RT_F, A,
                             (W, H, 1), 4, yrange=(r0, r1))
        parts = [None] * world
        dist.all_gather_object(parts, band)
        if rank == 0:
            full = orc.read_grid(img, True, orc.ADDRESS_REPEAT, orc.FILTER_LINEAR, orc.RT_F, A,
                                 (W, H, 1), 4)
            got = np.concatenate(parts, axis=1)
            q.put(bool(np.array_equal(got.view(np.uint32), full.view(np.uint32))))
    finally:
        dist.destroy_process_group()


def test_two_rank_plumbing_and_sharded_equality():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    mp.start_processes(_worker, args=(2, _free_port(), q), nprocs=2, join=True,
                       start_method="spawn")
    assert q.get(timeout=60) is True


@pytest.mark.parametrize("H,world", [(32768, 1), (32768, 2), (32768, 8), (37, 2), (5, 4), (3, 8)])
def test_row_bands_partition(H, world):
    bands = bdist.row_bands(H, world)
    assert len(bands) == world
    assert bands[0][0] == 0 and bands[-1][1] == H
    for (a0, a1), (b0, b1) in zip(bands, bands[1:]):
        assert a1 == b0 and a0 <= a1
    sizes = [b - a for a, b in bands]
    assert max(sizes) - min(sizes) <= 1


def test_linear_halo_rows():
    assert bdist.linear_halo(0, 10, 40, wrap=False) == [10]
    assert bdist.linear_halo(0, 10, 40, wrap=True) == [39, 10]
    assert bdist.linear_halo(30, 40, 40, wrap=True) == [29, 0]
    assert bdist.linear_halo(10, 20, 40, wrap=False) == [9, 20]
    assert bdist.ring_neighbors(0, 8) == (7, 1)
    assert bdist.ring_neighbors(7, 8) == (6, 0)
