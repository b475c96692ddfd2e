"""Host logic of the C5 multi-GPU path (bench.py run_c5), on CPU:
the texel rows each rank's output band taps (per pass), the shard interval,
and the region-copy plan that fills the shard from the owners' bands -- every
shard row exactly once, from the rank that owns it, at the right offsets.
The rows are checked against an independent count with the exact-rational
model of the addressing (tests/exact_model.py) on a small image, and a
world-size-2 gloo run exchanges the plans and checks that together the ranks
read every owned row the passes need."""
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_sc_kimdjjl15_b200 import synth  # noqa: E402
from tests import exact_model as em  # noqa: E402

MODE = {"repeat": (0x1133, 3), "mirrored": (0x1134, 4)}


def _plan(H, world, rank, mode):
    band = H // world
    A = synth.affine_translate_2d(H, H)
    need = bench._axis_taps(A[5], A[7], band, H, mode, start=rank * band)
    begin, count = bench.circular_interval(need, H)
    rows = [(begin + t) % H for t in range(count)]
    return need, rows, bench.shard_copy_plan(rows, band, world), band


@pytest.mark.parametrize("H,world", [(1024, 2), (2048, 4), (4096, 8), (32768, 8), (32768, 2)])
@pytest.mark.parametrize("mode", ["repeat", "mirrored"])
def test_plan_covers_the_shard_once_from_the_owners(H, world, mode):
    for rank in range(world):
        need, rows, plan, band = _plan(H, world, rank, mode)
        assert set(int(r) for r in need) <= set(rows)
        filled = np.zeros(len(rows), int)
        for d, sr, dr, n in plan:
            assert 0 <= sr and sr + n <= band and 0 <= d < world
            for t in range(n):
                assert rows[dr + t] == d * band + sr + t      # the right global row, from its owner
                filled[dr + t] += 1
        assert np.all(filled == 1)


@pytest.mark.parametrize("mode", ["repeat", "mirrored"])
def test_needed_rows_match_the_exact_model(mode):
    """The bench's float32 tap count equals the exact-rational model's rows."""
    H, world = 64, 4
    A = synth.affine_translate_2d(H, H)
    addr = MODE[mode][0]
    for rank in range(world):
        band = H // world
        need = set(int(r) for r in bench._axis_taps(A[5], A[7], band, H, mode, start=rank * band))
        exp = set()
        for y in range(rank * band, (rank + 1) * band):
            v = np.float32(np.float32(np.float32(A[5]) * np.float32(y)) + np.float32(A[7]))
            i0, i1, w = em.axis(v, H, True, addr, 0x1141)
            for i, wt in ((i0, 1 - w), (i1, w)):
                if i is not None and wt != 0:
                    exp.add(int(i))
        assert need == exp, (rank, sorted(need ^ exp))


def _worker(rank, world, port, H, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sc_kimdjjl15_b200 import dist as bdist
    ok = True
    for mode in ("repeat", "mirrored"):
        _, rows, plan, band = _plan(H, world, rank, mode)
        # what each owner serves to this rank, gathered on every rank
        served = bdist.exchange_bytes(repr([(d, sr, n) for d, sr, _, n in plan]).encode())
        for r, blob in enumerate(served):
            for d, sr, n in eval(blob.decode()):
                ok &= 0 <= sr and sr + n <= band and 0 <= d < world
        ok &= sum(n for *_, n in plan) == len(rows)
    q.put((rank, bool(ok)))
    dist.destroy_process_group()


def test_gloo_world2_plans():
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    ps = [ctx.Process(target=_worker, args=(r, 2, port, 8192, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    assert sorted(res) == [(0, True), (1, True)]
