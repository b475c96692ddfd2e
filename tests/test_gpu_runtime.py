"""Runtime semantics on the GPU (SURVEY §8(b) ownership, §8(e) multi-device):

* clReleaseMemObject is stream-ordered and deferred: releasing the source of a
  long copy right after enqueueing it returns without a host wait, and the
  copy still reads the right bytes (the storage is freed only after the
  queue's event for it completes);
* launches of one translated module from two queues that both set the
  module's global offset are chained, so each launch sees its own offset
  (symbol race);
* two processes sharing objects through CUDA IPC (tests/ipc_worker.py): region
  copies in place on the exporter's memory, whole-object pulls for sampling
  and migration, a wait-listed migration ordered after the write it waits for,
  and the copy-engine reference path."""
import ctypes
import os
import subprocess
import sys
import time

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_release_is_deferred_and_stream_ordered(sess):
    L = cl.lib()
    n = 1 << 30  # 1 GiB: the copy takes ~0.3 ms on the GPU
    g = np.random.default_rng(7)
    head = g.integers(0, 256, 1 << 20, dtype=np.uint8)
    src, dst = sess.buffer(n), sess.buffer(n)
    sess.write(src, head)                 # a recognisable first MiB
    pat = np.array([0x3C], np.uint8)
    cl.check(L.clEnqueueFillBuffer(sess.queue, src, pat.ctypes.data, 1, 1 << 20, n - (1 << 20), 0, None, None))
    sess.finish()
    # queue several long copies (~7 ms), then release the source while they run
    for _ in range(24):
        cl.check(L.clEnqueueCopyBuffer(sess.queue, src, dst, 0, 0, n, 0, None, None))
    t0 = time.perf_counter()
    cl.check(L.clReleaseMemObject(src))
    dt = time.perf_counter() - t0
    pending = L.clFinish(sess.queue)   # (reaps the deferred free)
    assert pending == 0
    assert dt < 2e-3, f"release blocked the host for {dt * 1e3:.2f} ms"
    got = sess.read(dst, 1 << 20)
    assert np.array_equal(got, head)
    assert np.all(sess.read(dst, 4096, offset=n - 4096) == 0x3C)
    # the handle is dead: a second release fails cleanly
    assert L.clReleaseMemObject(src) == -38  # CL_INVALID_MEM_OBJECT
    sess.release(dst)


def test_module_symbols_chained_across_queues(sess):
    from tests.test_gpu_kernels import _cubin_bytes
    L = cl.lib()
    prog = sess.program(_cubin_bytes())
    q2 = sess.queue_for(0)
    N = 1 << 22
    outs = [sess.buffer(N * 4), sess.buffer(N * 4)]
    offs = [7, 100003]
    ks = [sess.kernel(prog, "ids1d"), sess.kernel(prog, "ids1d")]
    for k, o in zip(ks, outs):
        sess.set_args(k, o)
    gws = cl.sz3((N, 0, 0))
    lws = cl.sz3((256, 0, 0))
    for it in range(20):
        for i, q in enumerate((sess.queue, q2)):
            cl.check(L.clEnqueueNDRangeKernel(q, ks[i], 1, cl.sz3((offs[i], 0, 0)), gws, lws, 0, None, None))
    cl.check(L.clFinish(q2))
    sess.finish()
    for i in range(2):
        got = sess.read(outs[i], N * 4, np.int32)
        gi = np.arange(offs[i], offs[i] + N, dtype=np.int64)
        assert np.array_equal(got, (gi * 10 + (gi - offs[i]) // 256).astype(np.int32)), f"queue {i}"
    for k in ks:
        L.clReleaseKernel(k)
    L.clReleaseCommandQueue(q2)
    L.clReleaseProgram(prog)
    sess.release(*outs)


def _free_port():
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def test_ipc_two_processes():
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr=127.0.0.1", f"--master-port={_free_port()}",
                        os.path.join(ROOT, "tests", "ipc_worker.py")],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]


def test_trace_log_names_command_and_kernel():
    """B2CL_LOG=1: one stderr line per enqueued command with the kernel used."""
    code = ("import numpy as np\n"
            "from paper_conf_sc_kimdjjl15_b200 import cl\n"
            "S = cl.Session(0)\n"
            "b = S.buffer(4096)\n"
            "p = np.arange(4, dtype=np.uint8)\n"
            "cl.check(cl.lib().clEnqueueFillBuffer(S.queue, b, p.ctypes.data, 4, 0, 4096, 0, None, None))\n"
            "S.finish()\n")
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=dict(os.environ, B2CL_LOG="1"),
                       capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    assert "[b2cl FILL_BUFFER" in r.stderr and "kernel=k_rect<FILL>" in r.stderr, r.stderr[-2000:]


def test_threads_share_the_runtime(sess):
    """Eight host threads (ctypes drops the GIL in every library call), each
    with its own queue, create / copy / fill / read back / release buffers and
    images concurrently -- objects released while their commands are still
    queued (deferred frees) -- and retain / release one shared buffer: every
    result exact, the shared object alive and intact, no error."""
    import threading
    L = cl.lib()
    base = np.arange(1 << 20, dtype=np.uint32).view(np.uint8)
    shared = sess.buffer(base.nbytes, base)
    errors = []

    def worker(tid):
        try:
            q = sess.queue_for(0)
            g = np.random.default_rng(100 + tid)
            for it in range(30):
                n = int(g.integers(1, 1 << 16)) * 16
                host = g.integers(0, 256, n, dtype=np.uint8)
                a = sess.buffer(n, host)
                b = sess.buffer(n)
                cl.check(L.clEnqueueCopyBuffer(q, a, b, 0, 0, n, 0, None, None))
                pat = np.array([tid, it, 7, 9], np.uint8)
                cl.check(L.clEnqueueFillBuffer(q, a, pat.ctypes.data, 4, 0, n, 0, None, None))
                cl.check(L.clReleaseMemObject(a))  # (its fill may still be queued)
                cl.check(L.clRetainMemObject(shared))
                out = np.empty(n, np.uint8)
                cl.check(L.clEnqueueReadBuffer(q, b, 1, 0, n, out.ctypes.data_as(ctypes.c_void_p), 0, None, None))
                cl.check(L.clReleaseMemObject(shared))
                assert np.array_equal(out, host), (tid, it)
                cl.check(L.clReleaseMemObject(b))
                if it % 5 == 0:
                    W, H = int(g.integers(1, 200)), int(g.integers(1, 100))
                    codes = g.integers(0, 256, (H, W, 4), dtype=np.uint8)
                    img = sess.image(cl.CL_RGBA, cl.CL_UNSIGNED_INT8, W, H, host=codes)
                    got = np.empty(W * H * 4, np.uint8)
                    cl.check(L.clEnqueueReadImage(q, img, 1, cl.sz3((0, 0, 0)), cl.sz3((W, H, 1)), 0, 0,
                                                  got.ctypes.data_as(ctypes.c_void_p), 0, None, None))
                    assert np.array_equal(got, codes.reshape(-1)), (tid, it, "image")
                    cl.check(L.clReleaseMemObject(img))
            assert L.clFinish(q) == 0
            cl.check(L.clReleaseCommandQueue(q))
        except Exception as exc:  # reported by the main thread
            errors.append(f"thread {tid}: {exc!r}")

    threads = [threading.Thread(target=worker, args=(t,)) for t in range(8)]
    for t in threads:
        t.start()
    for t in threads:
        t.join(timeout=300)
    assert not any(t.is_alive() for t in threads), "a thread hung"
    assert not errors, errors
    assert np.array_equal(sess.read(shared, base.nbytes), base)
    sess.release(shared)


def test_released_memory_is_reclaimed(sess):
    """800 buffers of 256 MiB (200 GiB in total, more than the device holds),
    each filled and released at once while its fill is still queued: the
    deferred frees are reaped as allocations proceed, so nothing runs out."""
    L = cl.lib()
    n = 256 << 20
    pat = np.array([1, 2, 3, 4], np.uint8)
    for it in range(800):
        b = sess.buffer(n)
        cl.check(L.clEnqueueFillBuffer(sess.queue, b, pat.ctypes.data, 4, 0, n, 0, None, None))
        cl.check(L.clReleaseMemObject(b))
    sess.finish()
