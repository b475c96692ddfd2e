"""Two-process worker for tests/test_gpu_runtime.py::test_ipc_two_processes
(launched with torch.distributed.run --nproc-per-node 2, gloo control plane;
both ranks may share one GPU -- CUDA IPC then maps the other process's memory
of the same device, which exercises the same library paths as NVLink peers).

rank 0 (exporter): an IPC-exportable RGBA32F image and a 64 MiB buffer with
seeded content; exports both handles.
rank 1 (importer): imports both (objects whose valid copy is rank 0's memory,
SURVEY §8(e)) and checks, through the C-ABI only:
  a. clEnqueueCopyImage of a row band from the imported image into a local
     image reads the region in place (bytes equal rank 0's rows);
  b. a read built-in on the imported image (whole-object pull first) equals
     the oracle on the same codes;
  c. clEnqueueFillBuffer on a region of the imported buffer writes rank 0's
     memory in place (rank 0 checks after a barrier);
  d. wait-list order of a pull: queue 1 fills the whole
     imported buffer and returns an event; queue 2 migrates it with that event
     in its wait list, then reads it back -- every byte is the new pattern;
  e. b2clEnqueueCopyBufferEngine (copy engines) from the imported buffer equals
     the SM copy kernel's result.
Exit status 0 iff every check passed on both ranks."""
import ctypes
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_kimdjjl15_b200 import cl, synth  # noqa: E402
from paper_conf_sc_kimdjjl15_b200 import dist as bdist  # noqa: E402

W, H = 300, 200
NB = 64 << 20


def main():
    dist.init_process_group("gloo")
    rank = dist.get_rank()
    torch.cuda.set_device(0)
    S = cl.Session(0)
    L = cl.lib()
    err = ctypes.c_int32()
    fmt = cl.ImageFormat(cl.CL_RGBA, cl.CL_FLOAT)
    desc = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE2D, W, H, 0, 0, 0, 0, 0, 0, None)
    codes = synth.image_codes(synth.rng(500), cl.CL_RGBA, cl.CL_FLOAT, W, H)
    ok = True
    if rank == 0:
        img = S.image(cl.CL_RGBA, cl.CL_FLOAT, W, H, host=codes,
                      flags=cl.CL_MEM_READ_WRITE | cl.B2CL_MEM_IPC_EXPORTABLE)
        buf = L.clCreateBuffer(S.ctx, cl.CL_MEM_READ_WRITE | cl.B2CL_MEM_IPC_EXPORTABLE, NB, None,
                               ctypes.byref(err))
        cl.check(err.value)
        pat = np.array([0x11], np.uint8)
        cl.check(L.clEnqueueFillBuffer(S.queue, buf, pat.ctypes.data, 1, 0, NB, 0, None, None))
        S.finish()
        hi, hb = (ctypes.c_uint8 * 64)(), (ctypes.c_uint8 * 64)()
        cl.check(L.b2clGetMemIpcHandle(img, hi))
        cl.check(L.b2clGetMemIpcHandle(buf, hb))
        bdist.exchange_bytes(bytes(hi) + bytes(hb))
        dist.barrier()          # rank 1 runs its checks
        dist.barrier()
        got = S.read(buf, NB)
        # c. rank 1 filled [1 MiB, 2 MiB) with 0x5A in place; d. then the whole buffer with 0xC3
        ok = bool(np.all(got == 0xC3))
        S.release(img, buf)
    else:
        hs = bdist.exchange_bytes(b"")
        hi = (ctypes.c_uint8 * 64).from_buffer_copy(hs[0][:64])
        hb = (ctypes.c_uint8 * 64).from_buffer_copy(hs[0][64:])
        dist.barrier()
        pimg = L.b2clCreateImageFromIpcHandle(S.ctx, S.device, cl.CL_MEM_READ_WRITE, ctypes.byref(fmt),
                                              ctypes.byref(desc), hi, ctypes.byref(err))
        cl.check(err.value, "b2clCreateImageFromIpcHandle")
        pbuf = L.b2clCreateBufferFromIpcHandle(S.ctx, S.device, hb, NB, ctypes.byref(err))
        cl.check(err.value, "b2clCreateBufferFromIpcHandle")
        # a. region copy reads the peer image in place
        loc = S.image(cl.CL_RGBA, cl.CL_FLOAT, W, H)
        cl.check(L.clEnqueueCopyImage(S.queue, pimg, loc, cl.sz3((0, 17, 0)), cl.sz3((0, 3, 0)),
                                      cl.sz3((W, 5, 1)), 0, None, None))
        band = S.read_image(loc, (0, 3, 0), (W, 5, 1)).view(np.float32).reshape(5, W, 4)
        ok &= bool(np.array_equal(band.view(np.uint32), codes[0, 17:22].view(np.uint32)))
        # b. a read built-in on the imported image (the whole image is pulled first)
        import oracle as orc
        oimg = orc.Image(codes.copy(), W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
        smp = S.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR)
        A = synth.affine_rotate_2d(W, H, 30.0)
        out = S.buffer(W * H * 16)
        Ac = (ctypes.c_float * 12)(*A.tolist())
        cl.check(L.b2clEnqueueReadImageGrid(S.queue, pimg, smp, 0, Ac, cl.sz3((W, H, 1)), 4, out, 0, 0,
                                            None, None))
        got = S.read(out, W * H * 16, np.float32).reshape(1, H, W, 4)
        exp = orc.read_grid(oimg, True, orc.ADDRESS_REPEAT, orc.FILTER_LINEAR, orc.RT_F, A, (W, H, 1), 4)
        ok &= bool(np.max(np.abs(got.astype(np.float64) - exp) / np.maximum(np.spacing(np.abs(exp)), 1e-30)
                          * (np.abs(exp) >= 2.0 ** -10)) <= 4.0)
        # c. in-place region fill of the peer buffer
        pat = np.array([0x5A], np.uint8)
        cl.check(L.clEnqueueFillBuffer(S.queue, pbuf, pat.ctypes.data, 1, 1 << 20, 1 << 20, 0, None, None))
        S.finish()
        # e. copy engines vs the SM kernel, from the peer buffer
        a, b = S.buffer(4 << 20), S.buffer(4 << 20)
        cl.check(L.b2clEnqueueCopyBufferEngine(S.queue, pbuf, a, 512 << 10, 0, 4 << 20, 0, None, None))
        cl.check(L.clEnqueueCopyBuffer(S.queue, pbuf, b, 512 << 10, 0, 4 << 20, 0, None, None))
        ra, rb = S.read(a, 4 << 20), S.read(b, 4 << 20)
        ok &= bool(np.array_equal(ra, rb) and ra[0] == 0x11 and ra[(1 << 20) - (512 << 10)] == 0x5A)
        # d. a pull waits for its wait list: fill (queue 1) -> migrate (queue 2)
        q2 = S.queue_for(0)
        ev = ctypes.c_void_p()
        pat2 = np.array([0xC3], np.uint8)
        cl.check(L.clEnqueueFillBuffer(S.queue, pbuf, pat2.ctypes.data, 1, 0, NB, 0, None, ctypes.byref(ev)))
        mems = (ctypes.c_void_p * 1)(pbuf)
        cl.check(L.clEnqueueMigrateMemObjects(q2, 1, mems, 0, 1, (ctypes.c_void_p * 1)(ev), None))
        host = np.zeros(NB, np.uint8)
        cl.check(L.clEnqueueReadBuffer(q2, pbuf, 1, 0, NB, host.ctypes.data, 0, None, None))
        ok &= bool(np.all(host == 0xC3))
        L.clReleaseEvent(ev)
        cl.check(L.clFinish(S.queue))
        L.clReleaseCommandQueue(q2)
        S.release(pimg, pbuf, loc, out, a, b)
        L.clReleaseSampler(smp)
        dist.barrier()
    res = [None, None]
    dist.all_gather_object(res, bool(ok))
    S.close()
    dist.destroy_process_group()
    if rank == 0:
        print("ipc checks:", res)
    sys.exit(0 if all(res) else 1)


if __name__ == "__main__":
    main()
