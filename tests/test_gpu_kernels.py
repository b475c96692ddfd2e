"""Launch glue for translated kernels (§3.5,
Fig. 5): kernels written in the translator's conventions against
include/b2cl_device.cuh are compiled with nvcc to a cubin and run through
clCreateProgramWithBinary / clBuildProgram / clCreateKernel / clSetKernelArg /
clEnqueueNDRangeKernel.  Results are compared with the oracle (image reads)
and with numpy (work-item indexing, __local carving)."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _cubin_bytes():
    """tests/kernels/translated.cu compiled with nvcc for sm_100a (cached per process)."""
    global _CUBIN
    if _CUBIN is None:
        import tempfile
        with tempfile.TemporaryDirectory() as d:
            out = os.path.join(d, "translated.cubin")
            nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
            subprocess.run([nvcc, "-cubin", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                            "-std=c++17", "-I", os.path.join(ROOT, "include"), "-o", out,
                            os.path.join(ROOT, "tests", "kernels", "translated.cu")], check=True)
            _CUBIN = open(out, "rb").read()
    return _CUBIN


_CUBIN = None


@pytest.fixture(scope="module")
def cubin():
    return _cubin_bytes()


@pytest.fixture(scope="module")
def prog(sess, cubin):
    p = sess.program(cubin)
    yield p
    cl.lib().clReleaseProgram(p)


def test_box3_image_read_and_local_memory(sess, orc, prog):
    W, H, LX = 96, 20, 32
    g = synth.rng(80)
    codes = synth.image_codes(g, cl.CL_RGBA, cl.CL_FLOAT, W, H)
    img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, W, H, host=codes)
    smp = sess.sampler(False, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    out = sess.buffer(W * H * 16)
    k = sess.kernel(prog, "box3")
    sess.set_args(k, img, smp, out, ("local", LX * 16), ctypes.c_int32(W))
    n0 = cl.launch_count()
    sess.ndrange(k, (W, H), (LX, 1))
    assert cl.launch_count() == n0 + 1
    got = sess.read(out, W * H * 16, np.float32).reshape(H, W, 4)
    # expected: oracle read at texel centres, then the work-group box sum in fp32 order
    oimg = orc.Image(codes, W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    xs, ys = np.meshgrid(np.arange(W) + 0.5, np.arange(H) + 0.5)
    co = np.stack([xs.ravel(), ys.ravel()], 1).astype(np.float32)
    t = orc.read_samples(oimg, False, orc.ADDRESS_CLAMP_TO_EDGE, orc.FILTER_LINEAR, orc.RT_F,
                         co).reshape(H, W // LX, LX, 4)
    left = np.concatenate([t[:, :, :1], t[:, :, :-1]], axis=2)
    right = np.concatenate([t[:, :, 1:], t[:, :, -1:]], axis=2)
    exp = ((left + t).astype(np.float32) + right).astype(np.float32).reshape(H, W, 4)
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))
    cl.lib().clReleaseKernel(k)
    sess.release(img, out)
    cl.lib().clReleaseSampler(smp)


def test_two_locals_offset_and_write_image(sess, prog):
    W, H, LX, LY, OX, OY = 32, 12, 8, 4, 3, 2
    g = synth.rng(81)
    codes = synth.image_codes(g, cl.CL_R, cl.CL_FLOAT, W + OX, H + OY)
    src = sess.image(cl.CL_R, cl.CL_FLOAT, W + OX, H + OY, host=codes)
    dst = sess.image(cl.CL_RGBA, cl.CL_FLOAT, W + OX, H + OY,
                     host=np.zeros((H + OY, W + OX, 4), np.float32))
    smp = sess.sampler(False, cl.CL_ADDRESS_NONE, cl.CL_FILTER_NEAREST)
    k = sess.kernel(prog, "two_locals")
    n = LX * LY
    sess.set_args(k, src, smp, dst, ("local", 4 * n), ("local", 4 * n), ctypes.c_float(2.5))
    sess.ndrange(k, (W, H), (LX, LY), offset=(OX, OY))
    got = sess.read_image(dst, (0, 0, 0), (W + OX, H + OY, 1)).view(np.float32).reshape(
        H + OY, W + OX, 4)
    exp = np.zeros_like(got)
    v = codes[0, :, :, 0]
    for y in range(OY, OY + H):
        for x in range(OX, OX + W):
            gx, gy = (x - OX) // LX, (y - OY) // LY
            lx, ly = (x - OX) % LX, (y - OY) % LY
            o = n - 1 - (ly * LX + lx)
            sx, sy = OX + gx * LX + o % LX, OY + gy * LY + o // LX
            exp[y, x] = [np.float32(v[sy, sx]) * np.float32(2.5), sx + 1000 * sy, 0.0, 1.0]
    assert np.array_equal(got, exp)
    cl.lib().clReleaseKernel(k)
    sess.release(src, dst)
    cl.lib().clReleaseSampler(smp)


def test_ids1d_default_local_size_and_offset(sess, prog):
    N, OFF = 1000, 7
    out = sess.buffer(N * 4)
    k = sess.kernel(prog, "ids1d")
    sess.set_args(k, out)
    sess.ndrange(k, (N,), None, offset=(OFF,))
    got = sess.read(out, N * 4, np.int32)
    g = np.arange(OFF, OFF + N)
    lsz = max(d for d in range(1, 257) if N % d == 0)  # the runtime's choice: largest divisor <= 256
    assert np.array_equal(got, g * 10 + (g - OFF) // lsz)
    cl.lib().clReleaseKernel(k)
    sess.release(out)


def test_launch_glue_errors(sess, prog):
    L = cl.lib()
    err = ctypes.c_int32()
    assert L.clCreateKernel(prog, b"no_such_kernel", ctypes.byref(err)) is None
    assert err.value == -46
    k = sess.kernel(prog, "box3")
    n = ctypes.c_uint32()
    assert L.clGetKernelInfo(k, 0x1191, 4, ctypes.byref(n), None) == 0 and n.value == 5
    v = ctypes.c_int32(1)
    assert L.clSetKernelArg(k, 9, 4, ctypes.byref(v)) == -49            # index
    assert L.clSetKernelArg(k, 4, 8, ctypes.byref(ctypes.c_int64(1))) == -51  # size
    assert L.clSetKernelArg(k, 3, 0, None) == -51                       # __local of 0 bytes
    gws = cl.sz3((64, 4, 1))
    assert L.clEnqueueNDRangeKernel(sess.queue, k, 2, None, gws, None, 0, None, None) == -52  # args
    out = sess.buffer(64 * 4 * 16)
    img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, 64, 4)
    smp = sess.sampler(False, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_NEAREST)
    sess.set_args(k, img, smp, out, ("local", 32 * 16), ctypes.c_int32(64))
    assert L.clEnqueueNDRangeKernel(sess.queue, k, 2, None, gws, cl.sz3((24, 1, 1)), 0, None,
                                    None) == -54                        # 24 does not divide 64
    assert L.clEnqueueNDRangeKernel(sess.queue, k, 4, None, gws, None, 0, None, None) == -53
    # a corrupt binary fails to build
    bad = b"\x7fELF not really a cubin" * 4
    buf = ctypes.create_string_buffer(bad, len(bad))
    bins = (ctypes.c_void_p * 1)(ctypes.cast(buf, ctypes.c_void_p))
    lens = (ctypes.c_size_t * 1)(len(bad))
    devs = (ctypes.c_void_p * 1)(sess.device)
    p2 = L.clCreateProgramWithBinary(sess.ctx, 1, devs, lens, bins, None, ctypes.byref(err))
    assert err.value == 0
    assert L.clBuildProgram(p2, 0, None, None, None, None) == -11
    assert L.clCreateKernel(p2, b"box3", ctypes.byref(err)) is None and err.value == -45
    L.clReleaseProgram(p2)
    L.clReleaseKernel(k)
    sess.release(out, img)
    L.clReleaseSampler(smp)


def test_dynamic_constant_arguments(sess, prog):
    """__constant buffers stay in global memory until the launch copies them into
    the module's constant array."""
    g = synth.rng(82)
    n1, n2, N = 37, 100, 1024
    lut1 = g.uniform(-1, 1, n1).astype(np.float32)
    lut2 = g.uniform(-1, 1, n2).astype(np.float32)
    b1, b2 = sess.buffer(lut1.nbytes, lut1), sess.buffer(lut2.nbytes, lut2)
    out = sess.buffer(N * 4)
    k = sess.kernel(prog, "const_lut")
    sess.set_args(k, out, b1, b2, ctypes.c_int32(n1), ctypes.c_int32(n2))
    sess.ndrange(k, (N,), (128,))
    i = np.arange(N)
    assert np.array_equal(sess.read(out, N * 4, np.float32), lut1[i % n1] + lut2[i % n2])
    # new contents are picked up by the next launch (copied at launch time)
    sess.write(b1, -lut1)
    sess.ndrange(k, (N,), (128,))
    assert np.array_equal(sess.read(out, N * 4, np.float32), -lut1[i % n1] + lut2[i % n2])
    # a non-buffer for a __constant argument is rejected
    v = ctypes.c_int64(5)
    assert cl.lib().clSetKernelArg(k, 1, 8, ctypes.byref(v)) == -50
    cl.lib().clReleaseKernel(k)
    sess.release(b1, b2, out)


def test_arrays_and_buffer_images_in_translated_kernel(sess, orc, prog):
    """image2d_array_t / image1d_buffer_t / image1d_array_t arguments: a weighted
    sum over layers, each layer read with the library's read built-in."""
    W, H, L = 40, 6, 5
    g = synth.rng(83)
    codes = synth.image_codes(g, cl.CL_RGBA, cl.CL_UNORM_INT8, W, H, L)
    arr = sess.image_array(cl.CL_RGBA, cl.CL_UNORM_INT8, W, L, H, host=codes)
    wts = g.uniform(-1, 1, 8).astype(np.float32)
    wb = sess.buffer(wts.nbytes, wts)
    wimg = sess.image_buffer(cl.CL_R, cl.CL_FLOAT, 8, wb)
    dst = sess.image_array(cl.CL_RGBA, cl.CL_FLOAT, W, H)
    smp = sess.sampler(False, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_NEAREST)
    k = sess.kernel(prog, "layer_mix")
    sess.set_args(k, arr, smp, wimg, dst)
    sess.ndrange(k, (W, H), (8, 2))
    got = sess.read_image(dst, (0, 0, 0), (W, H, 1)).view(np.float32).reshape(H, W, 4)
    oarr = orc.Image(codes.copy(), W, H, L, dims=2, order=orc.RGBA, type=orc.UNORM_INT8,
                     arrayed=True)
    xs, ys = np.meshgrid(np.arange(W) + 0.5, np.arange(H) + 0.5)
    exp = np.zeros((H * W, 4), np.float32)
    for l in range(L):
        co = np.stack([xs.ravel(), ys.ravel(), np.full(W * H, l), np.zeros(W * H)], 1)
        t = orc.read_samples(oarr, False, orc.ADDRESS_CLAMP_TO_EDGE, orc.FILTER_NEAREST, orc.RT_F,
                             co.astype(np.float32))
        exp = (exp + (t * wts[l]).astype(np.float32)).astype(np.float32)
    assert np.array_equal(got.reshape(-1, 4), exp)
    cl.lib().clReleaseKernel(k)
    cl.lib().clReleaseSampler(smp)
    sess.release(arr, wimg, wb, dst)
