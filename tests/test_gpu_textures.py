"""CUDA texture front end: translated
CUDA kernels fetch with tex1Dfetch / tex1D / tex2D / tex3D / tex2DLayered on
the image + sampler pair of b2clCreateTextureObject.

Each fetch is compared with two oracles on the same seeded inputs:
  * the OpenCL oracle's read_imageX with the mapped sampler and view type --
    the product's claim (bit-exact, LINEAR within 4 ulp / 1e-6);
  * the CUDA-side oracle (oracle_tex_fetch: the CUDA Programming Guide's
    texture-fetching formulas) -- the translation's fidelity; equal under the
    same bar except MIRROR off the dyadic lattices (reading A43, pinned on
    the CPU in tests/test_oracle_cuda_tex.py).
"""
import ctypes
import os
import subprocess

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth
from tests.gpu_helpers import assert_parity, parity_read

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CL_ADDR = {0: cl.CL_ADDRESS_REPEAT, 1: cl.CL_ADDRESS_CLAMP_TO_EDGE, 2: cl.CL_ADDRESS_MIRRORED_REPEAT,
           3: cl.CL_ADDRESS_CLAMP}
CL_FILT = {0: cl.CL_FILTER_NEAREST, 1: cl.CL_FILTER_LINEAR}


@pytest.fixture(scope="module")
def tprog(sess, tmp_path_factory):
    out = tmp_path_factory.mktemp("t") / "textures.cubin"
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    subprocess.run([nvcc, "-cubin", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                    "-std=c++17", "-I", os.path.join(ROOT, "include"), "-o", str(out),
                    os.path.join(ROOT, "tests", "kernels", "textures.cu")], check=True)
    p = sess.program(out.read_bytes())
    yield p
    cl.lib().clReleaseProgram(p)


def _run(sess, prog, name, tex, coords, out_bytes_per, sampler=True):
    n = coords.shape[0]
    cb = sess.buffer(max(coords.nbytes, 16), np.ascontiguousarray(coords))
    ob = sess.buffer(max(n * out_bytes_per, 16))
    k = sess.kernel(prog, name)
    args = [ctypes.c_void_p(tex.image)] + ([ctypes.c_void_p(tex.sampler)] if sampler else [])
    sess.set_args(k, *args, cb, ob, ctypes.c_int32(n))
    sess.ndrange(k, ((n + 127) // 128 * 128,), (128,))
    got = sess.read(ob, n * out_bytes_per)
    cl.lib().clReleaseKernel(k)
    sess.release(cb, ob)
    return got


def _coords(g, dims, sizes, norm, n_rand=1500):
    sp = synth.special_floats()
    lat = synth.coord_lattice(-2.0, 3.0, 1 / 32) if norm else synth.coord_lattice(-2.0, max(sizes) + 2.0, 1 / 8)
    pts = []
    for d in range(dims):
        vals = np.concatenate([lat, sp])
        c = g.uniform(-0.5, 1.5 if norm else max(sizes) + 1, (vals.size, dims)).astype(np.float32)
        c[:, d] = vals
        pts.append(c)
    pts.append(g.uniform(-1.5, 2.5, (n_rand, dims)).astype(np.float32) * np.float32(1 if norm else max(sizes)))
    return np.ascontiguousarray(np.concatenate(pts), np.float32)


def _dyadic(c):
    with np.errstate(invalid="ignore"):
        s = c.astype(np.float64) * 2.0 ** 20
        return np.all(np.isfinite(s) & (s == np.round(s)), axis=1)


def _check_both(orc, got, cl_img, tex_img, mode, filt, rmode, norm, rt, co, nch, what):
    """got: (n, nch) as uint32 bits; co: the coordinates (tex order)."""
    linear = filt == 1
    dt = np.float32 if rt == orc.RT_F else np.uint32
    rd = lambda im: np.ascontiguousarray(  # noqa: E731
        orc.read_samples(im, norm, CL_ADDR[mode], CL_FILT[filt], rt, co).view(np.uint32)[:, :nch]).view(dt)
    parity_read(got.view(dt), rd(cl_img), linear, what + " vs read_imageX", orc, cl_img, rd)
    keep = np.ones(co.shape[0], bool) if mode != 2 else _dyadic(co[:, :tex_img.dims])
    rt_ = lambda im: np.ascontiguousarray(  # noqa: E731
        orc.tex_fetch(im, [mode] * 3, filt, rmode, norm, co)[:, :nch][keep]).view(dt)
    parity_read(got[keep].view(dt), rt_(tex_img), linear, what + " vs CUDA", orc, tex_img, rt_)


@pytest.mark.parametrize("mode", [0, 1, 2, 3])
@pytest.mark.parametrize("filt", [0, 1])
def test_tex2D_float4_array_resource(sess, orc, tprog, mode, filt):
    W, H = 37, 21
    g = synth.rng(300 + 2 * mode + filt)
    data = synth.image_codes(g, cl.CL_RGBA, cl.CL_FLOAT, W, H)
    img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, W, H, host=data)
    o = orc.Image(data, W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    for norm in (True, False):
        if not norm and mode in (0, 2):
            continue
        res = cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, img)
        tex = sess.texture(res, cl.texture_desc([mode, mode], filt, 0, norm))
        assert tex.image == img and tex.rtype == 0   # element-type float: the image itself
        co = _coords(g, 2, (W, H), norm)
        got = _run(sess, tprog, "fetch2d_f4", tex, co, 16).view(np.uint32).reshape(-1, 4)
        _check_both(orc, got, o, o, mode, filt, 0, norm, orc.RT_F, co, 4, f"2D f4 m{mode} f{filt} n{norm}")
        cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(img)


def test_tex2D_normalized_read_of_uint8_view(sess, orc, tprog):
    """cudaReadModeNormalizedFloat over an UNSIGNED_INT8 image: a UNORM_INT8 view."""
    W, H = 40, 17
    g = synth.rng(310)
    data = synth.image_codes(g, cl.CL_R, cl.CL_UNSIGNED_INT8, W, H)
    img = sess.image(cl.CL_R, cl.CL_UNSIGNED_INT8, W, H, host=data)
    o = orc.Image(data, W, H, 1, dims=2, order=orc.R, type=orc.UNSIGNED_INT8)
    ov = orc.Image(data, W, H, 1, dims=2, order=orc.R, type=orc.UNORM_INT8)
    for mode in range(4):
        tex = sess.texture(cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, img),
                           cl.texture_desc([mode] * 2, 1, 1, True))
        assert tex.image != img
        fmt = cl.ImageFormat()
        cl.check(cl.lib().clGetImageInfo(tex.image, cl.CL_IMAGE_FORMAT, 8, ctypes.byref(fmt), None))
        assert (fmt.image_channel_order, fmt.image_channel_data_type) == (cl.CL_R, cl.CL_UNORM_INT8)
        co = _coords(g, 2, (W, H), True)
        got = _run(sess, tprog, "fetch2d_f1", tex, co, 4).view(np.uint32).reshape(-1, 1)
        _check_both(orc, got, ov, o, mode, 1, 1, True, orc.RT_F, co, 1, f"u8 normalized m{mode}")
        cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(img)


def test_tex2D_element_reads_uchar4_and_pitch2d_short2(sess, orc, tprog):
    g = synth.rng(311)
    # uchar4 element reads of an RGBA8 image (point filtering)
    W, H = 29, 13
    data = synth.image_codes(g, cl.CL_RGBA, cl.CL_UNSIGNED_INT8, W, H)
    img = sess.image(cl.CL_RGBA, cl.CL_UNSIGNED_INT8, W, H, host=data)
    o = orc.Image(data, W, H, 1, dims=2, order=orc.RGBA, type=orc.UNSIGNED_INT8)
    tex = sess.texture(cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, img), cl.texture_desc([3, 3], 0, 0, False))
    co = _coords(g, 2, (W, H), False)
    got = _run(sess, tprog, "fetch2d_uc4", tex, co, 4).reshape(-1, 4).astype(np.uint32)
    _check_both(orc, got, o, o, 3, 0, 0, False, orc.RT_UI, co, 4, "uchar4 border")
    cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(img)
    # PITCH2D: an RG SIGNED_INT16 view of a buffer at an offset with a caller pitch
    W, H, pitch, off = 37, 11, 37 * 4 + 20, 64
    rows = synth.image_codes(g, cl.CL_RG, cl.CL_SIGNED_INT16, W, H)
    host = np.zeros(off + pitch * H, np.uint8)
    for j in range(H):
        host[off + j * pitch: off + j * pitch + W * 4] = rows[0, j].view(np.uint8).reshape(-1)
    buf = sess.buffer(host.nbytes, host)
    res = cl.ResourceDesc(cl.B2CL_RESOURCE_PITCH2D, buf, off, cl.ChannelFormatDesc(16, 16, 0, 0, 0),
                          0, W, H, pitch)
    o = orc.Image(host[off:], W, H, 1, dims=2, order=orc.RG, type=orc.SIGNED_INT16, row_pitch=pitch)
    for mode in (1, 3):
        tex = sess.texture(res, cl.texture_desc([mode, mode], 0, 0, True))
        co = _coords(g, 2, (W, H), True)
        got = _run(sess, tprog, "fetch2d_s2", tex, co, 4).view(np.int16).reshape(-1, 2)
        _check_both(orc, got.astype(np.int32).view(np.uint32), o, o, mode, 0, 0, True, orc.RT_I, co, 2,
                    f"pitch2d short2 m{mode}")
        cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(buf)


def test_tex3D_half_rg_and_tex1D(sess, orc, tprog):
    g = synth.rng(312)
    W, H, D = 9, 7, 5
    data = synth.image_codes(g, cl.CL_RG, cl.CL_HALF_FLOAT, W, H, D)
    vol = sess.image(cl.CL_RG, cl.CL_HALF_FLOAT, W, H, D, host=data)
    o = orc.Image(data, W, H, D, dims=3, order=orc.RG, type=orc.HALF_FLOAT)
    for mode in range(4):
        tex = sess.texture(cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, vol), cl.texture_desc([mode] * 3, 1, 0, True))
        co = _coords(g, 3, (W, H, D), True)
        co4 = np.concatenate([co, np.zeros((co.shape[0], 1), np.float32)], 1)
        got = _run(sess, tprog, "fetch3d_f2", tex, co4, 8).view(np.uint32).reshape(-1, 2)
        _check_both(orc, got, o, o, mode, 1, 0, True, orc.RT_F, co4, 2, f"3D half m{mode}")
        cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(vol)
    W = 50
    data = synth.image_codes(g, cl.CL_RGBA, cl.CL_FLOAT, W)
    img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, W, host=data)
    o = orc.Image(data, W, 1, 1, dims=1, order=orc.RGBA, type=orc.FLOAT)
    for mode, filt in ((0, 1), (2, 0), (1, 1), (3, 0)):
        tex = sess.texture(cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, img), cl.texture_desc([mode], filt, 0, True))
        co = _coords(g, 1, (W,), True)
        got = _run(sess, tprog, "fetch1d_f4", tex, co, 16).view(np.uint32).reshape(-1, 4)
        _check_both(orc, got, o, o, mode, filt, 0, True, orc.RT_F, co, 4, f"1D m{mode} f{filt}")
        cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(img)


def test_tex1Dfetch_linear_resource_sees_later_writes(sess, orc, tprog):
    g = synth.rng(313)
    n, off = 3000, 256
    data = synth.image_codes(g, cl.CL_RGBA, cl.CL_FLOAT, n)
    host = np.zeros(off + n * 16, np.uint8)
    host[off:] = data.view(np.uint8).reshape(-1)
    buf = sess.buffer(host.nbytes, host)
    res = cl.ResourceDesc(cl.B2CL_RESOURCE_LINEAR, buf, off, cl.ChannelFormatDesc(32, 32, 32, 32, 2), n * 16)
    tex = sess.texture(res, cl.texture_desc([1], 0, 0, False))
    assert tex.sampler is None
    xs = np.concatenate([np.arange(n), [-1, n, n + 5, -2 ** 31, 2 ** 31 - 1]]).astype(np.int32)
    got = _run(sess, tprog, "fetch1dfetch_f4", tex, xs, 16, sampler=False).view(np.uint32).reshape(-1, 4)
    o = orc.Image(host[off:], n, 1, 1, dims=1, order=orc.RGBA, type=orc.FLOAT)
    exp = orc.tex1Dfetch(o, 0, xs)
    assert np.array_equal(got, exp)
    assert not got[n:].any()   # out of range: 0
    # a texture is a view: a later write to the buffer is what the next fetch sees
    pat = np.array([1.5, -2.0, 0.25, 7.0], np.float32)
    cl.check(cl.lib().clEnqueueFillBuffer(sess.queue, buf, pat.ctypes.data, 16, off + 16 * 10, 16 * 5,
                                          0, None, None))
    got = _run(sess, tprog, "fetch1dfetch_f4", tex, np.arange(8, 17, dtype=np.int32), 16,
               sampler=False).view(np.float32).reshape(-1, 4)
    assert np.array_equal(got[2:7], np.tile(pat, (5, 1)))
    assert np.array_equal(got[:2].view(np.uint32), data[0, 0, 8:10].view(np.uint32))
    cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(buf)


def test_tex2DLayered(sess, orc, tprog):
    g = synth.rng(314)
    W, H, L = 16, 9, 4
    data = synth.image_codes(g, cl.CL_R, cl.CL_FLOAT, W, H, L)
    arr = sess.image_array(cl.CL_R, cl.CL_FLOAT, W, L, H, host=data)
    o = orc.Image(data, W, H, L, dims=2, order=orc.R, type=orc.FLOAT, arrayed=True)
    for mode, filt in ((1, 1), (0, 1), (3, 0), (2, 1)):
        tex = sess.texture(cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, arr), cl.texture_desc([mode] * 2, filt, 0, True))
        co = _coords(g, 2, (W, H), True)
        co4 = np.concatenate([co, g.integers(-1, L + 1, (co.shape[0], 1)).astype(np.float32),
                              np.zeros((co.shape[0], 1), np.float32)], 1)
        got = _run(sess, tprog, "fetch2dlayered_f1", tex, co4, 4).view(np.uint32).reshape(-1, 1)
        _check_both(orc, got, o, o, mode, filt, 0, True, orc.RT_F, co4[:, :3], 1, f"layered m{mode}")
        cl.check(cl.lib().b2clDestroyTextureObject(ctypes.byref(tex)))
    sess.release(arr)


def test_texture_object_errors(sess):
    L = cl.lib()
    img = sess.image(cl.CL_RGBA, cl.CL_UNSIGNED_INT8, 8, 8)
    buf = sess.buffer(4096)
    t = cl.Texture()
    res = cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, img)
    mk = lambda r, d: L.b2clCreateTextureObject(sess.ctx, ctypes.byref(r), ctypes.byref(d), ctypes.byref(t))
    assert mk(res, cl.texture_desc([1, 3], 0, 0, True)) == -30          # modes differ (A40)
    assert mk(res, cl.texture_desc([1, 1], 1, 0, True)) == -59          # linear on an int read
    assert mk(res, cl.texture_desc([0, 0], 0, 0, False)) == -30         # wrap, unnormalized
    assert mk(res, cl.texture_desc([3, 3], 0, 1, True, (1, 0, 0, 0))) == -30  # border colour
    bad = cl.ResourceDesc(cl.B2CL_RESOURCE_LINEAR, buf, 8, cl.ChannelFormatDesc(32, 32, 32, 32, 2), 4096)
    assert mk(bad, cl.texture_desc([1], 0, 0, False)) == -30            # past the buffer end
    bad = cl.ResourceDesc(cl.B2CL_RESOURCE_PITCH2D, buf, 0, cl.ChannelFormatDesc(8, 8, 8, 8, 1), 0, 40, 4, 100)
    assert mk(bad, cl.texture_desc([1, 1], 0, 0, True)) == -30          # pitch < width * 4
    bad = cl.ResourceDesc(cl.B2CL_RESOURCE_ARRAY, buf)
    assert mk(bad, cl.texture_desc([1], 0, 0, True)) == -38             # ARRAY needs an image
    assert t.image is None and t.sampler is None                        # untouched on error
    sess.release(img, buf)
