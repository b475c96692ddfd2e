"""Tiled (block-linear) image storage (B2CL_MEM_TILED_IMAGE; north_star
"pitched and tiled image storage"): an internal layout of 2D images, invisible
through the API.  Every path that touches a tiled image is checked against the
oracle (reads, writes) or numpy (pixel boxes), on ragged sizes that span
several tiles, for several element sizes (the tile is 8 rows x 128 bytes)."""
import ctypes

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth
from tests.gpu_helpers import VALID_SAMPLERS, gpu_read_grid, gpu_read_samples, parity_read, rtype_of

pytestmark = pytest.mark.gpu
TILED = cl.CL_MEM_READ_WRITE | cl.B2CL_MEM_TILED_IMAGE
FORMATS = [(cl.CL_RGBA, cl.CL_FLOAT), (cl.CL_R, cl.CL_UNORM_INT8), (cl.CL_RG, cl.CL_HALF_FLOAT),
           (cl.CL_BGRA, cl.CL_UNORM_INT8), (cl.CL_RGBA, cl.CL_UNSIGNED_INT16), (cl.CL_R, cl.CL_FLOAT)]


def _pair(S, orc, order, type_, W, H, seed):
    codes = synth.image_codes(synth.rng(600 + seed), order, type_, W, H)
    tiled = S.image(order, type_, W, H, host=codes, flags=TILED)
    oimg = orc.Image(codes.copy(), W, H, 1, dims=2, order=order, type=type_)
    return tiled, oimg, codes


@pytest.mark.parametrize("fmt", FORMATS)
def test_tiled_upload_read_back_and_info(sess, orc, fmt):
    order, type_ = fmt
    W, H = 77, 43
    img, _, codes = _pair(sess, orc, order, type_, W, H, 1)
    es = sess.image_info(img, cl.CL_IMAGE_ELEMENT_SIZE)
    assert sess.image_info(img, cl.CL_IMAGE_ROW_PITCH) == W * es      # reading A46
    full = sess.read_image(img, (0, 0, 0), (W, H, 1))
    assert np.array_equal(full, codes.reshape(-1).view(np.uint8))
    # a sub-box with host pitches
    sub = sess.read_image(img, (5, 9, 0), (30, 17, 1), row_pitch=30 * es + 24)
    exp = codes[0, 9:26, 5:35].reshape(17, -1).view(np.uint8)
    got = sub.reshape(17, 30 * es + 24)[:, :30 * es]
    assert np.array_equal(got, exp)
    sess.release(img)


@pytest.mark.parametrize("fmt", FORMATS[:4])
def test_tiled_sampling_all_samplers(sess, orc, fmt):
    order, type_ = fmt
    W, H = 61, 35
    img, oimg, _ = _pair(sess, orc, order, type_, W, H, 2)
    rt = rtype_of(type_)
    g = synth.rng(610)
    for norm, addr, filt in VALID_SAMPLERS:
        lin = filt == cl.CL_FILTER_LINEAR
        if rt != cl.B2CL_RTYPE_FLOAT and lin:
            continue
        smp = sess.sampler(bool(norm), addr, filt)
        lo, hi = (-0.3, 1.3) if norm else (-3.0, max(W, H) + 3.0)
        co = g.uniform(lo, hi, (3000, 2)).astype(np.float32)
        got = gpu_read_samples(sess, img, smp, rt, co)
        rd = lambda im: orc.read_samples(im, bool(norm), addr, filt, rt, co)  # noqa: E731
        parity_read(got, rd(oimg), lin, f"tiled {fmt} {norm} {addr:#x} {filt:#x}", orc, oimg, rd)
        cl.lib().clReleaseSampler(smp)
    # grid mode, a rotation (the general kernel on tiled storage)
    smp = sess.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR if rt == cl.B2CL_RTYPE_FLOAT
                       else cl.CL_FILTER_NEAREST)
    A = synth.affine_rotate_2d(W, H, 30.0)
    filt = cl.CL_FILTER_LINEAR if rt == cl.B2CL_RTYPE_FLOAT else cl.CL_FILTER_NEAREST
    got = gpu_read_grid(sess, img, smp, rt, A, (W, H, 1), 4)
    rd = lambda im: orc.read_grid(im, True, cl.CL_ADDRESS_REPEAT, filt, rt, A, (W, H, 1), 4)  # noqa: E731
    parity_read(got, rd(oimg), filt == cl.CL_FILTER_LINEAR, f"tiled grid {fmt}", orc, oimg, rd)
    cl.lib().clReleaseSampler(smp)
    sess.release(img)


def test_tiled_copies_and_fill(sess, orc):
    L = cl.lib()
    W, H = 70, 29
    order, type_ = cl.CL_RGBA, cl.CL_UNORM_INT8
    t1, _, c1 = _pair(sess, orc, order, type_, W, H, 3)
    lin = sess.image(order, type_, W, H, host=synth.image_codes(synth.rng(620), order, type_, W, H))
    t2 = sess.image(order, type_, W, H, flags=TILED)
    z = (0, 0, 0)
    # tiled -> linear, linear -> tiled, tiled -> tiled, with offsets
    cl.check(L.clEnqueueCopyImage(sess.queue, t1, lin, cl.sz3((3, 4, 0)), cl.sz3((10, 1, 0)), cl.sz3((40, 20, 1)),
                                  0, None, None))
    cl.check(L.clEnqueueCopyImage(sess.queue, lin, t2, cl.sz3(z), cl.sz3(z), cl.sz3((W, H, 1)), 0, None, None))
    cl.check(L.clEnqueueCopyImage(sess.queue, t1, t2, cl.sz3((60, 20, 0)), cl.sz3((0, 0, 0)), cl.sz3((10, 9, 1)),
                                  0, None, None))
    exp_lin = synth.image_codes(synth.rng(620), order, type_, W, H)[0].copy()
    exp_lin[1:21, 10:50] = c1[0, 4:24, 3:43]
    exp_t2 = exp_lin.copy()
    exp_t2[0:9, 0:10] = c1[0, 20:29, 60:70]
    assert np.array_equal(sess.read_image(lin, z, (W, H, 1)).reshape(H, W, 4), exp_lin)
    assert np.array_equal(sess.read_image(t2, z, (W, H, 1)).reshape(H, W, 4), exp_t2)
    # image <-> buffer
    buf = sess.buffer(8 + 33 * 11 * 4)
    cl.check(L.clEnqueueCopyImageToBuffer(sess.queue, t1, buf, cl.sz3((30, 7, 0)), cl.sz3((33, 11, 1)), 8, 0,
                                          None, None))
    assert np.array_equal(sess.read(buf, 33 * 11 * 4, offset=8), c1[0, 7:18, 30:63].reshape(-1).view(np.uint8))
    cl.check(L.clEnqueueCopyBufferToImage(sess.queue, buf, t2, 8, cl.sz3((1, 15, 0)), cl.sz3((33, 11, 1)), 0,
                                          None, None))
    exp_t2[15:26, 1:34] = c1[0, 7:18, 30:63]
    assert np.array_equal(sess.read_image(t2, z, (W, H, 1)).reshape(H, W, 4), exp_t2)
    # fill (converted once with the write rules) and write_image samples
    col = np.array([1.0, 0.0, 0.5, 0.25], np.float32)
    cl.check(L.clEnqueueFillImage(sess.queue, t2, col.ctypes.data, cl.sz3((5, 3, 0)), cl.sz3((50, 12, 1)), 0,
                                  None, None))
    exp_t2[3:15, 5:55] = np.frombuffer(orc.convert_texel(orc.RGBA, orc.UNORM_INT8, orc.RT_F, col), np.uint8)
    assert np.array_equal(sess.read_image(t2, z, (W, H, 1)).reshape(H, W, 4), exp_t2)
    # host write into a tiled image, then read back
    host = synth.image_codes(synth.rng(621), order, type_, 23, 9)
    cl.check(L.clEnqueueWriteImage(sess.queue, t2, 1, cl.sz3((40, 19, 0)), cl.sz3((23, 9, 1)), 0, 0,
                                   host.ctypes.data, 0, None, None))
    exp_t2[19:28, 40:63] = host[0]
    assert np.array_equal(sess.read_image(t2, z, (W, H, 1)).reshape(H, W, 4), exp_t2)
    sess.release(t1, t2, lin, buf)


def test_tiled_write_samples_match_oracle(sess, orc):
    W, H = 50, 21
    order, type_ = cl.CL_RGBA, cl.CL_FLOAT
    img = sess.image(order, type_, W, H, host=np.zeros((1, H, W, 4), np.float32), flags=TILED)
    oimg = orc.Image(np.zeros((1, H, W, 4), np.float32), W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    g = synth.rng(630)
    ij = np.stack([g.integers(-3, W + 3, 500), g.integers(-3, H + 3, 500)], 1).astype(np.int32)
    cols = g.uniform(-2, 2, (500, 4)).astype(np.float32)
    # duplicates would race: keep the last writer of each texel only
    _, last = np.unique(ij[::-1], axis=0, return_index=True)
    keep = np.sort(len(ij) - 1 - last)
    ij, cols = np.ascontiguousarray(ij[keep]), np.ascontiguousarray(cols[keep])
    cb, kb = sess.buffer(ij.nbytes, ij), sess.buffer(cols.nbytes, cols)
    cl.check(cl.lib().b2clEnqueueWriteImageSamples(sess.queue, img, cl.B2CL_RTYPE_FLOAT, cb, 0, len(ij), kb, 0, 0,
                                                   None, None))
    orc.write_samples(oimg, orc.RT_F, ij, cols)
    got = sess.read_image(img, (0, 0, 0), (W, H, 1))
    assert np.array_equal(got, oimg.data)
    sess.release(img, cb, kb)


def test_tiled_rejections(sess):
    L = cl.lib()
    err = ctypes.c_int32()
    fmt = cl.ImageFormat(cl.CL_RGBA, cl.CL_FLOAT)
    for t, w, h, d in ((cl.CL_MEM_OBJECT_IMAGE3D, 8, 8, 8), (cl.CL_MEM_OBJECT_IMAGE1D, 8, 0, 0)):
        desc = cl.ImageDesc(t, w, h, d, 0, 0, 0, 0, 0, None)
        m = L.clCreateImage(sess.ctx, TILED, ctypes.byref(fmt), ctypes.byref(desc), None, ctypes.byref(err))
        assert not m and err.value == -30
    m = L.clCreateBuffer(sess.ctx, TILED, 64, None, ctypes.byref(err))
    assert not m and err.value == -30
    desc = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE2D, 64, 64, 0, 0, 0, 0, 0, 0, None)
    m = L.b2clCreateImageShard(sess.ctx, TILED, ctypes.byref(fmt), ctypes.byref(desc), 0, 16, 1, None,
                               ctypes.byref(err))
    assert not m and err.value == -30


def test_tiled_image_as_translated_kernel_argument(sess, orc):
    """A translated kernel (tests/kernels/translated.cu box3) reading a tiled
    image through the device header's built-ins: the same bits as a pitched one."""
    from tests.test_gpu_kernels import _cubin_bytes
    W, H, LX = 96, 20, 32
    codes = synth.image_codes(synth.rng(80), cl.CL_RGBA, cl.CL_FLOAT, W, H)
    prog = sess.program(_cubin_bytes())
    smp = sess.sampler(False, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    outs = []
    for flags in (cl.CL_MEM_READ_WRITE, TILED):
        img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, W, H, host=codes, flags=flags)
        out = sess.buffer(W * H * 16)
        k = sess.kernel(prog, "box3")
        sess.set_args(k, img, smp, out, ("local", LX * 16), ctypes.c_int32(W))
        sess.ndrange(k, (W, H), (LX, 1))
        outs.append(sess.read(out, W * H * 16, np.uint32))
        cl.lib().clReleaseKernel(k)
        sess.release(img, out)
    assert np.array_equal(outs[0], outs[1])
    cl.lib().clReleaseSampler(smp)
    cl.lib().clReleaseProgram(prog)
