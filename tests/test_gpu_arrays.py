"""GPU parity of image arrays and 1D image buffers (
[CL1.2 §5.3.1], §8.4) through the C-ABI against the CPU oracle: the read
built-ins (samples and grid), writes, host transfers with the 1D-array
slice-pitch rule, pixel-box copies/fills across layers, image info, and a 1D
image buffer wider than CUDA's 2^27-texel linear-texture limit."""
import ctypes

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth

from tests.gpu_helpers import (VALID_SAMPLERS, assert_parity, parity_read, gpu_read_grid,
                         gpu_read_samples, rtype_of)

pytestmark = pytest.mark.gpu

FORMATS = [(cl.CL_RGBA, cl.CL_FLOAT), (cl.CL_R, cl.CL_UNORM_INT8), (cl.CL_RG, cl.CL_HALF_FLOAT),
           (cl.CL_BGRA, cl.CL_UNORM_INT8), (cl.CL_RGBA, cl.CL_SIGNED_INT16),
           (cl.CL_LUMINANCE, cl.CL_SNORM_INT16), (cl.CL_RA, cl.CL_UNSIGNED_INT32)]


def _arrays(S, orc, order, type_, W, H, L, seed):
    """The same seeded codes as a GPU image array and an oracle array (H = 0: 1D array)."""
    g = synth.rng(400 + seed)
    if H:
        codes = synth.image_codes(g, order, type_, W, H, L)                 # (L, H, W, c)
        oimg = orc.Image(codes.copy(), W, H, L, dims=2, order=order, type=type_, arrayed=True)
    else:
        codes = synth.image_codes(g, order, type_, W, L)                    # (1, L, W, c)
        oimg = orc.Image(codes.copy(), W, L, 1, dims=1, order=order, type=type_, arrayed=True)
    img = S.image_array(order, type_, W, L, H, host=codes)
    return img, oimg, codes


def _coords(g, n, dims, W, H, L, norm, integer):
    ext = [W, H][:dims]
    if integer:
        cols = [g.integers(-2, e + 2, n) for e in ext] + [g.integers(-2, L + 2, n)]
        c = np.stack(cols, 1).astype(np.int32)
    else:
        cols = [(g.uniform(-0.4, 1.4, n) if norm else g.uniform(-3, e + 3, n)) for e in ext]
        lay = np.concatenate([g.uniform(-2, L + 1, n - 8),
                              [0.5, 1.5, 2.5, -0.5, L - 0.5, L + 0.5, np.nan, 1e9]])
        c = np.stack(cols + [lay], 1).astype(np.float32)
    if dims == 2:  # 2D arrays take 4-component coordinates
        c = np.concatenate([c, np.zeros((n, 1), c.dtype)], 1)
    return np.ascontiguousarray(c)


@pytest.mark.parametrize("dims", [1, 2])
@pytest.mark.parametrize("fmt", FORMATS)
def test_array_samples_all_samplers(sess, orc, dims, fmt):
    order, type_ = fmt
    W, H, L = 37, (11 if dims == 2 else 0), 5
    img, oimg, _ = _arrays(sess, orc, order, type_, W, H, L, dims)
    rt = rtype_of(type_)
    g = synth.rng(410 + dims)
    for norm, addr, filt in VALID_SAMPLERS:
        lin = filt == cl.CL_FILTER_LINEAR
        if rt != cl.B2CL_RTYPE_FLOAT and lin:
            continue
        smp = sess.sampler(bool(norm), addr, filt)
        co = _coords(g, 700, dims, W, H or 1, L, norm, False)
        got = gpu_read_samples(sess, img, smp, rt, co)
        rd = lambda im: orc.read_samples(im, bool(norm), addr, filt, rt, co)  # noqa: E731
        parity_read(got, rd(oimg), lin, f"{dims}D array {fmt} {norm} {addr:#x} {filt:#x}", orc, oimg, rd)
        if not norm and not lin:  # integer coordinates (reading A30)
            ci = _coords(g, 300, dims, W, H or 1, L, norm, True)
            got = gpu_read_samples(sess, img, smp, rt, ci, int_coords=True)
            exp = orc.read_samples(oimg, False, addr, filt, rt, ci)
            assert_parity(got, exp, False, f"{dims}D array int coords")
        cl.lib().clReleaseSampler(smp)
    sess.release(img)


@pytest.mark.parametrize("dims", [1, 2])
def test_array_grid(sess, orc, dims):
    W, H, L = 70, (45 if dims == 2 else 0), 6
    img, oimg, _ = _arrays(sess, orc, cl.CL_RGBA, cl.CL_FLOAT, W, H, L, 20 + dims)
    if dims == 2:  # layer = 0.6*z - 0.3 + 0.01*x: the layer coordinate may depend on x
        A = [1.02, 0.13, 0.0, -1.5, -0.07, 0.96, 0.0, 0.4, 0.01, 0.0, 0.6, -0.3]
        out = (W + 3, H + 2, 9)
    else:     # 1D array: coordinate 1 (the layer) from y
        A = [0.93, 0.0, 0.0, -2.2, 0.0, 0.55, 0.0, -0.8, 0, 0, 0, 0]
        out = (W + 5, 15, 1)
    for norm, addr, filt in VALID_SAMPLERS:
        if norm:
            continue  # unnormalized keeps the map readable; normalized is covered by samples
        smp = sess.sampler(False, addr, filt)
        got = gpu_read_grid(sess, img, smp, cl.B2CL_RTYPE_FLOAT, A, out, 4)
        rd = lambda im: orc.read_grid(im, False, addr, filt, orc.RT_F, np.array(A, np.float32), out, 4)  # noqa: E731
        parity_read(got, rd(oimg), filt == cl.CL_FILTER_LINEAR, f"grid {dims}D array {addr:#x}", orc, oimg, rd)
        cl.lib().clReleaseSampler(smp)
    sess.release(img)


def test_array_write_samples(sess, orc):
    W, H, L = 13, 7, 4
    for dims in (1, 2):
        img, oimg, codes = _arrays(sess, orc, cl.CL_RGBA, cl.CL_UNORM_INT8, W, H if dims == 2 else 0,
                                   L, 30 + dims)
        g = synth.rng(420 + dims)
        n = 500
        cols = [g.integers(-1, W + 1, n)] + ([g.integers(-1, H + 1, n)] if dims == 2 else [])
        cols.append(g.integers(-1, L + 1, n))
        co = np.stack(cols, 1).astype(np.int32)
        if dims == 2:
            co = np.concatenate([co, np.zeros((n, 1), np.int32)], 1)
        co = np.ascontiguousarray(co)
        # distinct targets so the result does not depend on write order
        _, first = np.unique(co, axis=0, return_index=True)
        co = np.ascontiguousarray(co[np.sort(first)])
        n = co.shape[0]
        colors = g.uniform(-0.2, 1.2, (n, 4)).astype(np.float32)
        cb, kb = sess.buffer(co.nbytes, co), sess.buffer(colors.nbytes, colors)
        cl.check(cl.lib().b2clEnqueueWriteImageSamples(sess.queue, img, cl.B2CL_RTYPE_FLOAT, cb, 0,
                                                       n, kb, 0, 0, None, None))
        orc.write_samples(oimg, orc.RT_F, co, colors)
        region = (W, H, L) if dims == 2 else (W, L, 1)
        got = sess.read_image(img, (0, 0, 0), region)
        assert np.array_equal(got, oimg.data[:got.size]), dims
        sess.release(img, cb, kb)


def test_1d_array_host_transfers_use_slice_pitch(sess, orc):
    W, L, es = 19, 9, 4
    g = synth.rng(430)
    codes = synth.image_codes(g, cl.CL_RGBA, cl.CL_UNORM_INT8, W, L)
    # creation from a host array whose layers are 160 bytes apart (image_slice_pitch:
    # >= image_row_pitch and a multiple of it, [CL1.2 §5.3.1])
    host = np.zeros(160 * L, np.uint8)
    for l in range(L):
        host[160 * l:160 * l + W * es] = codes[0, l].reshape(-1)
    err = ctypes.c_int32()
    fmt = cl.ImageFormat(cl.CL_RGBA, cl.CL_UNORM_INT8)
    bad = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE1D_ARRAY, W, 0, 0, L, 80, 100, 0, 0, None)
    assert cl.lib().clCreateImage(sess.ctx, cl.CL_MEM_COPY_HOST_PTR, ctypes.byref(fmt),
                                  ctypes.byref(bad), host.ctypes.data, ctypes.byref(err)) is None
    assert err.value == -65
    img = sess.image_array(cl.CL_RGBA, cl.CL_UNORM_INT8, W, L, host=host, host_row_pitch=80,
                           host_slice_pitch=160)
    oimg = orc.Image(codes.copy(), W, L, 1, dims=1, order=orc.RGBA, type=orc.UNORM_INT8,
                     arrayed=True)
    assert np.array_equal(sess.read_image(img, (0, 0, 0), (W, L, 1)), oimg.data)
    for origin, region, rp, sp in (((2, 1, 0), (5, 4, 1), 0, 0), ((0, 3, 0), (W, 6, 1), 0, 96),
                                   ((7, 0, 0), (4, 9, 1), 24, 40)):
        n = 2000
        got = np.full(n, 0xEE, np.uint8)
        cl.check(cl.lib().clEnqueueReadImage(sess.queue, img, 1, cl.sz3(origin), cl.sz3(region),
                                             rp, sp, got.ctypes.data, 0, None, None))
        exp = np.full(n, 0xEE, np.uint8)
        orc.read_image_rect(oimg, origin, region, rp, sp, exp)
        assert np.array_equal(got, exp), (origin, region, rp, sp)
        # write the host bytes back shifted by one layer, compare the whole array
        o2 = (origin[0], (origin[1] + 1) % (L - region[1] + 1), 0)
        cl.check(cl.lib().clEnqueueWriteImage(sess.queue, img, 1, cl.sz3(o2), cl.sz3(region), rp,
                                              sp, got.ctypes.data, 0, None, None))
        orc.write_image_rect(oimg, o2, region, rp, sp, got)
        assert np.array_equal(sess.read_image(img, (0, 0, 0), (W, L, 1)), oimg.data)
    # a 2D image's rule is unchanged: slice pitch must be 0 for it
    img2 = sess.image(cl.CL_RGBA, cl.CL_UNORM_INT8, W, L)
    buf = np.zeros(4000, np.uint8)
    assert cl.lib().clEnqueueReadImage(sess.queue, img2, 1, cl.sz3((0, 0, 0)), cl.sz3((W, L, 1)),
                                       0, 200, buf.ctypes.data, 0, None, None) == -30
    sess.release(img, img2)


def test_array_copies_and_fills(sess, orc):
    W, H, L = 24, 10, 6
    a2, oa2, _ = _arrays(sess, orc, cl.CL_RGBA, cl.CL_HALF_FLOAT, W, H, L, 40)
    g = synth.rng(440)
    codes3 = synth.image_codes(g, cl.CL_RGBA, cl.CL_HALF_FLOAT, W, H, L)
    v3 = sess.image(cl.CL_RGBA, cl.CL_HALF_FLOAT, W, H, L, host=codes3)
    ov3 = orc.Image(codes3.copy(), W, H, L, dims=3, order=orc.RGBA, type=orc.HALF_FLOAT)
    # layers 1..3 of the 2D array -> slices 2..4 of the 3D image, and back into layers 0..2
    cl.check(cl.lib().clEnqueueCopyImage(sess.queue, a2, v3, cl.sz3((3, 1, 1)), cl.sz3((0, 2, 2)),
                                         cl.sz3((17, 8, 3)), 0, None, None))
    orc.copy_image(oa2, ov3, (3, 1, 1), (0, 2, 2), (17, 8, 3))
    cl.check(cl.lib().clEnqueueCopyImage(sess.queue, v3, a2, cl.sz3((1, 0, 3)), cl.sz3((2, 2, 0)),
                                         cl.sz3((20, 8, 3)), 0, None, None))
    orc.copy_image(ov3, oa2, (1, 0, 3), (2, 2, 0), (20, 8, 3))
    # fill layers 4..5, then array -> buffer of layers 2..5
    color = np.array([0.25, -1.5, 65504.0, 3.0], np.float32)
    cl.check(cl.lib().clEnqueueFillImage(sess.queue, a2, color.ctypes.data, cl.sz3((5, 3, 4)),
                                         cl.sz3((9, 4, 2)), 0, None, None))
    orc.fill_image(oa2, orc.RT_F, color, (5, 3, 4), (9, 4, 2))
    nb = W * H * 4 * 8
    buf = sess.buffer(nb + 64)
    cl.check(cl.lib().clEnqueueCopyImageToBuffer(sess.queue, a2, buf, cl.sz3((0, 0, 2)),
                                                 cl.sz3((W, H, 4)), 64, 0, None, None))
    exp = np.zeros(nb + 64, np.uint8)
    orc.copy_image_to_buffer(oa2, exp, (0, 0, 2), (W, H, 4), 64)
    assert np.array_equal(sess.read(buf, nb + 64)[64:], exp[64:])
    assert np.array_equal(sess.read_image(a2, (0, 0, 0), (W, H, L)), oa2.data)
    assert np.array_equal(sess.read_image(v3, (0, 0, 0), (W, H, L)), ov3.data)
    # 1D array: CopyBufferToImage into layers 3..4
    a1, oa1, _ = _arrays(sess, orc, cl.CL_R, cl.CL_FLOAT, W, 0, L, 41)
    src = synth.rng(441).integers(0, 256, 4096, dtype=np.uint8)
    sb = sess.buffer(src.nbytes, src)
    cl.check(cl.lib().clEnqueueCopyBufferToImage(sess.queue, sb, a1, 12, cl.sz3((4, 3, 0)),
                                                 cl.sz3((15, 2, 1)), 0, None, None))
    orc.copy_buffer_to_image(src, oa1, 12, (4, 3, 0), (15, 2, 1))
    assert np.array_equal(sess.read_image(a1, (0, 0, 0), (W, L, 1)), oa1.data)
    # boxes beyond the layer count are rejected
    assert cl.lib().clEnqueueFillImage(sess.queue, a1, color.ctypes.data, cl.sz3((0, 5, 0)),
                                       cl.sz3((1, 2, 1)), 0, None, None) == -30
    sess.release(a2, v3, buf, a1, sb)


def test_array_and_buffer_image_info(sess):
    a1 = sess.image_array(cl.CL_RGBA, cl.CL_FLOAT, 100, 7)
    a2 = sess.image_array(cl.CL_R, cl.CL_UNORM_INT8, 30, 5, 20)
    b = sess.buffer(4096)
    ib = sess.image_buffer(cl.CL_RG, cl.CL_UNSIGNED_INT16, 1000, b)
    info = lambda m, n: sess.image_info(m, n)  # noqa: E731
    assert [info(a1, n) for n in (cl.CL_IMAGE_WIDTH, cl.CL_IMAGE_HEIGHT, cl.CL_IMAGE_DEPTH,
                                  cl.CL_IMAGE_ARRAY_SIZE)] == [100, 0, 0, 7]
    assert info(a1, cl.CL_IMAGE_SLICE_PITCH) == info(a1, cl.CL_IMAGE_ROW_PITCH) >= 1600
    assert [info(a2, n) for n in (cl.CL_IMAGE_WIDTH, cl.CL_IMAGE_HEIGHT, cl.CL_IMAGE_DEPTH,
                                  cl.CL_IMAGE_ARRAY_SIZE)] == [30, 20, 0, 5]
    assert info(a2, cl.CL_IMAGE_SLICE_PITCH) == 20 * info(a2, cl.CL_IMAGE_ROW_PITCH)
    assert [info(ib, n) for n in (cl.CL_IMAGE_WIDTH, cl.CL_IMAGE_HEIGHT, cl.CL_IMAGE_ARRAY_SIZE,
                                  cl.CL_IMAGE_ROW_PITCH, cl.CL_IMAGE_SLICE_PITCH)] == [1000, 0, 0,
                                                                                      4000, 0]
    assert info(ib, cl.CL_IMAGE_BUFFER) == b
    t = ctypes.c_uint32()
    cl.check(cl.lib().clGetMemObjectInfo(ib, 0x1100, 4, ctypes.byref(t), None))
    assert t.value == cl.CL_MEM_OBJECT_IMAGE1D_BUFFER
    # descriptor errors: a 1D buffer image larger than its buffer, a missing buffer,
    # a host pointer, an array of 0 layers
    err = ctypes.c_int32()
    fmt = cl.ImageFormat(cl.CL_RGBA, cl.CL_FLOAT)
    d = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE1D_BUFFER, 257, 0, 0, 0, 0, 0, 0, 0, b)
    assert cl.lib().clCreateImage(sess.ctx, 0, ctypes.byref(fmt), ctypes.byref(d), None,
                                  ctypes.byref(err)) is None and err.value == -40
    d = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE1D_BUFFER, 16, 0, 0, 0, 0, 0, 0, 0, None)
    assert cl.lib().clCreateImage(sess.ctx, 0, ctypes.byref(fmt), ctypes.byref(d), None,
                                  ctypes.byref(err)) is None and err.value == -65
    d = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE1D_ARRAY, 16, 0, 0, 0, 0, 0, 0, 0, None)
    assert cl.lib().clCreateImage(sess.ctx, 0, ctypes.byref(fmt), ctypes.byref(d), None,
                                  ctypes.byref(err)) is None and err.value == -65
    sess.release(a1, a2, ib, b)


def test_1d_image_buffer_aliases_its_buffer(sess, orc):
    W = 3000
    g = synth.rng(450)
    codes = synth.image_codes(g, cl.CL_RGBA, cl.CL_UNORM_INT16, W)
    b = sess.buffer(codes.nbytes + 100, np.concatenate([codes.view(np.uint8).reshape(-1),
                                                        np.zeros(100, np.uint8)]))
    ib = sess.image_buffer(cl.CL_RGBA, cl.CL_UNORM_INT16, W, b)
    sess.release(b)  # the image keeps its buffer alive
    oimg = orc.Image(codes.copy(), W, 1, 1, dims=1, order=orc.RGBA, type=orc.UNORM_INT16)
    smp = sess.sampler(False, cl.CL_ADDRESS_NONE, cl.CL_FILTER_NEAREST)
    ci = np.arange(-3, W + 3, dtype=np.int32)[:, None].copy()
    got = gpu_read_samples(sess, ib, smp, cl.B2CL_RTYPE_FLOAT, ci, int_coords=True)
    exp = orc.read_samples(oimg, False, orc.ADDRESS_NONE, orc.FILTER_NEAREST, orc.RT_F, ci)
    assert_parity(got, exp, False, "1D buffer image")
    # a write through the image is a write of the buffer's bytes
    co = np.array([[5], [W - 1], [W]], np.int32)
    col = np.array([[1, 0, 0.5, 2], [0, 0, 0, 0], [1, 1, 1, 1]], np.float32)
    cb, kb = sess.buffer(co.nbytes, co), sess.buffer(col.nbytes, col)
    cl.check(cl.lib().b2clEnqueueWriteImageSamples(sess.queue, ib, cl.B2CL_RTYPE_FLOAT, cb, 0, 3,
                                                   kb, 0, 0, None, None))
    orc.write_samples(oimg, orc.RT_F, co, col)
    got = sess.read_image(ib, (0, 0, 0), (W, 1, 1))
    assert np.array_equal(got, oimg.data)
    cl.lib().clReleaseSampler(smp)
    sess.release(ib, cb, kb)


def test_1d_image_buffer_beyond_cuda_texture_limit(sess, orc):
    """Width 2^28 + 1000 texels > the 2^27 CUDA 1D linear-texture limit the paper
    reports: read back at sampled coordinates, LINEAR too."""
    W = (1 << 28) + 1000
    g = synth.rng(460)
    b = sess.buffer(W)
    # fill with a byte ramp (FillBuffer with a 128-byte pattern: texel i = i mod 128)
    pat = np.arange(128, dtype=np.uint8)
    cl.check(cl.lib().clEnqueueFillBuffer(sess.queue, b, pat.ctypes.data, 128, 0, W // 128 * 128,
                                          0, None, None))
    ib = sess.image_buffer(cl.CL_R, cl.CL_UNORM_INT8, W // 128 * 128, b)
    n = W // 128 * 128
    idx = np.concatenate([g.integers(0, n, 2000), [0, 1, (1 << 27) - 1, 1 << 27, (1 << 27) + 1,
                                                    n - 2, n - 1]])
    smp = sess.sampler(False, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_NEAREST)
    got = gpu_read_samples(sess, ib, smp, cl.B2CL_RTYPE_FLOAT, idx.astype(np.int32)[:, None].copy(),
                           int_coords=True)
    exp = (idx % 128).astype(np.float32) / np.float32(255.0)
    assert np.array_equal(got[:, 0], exp.astype(np.float32))
    # LINEAR and normalized coordinates over the whole width against the oracle
    # on the same 256 MiB of texels (fp32 spacing at 2^28 is 32 texels: the
    # address arithmetic is what the spec's fp32 formulas give there)
    oimg = orc.Image(np.tile(np.arange(128, dtype=np.uint8), n // 128), n, 1, 1, dims=1,
                     order=orc.R, type=orc.UNORM_INT8)
    smp2 = sess.sampler(False, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    u = np.concatenate([g.uniform(0, n, 3000), n - g.uniform(0, 64, 100)]).astype(np.float32)
    got = gpu_read_samples(sess, ib, smp2, cl.B2CL_RTYPE_FLOAT, u[:, None].copy())
    exp = orc.read_samples(oimg, False, orc.ADDRESS_CLAMP_TO_EDGE, orc.FILTER_LINEAR, orc.RT_F,
                           u[:, None].copy())
    assert_parity(got, exp, True, "2^28 LINEAR")
    smp3 = sess.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR)
    s_ = g.uniform(-1, 2, 3000).astype(np.float32)
    got = gpu_read_samples(sess, ib, smp3, cl.B2CL_RTYPE_FLOAT, s_[:, None].copy())
    exp = orc.read_samples(oimg, True, orc.ADDRESS_REPEAT, orc.FILTER_LINEAR, orc.RT_F,
                           s_[:, None].copy())
    assert_parity(got, exp, True, "2^28 REPEAT")
    cl.lib().clReleaseSampler(smp3)
    cl.lib().clReleaseSampler(smp)
    cl.lib().clReleaseSampler(smp2)
    sess.release(ib, b)
