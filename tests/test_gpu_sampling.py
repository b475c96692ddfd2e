"""GPU parity of the read_image / write_image path (steps a1-a8) through the C-ABI
against the CPU oracle, on the same seeded inputs.

Bar (BASELINE.json north_star): NEAREST, integer formats and writes bit-exact;
LINEAR within 4 fp32 ulp or 1e-6 absolute, NaN iff NaN.
"""
import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth
from tests.gpu_helpers import (VALID_SAMPLERS, assert_parity, coord_stride, gpu_read_grid,
                               gpu_read_samples, make_images, parity_read, rtype_of)

pytestmark = pytest.mark.gpu

R, RG, RA, A_, RGBA, BGRA, ARGB, INT_, LUM = (cl.CL_R, cl.CL_RG, cl.CL_RA, cl.CL_A, cl.CL_RGBA,
                                              cl.CL_BGRA, cl.CL_ARGB, cl.CL_INTENSITY,
                                              cl.CL_LUMINANCE)
F32, F16, U8N, U16N, S8N, S16N = (cl.CL_FLOAT, cl.CL_HALF_FLOAT, cl.CL_UNORM_INT8,
                                  cl.CL_UNORM_INT16, cl.CL_SNORM_INT8, cl.CL_SNORM_INT16)

FLOAT_FORMATS = [(RGBA, F32), (R, F32), (RGBA, U8N), (BGRA, U8N), (RG, F16), (RGBA, U16N),
                 (R, S8N), (RA, S16N), (A_, U8N), (INT_, U8N), (LUM, F32), (ARGB, U8N),
                 (RGBA, F16), (RG, U8N),
                 # packed formats (NEXT row 4); CL_RGBx: border alpha 0 vs texel alpha 1
                 (cl.CL_RGB, cl.CL_UNORM_SHORT_565), (cl.CL_RGBx, cl.CL_UNORM_SHORT_555),
                 (cl.CL_RGBx, cl.CL_UNORM_INT_101010), (cl.CL_RGB, cl.CL_UNORM_INT_101010)]
INT_FORMATS = [(RGBA, cl.CL_UNSIGNED_INT8), (R, cl.CL_SIGNED_INT16), (RG, cl.CL_UNSIGNED_INT32),
               (RGBA, cl.CL_SIGNED_INT32), (BGRA, cl.CL_SIGNED_INT8), (RA, cl.CL_UNSIGNED_INT16)]
SHAPES = [(1, (37, 1, 1)), (2, (1, 1, 1)), (2, (3, 5, 1)), (2, (65, 33, 1)), (3, (7, 3, 2)),
          (3, (9, 6, 5))]


def _coords(g, dims, size, norm, n_rand=3000):
    W, H, D = size
    ns = np.array([W, H, D][:dims], np.float32)
    sp = synth.special_floats()
    lat = synth.coord_lattice(-2, 3, 1 / 32) if norm else synth.coord_lattice(-2, max(W, H, D) + 2, 1 / 16)
    lo, hi = (-1.5, 2.5) if norm else (-2.0, 1.0)
    if norm:
        rnd = g.uniform(lo, hi, (n_rand, dims)).astype(np.float32)
    else:
        rnd = (g.uniform(-0.2, 1.2, (n_rand, dims)) * ns).astype(np.float32)
    pts = [rnd]
    for d in range(dims):
        for vals in (lat, sp):
            c = rnd[:vals.size].copy() if vals.size <= n_rand else np.resize(rnd, (vals.size, dims))
            c[:, d] = vals
            pts.append(c)
    c = np.concatenate(pts).astype(np.float32)
    if dims == 3:
        c = np.concatenate([c, np.zeros((c.shape[0], 1), np.float32)], 1)
    return np.ascontiguousarray(c)


@pytest.mark.parametrize("order,type_", FLOAT_FORMATS)
@pytest.mark.parametrize("dims,size", SHAPES)
def test_read_imagef_all_samplers(sess, orc, order, type_, dims, size):
    W, H, D = size
    signed = type_ in (F32, F16)
    img, oimg, _ = make_images(sess, orc, order, type_, W, H, D, dims, seed=W * 7 + H + D,
                               signed=signed)
    g = synth.rng(77 + W + H + D)
    try:
        for norm, addr, filt in VALID_SAMPLERS:
            smp = sess.sampler(norm, addr, filt)
            co = _coords(g, dims, size, norm)
            got = gpu_read_samples(sess, img, smp, cl.B2CL_RTYPE_FLOAT, co)
            rd = lambda im: orc.read_samples(im, norm, addr, filt, orc.RT_F, co)  # noqa: E731
            # mixed-sign texels: the LINEAR bound counts ulps of the condition sum
            # |w|*|T| (the oracle's read of the |T| image), reading A10
            parity_read(got, rd(oimg), filt == cl.CL_FILTER_LINEAR,
                        f"fmt {hex(order)}/{hex(type_)} dims {dims} smp {norm},{hex(addr)},{hex(filt)}",
                        orc, oimg, rd)
            cl.lib().clReleaseSampler(smp)
    finally:
        sess.release(img)


@pytest.mark.parametrize("order,type_", INT_FORMATS)
@pytest.mark.parametrize("dims,size", [(1, (19, 1, 1)), (2, (13, 7, 1)), (3, (5, 4, 3))])
def test_read_imagei_ui_nearest(sess, orc, order, type_, dims, size):
    W, H, D = size
    img, oimg, _ = make_images(sess, orc, order, type_, W, H, D, dims, seed=3 * W + H)
    g = synth.rng(99)
    rt = rtype_of(type_)
    try:
        for norm, addr, filt in VALID_SAMPLERS:
            if filt != cl.CL_FILTER_NEAREST:
                continue
            smp = sess.sampler(norm, addr, filt)
            co = _coords(g, dims, size, norm, 1500)
            got = gpu_read_samples(sess, img, smp, rt, co)
            exp = orc.read_samples(oimg, norm, addr, filt, rt, co)
            assert_parity(got, exp, False, f"int fmt {hex(order)}/{hex(type_)} {norm},{hex(addr)}")
            cl.lib().clReleaseSampler(smp)
    finally:
        sess.release(img)


@pytest.mark.parametrize("dims", [1, 2, 3])
def test_integer_coordinates(sess, orc, dims):
    size = (11, 6, 4)
    W, H, D = size
    img, oimg, _ = make_images(sess, orc, RGBA, U8N, W, H, D, dims, seed=5)
    g = synth.rng(5)
    ic = g.integers(-3, 14, (2000, coord_stride(dims))).astype(np.int32)
    ic[:5, 0] = [-2 ** 31, 2 ** 31 - 1, 0, -1, W]
    for addr in (cl.CL_ADDRESS_NONE, cl.CL_ADDRESS_CLAMP, cl.CL_ADDRESS_CLAMP_TO_EDGE):
        smp = sess.sampler(False, addr, cl.CL_FILTER_NEAREST)
        got = gpu_read_samples(sess, img, smp, cl.B2CL_RTYPE_FLOAT, ic, int_coords=True)
        exp = orc.read_samples(oimg, False, addr, cl.CL_FILTER_NEAREST, orc.RT_F, ic)
        assert_parity(got, exp, False, f"icoord {hex(addr)}")
    sess.release(img)


def test_unorm_codes_exhaustive(sess, orc):
    """Every UNORM/SNORM 8/16 code through read_imagef equals IEEE c/d (A11)."""
    for type_, n in ((U8N, 256), (S8N, 256), (U16N, 65536), (S16N, 65536)):
        codes = np.arange(n, dtype=np.uint32).astype(np.uint8 if n == 256 else np.uint16)
        if type_ in (S8N, S16N):
            codes = codes.view(np.int8 if n == 256 else np.int16)
        W = 256
        Hh = n // W
        img = sess.image(R, type_, W, Hh, host=codes.reshape(Hh, W, 1))
        oimg = orc.Image(codes.reshape(1, Hh, W, 1).copy(), W, Hh, 1, dims=2, order=R, type=type_)
        smp = sess.sampler(False, cl.CL_ADDRESS_NONE, cl.CL_FILTER_NEAREST)
        xs, ys = np.meshgrid(np.arange(W) + 0.5, np.arange(Hh) + 0.5)
        co = np.stack([xs.ravel(), ys.ravel()], 1).astype(np.float32)
        got = gpu_read_samples(sess, img, smp, cl.B2CL_RTYPE_FLOAT, co)
        exp = orc.read_samples(oimg, False, cl.CL_ADDRESS_NONE, cl.CL_FILTER_NEAREST, orc.RT_F, co)
        assert_parity(got, exp, False, f"codes {hex(type_)}")
        sess.release(img)


@pytest.mark.parametrize("order", [cl.CL_RGB, cl.CL_RGBx])
def test_packed_words_exhaustive(sess, orc, order):
    """Every 565 / 555 word and 2^16 random 101010 words through read_imagef
    (NEXT row 4): bit-exact to the oracle, whose fields are pinned to numpy."""
    g = synth.rng(13)
    for type_ in (cl.CL_UNORM_SHORT_565, cl.CL_UNORM_SHORT_555, cl.CL_UNORM_INT_101010):
        if type_ == cl.CL_UNORM_INT_101010:
            words = g.integers(0, 1 << 32, 1 << 16, dtype=np.uint64).astype(np.uint32)
        else:
            words = np.arange(1 << 16, dtype=np.uint16)
        W, Hh = 256, words.size // 256
        img = sess.image(order, type_, W, Hh, host=words.reshape(Hh, W, 1))
        oimg = orc.Image(words.reshape(1, Hh, W, 1).copy(), W, Hh, 1, dims=2, order=order, type=type_)
        smp = sess.sampler(False, cl.CL_ADDRESS_NONE, cl.CL_FILTER_NEAREST)
        xs, ys = np.meshgrid(np.arange(W) + 0.5, np.arange(Hh) + 0.5)
        co = np.stack([xs.ravel(), ys.ravel()], 1).astype(np.float32)
        got = gpu_read_samples(sess, img, smp, cl.B2CL_RTYPE_FLOAT, co)
        exp = orc.read_samples(oimg, False, cl.CL_ADDRESS_NONE, cl.CL_FILTER_NEAREST, orc.RT_F, co)
        assert_parity(got, exp, False, f"packed {hex(order)}/{hex(type_)}")
        cl.lib().clReleaseSampler(smp)
        sess.release(img)


# ---------------------------------------------------------------- grid mode
GRID_CASES = [
    # (dims, order, type, img size, sampler, affine-maker, out dims, outc)
    (2, RGBA, F32, (97, 61, 1), (1, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR), "translate", (97, 61, 1), 4),
    (2, RGBA, F32, (97, 61, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "translate", (97, 61, 1), 4),
    (2, RGBA, F32, (64, 48, 1), (1, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR), "rotate", (70, 50, 1), 4),
    (2, RGBA, F32, (64, 48, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "rotate", (70, 50, 1), 4),
    (3, R, F32, (40, 33, 17), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil", (40, 33, 17), 1),
    (3, R, F32, (40, 40, 17), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d", (44, 37, 19), 1),
    (3, RGBA, F16, (12, 10, 9), (1, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR), "rotate3d", (17, 13, 11), 4),
    (2, RGBA, U8N, (64, 64, 1), (0, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_NEAREST), "rotate", (70, 66, 1), 4),
    (2, RG, F32, (33, 21, 1), (1, cl.CL_ADDRESS_NONE, cl.CL_FILTER_LINEAR), "translate", (40, 30, 3), 2),
    (2, cl.CL_RGBx, cl.CL_UNORM_SHORT_565, (33, 21, 1), (1, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_LINEAR), "rotate", (40, 30, 1), 4),
    (3, cl.CL_RGB, cl.CL_UNORM_INT_101010, (9, 6, 5), (1, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR), "rotate3d", (11, 7, 6), 4),
    # staged-footprint kernel: separable, non-wrapping, LINEAR (borders, scale != 1)
    (3, R, F32, (30, 20, 12), (1, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_LINEAR), "stencil", (30, 20, 12), 1),
    (3, R, F32, (30, 20, 12), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "scale2", (33, 21, 9), 1),
    (2, RGBA, F16, (50, 40, 1), (1, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_LINEAR), "scale2", (31, 27, 1), 4),
    (2, RGBA, F32, (64, 64, 1), (0, cl.CL_ADDRESS_NONE, cl.CL_FILTER_LINEAR), "unnorm", (96, 96, 1), 4),
    (1, RGBA, U8N, (70, 1, 1), (0, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_LINEAR), "unnorm", (100, 3, 1), 4),
    (2, R, S16N, (97, 61, 1), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "scale2", (300, 70, 1), 1),
    (2, RGBA, U8N, (64, 64, 1), (0, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_NEAREST), "unnorm", (96, 96, 1), 4),
    (2, BGRA, U8N, (31, 17, 1), (1, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_LINEAR), "rotate", (45, 29, 1), 3),
    (1, RG, F16, (50, 1, 1), (1, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR), "translate", (77, 1, 1), 2),
    (3, RGBA, U16N, (9, 8, 7), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "stencil", (12, 11, 10), 4),
    # config-3 kernel (k_sample_grid_walk4): 16-byte stencil rows in the interior
    # warps, texel-by-texel at the right edge and the ragged last warp, a ragged walk
    (3, R, F32, (300, 7, 37), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil", (300, 7, 37), 1),
    (3, R, F32, (1030, 3, 5), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil", (1030, 3, 5), 1),
    # shifted by one texel (i0 = x + 1: not 16-byte aligned) and by five (the 5th
    # texel of the last lane comes from the next 16 bytes), output width not /4
    (3, R, F32, (260, 4, 19), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil+1", (258, 4, 19), 1),
    (3, R, F32, (260, 4, 19), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil+4", (250, 4, 19), 1),
    # config-3 TMA kernel (k_sample_grid_vol): ragged tiles on every axis; a
    # 2x magnification (taps shared by neighbouring outputs and slices: scalar
    # slots, unchained rows, repeated z pairs); 2x minification (taps outside
    # the staged box: direct tiles); a z map running backwards (other kernel)
    (3, R, F32, (300, 37, 40), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil", (300, 37, 40), 1),
    (3, R, F32, (70, 45, 30), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "magnify", (150, 40, 50), 1),
    (3, R, F32, (300, 60, 40), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "scale2", (150, 33, 21), 1),
    (3, R, F32, (140, 20, 24), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil-zneg", (140, 20, 24), 1),
    # mirror-fold kernel (k_sample_grid_fold, MIRRORED_REPEAT with one fold per
    # axis): ragged primary tiles, unpaired columns past the mirror sum, an
    # exact and an inexact mirror, the fold near an edge, a 3-slice output
    (2, RGBA, F32, (300, 130, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "translate", (300, 130, 1), 4),
    (2, RGBA, F32, (257, 129, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "fold-exact", (257, 129, 1), 4),
    (2, RGBA, F32, (200, 150, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "fold-edge", (200, 150, 1), 4),
    (2, RGBA, F32, (160, 96, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "translate", (160, 96, 3), 4),
    # 1024 fold tiles (several waves of CTAs, tables turned into box / output
    # addresses per tile)
    (2, RGBA, F32, (2048, 2048, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "translate", (2048, 2048, 1), 4),
    # rotated-map staged kernel (k_sample_grid_volr): ragged tiles, the corners
    # clamped to the edges; 3x minification (footprint larger than the box:
    # direct tiles); z at half scale (repeated slice pairs)
    (3, R, F32, (90, 90, 21), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d", (100, 70, 25), 1),
    (3, R, F32, (90, 90, 21), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d-min", (70, 66, 9), 1),
    (3, R, F32, (90, 90, 21), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d-zhalf", (130, 33, 30), 1),
    (3, R, F32, (150, 150, 20), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d-wide", (160, 120, 24), 1),
    # several tiles and z chunks per CTA (the staging cursor crosses tiles)
    (3, R, F32, (200, 160, 300), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d", (256, 200, 300), 1),
    (3, R, F32, (120, 100, 200), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d-zhalf", (150, 120, 300), 1),
]


def _affine(kind, size, out):
    W, H, D = size
    if kind == "translate":
        return synth.affine_translate_2d(W, H)
    if kind == "rotate":
        return synth.affine_rotate_2d(W, H, 30.0)
    if kind == "scale2":  # 2x minification, separable, offset so edges hit the border
        A = np.zeros(12, np.float32)
        A[0], A[3] = 2.0 / W, -0.3 / W
        A[5], A[7] = 2.0 / H, 0.45 / H
        A[10], A[11] = 2.0 / D, -0.2 / D
        return A
    if kind == "fold-exact":  # mirror sum an integer: partners tap the same texels
        return synth.affine_translate_2d(W, H, dx=0.5, dy=0.5)
    if kind == "fold-edge":  # the fold 10 / 7 outputs from the right / bottom edge
        return synth.affine_translate_2d(W, H, dx=-10.3, dy=-7.6)
    if kind == "magnify":  # 2x magnification, separable, offset by a fraction of a texel
        A = np.zeros(12, np.float32)
        A[0], A[3] = 0.5 / W, 0.37 / W
        A[5], A[7] = 0.5 / H, 0.81 / H
        A[10], A[11] = 0.5 / D, 0.13 / D
        return A
    if kind == "stencil-zneg":  # z runs backwards through the volume
        A = synth.affine_stencil_3d(W)
        A[5], A[7] = 1.0 / H, (0.5 + 0.6) / H
        A[10], A[11] = -1.0 / D, (D - 0.5 + 0.2) / D
        return A
    if kind == "rotate3d-wide":  # 45 degrees at 1.5x minification: a box near the kernel's largest (fewer ring stages)
        A = synth.affine_rotate_3d(W, 45.0)
        A[[0, 1, 4, 5]] *= 1.5
        return A
    if kind.startswith("rotate3d-"):
        A = synth.affine_rotate_3d(W, 20.0)
        if kind.endswith("min"):
            A[[0, 1, 4, 5]] *= 3.0
        else:
            A[10] *= 0.5
        return A
    if kind == "rotate3d":
        return synth.affine_rotate_3d(W, 20.0)
    if kind.startswith("stencil"):
        A = synth.affine_stencil_3d(W)
        if "+" in kind:  # shift the x taps by whole texels
            A[3] = (0.5 + 0.3 + int(kind.split("+")[1])) / W
        A[5] = 1.0 / H
        A[7] = (0.5 + 0.6) / H
        A[10] = 1.0 / D
        A[11] = (0.5 + 0.2) / D
        return A
    return synth.affine_unnorm_2d(1 / 16 * 12, -2.0)


@pytest.mark.parametrize("case", GRID_CASES)
def test_grid_mode(sess, orc, case):
    dims, order, type_, size, (norm, addr, filt), kind, out, outc = case
    W, H, D = size
    img, oimg, _ = make_images(sess, orc, order, type_, W, H, D, dims, seed=sum(size))
    smp = sess.sampler(norm, addr, filt)
    A = _affine(kind, size, out)
    got = gpu_read_grid(sess, img, smp, cl.B2CL_RTYPE_FLOAT, A, out, outc)
    rd = lambda im: orc.read_grid(im, norm, addr, filt, orc.RT_F, A, out, outc)  # noqa: E731
    parity_read(got, rd(oimg), filt == cl.CL_FILTER_LINEAR, f"grid {case}", orc, oimg, rd)
    sess.release(img)


def test_config1_full_bruteforce(sess, orc):
    """BASELINE config 1: 64x64 RGBA8, unnormalized, CLAMP + NEAREST, every
    coordinate of a 1/16 lattice over [-2, 66)^2 (1088^2 samples), bit-exact."""
    img, oimg, _ = make_images(sess, orc, RGBA, U8N, 64, 64, 1, 2, seed=1)
    smp = sess.sampler(False, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_NEAREST)
    A = synth.affine_unnorm_2d(1 / 16, -2.0)
    out = (1088, 1088, 1)
    got = gpu_read_grid(sess, img, smp, cl.B2CL_RTYPE_FLOAT, A, out, 4)
    exp = orc.read_grid(oimg, False, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_NEAREST, orc.RT_F, A, out, 4,
                        nthreads=8)
    assert_parity(got, exp, False, "config1")
    # and the same through the coordinate-list entry point
    xs = (np.arange(1088) / 16 - 2).astype(np.float32)
    co = np.stack(np.meshgrid(xs, xs), -1).reshape(-1, 2)
    got2 = gpu_read_samples(sess, img, smp, cl.B2CL_RTYPE_FLOAT, co)
    assert_parity(got2, exp.reshape(-1, 4), False, "config1 list")
    sess.release(img)


@pytest.mark.parametrize("addr", [cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT])
@pytest.mark.parametrize("kind", ["translate", "rotate"])
def test_config2_full_size_sampled_rows(sess, orc, addr, kind):
    """BASELINE config 2 at full size (4096^2 RGBA32F, normalized, LINEAR), in the
    launch configuration bench.py times; rows sampled: all seam / edge rows and
    every 97th row, all columns, against the oracle."""
    N = 4096
    img, oimg, _ = make_images(sess, orc, RGBA, F32, N, N, 1, 2, seed=2)
    smp = sess.sampler(True, addr, cl.CL_FILTER_LINEAR)
    A = synth.affine_translate_2d(N, N) if kind == "translate" else synth.affine_rotate_2d(N, N, 30.0)
    got = gpu_read_grid(sess, img, smp, cl.B2CL_RTYPE_FLOAT, A, (N, N, 1), 4)
    rows = sorted(set([0, 1, N // 2 - 1, N // 2, N // 2 + 1, N - 2, N - 1] + list(range(5, N, 97))))
    for y in rows:
        exp = orc.read_grid(oimg, True, addr, cl.CL_FILTER_LINEAR, orc.RT_F, A, (N, N, 1), 4,
                            yrange=(y, y + 1))
        assert_parity(got[0, y:y + 1], exp[0], True, f"config2 row {y}")
    sess.release(img)


@pytest.mark.parametrize("kind", ["stencil", "rotate3d"])
def test_config3_full_size_sampled_slices(sess, orc, kind):
    """BASELINE config 3 at full size (512^3 R32F, trilinear, CLAMP_TO_EDGE; stencil map
    (separable kernel) and volume-render rotation (general kernel)): sampled rows of
    first / middle / last slices against the oracle."""
    N = 512
    img, oimg, _ = make_images(sess, orc, R, F32, N, N, N, 3, seed=3)
    smp = sess.sampler(True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    A = synth.affine_stencil_3d(N) if kind == "stencil" else synth.affine_rotate_3d(N, 20.0)
    got = gpu_read_grid(sess, img, smp, cl.B2CL_RTYPE_FLOAT, A, (N, N, N), 1)
    for z in (0, 1, 255, 510, 511):
        for y in (0, 1, 100, 256, 511):
            exp = orc.read_grid(oimg, True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR,
                                orc.RT_F, A, (N, N, N), 1, zrange=(z, z + 1), yrange=(y, y + 1))
            assert_parity(got[z:z + 1, y:y + 1], exp, True, f"config3 z{z} y{y}")
    # property at any size: the trilinear read of a [0,1) volume stays in [0,1]
    assert np.all((got >= 0) & (got <= 1))
    sess.release(img)


# ---------------------------------------------------------------- write_image
WRITE_FORMATS = [(RGBA, U8N, cl.B2CL_RTYPE_FLOAT), (BGRA, U8N, cl.B2CL_RTYPE_FLOAT),
                 (RGBA, S8N, cl.B2CL_RTYPE_FLOAT), (RG, U16N, cl.B2CL_RTYPE_FLOAT),
                 (R, S16N, cl.B2CL_RTYPE_FLOAT), (RGBA, F16, cl.B2CL_RTYPE_FLOAT),
                 (RGBA, F32, cl.B2CL_RTYPE_FLOAT), (A_, U8N, cl.B2CL_RTYPE_FLOAT),
                 (ARGB, U8N, cl.B2CL_RTYPE_FLOAT), (RA, F16, cl.B2CL_RTYPE_FLOAT),
                 (INT_, F32, cl.B2CL_RTYPE_FLOAT), (LUM, U8N, cl.B2CL_RTYPE_FLOAT),
                 (cl.CL_RGB, cl.CL_UNORM_SHORT_565, cl.B2CL_RTYPE_FLOAT),
                 (cl.CL_RGBx, cl.CL_UNORM_SHORT_555, cl.B2CL_RTYPE_FLOAT),
                 (cl.CL_RGB, cl.CL_UNORM_INT_101010, cl.B2CL_RTYPE_FLOAT),
                 (RGBA, cl.CL_SIGNED_INT8, cl.B2CL_RTYPE_INT), (RG, cl.CL_SIGNED_INT16, cl.B2CL_RTYPE_INT),
                 (R, cl.CL_SIGNED_INT32, cl.B2CL_RTYPE_INT), (RGBA, cl.CL_UNSIGNED_INT8, cl.B2CL_RTYPE_UINT),
                 (RA, cl.CL_UNSIGNED_INT16, cl.B2CL_RTYPE_UINT), (R, cl.CL_UNSIGNED_INT32, cl.B2CL_RTYPE_UINT)]


@pytest.mark.parametrize("order,type_,rt", WRITE_FORMATS)
@pytest.mark.parametrize("dims", [1, 2, 3])
def test_write_image(sess, orc, order, type_, rt, dims):
    W, H, D = 23, (9 if dims > 1 else 1), (4 if dims > 2 else 1)
    img, oimg, codes = make_images(sess, orc, order, type_, W, H, D, dims, seed=11)
    g = synth.rng(12)
    n = W * H * D
    # unique in-range coordinates (a permutation) plus out-of-range no-ops
    perm = g.permutation(n)
    ic = np.zeros((n + 40, {1: 1, 2: 2, 3: 4}[dims]), np.int32)
    ic[:n, 0] = perm % W
    if dims > 1:
        ic[:n, 1] = (perm // W) % H
    if dims > 2:
        ic[:n, 2] = perm // (W * H)
    ic[n:, 0] = g.integers(-5, 0, 40)
    if rt == cl.B2CL_RTYPE_FLOAT:
        col = g.uniform(-1.5, 1.5, (n + 40, 4)).astype(np.float32)
        col[:8] = [[np.nan, 0.5, 1 / 510, 3 / 510], [2.0, -0.3, 65520.0, 6e-8], [1.0, 0.0, -0.0, 1e-40],
                   [np.inf, -np.inf, 0.49999997, 254.5 / 255], [0.5, 0.25, 0.125, 0.0625],
                   [-1.0, -0.999, 1.0001, 100.0], [1.5 / 255, 2.5 / 255, 1e-5, 0.9999],
                   [65504.0, 65519.0, -65520.0, 2 ** -24]]
        if type_ == F16:  # half NaN payloads are unspecified (reading A13): compared separately
            col[0, 0] = 0.5
    else:
        col = g.integers(-2 ** 31, 2 ** 31, (n + 40, 4), dtype=np.int64).astype(np.int32)
        col[:4] = [[300, -300, 127, -128], [70000, -70000, 32767, -32768], [255, 256, 65535, 65536],
                   [-1, 0, 1, 2 ** 31 - 1]]
        if rt == cl.B2CL_RTYPE_UINT:
            col = col.view(np.uint32)
    cbuf = sess.buffer(ic.nbytes, ic)
    kbuf = sess.buffer(col.nbytes, col)
    cl.check(cl.lib().b2clEnqueueWriteImageSamples(sess.queue, img, rt, cbuf, 0, ic.shape[0], kbuf, 0,
                                                   0, None, None))
    orc.write_samples(oimg, rt, ic, col)
    got = sess.read_image(img, (0, 0, 0), (W, H, D))
    assert np.array_equal(got, oimg.data[:got.size]), f"write {hex(order)}/{hex(type_)}"
    sess.release(img, cbuf, kbuf)


def test_supported_formats_match_the_legal_table(sess, orc):
    """clGetSupportedImageFormats lists exactly the (order, type) pairs the oracle
    accepts ([CL1.2 §5.3.1.1], packed formats included; CL_Rx / CL_RGx not, A37)."""
    import ctypes
    L = cl.lib()
    n = ctypes.c_uint32()
    cl.check(L.clGetSupportedImageFormats(sess.ctx, 0, 0x10F1, 0, None, ctypes.byref(n)))
    fmts = (ctypes.c_uint32 * (2 * n.value))()
    cl.check(L.clGetSupportedImageFormats(sess.ctx, 0, 0x10F1, n.value, fmts, None))
    got = {(fmts[2 * i], fmts[2 * i + 1]) for i in range(n.value)}
    exp = {(o, t) for o in range(0x10B0, 0x10BD) for t in range(0x10D0, 0x10DF)
           if orc.elem_size(o, t) > 0}
    assert got == exp
    assert (cl.CL_RGBx, cl.CL_UNORM_INT_101010) in got and (cl.CL_RGB, cl.CL_UNORM_SHORT_565) in got


@pytest.mark.parametrize("case", ["inf_x", "nan_y", "huge_z", "zero_scale", "neg_zero"])
def test_config3_kernels_degenerate_maps(sess, orc, case):
    """The config-3 format and sampler with degenerate separable and rotated
    maps (infinite / NaN / huge coefficients, zero scale, -0): whichever kernel
    the library picks (staged, walk or general) agrees with the oracle."""
    W, H, D = 70, 20, 12
    img, oimg, _ = make_images(sess, orc, R, F32, W, H, D, 3, seed=99)
    smp = sess.sampler(True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    for rotated in (False, True):
        A = synth.affine_rotate_3d(W, 20.0) if rotated else _affine("stencil", (W, H, D), (W, H, D))
        A = A.copy()
        if case == "inf_x":
            A[0] = np.float32(np.inf)
        elif case == "nan_y":
            A[7] = np.float32(np.nan)
        elif case == "huge_z":
            A[11] = np.float32(3e9)
        elif case == "zero_scale":
            A[0] = A[5] = A[10] = np.float32(0.0)
        else:
            A[10] = np.float32(-0.0)
        out = (W, H, D)
        got = gpu_read_grid(sess, img, smp, cl.B2CL_RTYPE_FLOAT, A, out, 1)
        exp = orc.read_grid(oimg, True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR, orc.RT_F, A, out, 1)
        assert_parity(got, exp, True, f"{case} rotated={rotated}")
    sess.release(img)


@pytest.mark.parametrize("n", [1, 2, 255, 256, 257, 511, 512, 513, 1000, 131073])
def test_list_lengths(sess, orc, n):
    """k_sample_list takes two samples per thread, strided by the grid: every
    list length (one block, a partial second sample, an odd tail) maps each
    coordinate to its own output slot and nothing past the end is written."""
    W, H = 67, 45
    img, oimg, _ = make_images(sess, orc, RGBA, F32, W, H, 1, 2, seed=n % 97)
    g = synth.rng(500 + n)
    co = g.uniform(-0.3, 1.3, size=(n, 2)).astype(np.float32)
    for addr in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_CLAMP_TO_EDGE):
        smp = sess.sampler(1, addr, cl.CL_FILTER_LINEAR)
        L = cl.lib()
        cbuf = sess.buffer(co.nbytes, co)
        guard = 64
        obuf = sess.buffer(16 * (n + guard), np.full(16 * (n + guard), 0xA5, np.uint8))
        cl.check(L.b2clEnqueueReadImageSamples(sess.queue, img, smp, cl.B2CL_RTYPE_FLOAT, cl.B2CL_COORD_FLOAT,
                                               cbuf, 0, n, obuf, 0, 0, None, None))
        raw = sess.read(obuf, 16 * (n + guard), np.uint8)
        assert np.all(raw[16 * n:] == 0xA5), "a store past the list's end"
        got = raw[:16 * n].view(np.float32).reshape(n, 4)
        exp = orc.read_samples(oimg, 1, addr, cl.CL_FILTER_LINEAR, orc.RT_F, co)
        assert_parity(got, exp, True, f"list n={n} addr {hex(addr)}")
        sess.release(cbuf, obuf)
        L.clReleaseSampler(smp)
    sess.release(img)
