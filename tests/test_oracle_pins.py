"""Pins of the CPU oracle against things other than itself.

Each test names what fixes the expected value: a hand-worked example stored in
tests/golden/ with its derivation, a closed form, an invariant, an exhaustive
table checked against numpy's IEEE arithmetic, or a library routine
(torch.nn.functional.grid_sample, numpy slicing / np.tile, numpy float16).
No expected value comes from the CUDA path.
"""
import os

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

ADDR = {"NONE": 0x1130, "CLAMP_TO_EDGE": 0x1131, "CLAMP": 0x1132, "REPEAT": 0x1133,
        "MIRRORED_REPEAT": 0x1134}
FILT = {"NEAREST": 0x1140, "LINEAR": 0x1141}
VALID_SAMPLERS = [(norm, a, f) for norm in (0, 1) for a in ADDR.values() for f in FILT.values()
                  if norm or a in (0x1130, 0x1131, 0x1132)]


def f32bits(x):
    return np.asarray(x, dtype=np.float32).view(np.uint32)


def _golden_lines(name):
    with open(os.path.join(GOLDEN, name)) as fh:
        for line in fh:
            line = line.split("|")[0].strip()
            if line and not line.startswith("#"):
                yield line.split()


# ---------------------------------------------------------------- P1
def test_p1_axis_examples(orc):
    img = orc.Image(np.array([10, 20, 30, 40], np.float32), 4, 1, 1, dims=1,
                    order=orc.R, type=orc.FLOAT)
    n = 0
    for norm, addr, filt, s, exp in _golden_lines("p1_axis_1d.txt"):
        out = orc.read_samples(img, bool(int(norm)), ADDR[addr], FILT[filt], orc.RT_F,
                               np.array([[float(s)]], np.float32))[0]
        assert out.tolist() == [float(exp), 0.0, 0.0, 1.0], (norm, addr, filt, s, out)
        n += 1
    assert n >= 40


def test_p1_rgba8_2x2(orc):
    codes = np.array([[[255, 128, 0, 255], [0, 128, 10, 255]],
                      [[0, 128, 20, 0], [255, 128, 30, 0]]], np.uint8)
    img = orc.Image(codes, 2, 2, 1, dims=2, order=orc.RGBA, type=orc.UNORM_INT8)
    for addr, s, t, *hexes in _golden_lines("p1_rgba8_2x2.txt"):
        out = orc.read_samples(img, False, ADDR[addr], FILT["LINEAR"], orc.RT_F,
                               np.array([[float(s), float(t)]], np.float32))[0]
        assert f32bits(out).tolist() == [int(h, 16) for h in hexes], (addr, s, t, out)


# ---------------------------------------------------------------- P2 closed forms
@pytest.mark.parametrize("dims", [1, 2, 3])
def test_p2_constant_image_linear_is_exact(orc, dims):
    """A constant image c: every LINEAR read that cannot reach the border is c exactly."""
    W, H, D = 7, (5 if dims > 1 else 1), (3 if dims > 2 else 1)
    c = np.float32(0.3183099)
    data = np.full((D, H, W, 1), c, np.float32)
    img = orc.Image(data, W, H, D, dims=dims, order=orc.R, type=orc.FLOAT)
    g = synth.rng(1)
    co = g.uniform(-3, 3, size=(3000, 4)).astype(np.float32)[:, :max(dims, 1) if dims < 3 else 4]
    for a in ("CLAMP_TO_EDGE", "REPEAT", "MIRRORED_REPEAT"):
        out = orc.read_samples(img, True, ADDR[a], FILT["LINEAR"], orc.RT_F, co)
        assert np.all(out[:, 0] == c), a
        assert np.all(out[:, 3] == 1.0)


def test_p2_ramp_linear_closed_form(orc):
    """Ramp T(i,j) = i + W*j (exact integers): bilinear interpolation reproduces a
    linear function, so an interior LINEAR read equals RN(t_x + W*t_y) with
    t = fl(u - 1/2); NEAREST equals floor(u) + W*floor(v)."""
    W, H = 37, 23
    ii, jj = np.meshgrid(np.arange(W), np.arange(H))
    data = (ii + W * jj).astype(np.float32)[None, :, :, None]
    img = orc.Image(data, W, H, 1, dims=2, order=orc.R, type=orc.FLOAT)
    g = synth.rng(2)
    u = g.uniform(1.0, W - 1.0, 20000).astype(np.float32)
    v = g.uniform(1.0, H - 1.0, 20000).astype(np.float32)
    out = orc.read_samples(img, False, ADDR["CLAMP_TO_EDGE"], FILT["LINEAR"], orc.RT_F,
                           np.stack([u, v], 1))
    tx = (u - np.float32(0.5)).astype(np.float64)
    ty = (v - np.float32(0.5)).astype(np.float64)
    exp = (tx + W * ty).astype(np.float32)
    assert np.array_equal(out[:, 0], exp)
    out = orc.read_samples(img, False, ADDR["CLAMP_TO_EDGE"], FILT["NEAREST"], orc.RT_F,
                           np.stack([u, v], 1))
    assert np.array_equal(out[:, 0], (np.floor(u) + W * np.floor(v)).astype(np.float32))


def test_p2_ramp_3d_linear_closed_form(orc):
    W, H, D = 9, 7, 5
    k, j, i = np.meshgrid(np.arange(D), np.arange(H), np.arange(W), indexing="ij")
    data = (i + W * j + W * H * k).astype(np.float32)[..., None]
    img = orc.Image(data, W, H, D, dims=3, order=orc.R, type=orc.FLOAT)
    g = synth.rng(3)
    n = 5000
    c = np.stack([g.uniform(1, W - 1, n), g.uniform(1, H - 1, n), g.uniform(1, D - 1, n),
                  np.zeros(n)], 1).astype(np.float32)
    out = orc.read_samples(img, False, ADDR["CLAMP_TO_EDGE"], FILT["LINEAR"], orc.RT_F, c)
    # exact value t_x + W*t_y + W*H*t_z (Fractions); the fp64-evaluated oracle blend
    # must be within half an ulp of it (faithful; it may pick either neighbour only
    # at an exact tie, which this integer ramp makes common).
    from fractions import Fraction
    t = c[:, :3] - np.float32(0.5)
    n_exact = 0
    for s in range(n):
        ex = (Fraction(float(t[s, 0])) + W * Fraction(float(t[s, 1]))
              + W * H * Fraction(float(t[s, 2])))
        got = Fraction(float(out[s, 0]))
        ulp = Fraction(float(np.spacing(np.float32(float(ex)))))
        assert abs(got - ex) <= ulp / 2, s
        n_exact += got == Fraction(float(np.float32(float(ex))))
    assert n_exact >= n * 0.99


def test_p2_one_by_one_image(orc):
    """A 1x1 image under CTE/REPEAT/MIRRORED returns T0 for any finite coordinate."""
    img = orc.Image(np.array([[0.1, 0.2, 0.3, 0.4]], np.float32), 1, 1, 1, dims=2,
                    order=orc.RGBA, type=orc.FLOAT)
    g = synth.rng(4)
    co = g.uniform(-5, 5, (3000, 2)).astype(np.float32)
    for a in ("CLAMP_TO_EDGE", "REPEAT", "MIRRORED_REPEAT"):
        for f in FILT.values():
            out = orc.read_samples(img, True, ADDR[a], f, orc.RT_F, co)
            assert np.all(out == np.array([0.1, 0.2, 0.3, 0.4], np.float32)), (a, f)


# ---------------------------------------------------------------- P3 invariants
WIDTHS = [1, 3, 4, 7, 64, 1000]


@pytest.mark.parametrize("n", WIDTHS)
def test_p3_addressing_invariants(orc, n):
    g = synth.rng(5 + n)
    ss = np.concatenate([g.uniform(-3, 3, 1500), synth.special_floats()[:20]]).astype(np.float32)
    M, R, CTE = ADDR["MIRRORED_REPEAT"], ADDR["REPEAT"], ADDR["CLAMP_TO_EDGE"]
    for s in ss:
        s = float(s)
        # MIRRORED(-s) == MIRRORED(s), indices and weights
        assert orc.axis_nearest(s, n, True, M) == orc.axis_nearest(-s, n, True, M)
        assert orc.axis_linear(s, n, True, M) == orc.axis_linear(-s, n, True, M)
        # REPEAT indices always in range
        i = orc.axis_nearest(s, n, True, R)
        i0, i1, _ = orc.axis_linear(s, n, True, R)
        if np.isfinite(s):
            assert 0 <= i < n and 0 <= i0 < n and 0 <= i1 < n
        # MIRRORED == CLAMP_TO_EDGE on [0, 1]
        if 0.0 <= s <= 1.0:
            assert orc.axis_nearest(s, n, True, M) == orc.axis_nearest(s, n, True, CTE)
            assert orc.axis_linear(s, n, True, M) == orc.axis_linear(s, n, True, CTE)


def test_p3_repeat_periodic_dyadic(orc):
    for n in WIDTHS:
        for s in synth.coord_lattice(-2, 2, 1 / 64):
            s = float(s)
            assert orc.axis_nearest(s, n, True, ADDR["REPEAT"]) == \
                orc.axis_nearest(s + 1.0, n, True, ADDR["REPEAT"])
            assert orc.axis_linear(s, n, True, ADDR["REPEAT"]) == \
                orc.axis_linear(s + 1.0, n, True, ADDR["REPEAT"])


def test_p3_linear_at_texel_centres_equals_nearest(orc):
    g = synth.rng(6)
    W, H = 13, 6
    data = synth.image_codes(g, orc.RGBA, orc.FLOAT, W, H)
    img = orc.Image(data, W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    xs, ys = np.meshgrid(np.arange(-2, W + 2) + 0.5, np.arange(-2, H + 2) + 0.5)
    co = np.stack([xs.ravel(), ys.ravel()], 1).astype(np.float32)
    for a in ("NONE", "CLAMP_TO_EDGE", "CLAMP"):
        lin = orc.read_samples(img, False, ADDR[a], FILT["LINEAR"], orc.RT_F, co)
        near = orc.read_samples(img, False, ADDR[a], FILT["NEAREST"], orc.RT_F, co)
        assert np.array_equal(f32bits(lin), f32bits(near)), a


ORDERS = ["R", "A", "RG", "RA", "RGBA", "BGRA", "ARGB", "INTENSITY", "LUMINANCE"]


@pytest.mark.parametrize("order", ORDERS)
def test_p3_border_is_map_of_zero_texel(orc, order):
    """Reading A8: for every in-scope order the CLAMP border colour equals the
    channel map of an all-zero texel (so TMA zero fill is exact)."""
    o = getattr(orc, order)
    t = orc.UNORM_INT8
    es = orc.elem_size(o, t)
    img = orc.Image(np.zeros(es, np.uint8), 1, 1, 1, dims=2, order=o, type=t)
    inside = orc.read_samples(img, False, ADDR["CLAMP"], FILT["NEAREST"], orc.RT_F,
                              np.array([[0.5, 0.5]], np.float32))
    border = orc.read_samples(img, False, ADDR["CLAMP"], FILT["NEAREST"], orc.RT_F,
                              np.array([[-0.5, 0.5]], np.float32))
    assert np.array_equal(inside, border)
    exp_w = 1.0 if order in ("R", "RG", "LUMINANCE") else 0.0
    assert border[0].tolist() == [0.0, 0.0, 0.0, exp_w]


def test_p3_channel_map_orders(orc):
    """[CL1.2 §8.3] channel mapping for each order, on a texel of distinct codes."""
    exp = {"R": (10, 0, 0, 255), "A": (0, 0, 0, 10), "RG": (10, 20, 0, 255),
           "RA": (10, 0, 0, 20), "RGBA": (10, 20, 30, 40), "BGRA": (30, 20, 10, 40),
           "ARGB": (20, 30, 40, 10), "INTENSITY": (10, 10, 10, 10),
           "LUMINANCE": (10, 10, 10, 255)}
    for order, e in exp.items():
        o = getattr(orc, order)
        es = orc.elem_size(o, orc.UNORM_INT8)
        img = orc.Image(np.array([10, 20, 30, 40][:es], np.uint8), 1, 1, 1, dims=2, order=o,
                        type=orc.UNORM_INT8)
        out = orc.read_samples(img, False, ADDR["NONE"], FILT["NEAREST"], orc.RT_F,
                               np.array([[0.5, 0.5]], np.float32))[0]
        assert out.tolist() == [np.float32(c) / np.float32(255) for c in e], order


# ---------------------------------------------------------------- P4 conversions
@pytest.mark.parametrize("tname,d,bits,signed", [("UNORM_INT8", 255, 8, False),
                                                 ("UNORM_INT16", 65535, 16, False),
                                                 ("SNORM_INT8", 127, 8, True),
                                                 ("SNORM_INT16", 32767, 16, True)])
def test_p4_norm_read_is_ieee_division(orc, tname, d, bits, signed):
    t = getattr(orc, tname)
    codes = np.arange(-(1 << (bits - 1)), 1 << (bits - 1)) if signed else np.arange(1 << bits)
    L = orc.lib()
    got = np.array([L.oracle_norm_to_float(t, int(c)) for c in codes], np.float32)
    exp = codes.astype(np.float32) / np.float32(d)       # numpy: IEEE fp32 division
    if signed:
        exp = np.maximum(np.float32(-1.0), exp)
    assert np.array_equal(f32bits(got), f32bits(exp))
    # read -> write round trip is the identity (SNORM: min code -> -d, reading A17)
    back = np.array([L.oracle_float_to_norm(t, float(v)) for v in got])
    exp_back = np.maximum(codes, -d) if signed else codes
    assert np.array_equal(back, exp_back)


def test_p4_norm_write_special_values(orc):
    L = orc.lib()
    cases = [("UNORM_INT8", 0.5, 128), ("SNORM_INT8", 0.5, 64), ("UNORM_INT16", 0.5, 32768),
             ("UNORM_INT8", float("nan"), 0), ("UNORM_INT8", 2.0, 255), ("UNORM_INT8", -0.3, 0),
             ("SNORM_INT8", -2.0, -128), ("SNORM_INT16", -1.0, -32767),
             ("UNORM_INT8", 1.0 / 510, 0),   # 0.5 exactly -> half-even -> 0
             ("UNORM_INT8", 3.0 / 510, 2)]   # 1.5 -> 2
    for tname, f, exp in cases:
        got = L.oracle_float_to_norm(getattr(orc, tname), f)
        assert got == exp, (tname, f, got)
    # UNORM8(128) read = RN(128/255) = 0x3F008081
    assert f32bits(L.oracle_norm_to_float(orc.UNORM_INT8, 128)) == 0x3F008081


def test_p4_half_read_all_codes(orc):
    L = orc.lib()
    codes = np.arange(65536, dtype=np.uint16)
    exp = codes.view(np.float16).astype(np.float32)
    got = np.array([L.oracle_half_to_float(int(c)) for c in codes], np.float32)
    nan = np.isnan(exp)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(f32bits(got[~nan]), f32bits(exp[~nan]))


def test_p4_half_write_matches_numpy(orc):
    """float -> half RTE with subnormals kept (reading A13) == numpy astype(float16)."""
    L = orc.lib()
    g = synth.rng(7)
    bits = g.integers(0, 1 << 32, 60000, dtype=np.uint64).astype(np.uint32)
    vals = bits.view(np.float32)
    # dense coverage of the half range, ties and the overflow boundary
    h = np.arange(65536, dtype=np.uint16).view(np.float16).astype(np.float32)
    h = h[np.isfinite(h)]
    nxt = np.nextafter(h, np.float32(np.inf))
    mids = ((h.astype(np.float64) + np.roll(h, -1).astype(np.float64)) / 2).astype(np.float32)
    extra = np.array([65520.0, 65519.996, 6e-8, 1 + 2 ** -11, 2 ** -25, 2 ** -24 * 1.5, -0.0],
                     np.float32)
    vals = np.concatenate([vals, h, nxt, mids, extra]).astype(np.float32)
    got = np.array([L.oracle_float_to_half_rte(float(v)) for v in vals], np.uint16)
    with np.errstate(over="ignore"):
        exp = vals.astype(np.float16).view(np.uint16)
    nan = np.isnan(vals)
    assert np.array_equal(got[~nan], exp[~nan])
    assert np.all((got[nan] & 0x7C00) == 0x7C00) and np.all((got[nan] & 0x3FF) != 0)
    assert L.oracle_float_to_half_rte(65520.0) == 0x7C00
    assert L.oracle_float_to_half_rte(6e-8) == 0x0001
    assert L.oracle_float_to_half_rte(1 + 2 ** -11) == 0x3C00


def test_p4_integer_write_saturation(orc):
    cases = [("SIGNED_INT8", orc.RT_I, 300, 127), ("SIGNED_INT8", orc.RT_I, -300, -128),
             ("SIGNED_INT16", orc.RT_I, 40000, 32767), ("SIGNED_INT32", orc.RT_I, -7, -7),
             ("UNSIGNED_INT8", orc.RT_UI, 256, 255), ("UNSIGNED_INT16", orc.RT_UI, 70000, 65535),
             ("UNSIGNED_INT32", orc.RT_UI, 0xFFFFFFFF, 0xFFFFFFFF)]
    for tname, rt, v, exp in cases:
        t = getattr(orc, tname)
        dt = np.int32 if rt == orc.RT_I else np.uint32
        col = np.array([v, 0, 0, 0], dtype=np.int64).astype(dt)
        texel = orc.convert_texel(orc.R, t, rt, col)
        got = np.frombuffer(texel, dtype=synth.texel_dtype(t))[0]
        assert int(got) == exp, (tname, v, got)


# ---------------------------------------------------------------- P6 library routines
torch = pytest.importorskip("torch")


@pytest.mark.parametrize("addr,pad", [("CLAMP", "zeros"), ("CLAMP_TO_EDGE", "border"),
                                      ("MIRRORED_REPEAT", "reflection")])
def test_p6_grid_sample_bilinear_2d(orc, addr, pad):
    """torch grid_sample(align_corners=False) bilinear equals LINEAR to ~1e-6:
    zeros <-> CLAMP, border <-> CLAMP_TO_EDGE, reflection <-> MIRRORED_REPEAT."""
    import torch.nn.functional as F
    g = synth.rng(8)
    W, H = 19, 11
    data = synth.image_codes(g, orc.RGBA, orc.FLOAT, W, H)
    img = orc.Image(data, W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    lo, hi = (-0.4, 1.4) if addr != "MIRRORED_REPEAT" else (-0.9, 0.9)
    st = g.uniform(lo, hi, (4000, 2)).astype(np.float32)
    out = orc.read_samples(img, True, ADDR[addr], FILT["LINEAR"], orc.RT_F, st)
    inp = torch.from_numpy(data[0].astype(np.float64)).permute(2, 0, 1)[None]
    grid = torch.from_numpy(st.astype(np.float64) * 2 - 1)[None, None]
    ref = F.grid_sample(inp, grid, mode="bilinear", padding_mode=pad,
                        align_corners=False)[0, :, 0].T.numpy()
    assert np.max(np.abs(out - ref)) < 1e-6


def test_p6_grid_sample_trilinear_3d(orc):
    import torch.nn.functional as F
    g = synth.rng(9)
    W, H, D = 9, 6, 5
    data = synth.image_codes(g, orc.R, orc.FLOAT, W, H, D)
    img = orc.Image(data, W, H, D, dims=3, order=orc.R, type=orc.FLOAT)
    c = g.uniform(-0.3, 1.3, (3000, 4)).astype(np.float32)
    out = orc.read_samples(img, True, ADDR["CLAMP_TO_EDGE"], FILT["LINEAR"], orc.RT_F, c)
    inp = torch.from_numpy(data[..., 0].astype(np.float64))[None, None]
    grid = torch.from_numpy(c[:, :3].astype(np.float64) * 2 - 1)[None, None, None]
    ref = F.grid_sample(inp, grid, mode="bilinear", padding_mode="border",
                        align_corners=False)[0, 0, 0, 0].numpy()
    assert np.max(np.abs(out[:, 0] - ref)) < 1e-6


# ---------------------------------------------------------------- bulk ops vs numpy
def test_copy_rect_matches_numpy_slicing(orc):
    g = synth.rng(10)
    for _ in range(60):
        so, do, region, srp, ssp, drp, dsp = synth.random_rect(g)
        src = g.integers(0, 256, ssp * (so[2] + region[2]) + 64, dtype=np.uint8)
        dst = g.integers(0, 256, dsp * (do[2] + region[2]) + 64, dtype=np.uint8)
        exp = dst.copy()
        s3 = np.lib.stride_tricks.as_strided(src[so[2] * ssp + so[1] * srp + so[0]:],
                                             (region[2], region[1], region[0]), (ssp, srp, 1))
        d3 = np.lib.stride_tricks.as_strided(exp[do[2] * dsp + do[1] * drp + do[0]:],
                                             (region[2], region[1], region[0]), (dsp, drp, 1))
        d3[...] = s3
        orc.copy_rect(src, dst, so, do, region, srp, ssp, drp, dsp)
        assert np.array_equal(dst, exp)


def test_copy_rect_default_pitches(orc):
    src = np.arange(2 * 3 * 5, dtype=np.uint8)
    dst = np.zeros_like(src)
    orc.copy_rect(src, dst, (0, 0, 0), (0, 0, 0), (5, 3, 2))
    assert np.array_equal(src, dst)


@pytest.mark.parametrize("p", [1, 2, 4, 8, 16, 32, 64, 128])
def test_fill_buffer_matches_np_tile(orc, p):
    g = synth.rng(11)
    pat = g.integers(0, 256, p, dtype=np.uint8)
    buf = np.zeros(p * 40, np.uint8)
    off, size = 3 * p, 20 * p
    orc.fill_buffer(buf, pat.tobytes(), off, size)
    exp = np.zeros_like(buf)
    exp[off:off + size] = np.tile(pat, size // p)
    assert np.array_equal(buf, exp)


def test_image_buffer_copies_match_numpy(orc):
    g = synth.rng(12)
    W, H, D = 11, 7, 3
    codes = synth.image_codes(g, orc.RGBA, orc.UNORM_INT8, W, H, D)
    # pitched source image: row pitch 64 B, slice pitch 8 rows
    rp, sp = 64, 64 * 8
    raw = np.zeros(sp * D, np.uint8)
    for k in range(D):
        for j in range(H):
            raw[k * sp + j * rp: k * sp + j * rp + W * 4] = codes[k, j].ravel()
    img = orc.Image(raw, W, H, D, dims=3, order=orc.RGBA, type=orc.UNORM_INT8, row_pitch=rp,
                    slice_pitch=sp)
    buf = np.zeros(5 + 4 * 4 * 3 * 2, np.uint8)
    orc.copy_image_to_buffer(img, buf, (2, 1, 1), (4, 3, 2), 5)
    assert np.array_equal(buf[5:], codes[1:3, 1:4, 2:6].ravel())
    # and back into a second, tightly pitched image
    raw2 = np.zeros(W * H * D * 4, np.uint8)
    img2 = orc.Image(raw2, W, H, D, dims=3, order=orc.RGBA, type=orc.UNORM_INT8)
    orc.copy_buffer_to_image(buf, img2, 5, (0, 0, 0), (4, 3, 2))
    got = raw2.reshape(D, H, W, 4)
    assert np.array_equal(got[0:2, 0:3, 0:4], codes[1:3, 1:4, 2:6])
    # copy image -> image
    raw3 = np.zeros(W * H * D * 4, np.uint8)
    img3 = orc.Image(raw3, W, H, D, dims=3, order=orc.RGBA, type=orc.UNORM_INT8)
    orc.copy_image(img, img3, (1, 2, 0), (3, 0, 1), (5, 4, 2))
    assert np.array_equal(raw3.reshape(D, H, W, 4)[1:3, 0:4, 3:8], codes[0:2, 2:6, 1:6])
    # read image rect with host pitches
    host = np.zeros(100 * 10, np.uint8)
    orc.read_image_rect(img, (1, 1, 0), (3, 2, 2), 20, 100, host)
    for k in range(2):
        for j in range(2):
            assert np.array_equal(host[k * 100 + j * 20: k * 100 + j * 20 + 12],
                                  codes[k, 1 + j, 1:4].ravel())


def test_fill_image_matches_convert(orc):
    W, H = 6, 4
    raw = np.zeros(W * H * 4, np.uint8)
    img = orc.Image(raw, W, H, 1, dims=2, order=orc.BGRA, type=orc.UNORM_INT8)
    orc.fill_image(img, orc.RT_F, np.array([1.0, 0.5, 0.0, 0.25], np.float32), (1, 1, 0),
                   (3, 2, 1))
    px = raw.reshape(H, W, 4)
    assert px[1, 1].tolist() == [0, 128, 255, 64]      # stored B, G, R, A
    assert px[0].sum() == 0 and px[3].sum() == 0 and px[1, 0].sum() == 0


def test_p7_rect_overlap_matches_byte_sets(orc):
    g = synth.rng(13)
    for _ in range(300):
        region = [int(g.integers(1, 6)), int(g.integers(1, 4)), int(g.integers(1, 3))]
        rp = region[0] + int(g.integers(0, 4))
        sp = rp * (region[1] + int(g.integers(0, 2)))
        so = [int(g.integers(0, 6)), int(g.integers(0, 3)), int(g.integers(0, 2))]
        do = [int(g.integers(0, 6)), int(g.integers(0, 3)), int(g.integers(0, 2))]

        def byteset(o):
            base = o[2] * sp + o[1] * rp + o[0]
            return {base + z * sp + y * rp + x for z in range(region[2])
                    for y in range(region[1]) for x in range(region[0])}
        exp = bool(byteset(so) & byteset(do))
        assert orc.rect_overlap(so, do, region, rp, sp, rp, sp) == exp


# ---------------------------------------------------------------- validation of combos
def test_oracle_rejects_undefined_combinations(orc):
    img = orc.Image(np.zeros(16, np.uint8), 2, 2, 1, dims=2, order=orc.RGBA,
                    type=orc.UNSIGNED_INT8)
    c = np.zeros((1, 2), np.float32)
    with pytest.raises(orc.OracleError) as e:                     # A7
        orc.read_samples(img, False, ADDR["CLAMP"], FILT["NEAREST"], orc.RT_F, c)
    assert e.value.code == -59
    with pytest.raises(orc.OracleError) as e:                     # A6
        orc.read_samples(img, False, ADDR["CLAMP"], FILT["LINEAR"], orc.RT_UI, c)
    assert e.value.code == -59
    with pytest.raises(orc.OracleError) as e:                     # A5
        orc.read_samples(img, False, ADDR["REPEAT"], FILT["NEAREST"], orc.RT_UI, c)
    assert e.value.code == -30
