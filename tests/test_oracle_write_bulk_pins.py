"""Pins P11 / P12 of the oracle's write side and bulk operations.

P11: the bytes write_image{f,i,ui} stores for every channel order (the inverse
channel map) and the low/high saturation of the signed conversions -- from the
hand-worked golden tests/golden/p11_write_slots.txt ([CL1.2 §5.3.1.1, §8.3.1,
§6.12.14.4]), plus the round trip "write then NEAREST-read gives the channel
map of the colour" (the forward map is pinned by P3).

P12: bulk operations at the corners the earlier pins left open --
FillImage / CopyBufferToImage / CopyImage into a 3D image at a non-zero
origin[2] with padded pitches, CopyBufferRect with an explicit row pitch and
slice pitch 0 (default region[1] * row_pitch, [CL1.2 §5.2.2]), and the
write_image out-of-range no-op (reading A15) on each axis, checked with guard
bands before and after the image and padding bytes between rows and slices so
a stray write anywhere is visible.

Every expected value comes from the golden file, numpy slicing/strides or the
spec's definition restated here -- never from the oracle or the CUDA path.
"""
import os

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
RT = {"f": 0, "i": 1, "ui": 2}


def _golden(section):
    with open(os.path.join(GOLDEN, "p11_write_slots.txt")) as fh:
        for line in fh:
            line = line.split("|")[0].strip()
            if line.startswith(section + " "):
                lhs, rhs = line[len(section) + 1:].split("->")
                yield lhs.split(), bytes(int(b, 16) for b in rhs.split())


def _color(rt, vals):
    if rt == "f":
        return np.array([float(v) for v in vals] + [0.0] * (4 - len(vals)), np.float32)
    dt = np.int32 if rt == "i" else np.uint32
    return np.array([int(v) for v in vals] + [0] * (4 - len(vals)), np.int64).astype(dt)


def test_p11_golden_write_slots(orc):
    n = 0
    for (order, typ, rt, *vals), exp in _golden("slot"):
        got = orc.convert_texel(getattr(orc, order), getattr(orc, typ), RT[rt], _color(rt, vals))
        assert got == exp, (order, typ, vals, got.hex(), exp.hex())
        n += 1
    assert n == 20


def test_p11_golden_saturation(orc):
    n = 0
    for (typ, rt, v), exp in _golden("sat"):
        got = orc.convert_texel(orc.R, getattr(orc, typ), RT[rt], _color(rt, [v]))
        assert got == exp, (typ, v, got.hex(), exp.hex())
        n += 1
    assert n == 14


# the channel map (x,y,z,w) a NEAREST read returns for a stored colour c, per
# order ([CL1.2 §8.3] table; INTENSITY / LUMINANCE store x, reading A16)
def _mapped(order, c, one):
    x, y, z, w = c
    return {"R": (x, 0, 0, one), "A": (0, 0, 0, w), "RG": (x, y, 0, one), "RA": (x, 0, 0, w),
            "RGBA": (x, y, z, w), "BGRA": (x, y, z, w), "ARGB": (x, y, z, w),
            "INTENSITY": (x, x, x, x), "LUMINANCE": (x, x, x, one)}[order]


@pytest.mark.parametrize("order,typ,rt", [
    ("R", "FLOAT", "f"), ("A", "FLOAT", "f"), ("RG", "FLOAT", "f"), ("RA", "FLOAT", "f"),
    ("RGBA", "FLOAT", "f"), ("INTENSITY", "FLOAT", "f"), ("LUMINANCE", "FLOAT", "f"),
    ("BGRA", "UNSIGNED_INT8", "ui"), ("ARGB", "UNSIGNED_INT8", "ui"), ("ARGB", "SIGNED_INT8", "i"),
    ("A", "UNSIGNED_INT16", "ui"), ("RA", "SIGNED_INT32", "i"), ("BGRA", "UNORM_INT8", "f"),
    ("ARGB", "UNORM_INT8", "f")])
def test_p11_write_then_read_is_the_channel_map(orc, order, typ, rt):
    """write_image at (i, j) then read_image there (NEAREST, texel centre) returns
    the channel map of the colour, for colours exactly representable in the type."""
    W, H = 4, 3
    es = orc.elem_size(getattr(orc, order), getattr(orc, typ))
    img = orc.Image(np.zeros(W * H * es, np.uint8), W, H, 1, dims=2, order=getattr(orc, order),
                    type=getattr(orc, typ))
    g = synth.rng(40)
    if typ == "FLOAT":
        cols = g.uniform(-4, 4, (W * H, 4)).astype(np.float32)
    elif typ == "UNORM_INT8":   # c / 255 round-trips exactly through the conversions
        cols = (g.integers(0, 256, (W * H, 4)).astype(np.float32) / np.float32(255))
    elif rt == "i":
        cols = g.integers(-100, 100, (W * H, 4)).astype(np.int32)
    else:
        cols = g.integers(0, 200, (W * H, 4)).astype(np.uint32)
    ij = np.array([(i, j) for j in range(H) for i in range(W)], np.int32)
    orc.write_samples(img, RT[rt], ij, cols)
    co = (ij + 0.5).astype(np.float32)
    got = orc.read_samples(img, False, orc.ADDRESS_CLAMP_TO_EDGE, orc.FILTER_NEAREST, RT[rt], co)
    one = 1.0 if rt == "f" else 1
    exp = np.array([_mapped(order, c, one) for c in cols.tolist()], dtype=got.dtype)
    assert np.array_equal(got, exp), (order, typ)


# ---------------------------------------------------------------- P12 bulk corners
def _pitched_3d(codes, rp, sp, guard):
    """codes (D, H, W, es bytes) laid out with row pitch rp and slice pitch sp
    after `guard` sentinel bytes, followed by `guard` more; padding = 0xA5."""
    D, H, W = codes.shape[:3]
    b = codes.reshape(D, H, -1).view(np.uint8).reshape(D, H, -1)
    raw = np.full(guard + sp * D + guard, 0xA5, np.uint8)
    view = np.lib.stride_tricks.as_strided(raw[guard:], (D, H, b.shape[2]), (sp, rp, 1))
    view[...] = b
    return raw, view


def _image(orc, raw, guard, W, H, D, order, typ, rp, sp):
    return orc.Image(raw[guard:], W, H, D, dims=3, order=order, type=typ, row_pitch=rp, slice_pitch=sp)


def test_p12_fill_image_3d_nonzero_z_origin(orc):
    g = synth.rng(41)
    W, H, D, es = 7, 5, 4, 4
    codes = synth.image_codes(g, orc.RGBA, orc.UNORM_INT8, W, H, D)
    rp, sp, guard = 40, 40 * 6, 256
    raw, view = _pitched_3d(codes, rp, sp, guard)
    exp = raw.copy()
    img = _image(orc, raw, guard, W, H, D, orc.RGBA, orc.UNORM_INT8, rp, sp)
    orc.fill_image(img, orc.RT_F, np.array([1.0, 0.0, 0.5, 0.25], np.float32), (2, 1, 1), (3, 3, 2))
    ev = np.lib.stride_tricks.as_strided(exp[guard:], (D, H, W, es), (sp, rp, es, 1))
    ev[1:3, 1:4, 2:5] = np.array([255, 0, 128, 64], np.uint8)   # P11 golden RGBA bytes
    assert np.array_equal(raw, exp)


def test_p12_buffer_to_image_and_image_copies_at_z_origin(orc):
    g = synth.rng(42)
    W, H, D, es = 6, 4, 5, 8
    rp, sp, guard = 64, 64 * 5, 512
    codes = synth.image_codes(g, orc.RG, orc.FLOAT, W, H, D)
    raw, _ = _pitched_3d(codes, rp, sp, guard)
    exp = raw.copy()
    img = _image(orc, raw, guard, W, H, D, orc.RG, orc.FLOAT, rp, sp)
    region, org, off = (3, 2, 3), (1, 2, 2), 24
    buf = g.integers(0, 256, off + 3 * 2 * 3 * es + 16, dtype=np.uint8)
    orc.copy_buffer_to_image(buf, img, off, org, region)
    ev = np.lib.stride_tricks.as_strided(exp[guard:], (D, H, W, es), (sp, rp, es, 1))
    ev[2:5, 2:4, 1:4] = buf[off:off + 3 * 2 * 3 * es].reshape(3, 2, 3, es)
    assert np.array_equal(raw, exp)
    # image -> image: both origins with z != 0, destination pitched differently
    rp2, sp2 = 56, 56 * 4
    raw2 = np.full(guard + sp2 * D + guard, 0x5A, np.uint8)
    exp2 = raw2.copy()
    dst = _image(orc, raw2, guard, W, H, D, orc.RG, orc.FLOAT, rp2, sp2)
    orc.copy_image(img, dst, (2, 1, 3), (0, 2, 1), (4, 2, 2))
    sv = np.lib.stride_tricks.as_strided(raw[guard:], (D, H, W, es), (sp, rp, es, 1))
    dv = np.lib.stride_tricks.as_strided(exp2[guard:], (D, H, W, es), (sp2, rp2, es, 1))
    dv[1:3, 2:4, 0:4] = sv[3:5, 1:3, 2:6]
    assert np.array_equal(raw2, exp2)
    # image -> buffer from z origin 2
    out = np.full(off + 4 * 3 * 2 * es + 8, 0x33, np.uint8)
    exp3 = out.copy()
    orc.copy_image_to_buffer(img, out, (1, 1, 2), (4, 3, 2), off)
    exp3[off:off + 4 * 3 * 2 * es] = sv[2:4, 1:4, 1:5].reshape(-1)
    assert np.array_equal(out, exp3)


@pytest.mark.parametrize("side", ["src", "dst", "both"])
def test_p12_copy_rect_slice_pitch_defaults_to_region1_times_row_pitch(orc, side):
    """[CL1.2 §5.2.2]: 'If src_slice_pitch is 0, src_slice_pitch is computed as
    region[1] * src_row_pitch' (likewise dst) -- with an explicit row pitch."""
    g = synth.rng(43)
    region, so, do = (5, 3, 4), (2, 1, 1), (1, 2, 2)
    srp, drp = 9, 11
    ssp_true, dsp_true = region[1] * srp, region[1] * drp
    src = g.integers(0, 256, ssp_true * (so[2] + region[2]) + 64, dtype=np.uint8)
    dst = g.integers(0, 256, dsp_true * (do[2] + region[2]) + 64, dtype=np.uint8)
    exp = dst.copy()
    s3 = np.lib.stride_tricks.as_strided(src[so[2] * ssp_true + so[1] * srp + so[0]:],
                                         (region[2], region[1], region[0]), (ssp_true, srp, 1))
    d3 = np.lib.stride_tricks.as_strided(exp[do[2] * dsp_true + do[1] * drp + do[0]:],
                                         (region[2], region[1], region[0]), (dsp_true, drp, 1))
    d3[...] = s3
    ssp = 0 if side in ("src", "both") else ssp_true
    dsp = 0 if side in ("dst", "both") else dsp_true
    orc.copy_rect(src, dst, so, do, region, srp, ssp, drp, dsp)
    assert np.array_equal(dst, exp)


@pytest.mark.parametrize("dims", [1, 2, 3])
def test_p12_write_out_of_range_is_a_no_op(orc, dims):
    """Reading A15: write_image outside [0, n) on ANY axis writes nothing --
    guard bands one slice long before and after the image and padded row and
    slice pitches make a stray write anywhere visible."""
    W, H, D = 5, (4 if dims > 1 else 1), (3 if dims > 2 else 1)
    es, rp = 4, 24
    sp = rp * (H + 1)
    guard = sp + rp
    raw = np.full(guard + sp * D + guard, 0xA5, np.uint8)
    img = orc.Image(raw[guard:], W, H, D, dims=dims, order=orc.RGBA, type=orc.UNSIGNED_INT8,
                    row_pitch=rp, slice_pitch=sp)
    coords, cols = [], []
    n = [W, H, D]
    # every coordinate one step outside each face, plus far outside, plus in-range writes
    for ax in range(dims):
        for bad in (-1, n[ax], -1000, n[ax] + 7):
            c = [1, min(1, H - 1), min(1, D - 1)]
            c[ax] = bad
            coords.append(c)
            cols.append([7, 7, 7, 7])
    inside = [(0, 0, 0), (W - 1, H - 1, D - 1), (2, H // 2, D // 2)]
    for k, c in enumerate(inside):
        coords.append(list(c))
        cols.append([10 + k, 20 + k, 30 + k, 40 + k])
    if dims == 3:
        icoords = np.array([c + [0] for c in coords], np.int32)   # int4, w ignored (A20)
    else:
        icoords = np.array([c[:dims] for c in coords], np.int32)
    exp = raw.copy()
    for k, c in enumerate(inside):
        o = guard + c[2] * sp + c[1] * rp + c[0] * es
        exp[o:o + es] = [10 + k, 20 + k, 30 + k, 40 + k]
    orc.write_samples(img, orc.RT_UI, icoords, np.array(cols, np.uint32))
    assert np.array_equal(raw, exp)


@pytest.mark.parametrize("host_rp,host_sp", [(0, 0), (40, 0), (40, 200)])
def test_p12_read_write_image_host_pitch_defaults(orc, host_rp, host_sp):
    """[CL1.2 §5.3.3]: row_pitch 0 -> region[0] * elem_size; slice_pitch 0 ->
    row_pitch * region[1] (a 3D image, region[2] > 1, z origin != 0)."""
    g = synth.rng(44)
    W, H, D, es = 6, 5, 4, 4
    rp, sp, guard = 32, 32 * 6, 64
    codes = synth.image_codes(g, orc.RGBA, orc.UNORM_INT8, W, H, D)
    raw, _ = _pitched_3d(codes, rp, sp, guard)
    img = _image(orc, raw, guard, W, H, D, orc.RGBA, orc.UNORM_INT8, rp, sp)
    org, region = (1, 1, 1), (4, 3, 2)
    hr = host_rp or region[0] * es
    hs = host_sp or hr * region[1]
    host = np.full(hs * region[2] + 16, 0x77, np.uint8)
    exp = host.copy()
    hv = np.lib.stride_tricks.as_strided(exp, (region[2], region[1], region[0] * es), (hs, hr, 1))
    hv[...] = codes[1:3, 1:4, 1:5].reshape(2, 3, -1)
    orc.read_image_rect(img, org, region, host_rp, host_sp, host)
    assert np.array_equal(host, exp)
    # and back: write the host box into a cleared image at the same origin
    raw2 = np.full_like(raw, 0xA5)
    img2 = _image(orc, raw2, guard, W, H, D, orc.RGBA, orc.UNORM_INT8, rp, sp)
    orc.write_image_rect(img2, org, region, host_rp, host_sp, host)
    iv = np.lib.stride_tricks.as_strided(raw2[guard:], (D, H, W * es), (sp, rp, 1))
    assert np.array_equal(iv[1:3, 1:4, es:5 * es].reshape(2, 3, 4, es), codes[1:3, 1:4, 1:5])
    assert np.array_equal(raw2[:guard], np.full(guard, 0xA5, np.uint8))
