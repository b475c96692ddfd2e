"""Pins of the oracle's CUDA texture fetches (NEXT row 3: the CUDA side of the
paper's CUDA-to-OpenCL texture translation).

What fixes the expected values:
  * hand-worked examples of the CUDA C Programming Guide's "Texture Fetching"
    formulas (tests/golden/p10_cuda_tex.txt) and a per-axis-mode example;
  * every 8/16-bit code of cudaReadModeNormalizedFloat against numpy float32
    division (unsigned c/(2^b-1), signed c/(2^(b-1)-1) clamped to -1);
  * the translation claim itself: a fetch equals read_imageX of the OpenCL
    oracle (pinned separately, P1-P7) with the mapped sampler and image type,
    bit for bit on the texture's channels, by brute force over lattices,
    specials and random coordinates for every mode, filter and shape (MIRROR
    off the dyadic lattices: within the rounding of CUDA's own mirror formula,
    reading A43).
"""
import os

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
MODES = {"WRAP": 0, "CLAMP": 1, "MIRROR": 2, "BORDER": 3}
FILTERS = {"POINT": 0, "LINEAR": 1}
# the paper's translation: texture -> (image, sampler)
CL_ADDR = {0: 0x1133, 1: 0x1131, 2: 0x1134, 3: 0x1132}   # REPEAT, CLAMP_TO_EDGE, MIRRORED, CLAMP
CL_FILT = {0: 0x1140, 1: 0x1141}


def _lines(name):
    with open(os.path.join(GOLDEN, name)) as fh:
        for line in fh:
            line = line.split("|")[0].strip()
            if line and not line.startswith("#"):
                yield line.split()


def test_p10_golden_1d(orc):
    img = orc.Image(np.array([10, 20, 30, 40], np.float32), 4, 1, 1, dims=1, order=orc.R,
                    type=orc.FLOAT)
    n = 0
    for mode, filt, norm, x, v in _lines("p10_cuda_tex.txt"):
        out = orc.tex_fetch(img, [MODES[mode]], FILTERS[filt], orc.TEX_ELEMENT, bool(int(norm)),
                            np.array([[float(x)]], np.float32))[0]
        assert out.view(np.float32).tolist() == [float(v), 0.0, 0.0, 0.0], (mode, filt, norm, x, out.view(np.float32))
        n += 1
    assert n >= 35


def test_p10_per_axis_modes(orc):
    """CUDA modes are per axis (OpenCL has one per sampler, reading A40): x wraps, y borders."""
    img = orc.Image(np.array([[1, 2], [3, 4]], np.float32), 2, 2, 1, dims=2, order=orc.R,
                    type=orc.FLOAT)
    co = np.array([[1.25, 0.25], [1.75, 1.25], [-0.25, 0.75]], np.float32)
    out = orc.tex_fetch(img, [orc.TEX_WRAP, orc.TEX_BORDER], orc.TEX_POINT, orc.TEX_ELEMENT, True, co)
    # (1.25, .25): x frac .25 -> i 0, y .5 -> j 0: T = 1; (1.75, 1.25): i 1, y 2.5 -> border 0;
    # (-0.25, .75): frac .75 -> i 1, j 1: T = 4
    assert out[:, 0].view(np.float32).tolist() == [1.0, 0.0, 4.0]


@pytest.mark.parametrize("stored,bits,signed", [("UNSIGNED_INT8", 8, False), ("SIGNED_INT8", 8, True),
                                                ("UNSIGNED_INT16", 16, False), ("SIGNED_INT16", 16, True)])
def test_p10_read_modes_every_code(orc, stored, bits, signed):
    t = getattr(orc, stored)
    dt = {8: np.int8 if signed else np.uint8, 16: np.int16 if signed else np.uint16}[bits]
    codes = np.arange(1 << bits, dtype=np.int64) - ((1 << (bits - 1)) if signed else 0)
    img = orc.Image(codes.astype(dt), codes.size, 1, 1, dims=1, order=orc.R, type=t)
    xs = np.arange(codes.size, dtype=np.int32)
    norm = orc.tex1Dfetch(img, orc.TEX_NORMALIZED, xs)[:, 0].view(np.float32)
    d = np.float32((1 << (bits - 1)) - 1 if signed else (1 << bits) - 1)
    exp = np.maximum(codes.astype(np.float32) / d, np.float32(-1.0))
    assert np.array_equal(norm.view(np.uint32), exp.astype(np.float32).view(np.uint32))
    elem = orc.tex1Dfetch(img, orc.TEX_ELEMENT, xs)[:, 0].view(np.int32)
    assert np.array_equal(elem, codes.astype(np.int32))
    # out of range: 0
    assert orc.tex1Dfetch(img, orc.TEX_NORMALIZED, [-1, codes.size]).tolist() == [[0] * 4] * 2


def test_p10_rejects_what_cuda_rejects(orc):
    img = orc.Image(np.zeros(4, np.uint8), 4, 1, 1, dims=1, order=orc.R, type=orc.UNSIGNED_INT8)
    co = np.zeros((1, 1), np.float32)
    with pytest.raises(orc.OracleError):   # wrap with unnormalized coordinates
        orc.tex_fetch(img, [orc.TEX_WRAP], orc.TEX_POINT, orc.TEX_ELEMENT, False, co)
    with pytest.raises(orc.OracleError):   # linear filtering of an element-type integer read
        orc.tex_fetch(img, [orc.TEX_CLAMP], orc.TEX_LINEAR, orc.TEX_ELEMENT, True, co)
    f = orc.Image(np.zeros(4, np.float32), 4, 1, 1, dims=1, order=orc.R, type=orc.FLOAT)
    with pytest.raises(orc.OracleError):   # normalized-float read of a float channel
        orc.tex_fetch(f, [orc.TEX_CLAMP], orc.TEX_POINT, orc.TEX_NORMALIZED, True, co)


# ---------------------------------------------------------------- the translation
# stored type x read mode -> the OpenCL image type of the translated image, return class
def _cl_type(orc, stored, read_mode):
    if read_mode == orc.TEX_NORMALIZED:
        return {orc.UNSIGNED_INT8: orc.UNORM_INT8, orc.SIGNED_INT8: orc.SNORM_INT8,
                orc.UNSIGNED_INT16: orc.UNORM_INT16, orc.SIGNED_INT16: orc.SNORM_INT16}[stored], orc.RT_F
    rt = {orc.UNSIGNED_INT8: orc.RT_UI, orc.UNSIGNED_INT16: orc.RT_UI, orc.UNSIGNED_INT32: orc.RT_UI,
          orc.SIGNED_INT8: orc.RT_I, orc.SIGNED_INT16: orc.RT_I, orc.SIGNED_INT32: orc.RT_I}.get(stored, orc.RT_F)
    return stored, rt


def _coords(g, dims, sizes, norm, arrayed, n_layers):
    sp = synth.special_floats()
    lat = synth.coord_lattice(-2.0, 3.0, 1 / 32) if norm else synth.coord_lattice(-2.0, max(sizes) + 2.0, 1 / 16)
    pts = []
    for d in range(dims):
        vals = np.concatenate([lat, sp])
        c = g.uniform(-0.5, 1.5 if norm else max(sizes) + 1, (vals.size, dims)).astype(np.float32)
        c[:, d] = vals
        pts.append(c)
    pts.append(g.uniform(-1.5, 2.5, (300, dims)).astype(np.float32) * np.float32(1 if norm else max(sizes)))
    c = np.concatenate(pts)
    if arrayed:
        c = np.concatenate([c, g.integers(-1, n_layers + 1, (c.shape[0], 1)).astype(np.float32)], 1)
    return np.ascontiguousarray(c, np.float32)


CASES = [  # (dims, arrayed, (W, H, D), order, stored type, read mode)
    (1, False, (5, 1, 1), "RGBA", "FLOAT", 0), (2, False, (4, 3, 1), "R", "UNSIGNED_INT8", 1),
    (3, False, (3, 4, 2), "RG", "SIGNED_INT16", 1), (2, False, (5, 2, 1), "RGBA", "HALF_FLOAT", 0),
    (1, True, (6, 3, 1), "R", "FLOAT", 0), (2, True, (3, 2, 3), "RGBA", "UNSIGNED_INT16", 1),
    (2, False, (4, 3, 1), "RGBA", "UNSIGNED_INT8", 0), (3, False, (2, 3, 2), "R", "SIGNED_INT32", 0)]


def _dyadic(c):
    """coordinates whose every component is a multiple of 2^-20 (the lattices):
    there frac(x), 1 - frac(x) and the OpenCL mirror |s - 2 rint(s/2)| are all exact"""
    with np.errstate(invalid="ignore"):
        s = c.astype(np.float64) * 2.0 ** 20
        return np.all(np.isfinite(s) & (s == np.round(s)), axis=1)


def _mirror_close(orc, cl_img, norm, rt, filt, co, got, exp, nch, vals):
    """MIRROR off the lattice (reading A43): CUDA's mirrored coordinate
    1 - frac(x) rounds where OpenCL's |s - 2 rint(s/2)| does not, by at most
    2^-24 of the unit interval.  LINEAR: the results differ by at most that
    coordinate error times N times the texel range (+ 4 ulp); NEAREST: the
    fetch equals the translated read at a coordinate within 2^-22 of s."""
    n = max(cl_img.width, cl_img.height, cl_img.depth)
    if filt == 1:
        g, e = got[:, :nch].view(np.float32).astype(np.float64), exp[:, :nch].view(np.float32).astype(np.float64)
        tol = n * 2.0 ** -22 * float(np.ptp(vals)) + 4 * np.spacing(np.abs(e).astype(np.float32)).astype(np.float64)
        ok = (np.abs(g - e) <= tol) | (np.isnan(g) & np.isnan(e))
        return np.all(ok, axis=1)
    ok = np.zeros(co.shape[0], bool)
    dims = cl_img.dims
    for delta in (0.0, 2.0 ** -24, -2.0 ** -24, 2.0 ** -23, -2.0 ** -23, 2.0 ** -22, -2.0 ** -22):
        for d in range(dims):
            c2 = co.copy()
            c2[:, d] = (c2[:, d].astype(np.float64) + delta).astype(np.float32)
            e2 = orc.read_samples(cl_img, norm, CL_ADDR[2], CL_FILT[0], rt, c2).view(np.uint32)
            ok |= np.all(e2[:, :nch] == got[:, :nch], axis=1)
    return ok


@pytest.mark.parametrize("case", CASES)
def test_p10_fetch_equals_translated_read_image(orc, case):
    """The paper's translation: tex*(tex, coords) equals
    read_imageX(image, sampler, coords) with the mapped sampler and image type,
    bit for bit -- for MIRROR on dyadic coordinates (off them, within the
    rounding of CUDA's mirror formula, reading A43)."""
    dims, arrayed, sizes, order, stored, rmode = case
    W, H, D = sizes
    g = synth.rng(70 + dims + 3 * W + H)
    order, stored = getattr(orc, order), getattr(orc, stored)
    data = synth.image_codes(g, order, stored, W, H, D, signed=True)
    tex_img = orc.Image(data, W, H, D, dims=dims, order=order, type=stored, arrayed=arrayed)
    cl_type, rt = _cl_type(orc, stored, rmode)
    cl_img = orc.Image(data, W, H, D, dims=dims, order=order, type=cl_type, arrayed=arrayed)
    nch = orc.lib().oracle_channels(order)
    n_layers = (H if dims == 1 else D) if arrayed else 1
    filters = [0, 1] if rt == orc.RT_F else [0]
    checked = 0
    for norm in (False, True):
        for mode in range(4):
            if not norm and mode in (orc.TEX_WRAP, orc.TEX_MIRROR):
                continue
            for filt in filters:
                co = _coords(g, dims, sizes, norm, arrayed, n_layers)
                got = orc.tex_fetch(tex_img, [mode] * dims, filt, rmode, norm, co)
                exp = orc.read_samples(cl_img, norm, CL_ADDR[mode], CL_FILT[filt], rt, co).view(np.uint32)
                bad = np.nonzero((got[:, :nch] != exp[:, :nch]).any(1))[0]
                if rt == orc.RT_F:  # NaN iff NaN (non-finite coordinates, reading A26)
                    gf, ef = got[:, :nch].view(np.float32), exp[:, :nch].view(np.float32)
                    bad = np.array([b for b in bad if not (np.isnan(gf[b]) & np.isnan(ef[b])).any()
                                    or (np.isnan(gf[b]) != np.isnan(ef[b])).any()], np.int64)
                if mode == orc.TEX_MIRROR and len(bad):
                    dy = _dyadic(co[:, :dims])
                    assert not dy[bad].any(), (norm, filt, co[bad[dy[bad]][0]])
                    vals = exp[:, :nch].view(np.float32)
                    close = _mirror_close(orc, cl_img, norm, rt, filt, co[bad], got[bad], exp[bad], nch,
                                          vals[np.isfinite(vals)])
                    assert close.all(), (norm, filt, co[bad[~close][0]], got[bad[~close][0]])
                    bad = []
                assert len(bad) == 0, (norm, mode, filt, co[bad[0]], got[bad[0]], exp[bad[0]])
                checked += co.shape[0]
    assert checked > 2000
