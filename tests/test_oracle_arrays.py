"""Pins of the oracle's image-array and 1D-buffer rules (
[CL1.2 §5.3.1], §8.4 "Selecting an Image from an Image Array").

What fixes the expected values: the hand-worked reads of
tests/golden/p8_array_layers.txt; numpy's round-half-to-even `np.rint` for the
layer index; the reduction of an array read to a read of the selected layer
as a plain image (whose rules are pinned in test_oracle_pins.py); numpy
slicing for the host-pitch quirk of 1D arrays.
"""
import os

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
ADDR = {"NONE": 0x1130, "CLAMP_TO_EDGE": 0x1131, "CLAMP": 0x1132, "REPEAT": 0x1133,
        "MIRRORED_REPEAT": 0x1134}
FILT = {"NEAREST": 0x1140, "LINEAR": 0x1141}
SAMPLERS = [(norm, a, f) for norm in (0, 1) for a in ADDR.values() for f in FILT.values()
            if norm or a in (0x1130, 0x1131, 0x1132)]


def _lines(name):
    with open(os.path.join(GOLDEN, name)) as fh:
        for line in fh:
            line = line.split("|")[0].strip()
            if line and not line.startswith("#"):
                yield line.split()


def test_p8_golden_1d_array(orc):
    W, L = 4, 4
    data = np.array([[10 * (i + 1) + 100 * l for i in range(W)] for l in range(L)], np.float32)
    img = orc.Image(data, W, L, 1, dims=1, order=orc.R, type=orc.FLOAT, arrayed=True)
    n = 0
    for norm, addr, filt, s, layer, exp in _lines("p8_array_layers.txt"):
        out = orc.read_samples(img, bool(int(norm)), ADDR[addr], FILT[filt], orc.RT_F,
                               np.array([[float(s), float(layer)]], np.float32))[0]
        assert out.tolist() == [float(exp), 0.0, 0.0, 1.0], (norm, addr, filt, s, layer, out)
        n += 1
    assert n >= 12


def test_p8_layer_index_is_rint_then_clamp(orc):
    g = synth.rng(300)
    c = np.concatenate([np.arange(-4, 12, 0.5, dtype=np.float32),
                        g.uniform(-20, 20, 2000).astype(np.float32),
                        np.array([np.inf, -np.inf, 3e9, -3e9, 7.4999995, 8.5000005],
                                 np.float32)])
    for n in (1, 2, 7, 8):
        exp = np.clip(np.rint(c.astype(np.float64)), 0, n - 1).astype(np.int64)
        got = np.array([orc.layer_index(float(v), n) for v in c])
        assert np.array_equal(got, exp), n
    assert orc.layer_index(float("nan"), 5) == 0  # reading A35


def _layer_image(orc, data, W, H, dims, order, typ, layer):
    """layer `layer` of an array, as a plain image (the reduction of §8.4)."""
    if dims == 1:
        return orc.Image(np.ascontiguousarray(data[layer]), W, 1, 1, dims=1, order=order, type=typ)
    return orc.Image(np.ascontiguousarray(data[layer]), W, H, 1, dims=2, order=order, type=typ)


@pytest.mark.parametrize("dims", [1, 2])
@pytest.mark.parametrize("fmt", [("RGBA", "FLOAT"), ("R", "UNORM_INT8"), ("RG", "HALF_FLOAT"),
                                 ("RGBA", "SIGNED_INT16"), ("BGRA", "UNORM_INT8")])
def test_p8_array_read_reduces_to_layer_read(orc, dims, fmt):
    order, typ = getattr(orc, fmt[0]), getattr(orc, fmt[1])
    ordn = {orc.R: 0x10B0, orc.RG: 0x10B2, orc.RGBA: 0x10B5, orc.BGRA: 0x10B6}[order]
    W, H, L = 9, (5 if dims == 2 else 1), 6
    g = synth.rng(301 + dims)
    if dims == 1:
        data = synth.image_codes(g, ordn, typ, W, L)[0]              # (L, W, ch)
        img = orc.Image(data, W, L, 1, dims=1, order=order, type=typ, arrayed=True)
        data = data.reshape(L, 1, W, -1)
    else:
        data = synth.image_codes(g, ordn, typ, W, H, L)               # (L, H, W, ch)
        img = orc.Image(data, W, H, L, dims=2, order=order, type=typ, arrayed=True)
    integer = typ in (orc.SIGNED_INT16,)
    rt = orc.RT_I if integer else orc.RT_F
    n = 400
    for norm, addr, filt in SAMPLERS:
        if integer and filt == FILT["LINEAR"]:
            continue
        sc = g.uniform(-0.3, 1.3, (n, dims)) if norm else g.uniform(-2, W + 2, (n, dims))
        lc = np.concatenate([g.uniform(-2, L + 1, n - 6), [0.5, 1.5, 2.5, -0.5, L - 0.5, L + 0.5]])
        co = np.concatenate([sc, lc[:, None]], 1).astype(np.float32)
        got = orc.read_samples(img, bool(norm), addr, filt, rt, co)
        lay = np.clip(np.rint(co[:, dims].astype(np.float64)), 0, L - 1).astype(int)
        for l in np.unique(lay):
            m = lay == l
            ref = orc.read_samples(_layer_image(orc, data, W, H, dims, order, typ, l), bool(norm),
                                   addr, filt, rt, np.ascontiguousarray(co[m, :dims]))
            assert np.array_equal(got[m].view(np.uint32), ref.view(np.uint32)), (norm, addr, filt, l)


def test_p8_array_int_coords_and_writes(orc):
    W, H, L = 5, 3, 4
    data = np.zeros((L, H, W, 4), np.uint8)
    img = orc.Image(data, W, H, L, dims=2, order=orc.RGBA, type=orc.UNSIGNED_INT8, arrayed=True)
    co = np.array([[1, 2, 3, 0], [4, 0, 0, 0], [0, 0, 4, 0], [0, 0, -1, 0], [5, 0, 1, 0]],
                  np.int32)
    col = np.array([[1, 2, 3, 4], [5, 6, 7, 8], [9, 9, 9, 9], [7, 7, 7, 7], [6, 6, 6, 6]],
                   np.uint32)
    orc.write_samples(img, orc.RT_UI, co, col)
    exp = np.zeros_like(data)
    exp[3, 2, 1] = [1, 2, 3, 4]
    exp[0, 0, 4] = [5, 6, 7, 8]        # layers 4 and -1 and x = 5 are out of range: no-ops (A15)
    assert np.array_equal(img.data.reshape(L, H, W, 4), exp)
    # integer-coordinate reads (A30): the layer is selected like a float one
    got = orc.read_samples(img, False, ADDR["CLAMP_TO_EDGE"], FILT["NEAREST"], orc.RT_UI,
                           np.array([[1, 2, 3, 0], [1, 2, 9, 0], [4, 0, -5, 0]], np.int32))
    assert got.tolist() == [[1, 2, 3, 4], [1, 2, 3, 4], [5, 6, 7, 8]]


def test_p8_1d_array_host_rect_uses_slice_pitch(orc):
    """clEnqueueRead/WriteImage on a 1D image array: region[1] counts layers and
    host layers are slice_pitch apart (default row_pitch)."""
    W, L, es = 6, 5, 4
    data = np.arange(L * W * es, dtype=np.uint8).reshape(L, W * es)
    img = orc.Image(data.copy(), W, L, 1, dims=1, order=orc.RGBA, type=orc.UNORM_INT8,
                    arrayed=True)
    origin, region = (2, 1, 0), (3, 3, 1)
    for rp, sp in ((0, 0), (16, 0), (12, 20), (0, 40)):
        host = np.full(200, 0xEE, np.uint8)
        orc.read_image_rect(img, origin, region, rp, sp, host)
        rpe = rp or region[0] * es
        spe = sp or rpe
        exp = np.full(200, 0xEE, np.uint8)
        for y in range(region[1]):
            exp[y * spe:y * spe + region[0] * es] = data[origin[1] + y, origin[0] * es:(origin[0] + region[0]) * es]
        assert np.array_equal(host, exp), (rp, sp)
        # the write is the inverse
        img2 = orc.Image(np.zeros_like(data), W, L, 1, dims=1, order=orc.RGBA,
                         type=orc.UNORM_INT8, arrayed=True)
        orc.write_image_rect(img2, origin, region, rp, sp, host)
        ref = np.zeros_like(data)
        ref[1:4, 8:20] = data[1:4, 8:20]
        assert np.array_equal(img2.data.reshape(L, -1), ref)


def test_p8_grid_mode_on_arrays(orc):
    """Grid reads of a 2D array: coordinate 2 of the affine map is the layer."""
    W, H, L = 8, 6, 3
    g = synth.rng(305)
    data = synth.image_codes(g, 0x10B5, orc.FLOAT, W, H, L)
    img = orc.Image(data, W, H, L, dims=2, order=orc.RGBA, type=orc.FLOAT, arrayed=True)
    A = np.array([0.9, 0.1, 0.0, -0.3, 0.05, 1.1, 0.0, 0.2, 0.0, 0.0, 0.75, -0.2], np.float32)
    got = orc.read_grid(img, False, ADDR["CLAMP"], FILT["LINEAR"], orc.RT_F, A, (W, H, 4), 4)
    z, y, x = np.meshgrid(np.arange(4), np.arange(H), np.arange(W), indexing="ij")
    xf, yf, zf = (v.astype(np.float32).ravel() for v in (x, y, z))
    co = []
    for k in range(3):
        a = A[4 * k:4 * k + 4]
        v = (a[0] * xf).astype(np.float32)
        v = (v + (a[1] * yf).astype(np.float32)).astype(np.float32)
        v = (v + (a[2] * zf).astype(np.float32)).astype(np.float32)
        co.append((v + a[3]).astype(np.float32))
    co = np.stack(co, 1)
    ref = orc.read_samples(img, False, ADDR["CLAMP"], FILT["LINEAR"], orc.RT_F, co)
    assert np.array_equal(got.reshape(-1, 4).view(np.uint32), ref.view(np.uint32))


def test_p8_integer_coordinates_are_exact_indices(orc):
    """Reading A30: an integer coordinate is the texel index itself -- equal to
    the float path at u = (float)i while i is exactly representable (|i| <= 2^24),
    and still the texel at i beyond (a 1D image buffer reaches 2^31 - 1)."""
    n = (1 << 25) + 64
    data = (np.arange(n, dtype=np.int64) * 2654435761 % 251).astype(np.uint8)
    img = orc.Image(data, n, 1, 1, dims=1, order=orc.R, type=orc.UNSIGNED_INT8)
    g = synth.rng(306)
    big = np.concatenate([g.integers((1 << 24) + 1, n, 500), [n - 1, (1 << 24) + 1, (1 << 25) + 1]])
    for addr in (ADDR["NONE"], ADDR["CLAMP_TO_EDGE"], ADDR["CLAMP"]):
        got = orc.read_samples(img, False, addr, FILT["NEAREST"], orc.RT_UI,
                               big.astype(np.int32)[:, None].copy())
        assert np.array_equal(got[:, 0], data[big]), addr          # the definition: texel i
        small = np.concatenate([g.integers(-5, 1 << 24, 500), [1 << 24, -1, n, n + 7]])
        gi = orc.read_samples(img, False, addr, FILT["NEAREST"], orc.RT_UI,
                              small.astype(np.int32)[:, None].copy())
        gf = orc.read_samples(img, False, addr, FILT["NEAREST"], orc.RT_UI,
                              small.astype(np.float32)[:, None].copy())
        ok = np.abs(small) <= (1 << 24)
        assert np.array_equal(gi[ok], gf[ok]), addr
    # out of range under CLAMP_TO_EDGE: the edge texel; under NONE/CLAMP: the border (0,0,0,1)
    got = orc.read_samples(img, False, ADDR["CLAMP_TO_EDGE"], FILT["NEAREST"], orc.RT_UI,
                           np.array([[n + 100], [-7]], np.int32))
    assert got[:, 0].tolist() == [data[n - 1], data[0]]
    got = orc.read_samples(img, False, ADDR["CLAMP"], FILT["NEAREST"], orc.RT_UI,
                           np.array([[n + 100]], np.int32))
    assert got.tolist() == [[0, 0, 0, 1]]
