"""Pins of the oracle's packed formats (NEXT row 4): CL_UNORM_SHORT_565,
CL_UNORM_SHORT_555 and CL_UNORM_INT_101010 with CL_RGB / CL_RGBx
([CL1.2 §5.3.1.1, §8.3.1.1], border colours [CL1.2 §6.12.14.1]).

Expected values come from the hand-worked golden tests/golden/p9_packed.txt,
from numpy bit-field extraction and IEEE float32 division written here from
the spec's bit layout (exhaustive over every 16-bit word), and from the
exact-rational sampling model tests/exact_model.py (pin P5) -- never from the
oracle itself or the CUDA path.
"""
import os
from fractions import Fraction

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import synth
from tests import exact_model as em

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
P565, P555, P101010 = 0x10D4, 0x10D5, 0x10D6
RGB, RGBX = 0x10B4, 0x10BC
TYPES = {"565": P565, "555": P555, "101010": P101010}
# [CL1.2 §5.3.1.1] layout: (bits, lowest bit) of R, G, B
LAYOUT = {P565: ((5, 11), (6, 5), (5, 0)), P555: ((5, 10), (5, 5), (5, 0)),
          P101010: ((10, 20), (10, 10), (10, 0))}
WORD = {P565: np.uint16, P555: np.uint16, P101010: np.uint32}


def _lines(section):
    with open(os.path.join(GOLDEN, "p9_packed.txt")) as fh:
        for line in fh:
            line = line.split("|")[0].strip()
            if line.startswith(section + " "):
                yield line.split()[1:]


def _expected_read(words, type_):
    """(R, G, B, 1) per word: numpy bit fields, float32 c / (2^bits - 1)."""
    w = words.astype(np.uint64)
    out = np.ones((w.size, 4), np.float32)
    for c, (bits, sh) in enumerate(LAYOUT[type_]):
        code = ((w >> np.uint64(sh)) & np.uint64((1 << bits) - 1)).astype(np.float32)
        out[:, c] = code / np.float32((1 << bits) - 1)
    return out


def _read_words(orc, words, type_, order=RGB):
    """NEAREST read at every texel centre of a W x 1 image of these words."""
    img = orc.Image(np.ascontiguousarray(words, WORD[type_]), words.size, 1, 1, dims=2,
                    order=order, type=type_)
    co = np.stack([np.arange(words.size) + 0.5, np.full(words.size, 0.5)], 1).astype(np.float32)
    return orc.read_samples(img, False, orc.ADDRESS_CLAMP_TO_EDGE, orc.FILTER_NEAREST, orc.RT_F, co)


def test_p9_golden_reads(orc):
    n = 0
    for t, code, *hexes in _lines("read"):
        for order in (RGB, RGBX):
            got = _read_words(orc, np.array([int(code, 16)]), TYPES[t], order)[0]
            assert got.view(np.uint32).tolist() == [int(h, 16) for h in hexes], (t, code, order)
        n += 1
    assert n == 12


def test_p9_golden_writes(orc):
    n = 0
    for t, x, y, z, w, word in _lines("write"):
        col = np.array([float(x), float(y), float(z), float(w)], np.float32)
        for order in (RGB, RGBX):
            got = orc.convert_texel(order, TYPES[t], orc.RT_F, col)
            assert int.from_bytes(got, "little") == int(word, 16), (t, col, order)
        n += 1
    assert n == 6


def test_p9_golden_border(orc):
    img = {o: orc.Image(np.array([0xFFFF], np.uint16), 1, 1, 1, dims=2, order=o, type=P565)
           for o in (RGB, RGBX)}
    n = 0
    for o, f, s, t, *hexes in _lines("border"):
        out = orc.read_samples(img[RGB if o == "RGB" else RGBX], False, orc.ADDRESS_CLAMP,
                               orc.FILTER_LINEAR if f == "LINEAR" else orc.FILTER_NEAREST, orc.RT_F,
                               np.array([[float(s), float(t)]], np.float32))[0]
        assert out.view(np.uint32).tolist() == [int(h, 16) for h in hexes], (o, f, s, t, out)
        n += 1
    assert n == 5


@pytest.mark.parametrize("type_", [P565, P555])
def test_p9_every_16bit_word(orc, type_):
    words = np.arange(1 << 16, dtype=np.uint16)
    got = _read_words(orc, words, type_)
    assert np.array_equal(got.view(np.uint32), _expected_read(words, type_).view(np.uint32))


def test_p9_101010_every_field_value_and_random_words(orc):
    g = synth.rng(60)
    fields = np.arange(1024, dtype=np.uint32)
    words = np.concatenate([fields << 20, fields << 10, fields, (fields << 20) | (3 << 30),
                            g.integers(0, 1 << 32, 50000, dtype=np.uint64).astype(np.uint32)])
    got = _read_words(orc, words, P101010)
    assert np.array_equal(got.view(np.uint32), _expected_read(words, P101010).view(np.uint32))


@pytest.mark.parametrize("type_", [P565, P555, P101010])
def test_p9_write_read_round_trip_clears_x_bits(orc, type_):
    """write_imagef(read_imagef(word)) = the word with its unused bits cleared."""
    g = synth.rng(61)
    if type_ == P101010:
        words = g.integers(0, 1 << 32, 20000, dtype=np.uint64).astype(np.uint32)
    else:
        words = np.arange(1 << 16, dtype=np.uint16)
    vals = _expected_read(words, type_)
    used = sum(((1 << b) - 1) << sh for b, sh in LAYOUT[type_])
    for k in range(0, words.size, max(1, words.size // 3000)):
        got = int.from_bytes(orc.convert_texel(RGB, type_, orc.RT_F, vals[k]), "little")
        assert got == int(words[k]) & used, (hex(int(words[k])), hex(got))


def test_p9_legal_pairs(orc):
    for t in (P565, P555, P101010):
        assert orc.elem_size(RGB, t) == (4 if t == P101010 else 2)
        assert orc.elem_size(RGBX, t) == (4 if t == P101010 else 2)
        for o in (orc.R, orc.RG, orc.RGBA, orc.BGRA, orc.LUMINANCE):
            assert orc.elem_size(o, t) == -1
    for t in (orc.UNORM_INT8, orc.FLOAT, orc.UNSIGNED_INT8):
        assert orc.elem_size(RGB, t) == -1 and orc.elem_size(RGBX, t) == -1
    for o in (orc.Rx, orc.RGx):  # reading A37: not supported
        assert orc.elem_size(o, orc.FLOAT) == -1 and orc.elem_size(o, orc.UNORM_INT8) == -1
    with pytest.raises(orc.OracleError):  # read_imagei on a packed (normalized) image: A7
        img = orc.Image(np.zeros(4, np.uint16), 4, 1, 1, dims=1, order=RGB, type=P565)
        orc.read_samples(img, False, orc.ADDRESS_NONE, orc.FILTER_NEAREST, orc.RT_I,
                         np.zeros((1, 1), np.float32))


SAMPLERS = [(norm, a, f) for norm in (0, 1) for a in range(0x1130, 0x1135)
            for f in (0x1140, 0x1141) if norm or a <= 0x1132]


@pytest.mark.parametrize("order", [RGB, RGBX])
@pytest.mark.parametrize("dims,sizes", [(2, (3, 2, 1)), (3, (2, 3, 2))])
def test_p9_exact_model_all_samplers(orc, order, dims, sizes):
    """Pin P5 on packed images: every sampler, dyadic lattices + random points; the
    exact model gets numpy-converted texels and the spec's border for the order."""
    g = synth.rng(62 + dims + (order & 0xF))
    W, H, D = sizes
    words = g.integers(0, 1 << 16, W * H * D, dtype=np.uint64).astype(np.uint16)
    img = orc.Image(words, W, H, D, dims=dims, order=order, type=P565)
    tex = _expected_read(words, P565).reshape(D, H, W, 4)
    border = [0.0, 0.0, 0.0, 1.0 if order == RGB else 0.0]
    for norm, addr, filt in SAMPLERS:
        lat = synth.coord_lattice(-1.0, 2.0, 1 / 8) if norm else synth.coord_lattice(-1.5, 4.5, 1 / 4)
        co = np.zeros((lat.size + 200, 4 if dims == 3 else 2), np.float32)
        for d in range(dims):
            co[:lat.size, d] = np.roll(lat, 7 * d)
        co[lat.size:, :dims] = g.uniform(-0.5, 1.5 if norm else 4.0, (200, dims))
        out = orc.read_samples(img, bool(norm), addr, filt, orc.RT_F, co)
        for s in range(co.shape[0]):
            val, kind = em.sample_exact(tex, dims, sizes, norm, addr, filt, co[s], border)
            if kind == "nearest":
                assert np.array_equal(out[s].view(np.uint32), np.asarray(val, np.float32).view(np.uint32))
            else:
                for c in range(4):
                    exp = em.round_f32(val[c])
                    if out[s, c] != exp:
                        assert em.is_tie(val[c]) and abs(Fraction(float(out[s, c])) - val[c]) <= \
                            abs(Fraction(float(exp)) - val[c]), (norm, addr, filt, co[s], c)
