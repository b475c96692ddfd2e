"""Pin P5: brute-force enumeration on tiny images against an exact-rational model.

For every valid sampler (16), tiny 1D/2D/3D images and every coordinate on a
dyadic lattice plus special values, the C oracle must equal tests/exact_model.py:
bit-exact for NEAREST, and the correctly rounded exact blend for LINEAR (at an
exact tie either neighbour, reading A10/O6).
"""
from fractions import Fraction

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import synth
from tests import exact_model as em

SAMPLERS = [(norm, a, f) for norm in (0, 1) for a in range(0x1130, 0x1135)
            for f in (0x1140, 0x1141) if norm or a <= 0x1132]
SHAPES = [(1, (1, 1, 1)), (1, (5, 1, 1)), (2, (1, 1, 1)), (2, (2, 3, 1)), (2, (4, 4, 1)),
          (2, (5, 7, 1)), (3, (2, 2, 2)), (3, (3, 4, 5))]


def _coords(dims, n_axes, norm, g):
    sp = synth.special_floats()
    if norm:
        lat = synth.coord_lattice(-2.0, 3.0, 1 / 32)
    else:
        lat = synth.coord_lattice(-2.0, max(n_axes) + 2.0, 1 / 16)
    pts = []
    if dims == 1:
        vals = np.concatenate([lat, sp])
        pts = vals[:, None]
    else:
        # lattice along each axis crossed with a random partner + specials per axis
        for d in range(dims):
            vals = np.concatenate([lat, sp])
            c = g.uniform(-0.5, 1.5 if norm else n_axes[1] + 1, (vals.size, dims)).astype(np.float32)
            c[:, d] = vals
            pts.append(c)
        pts = np.concatenate(pts)
        pts = np.concatenate([pts, g.uniform(-1.5, 2.5, (400, dims)).astype(np.float32) *
                              (1 if norm else np.float32(max(n_axes)))])
    if dims == 3:
        pts = np.concatenate([pts, np.zeros((pts.shape[0], 1), np.float32)], 1)
    return np.ascontiguousarray(pts, dtype=np.float32)


@pytest.mark.parametrize("dims,sizes", SHAPES)
def test_p5_oracle_equals_exact_model(orc, dims, sizes):
    g = synth.rng(100 + sum(sizes) * dims)
    W, H, D = sizes
    data = synth.image_codes(g, orc.RGBA, orc.FLOAT, W, H, D)
    img = orc.Image(data, W, H, D, dims=dims, order=orc.RGBA, type=orc.FLOAT)
    border = [0.0, 0.0, 0.0, 0.0]
    n_checked = 0
    for norm, addr, filt in SAMPLERS:
        co = _coords(dims, sizes, norm, g)
        out = orc.read_samples(img, bool(norm), addr, filt, orc.RT_F, co)
        for s in range(co.shape[0]):
            val, kind = em.sample_exact(data, dims, sizes, norm, addr, filt, co[s], border)
            if kind == "nearest":
                assert np.array_equal(out[s].view(np.uint32), np.asarray(val, np.float32).view(np.uint32)), \
                    (norm, addr, filt, co[s])
            elif kind == "nan":
                assert np.all(np.isnan(out[s])), (norm, addr, filt, co[s])
            else:
                for c in range(4):
                    exp = em.round_f32(val[c])
                    if out[s, c] != exp:
                        assert em.is_tie(val[c]) and abs(Fraction(float(out[s, c])) - val[c]) <= \
                            abs(Fraction(float(exp)) - val[c]), (norm, addr, filt, co[s], c)
            n_checked += 1
    assert n_checked > 1000


def test_p5_exact_model_self_check():
    """The exact model itself reproduces two P1 hand examples."""
    tex = np.zeros((1, 1, 4, 4), np.float32)
    tex[0, 0, :, 0] = [10, 20, 30, 40]
    val, _ = em.sample_exact(tex, 1, (4, 1, 1), 1, em.REPEAT, em.LINEAR, [0.9375], [0, 0, 0, 1])
    assert val[0] == Fraction(65, 2)
    val, _ = em.sample_exact(tex, 1, (4, 1, 1), 0, em.CLAMP, em.LINEAR, [0.25], [0, 0, 0, 1])
    assert val[0] == Fraction(15, 2)
