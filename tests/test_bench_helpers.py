"""bench.py's measurement bookkeeping (CPU): the distinct-texel count of a
2D map, used for the algorithmic bytes of non-separable maps, equals the
product of the per-axis counts on separable maps."""
import numpy as np
import pytest

import bench
from paper_conf_sc_kimdjjl15_b200 import synth


@pytest.mark.parametrize("mode", ["repeat", "mirrored", "clamp_to_edge"])
@pytest.mark.parametrize("n", [64, 300])
def test_distinct_texels_2d_matches_separable_count(mode, n):
    maps = [synth.affine_translate_2d(n, n), synth.affine_translate_2d(n, n, dx=0.5, dy=0.0)]
    if mode == "clamp_to_edge":  # shifted so the clamped edges lose texels
        maps = [synth.affine_stencil_3d(n), synth.affine_stencil_3d(n, delta=(7.3, -5.6, 0.0))]
    for A in maps:
        cols = bench._axis_taps(A[0], A[3], n, n, mode).size
        rows = bench._axis_taps(A[5], A[7], n, n, mode).size
        assert bench._distinct_texels_2d(A, n, n, mode, chunk=37) == cols * rows


def test_distinct_texels_2d_rotation_bounds():
    n = 256
    A = synth.affine_rotate_2d(n, n, 30.0)
    for mode in ("repeat", "mirrored"):
        k = bench._distinct_texels_2d(A, n, n, mode)
        # a unit-scale rotation reads at most every texel and at least the
        # inscribed disc's worth of them
        assert np.pi / 4 * n * n * 0.9 < k <= n * n
