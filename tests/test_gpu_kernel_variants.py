"""Every grid-kernel family against the oracle, not only the default choice.

The library picks one kernel per hot configuration (sample.cu:
launch_sample); B2CL_GRID_KERNEL forces a family for the whole process
(g = one thread per sample, s = separable, w = walk, 4 = the 3D walk of
16-byte rows, t = the staged 2D tile, b = the TMA footprint box for every
2D RGBA32F LINEAR map, separable ones included).  Each forced run repeats the grid-mode
parity cases and the full-size config-2/3 checks in a subprocess, so the
kernels the default no longer selects stay parity-green.
"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.gpu
@pytest.mark.parametrize("family", ["g", "s", "w", "4", "t", "b"])
def test_forced_grid_kernel_family(family):
    env = dict(os.environ, B2CL_GRID_KERNEL=family)
    r = subprocess.run(
        [sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
         os.path.join(ROOT, "tests", "test_gpu_sampling.py"), "-k", "grid_mode or config2 or config3"],
        cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0, r.stdout[-4000:] + r.stderr[-2000:]
