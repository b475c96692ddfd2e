"""Probe the config-3 TMA kernel on assorted shapes, one subprocess each:
    python tools/vol_probe.py            (prints OK / FAIL per case)"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, numpy as np
sys.path.insert(0, ROOT)
import oracle as orc
from paper_conf_sc_kimdjjl15_b200 import cl, synth
from tests.gpu_helpers import gpu_read_grid, make_images, assert_parity
W, H, D, sh, ow = map(int, sys.argv[1:6])
S = cl.Session(0)
img, oimg, _ = make_images(S, orc, cl.CL_R, cl.CL_FLOAT, W, H, D, 3, seed=5)
smp = S.sampler(True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
A = synth.affine_stencil_3d(W)
A[3] = (0.5 + 0.3 + sh) / W
A[5], A[7] = 1.0 / H, 1.1 / H
A[10], A[11] = 1.0 / D, 0.7 / D
got = gpu_read_grid(S, img, smp, cl.B2CL_RTYPE_FLOAT, A, (ow, H, D), 1)
exp = orc.read_grid(oimg, True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR, orc.RT_F, A, (ow, H, D), 1)
assert_parity(got, exp, True, "probe")
'''.replace("ROOT", repr(ROOT))
CASES = [(260, 4, 19, 0, 260), (260, 4, 19, 1, 258), (260, 4, 19, 1, 260), (260, 4, 19, 0, 258),
         (264, 4, 19, 1, 262), (388, 4, 19, 1, 386), (260, 20, 19, 1, 258), (300, 7, 37, 0, 300),
         (260, 4, 19, 4, 250), (1030, 3, 5, 0, 1030), (512, 16, 16, 1, 510), (512, 16, 16, 3, 509)]
for c in CASES:
    r = subprocess.run([sys.executable, "-c", CHILD, *map(str, c)], capture_output=True, text=True, timeout=300)
    print(c, "OK" if r.returncode == 0 else "FAIL " + (r.stderr.strip().splitlines() or [""])[-1][:150], flush=True)
