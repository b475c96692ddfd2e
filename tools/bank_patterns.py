"""Warp address patterns of the rotated-map kernel's tap loads (lanes = 32
consecutive output x at one y; 20-degree rotation; box pitch P words) for
tools/bank_probe.cu.   python tools/bank_patterns.py P out.bin"""
import sys

import numpy as np

P = int(sys.argv[1])
th = np.deg2rad(20)
c, s = np.cos(th), np.sin(th)
rng = np.random.default_rng(0)
pats = []
for _ in range(500):
    x0, y0 = rng.uniform(0, 512, 2)
    l = np.arange(32)
    u = c * (x0 + l) - s * y0
    v = s * (x0 + l) + c * y0
    i = np.floor(u).astype(int)
    j = np.floor(v).astype(int)
    i -= i.min()
    j -= j.min()
    for di, dj in ((0, 0), (1, 0), (0, 1), (1, 1)):
        pats.append((j + dj) * P + i + di)
np.array(pats, np.int32).tofile(sys.argv[2])
