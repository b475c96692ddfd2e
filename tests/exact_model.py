"""An independent, exact-rational Python model of [CL1.2 §8.2] sampling (pin P5).

Written separately from oracle/oracle.c (no shared code): numpy float32 scalar
operations for the address path (each one IEEE RN op, as reading A2 requires)
and fractions.Fraction for the LINEAR blend, so the blend is the exact real
value rounded once to fp32.  Used only on tiny images.
"""
from fractions import Fraction

import numpy as np

f32 = np.float32
I32_MAX, I32_MIN = 2 ** 31 - 1, -2 ** 31
NONE, CTE, CLAMP, REPEAT, MIRROR = range(0x1130, 0x1135)
NEAREST, LINEAR = 0x1140, 0x1141


def ifloor(x):
    if np.isnan(x):
        return 0
    f = np.floor(x)
    if f >= 2.0 ** 31:
        return I32_MAX
    if f < -2.0 ** 31:
        return I32_MIN
    return int(f)


def _am(mode, i, n):
    if mode == CTE:
        return min(max(i, 0), n - 1)
    if mode == CLAMP:
        return min(max(i, -1), n)
    return i


def axis(s, n, norm, mode, filt):
    """Returns (i0, i1, a) with a as float32 (i1/a unused for NEAREST)."""
    s = f32(s)
    fn = f32(n)
    with np.errstate(invalid="ignore", over="ignore"):
        if mode == REPEAT:
            u = f32(f32(s - np.floor(s)) * fn)
            if filt == NEAREST:
                i = ifloor(u)
                return (i - n if i > n - 1 else i), None, None
            t = f32(u - f32(0.5))
            i0 = ifloor(t)
            i1 = i0 + 1
            i0 = i0 + n if i0 < 0 else i0
            i1 = i1 - n if i1 > n - 1 else i1
            return i0, i1, f32(t - np.floor(t))
        if mode == MIRROR:
            sp = f32(f32(2.0) * np.rint(f32(f32(0.5) * s)))
            sp = np.abs(f32(s - sp))
            u = f32(sp * fn)
            if filt == NEAREST:
                return min(ifloor(u), n - 1), None, None
            t = f32(u - f32(0.5))
            i0 = ifloor(t)
            return max(i0, 0), min(i0 + 1, n - 1), f32(t - np.floor(t))
        u = f32(s * fn) if norm else s
        if filt == NEAREST:
            return _am(mode, ifloor(u), n), None, None
        t = f32(u - f32(0.5))
        b = ifloor(t)
        return _am(mode, b, n), _am(mode, b + 1, n), f32(t - np.floor(t))


def round_f32(q: Fraction) -> np.float32:
    """Correctly rounded (half-even) fp32 of an exact rational."""
    c = f32(float(q))
    best = None
    for cand in (np.nextafter(c, f32(-np.inf)), c, np.nextafter(c, f32(np.inf))):
        if not np.isfinite(cand):
            continue
        d = abs(Fraction(float(cand)) - q)
        if best is None or d < best[0] or (d == best[0] and
                                            (int(f32(cand).view(np.uint32)) & 1) == 0):
            best = (d, f32(cand))
    return best[1]


def is_tie(q: Fraction) -> bool:
    c = f32(float(q))
    lo, hi = (np.nextafter(c, f32(-np.inf)), c) if Fraction(float(c)) > q else \
        (c, np.nextafter(c, f32(np.inf)))
    return Fraction(float(lo)) + Fraction(float(hi)) == 2 * q


def sample_exact(texels, dims, sizes, norm, mode, filt, coord, border):
    """texels: float32 array (D, H, W, 4) of already-converted, channel-mapped
    texels; border: 4 floats.  Returns (values_as_Fraction_or_float32[4], kind)."""
    W, H, D = sizes

    def get(i, j, k):
        if 0 <= i < W and 0 <= j < H and 0 <= k < D:
            return texels[k, j, i]
        return np.asarray(border, np.float32)

    ns = [W, H, D][:dims]
    if filt == NEAREST:
        ix = [axis(coord[d], ns[d], norm, mode, NEAREST)[0] for d in range(dims)] + [0] * (3 - dims)
        return get(*ix), "nearest"
    ax = [axis(coord[d], ns[d], norm, mode, LINEAR) for d in range(dims)]
    if any(np.isnan(a[2]) for a in ax):
        return None, "nan"
    while len(ax) < 3:
        ax.append((0, 0, f32(0.0)))
    acc = [Fraction(0)] * 4
    for kk in range(2 if dims > 2 else 1):
        for jj in range(2 if dims > 1 else 1):
            for ii in range(2):
                w = Fraction(1)
                for d, sel in zip(range(dims), (ii, jj, kk)):
                    a = Fraction(float(ax[d][2]))
                    w *= a if sel else (1 - a)
                t = get(ax[0][ii], ax[1][jj], ax[2][kk])
                for c in range(4):
                    acc[c] += w * Fraction(float(t[c]))
    return acc, "linear"
