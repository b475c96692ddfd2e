"""Seeded synthetic inputs shared by the tests, the bench and the oracle runs.

This module holds NO arithmetic of the method: it only draws random texel
codes, coordinates and copy boxes, and writes down the affine coordinate maps
of the benchmark workloads ("input recipe").  Both the CUDA path
and the oracle receive exactly the arrays produced here.

Recipe: numpy.random.default_rng(SEED), SEED = 20151115.
Float images are U[0,1) (a second, signed dataset uses U[-1,1)); half images
are U[0,1) rounded by numpy to float16; integer and normalized-integer images
are uniform over their full code range.
"""
from __future__ import annotations

import numpy as np

SEED = 20151115

# Khronos values (public cl.h); the product binding has its own copy.
_CHANNELS = {0x10B0: 1, 0x10B1: 1, 0x10B2: 2, 0x10B3: 2, 0x10B5: 4, 0x10B6: 4, 0x10B7: 4,
             0x10B8: 1, 0x10B9: 1, 0x10B4: 1, 0x10BC: 1}  # CL_RGB / CL_RGBx: one packed word
_TYPE_DTYPE = {0x10D0: np.int8, 0x10D1: np.int16, 0x10D2: np.uint8, 0x10D3: np.uint16,
               0x10D7: np.int8, 0x10D8: np.int16, 0x10D9: np.int32,
               0x10DA: np.uint8, 0x10DB: np.uint16, 0x10DC: np.uint32,
               0x10DD: np.float16, 0x10DE: np.float32,
               0x10D4: np.uint16, 0x10D5: np.uint16, 0x10D6: np.uint32}  # packed words


def rng(offset: int = 0) -> np.random.Generator:
    return np.random.default_rng(SEED + offset)


def texel_dtype(type_: int):
    return _TYPE_DTYPE[type_]


def image_codes(g: np.random.Generator, order: int, type_: int, width: int, height: int = 1,
                depth: int = 1, signed: bool = False) -> np.ndarray:
    """Tightly packed texel codes, shape (depth, height, width, channels)."""
    nc = _CHANNELS[order]
    dt = _TYPE_DTYPE[type_]
    shape = (depth, height, width, nc)
    if dt == np.float32:
        lo = -1.0 if signed else 0.0
        return g.uniform(lo, 1.0, size=shape).astype(np.float32)
    if dt == np.float16:
        lo = -1.0 if signed else 0.0
        return g.uniform(lo, 1.0, size=shape).astype(np.float16)
    nbytes = int(np.prod(shape)) * np.dtype(dt).itemsize
    return g.integers(0, 256, size=nbytes, dtype=np.uint8).view(dt).reshape(shape)


def image_rows(order: int, type_: int, width: int, rows, key: int = 5,
               signed: bool = False) -> np.ndarray:
    """Rows of a large virtual 2D image whose row j is drawn from its own
    generator default_rng([SEED, key, j]) -- so any rank can materialise any
    band (or shard) of a global image without generating the rest.
    Returns shape (1, len(rows), width, channels)."""
    out = [image_codes(np.random.default_rng([SEED, key, int(j)]), order, type_, width,
                       signed=signed)[0, 0] for j in rows]
    return np.stack(out)[None]


def special_floats() -> np.ndarray:
    """Coordinates that stress the address path."""
    f32 = np.float32
    vals = [0.0, -0.0, -1e-9, 1e-9, 1.0, -1.0, 0.5, -0.5, 1.5, 2.0, 3.0, 0.25, 0.75,
            np.nextafter(f32(1.0), f32(0.0)), np.nextafter(f32(0.0), f32(1.0)),
            -np.nextafter(f32(0.0), f32(1.0)), np.nextafter(f32(1.0), f32(2.0)),
            1e30, -1e30, 3e9, -3e9, np.inf, -np.inf, np.nan, 65536.0, 1e-38]
    return np.array(vals, dtype=np.float32)


def coord_lattice(lo: float, hi: float, step: float) -> np.ndarray:
    """lo, lo+step, ... < hi as float32 (dyadic steps are exact)."""
    n = int(np.floor((hi - lo) / step))
    return (np.float32(lo) + np.arange(n, dtype=np.float64) * step).astype(np.float32)


def random_coords(g: np.random.Generator, n: int, dims: int, lo: float, hi: float) -> np.ndarray:
    c = g.uniform(lo, hi, size=(n, dims)).astype(np.float32)
    if dims == 3:  # float4 per sample, w ignored (reading A20)
        c = np.concatenate([c, np.zeros((n, 1), np.float32)], axis=1)
    return c


# ---- affine coordinate maps of the benchmark workloads (coord = A.(x,y,z,1)) ----

def affine_translate_2d(width: int, height: int, dx: float = 0.3, dy: float = 0.7,
                        half_period: bool = True) -> np.ndarray:
    """C2 map (A): normalized s = (x + dx [+ W/2]) / W, t = (y + dy [+ H/2]) / H.

    The half-period shift puts the REPEAT / MIRRORED seam through the middle
    of the output so seam tiles are exercised."""
    ox = dx + (width / 2 if half_period else 0.0)
    oy = dy + (height / 2 if half_period else 0.0)
    A = np.zeros(12, dtype=np.float32)
    A[0] = 1.0 / width
    A[3] = ox / width
    A[5] = 1.0 / height
    A[7] = oy / height
    return A


def affine_rotate_2d(width: int, height: int, degrees: float = 30.0,
                     scale: float = 1.0) -> np.ndarray:
    """C2 map (B): rotation about the image centre at unit scale, normalized.

    Output pixel (x,y) maps to s,t covering about [-0.2, 1.2]^2 (wraps)."""
    th = np.deg2rad(degrees)
    c, s = np.cos(th) * scale, np.sin(th) * scale
    cx, cy = width / 2.0, height / 2.0
    A = np.zeros(12, dtype=np.float32)
    # s = (c*(x+0.5-cx) - s*(y+0.5-cy) + cx) / W
    A[0] = c / width
    A[1] = -s / width
    A[3] = (c * (0.5 - cx) - s * (0.5 - cy) + cx) / width
    A[4] = s / height
    A[5] = c / height
    A[7] = (s * (0.5 - cx) + c * (0.5 - cy) + cy) / height
    return A


def affine_stencil_3d(n: int, delta=(0.3, 0.6, 0.2)) -> np.ndarray:
    """C3 map (A): s = (x + 0.5 + dx)/n, t = (y + 0.5 + dy)/n, r = (z + 0.5 + dz)/n."""
    A = np.zeros(12, dtype=np.float32)
    for k in range(3):
        A[4 * k + k] = 1.0 / n
        A[4 * k + 3] = (0.5 + delta[k]) / n
    return A


def affine_rotate_3d(n: int, degrees: float = 20.0) -> np.ndarray:
    """C3 map (B), volume-render shaped: rotation about the z axis through the
    volume centre, normalized coordinates (non-separable)."""
    th = np.deg2rad(degrees)
    c, s = np.cos(th), np.sin(th)
    h = n / 2.0
    A = np.zeros(12, dtype=np.float32)
    A[0], A[1], A[3] = c / n, -s / n, (c * (0.5 - h) - s * (0.5 - h) + h) / n
    A[4], A[5], A[7] = s / n, c / n, (s * (0.5 - h) + c * (0.5 - h) + h) / n
    A[10], A[11] = 1.0 / n, 0.5 / n
    return A


def affine_unnorm_2d(step: float, origin: float) -> np.ndarray:
    """C1 brute-force map: unnormalized (u, v) = (origin + step*x, origin + step*y)."""
    A = np.zeros(12, dtype=np.float32)
    A[0] = step
    A[3] = origin
    A[5] = step
    A[7] = origin
    return A


def random_rect(g: np.random.Generator, max_region=(64, 8, 4), max_pad=(40, 3, 2)):
    """A random pitched rect-copy box: (src_origin, dst_origin, region, srp, ssp, drp, dsp)."""
    region = [int(g.integers(1, m + 1)) for m in max_region]
    so = [int(g.integers(0, p + 1)) for p in max_pad]
    do = [int(g.integers(0, p + 1)) for p in max_pad]
    srp = region[0] + so[0] + int(g.integers(0, 17))
    drp = region[0] + do[0] + int(g.integers(0, 17))
    ssp = srp * (region[1] + so[1] + int(g.integers(0, 3)))
    dsp = drp * (region[1] + do[1] + int(g.integers(0, 3)))
    return so, do, region, srp, ssp, drp, dsp
