"""Shared helpers for the -m gpu parity tests (CUDA path through the C-ABI vs the oracle)."""
import ctypes

import numpy as np

from paper_conf_sc_kimdjjl15_b200 import cl, synth

RT_DTYPE = {cl.B2CL_RTYPE_FLOAT: np.float32, cl.B2CL_RTYPE_INT: np.int32,
            cl.B2CL_RTYPE_UINT: np.uint32}
INT_TYPES = {cl.CL_SIGNED_INT8: cl.B2CL_RTYPE_INT, cl.CL_SIGNED_INT16: cl.B2CL_RTYPE_INT,
             cl.CL_SIGNED_INT32: cl.B2CL_RTYPE_INT, cl.CL_UNSIGNED_INT8: cl.B2CL_RTYPE_UINT,
             cl.CL_UNSIGNED_INT16: cl.B2CL_RTYPE_UINT, cl.CL_UNSIGNED_INT32: cl.B2CL_RTYPE_UINT}
VALID_SAMPLERS = [(norm, a, f) for norm in (0, 1) for a in range(0x1130, 0x1135)
                  for f in (0x1140, 0x1141) if norm or a <= 0x1132]


def rtype_of(type_):
    return INT_TYPES.get(type_, cl.B2CL_RTYPE_FLOAT)


def coord_stride(dims):
    return {1: 1, 2: 2, 3: 4}[dims]


def make_images(S, orc, order, type_, W, H=1, D=1, dims=2, seed=0, signed=False):
    """The same seeded texel codes as a GPU image and an oracle image."""
    g = synth.rng(1000 + seed)
    codes = synth.image_codes(g, order, type_, W, H, D, signed=signed)
    img = S.image(order, type_, W, H if dims > 1 else 0, D if dims > 2 else 0, host=codes)
    oimg = orc.Image(codes.copy(), W, H, D, dims=dims, order=order, type=type_)
    return img, oimg, codes


def gpu_read_samples(S, img, smp, rtype, coords, int_coords=False):
    coords = np.ascontiguousarray(coords)
    n = coords.shape[0]
    cbuf = S.buffer(max(coords.nbytes, 16), coords if n else None)
    obuf = S.buffer(max(16 * n, 16))
    cl.check(cl.lib().b2clEnqueueReadImageSamples(
        S.queue, img, smp, rtype, cl.B2CL_COORD_INT if int_coords else cl.B2CL_COORD_FLOAT,
        cbuf, 0, n, obuf, 0, 0, None, None), "b2clEnqueueReadImageSamples")
    out = S.read(obuf, 16 * n, RT_DTYPE[rtype]).reshape(n, 4) if n else np.zeros((0, 4))
    S.release(cbuf, obuf)
    return out


def gpu_read_grid(S, img, smp, rtype, affine, out_dims, outc):
    w, h, d = out_dims
    nbytes = w * h * d * outc * 4
    obuf = S.buffer(max(nbytes, 16))
    A = (ctypes.c_float * 12)(*[float(x) for x in np.asarray(affine, np.float32)])
    cl.check(cl.lib().b2clEnqueueReadImageGrid(S.queue, img, smp, rtype, A, cl.sz3(out_dims), outc,
                                               obuf, 0, 0, None, None), "b2clEnqueueReadImageGrid")
    out = S.read(obuf, nbytes, RT_DTYPE[rtype]).reshape(d, h, w, outc)
    S.release(obuf)
    return out


def assert_parity(got, exp, linear, what=""):
    """Bit-exact unless LINEAR; LINEAR: |g-o| <= 4 ulp(o) or <= 1e-6, NaN iff NaN
    (north_star tolerance; reading A10)."""
    got = np.asarray(got)
    exp = np.asarray(exp)
    assert got.shape == exp.shape, (got.shape, exp.shape)
    if not linear or got.dtype != np.float32:
        bad = got.view(np.uint32) != exp.view(np.uint32)
        if bad.any():
            idx = np.argwhere(bad)[:5]
            raise AssertionError(f"{what}: {bad.sum()} bit mismatches, first at {idx.tolist()}: "
                                 f"got {got[tuple(idx[0])]} exp {exp[tuple(idx[0])]}")
        return
    gn, en = np.isnan(got), np.isnan(exp)
    assert np.array_equal(gn, en), f"{what}: NaN pattern differs ({(gn != en).sum()})"
    g, e = got[~en].astype(np.float64), exp[~en].astype(np.float64)
    tol = np.maximum(4.0 * np.spacing(np.abs(exp[~en])).astype(np.float64), 1e-6)
    err = np.abs(g - e)
    bad = err > tol
    assert not bad.any(), (f"{what}: {bad.sum()} of {bad.size} beyond 4 ulp / 1e-6; "
                           f"max err {err.max()}")
