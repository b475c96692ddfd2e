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


# reading A10 (north_star): LINEAR passes iff |g - o| <= 4 ulp(o), where the
# 1e-6 absolute floor applies only NEAR ZERO, |o| < 2^-10.  For mixed-sign
# data the fp32 blend's error scales with the condition sum |w|*|T|, not with
# |o| (cancellation), so callers with signed texels pass
# `scale` = the oracle's LINEAR read of the |T| image (same sampler and
# coordinates): then ulps are counted against max(|o|, scale).
NEAR_ZERO = 2.0 ** -10
ULP_BOUND = 4.0
WORST = {}   # what -> worst LINEAR error in ulps (printed in the session summary)


def abs_codes(codes, type_):
    """|T| per texel for the condition scale: SNORM's most negative code maps to
    -1.0 like its neighbour, so its magnitude is the largest positive code."""
    c = np.asarray(codes)
    if c.dtype in (np.int8, np.int16):
        top = np.iinfo(c.dtype).max
        return np.where(c == np.iinfo(c.dtype).min, top, np.abs(c)).astype(c.dtype)
    return np.abs(c)


_SIGNED_TYPES = {0x10D0: np.int8, 0x10D1: np.int16, 0x10D7: np.int8, 0x10D8: np.int16,
                 0x10DD: np.float16, 0x10DE: np.float32}  # SNORM, SINT (CUDA normalized reads), HALF, FLOAT


def abs_image(orc, oimg):
    """The oracle image of |T| (same layout, same format), or None for formats
    whose texels are never negative -- its LINEAR read is the condition scale
    sum |w|*|T| of reading A10.  Bytes outside the texels are copied unchanged."""
    dt = _SIGNED_TYPES.get(oimg.type)
    if dt is None:
        return None
    data = oimg.data.copy()
    n = data.size // np.dtype(dt).itemsize
    v = data[:n * np.dtype(dt).itemsize].view(dt)
    v[...] = abs_codes(v, oimg.type)
    return orc.Image(data, oimg.width, oimg.height, oimg.depth, dims=oimg.dims, order=oimg.order,
                     type=oimg.type, row_pitch=oimg.row_pitch, slice_pitch=oimg.slice_pitch,
                     arrayed=oimg.arrayed)


def parity_read(got, exp, linear, what, orc, oimg, read):
    """assert_parity for a read of oracle image `oimg`; `read(img)` repeats the
    oracle read on another image (the |T| image gives the LINEAR scale)."""
    scale = None
    if linear:
        a = abs_image(orc, oimg)
        if a is not None:
            scale = read(a)
    return assert_parity(got, exp, linear, what, scale=scale)


def assert_parity(got, exp, linear, what="", scale=None):
    """Bit-exact unless LINEAR; LINEAR: <= 4 ulp (reading A10, above), NaN iff NaN.
    Returns the worst LINEAR error in ulps (0 for exact comparisons)."""
    got = np.asarray(got)
    exp = np.asarray(exp)
    assert got.shape == exp.shape, (got.shape, exp.shape)
    if not linear or got.dtype != np.float32:
        bad = got.view(np.uint32) != exp.view(np.uint32)
        if bad.any():
            idx = np.argwhere(bad)[:5]
            raise AssertionError(f"{what}: {bad.sum()} bit mismatches, first at {idx.tolist()}: "
                                 f"got {got[tuple(idx[0])]} exp {exp[tuple(idx[0])]}")
        return 0.0
    gn, en = np.isnan(got), np.isnan(exp)
    assert np.array_equal(gn, en), f"{what}: NaN pattern differs ({(gn != en).sum()})"
    keep = ~en
    g, e = got[keep].astype(np.float64), exp[keep].astype(np.float64)
    mag = np.abs(exp[keep])
    if scale is not None:
        mag = np.maximum(mag, np.abs(np.asarray(scale, np.float32)[keep]))
    err = np.abs(g - e)
    if err.size == 0:
        return 0.0
    ulp = np.spacing(mag).astype(np.float64)
    near = mag < NEAR_ZERO
    bad = np.where(near, err > 1e-6, err > ULP_BOUND * ulp)
    far = ~near
    worst = float((err[far] / ulp[far]).max()) if far.any() else 0.0
    WORST[what] = max(WORST.get(what, 0.0), worst)
    if bad.any():
        k = int(np.argmax(np.where(bad, err / np.where(near, 1e-6, ULP_BOUND * ulp), 0)))
        raise AssertionError(f"{what}: {bad.sum()} of {bad.size} beyond 4 ulp (1e-6 below 2^-10); "
                             f"worst at |o|={mag[k]:.3g}: err {err[k]:.3g} = {err[k] / ulp[k]:.2f} ulp")
    return worst
