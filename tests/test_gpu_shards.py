"""Image shards: a band of output rows read from a shard that
stores only the texel rows the band needs must be BIT-IDENTICAL to the same
rows read from the whole image -- sharding changes no value -- for every grid
kernel (separable, walk, general) and for wrapping and non-wrapping modes.
The rows a band needs are computed with tests/exact_model.py (independent of
the product), and stored as the minimal circular interval."""
import ctypes

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth
from tests import exact_model as em
from tests.gpu_helpers import assert_parity, gpu_read_grid

pytestmark = pytest.mark.gpu

RGBA, R, RG = cl.CL_RGBA, cl.CL_R, cl.CL_RG
F32, F16 = cl.CL_FLOAT, cl.CL_HALF_FLOAT


def _needed(A, out_region, origin, sizes, dims, norm, addr, filt):
    """Set of outer-axis texel indices (rows in 2D, slices in 3D) touched."""
    W, H, D = sizes
    k = dims - 1  # outer axis
    n = [W, H, D][k]
    need = set()
    xs = range(origin[0], origin[0] + out_region[0])
    ys = range(origin[1], origin[1] + out_region[1])
    zs = range(origin[2], origin[2] + out_region[2])
    f32 = np.float32
    for z in zs:
        for y in ys:
            for x in xs:
                row = A[4 * k: 4 * k + 4].astype(np.float32)
                v = f32(f32(row[0] * f32(x)) + f32(row[1] * f32(y)))
                v = f32(v + f32(row[2] * f32(z)))
                v = f32(v + row[3])
                i0, i1, _ = em.axis(v, n, norm, addr, filt)
                for i in (i0, i1):
                    if i is not None and 0 <= i < n:
                        need.add(int(i))
    return need, n


def _circular_interval(need, n):
    """Smallest (begin, count) with {(begin + s) mod n : s < count} covering `need`."""
    rows = sorted(need)
    if not rows:
        return 0, 1
    gaps = [(rows[(i + 1) % len(rows)] - rows[i]) % n for i in range(len(rows))]
    i = int(np.argmax(gaps)) if len(rows) > 1 else 0
    begin = rows[(i + 1) % len(rows)]
    count = (rows[i] - begin) % n + 1
    return begin, count


def _read_region(S, img, smp, A, origin, region, outc):
    w, h, d = region
    nbytes = w * h * d * outc * 4
    buf = S.buffer(max(nbytes, 16))
    Af = (ctypes.c_float * 12)(*[float(v) for v in np.asarray(A, np.float32)])
    cl.check(cl.lib().b2clEnqueueReadImageGridRegion(S.queue, img, smp, 0, Af, cl.sz3(origin),
                                                     cl.sz3(region), outc, buf, 0, 0, None, None))
    out = S.read(buf, nbytes, np.float32).reshape(d, h, w, outc)
    S.release(buf)
    return out


CASES = [
    # dims, order, type, sizes, (norm, addr, filt), map, outc
    (2, RGBA, F32, (64, 48, 1), (1, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR), "translate", 4),
    (2, RGBA, F32, (64, 48, 1), (1, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR), "translate", 4),
    (2, RGBA, F32, (40, 36, 1), (1, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR), "rotate", 4),
    (2, RG, F16, (33, 30, 1), (1, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_LINEAR), "translate", 2),
    (2, RGBA, cl.CL_UNORM_INT8, (50, 41, 1), (0, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_NEAREST), "unnorm", 4),
    (3, R, F32, (24, 20, 18), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "stencil", 1),
    (3, R, F32, (24, 24, 16), (1, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR), "rotate3d", 1),
]


def _affine(kind, W, H, D):
    if kind == "translate":
        return synth.affine_translate_2d(W, H)
    if kind == "rotate":
        return synth.affine_rotate_2d(W, H, 30.0)
    if kind == "unnorm":
        return synth.affine_unnorm_2d(0.75, -2.0)
    if kind == "stencil":
        A = synth.affine_stencil_3d(W)
        A[5], A[7] = 1.0 / H, 1.1 / H
        A[10], A[11] = 1.0 / D, 0.7 / D
        return A
    return synth.affine_rotate_3d(W, 20.0)


@pytest.mark.parametrize("case", CASES)
@pytest.mark.parametrize("G", [2, 3])
def test_sharded_read_is_bit_identical(sess, case, G):
    dims, order, type_, sizes, (norm, addr, filt), kind, outc = case
    W, H, D = sizes
    g = synth.rng(70 + W + G)
    codes = synth.image_codes(g, order, type_, W, H, D)  # (D, H, W, c)
    full = sess.image(order, type_, W, H, D if dims == 3 else 0, host=codes)
    smp = sess.sampler(norm, addr, filt)
    A = _affine(kind, W, H, D)
    out_dims = (W, H, D if dims == 3 else 1)
    ref = gpu_read_grid(sess, full, smp, 0, A, out_dims, outc)
    outer = out_dims[dims - 1]
    for r0, r1 in [(b * outer // G, (b + 1) * outer // G) for b in range(G)]:
        origin = [0, 0, 0]
        region = list(out_dims)
        origin[dims - 1], region[dims - 1] = r0, r1 - r0
        need, n = _needed(A, region, origin, sizes, dims, norm, addr, filt)
        begin, count = _circular_interval(need, n)    # the band: exactly the rows needed
        halo = 1 if count + 2 <= n else 0              # plus one spare row each side
        idx = [(begin - halo + s) % n for s in range(count + 2 * halo)]
        host = codes[:, idx] if dims == 2 else codes[idx]
        shard = sess.image_shard(order, type_, W, H, D if dims == 3 else 0, begin, count, halo,
                                 host=host)
        got = _read_region(sess, shard, smp, A, origin, region, outc)
        if dims == 2:
            exp = ref[:, r0:r1]
        else:
            exp = ref[r0:r1]
        assert np.array_equal(got.view(np.uint32), exp.view(np.uint32)), (kind, G, r0, r1)
        sess.release(shard)
    sess.release(full)
    cl.lib().clReleaseSampler(smp)


def test_region_origin_equals_full_grid_rows(sess):
    """A region of the output grid equals the same sub-box of the whole grid."""
    W, H = 70, 50
    codes = synth.image_codes(synth.rng(71), RGBA, F32, W, H)
    img = sess.image(RGBA, F32, W, H, host=codes)
    for addr, kind in ((cl.CL_ADDRESS_REPEAT, "rotate"), (cl.CL_ADDRESS_MIRRORED_REPEAT, "translate")):
        smp = sess.sampler(True, addr, cl.CL_FILTER_LINEAR)
        A = _affine(kind, W, H, 1)
        ref = gpu_read_grid(sess, img, smp, 0, A, (W, H, 1), 4)
        got = _read_region(sess, img, smp, A, (13, 7, 0), (41, 29, 1), 4)
        assert np.array_equal(got.view(np.uint32), ref[:, 7:36, 13:54].view(np.uint32))
        cl.lib().clReleaseSampler(smp)
    sess.release(img)


def test_shard_argument_errors(sess):
    L = cl.lib()
    fmt = cl.ImageFormat(RGBA, F32)
    err = ctypes.c_int32()
    for dims, begin, count, halo in ((2, 0, 0, 0), (2, 10, 8, 0), (2, 0, 9, 1), (1, 0, 2, 0)):
        itype = cl.CL_MEM_OBJECT_IMAGE2D if dims == 2 else cl.CL_MEM_OBJECT_IMAGE1D
        desc = cl.ImageDesc(itype, 16, 10 if dims == 2 else 0, 0, 0, 0, 0, 0, 0, None)
        m = L.b2clCreateImageShard(sess.ctx, 1, ctypes.byref(fmt), ctypes.byref(desc), begin, count,
                                   halo, None, ctypes.byref(err))
        assert m is None and err.value in (-30, -65), (dims, begin, count, halo, err.value)


@pytest.mark.parametrize("kind", ["stencil", "rotate3d"])
def test_region_origin_3d_staged_kernels(sess, orc, kind):
    """3D regions (origin on every axis, ragged sizes) through the staged
    config-3 kernels equal the same sub-box of the whole grid, and the oracle."""
    W, H, D = 300, 70, 24
    codes = synth.image_codes(synth.rng(72), R, F32, W, H, D)
    img = sess.image(R, F32, W, H, D, host=codes)
    oimg = orc.Image(codes.copy(), W, H, D, dims=3, order=R, type=F32)
    smp = sess.sampler(True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    A = _affine(kind, W, H, D)
    ref = gpu_read_grid(sess, img, smp, 0, A, (W, H, D), 1)
    for origin, region in (((37, 5, 3), (150, 20, 11)), ((0, 33, 17), (300, 37, 7)), ((261, 0, 0), (39, 70, 24))):
        got = _read_region(sess, img, smp, A, origin, region, 1)
        (x0, y0, z0), (w, h, d) = origin, region
        exp = ref[z0:z0 + d, y0:y0 + h, x0:x0 + w]
        assert np.array_equal(got.view(np.uint32), exp.view(np.uint32)), (kind, origin)
    full = orc.read_grid(oimg, True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR, orc.RT_F, A, (W, H, D), 1)
    assert_parity(ref, full, True, f"3D region base {kind}")
    sess.release(img)
    cl.lib().clReleaseSampler(smp)
