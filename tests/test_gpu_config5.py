"""BASELINE config 5's image at full size on one B200: 32768 x 32768 RGBA32F
(16 GiB, so texel offsets pass 2^32 bytes), read with the config-2 map (A)
under REPEAT and MIRRORED_REPEAT through the kernels bench.py times; sampled
output rows (first, last, both shard seams of 2/4/8-way row bands, middle)
against the oracle on every column.

The oracle's copy of the image is a 16 GiB anonymous mapping of which only
the texel rows the sampled outputs can tap (their estimated row +- 3) are
written, from the same per-row seeded generator (synth.image_rows) that
filled the GPU image; an untouched row reads as zeros, so a wrong estimate
fails the comparison instead of hiding anything."""
import ctypes
import mmap

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth
from tests.gpu_helpers import assert_parity

pytestmark = pytest.mark.gpu

N = 32768
ES = 16
ROW = N * ES


def _rows_near(A, ys, addr):
    """Texel rows within 3 of the taps of output rows ys (numpy float32, an
    estimate only: the oracle and the GPU both compute the real taps)."""
    f = np.float32
    need = set()
    for y in ys:
        s = f(A[5]) * f(y) + f(A[7])
        if addr == cl.CL_ADDRESS_REPEAT:
            u = (s - np.floor(s)) * f(N)
        else:
            u = abs(s - f(2) * np.rint(f(0.5) * s)) * f(N)
        j = int(np.floor(u - f(0.5)))
        need.update((j + d) % N for d in range(-3, 4))
    return sorted(need)


def test_config5_full_size_image_sampled_rows(sess, orc):
    img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, N, N)
    band = 512
    for y0 in range(0, N, band):
        rows = np.ascontiguousarray(synth.image_rows(cl.CL_RGBA, cl.CL_FLOAT, N, range(y0, y0 + band)))
        cl.check(cl.lib().clEnqueueWriteImage(sess.queue, img, 1, cl.sz3((0, y0, 0)), cl.sz3((N, band, 1)), 0, 0,
                                              rows.ctypes.data, 0, None, None), "clEnqueueWriteImage")
    A = synth.affine_translate_2d(N, N)
    ys = [0, 1, N // 8 - 1, N // 8, N // 4 - 1, N // 4, N // 2 - 1, N // 2, 3 * N // 4, 12345, N - 2, N - 1]
    Ac = (ctypes.c_float * 12)(*[float(x) for x in A])
    out = sess.buffer(N * ROW)  # 16 GiB; only the sampled rows come back
    for addr in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT):
        smp = sess.sampler(True, addr, cl.CL_FILTER_LINEAR)
        cl.check(cl.lib().b2clEnqueueReadImageGrid(sess.queue, img, smp, cl.B2CL_RTYPE_FLOAT, Ac, cl.sz3((N, N, 1)),
                                                   4, out, 0, 0, None, None), "b2clEnqueueReadImageGrid")
        got = np.stack([sess.read(out, ROW, offset=y * ROW).view(np.float32).reshape(1, N, 4) for y in ys])
        mm = mmap.mmap(-1, N * ROW)
        host = np.frombuffer(mm, dtype=np.uint8)
        need = _rows_near(A, ys, addr)
        for j in need:
            host[j * ROW:(j + 1) * ROW] = synth.image_rows(cl.CL_RGBA, cl.CL_FLOAT, N, [j]).view(np.uint8).reshape(-1)
        oimg = orc.Image(host, N, N, 1, dims=2, order=cl.CL_RGBA, type=cl.CL_FLOAT)
        for k, y in enumerate(ys):
            exp = orc.read_grid(oimg, True, addr, cl.CL_FILTER_LINEAR, orc.RT_F, A, (N, N, 1), 4,
                                yrange=(y, y + 1), nthreads=8)
            assert_parity(got[k], exp[0], True, f"config5 {hex(addr)} row {y}")
        del oimg, host
        mm.close()
        cl.lib().clReleaseSampler(smp)
    sess.release(img, out)
