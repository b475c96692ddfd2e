"""Launch each hot kernel a few times, for ncu captures on the GPU box.

    ncu --set full -k regex:<kernel> -c N -o gpurun_out/prof python tools/prof_kernels.py [which...]

which: c2r / c2m (ONE map (A) REPEAT / MIRRORED launch each: bench.py's
in-run traffic capture), c2 (REPEAT + MIRRORED 4096^2 RGBA32F, maps A and B), c3 (512^3 R32F stencil + rotated),
copy (8 GiB pitched rect, aligned + misaligned), fill (8 GiB).  Each launch is
preceded by one untimed warm-up launch of the same kernel.
"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_sc_kimdjjl15_b200 import build, cl, synth  # noqa: E402


def main(which):
    build.build()
    S = cl.Session(0)
    L = cl.lib()
    if "c2r" in which or "c2m" in which:
        # the bench's in-run traffic capture: ONE launch of each named map (A) pass
        n = 4096
        img = S.image(cl.CL_RGBA, cl.CL_FLOAT, n, n,
                      host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n, n))
        out = S.buffer(n * n * 16)
        A = (ctypes.c_float * 12)(*synth.affine_translate_2d(n, n).tolist())
        for key, addr in (("c2r", cl.CL_ADDRESS_REPEAT), ("c2m", cl.CL_ADDRESS_MIRRORED_REPEAT)):
            if key in which:
                smp = S.sampler(True, addr, cl.CL_FILTER_LINEAR)
                cl.check(L.b2clEnqueueReadImageGrid(S.queue, img, smp, 0, A, cl.sz3((n, n, 1)), 4,
                                                    out, 0, 0, None, None))
        S.finish()
        S.release(img, out)
    if "c2" in which:
        n = 4096
        img = S.image(cl.CL_RGBA, cl.CL_FLOAT, n, n,
                      host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n, n))
        out = S.buffer(n * n * 16)
        A = (ctypes.c_float * 12)(*synth.affine_translate_2d(n, n).tolist())
        Ar = (ctypes.c_float * 12)(*synth.affine_rotate_2d(n, n, 30.0).tolist())
        for addr in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT):
            smp = S.sampler(True, addr, cl.CL_FILTER_LINEAR)
            for aff in (A, A, Ar, Ar):
                cl.check(L.b2clEnqueueReadImageGrid(S.queue, img, smp, 0, aff, cl.sz3((n, n, 1)), 4,
                                                    out, 0, 0, None, None))
        S.finish()
        S.release(img, out)
    if "c3" in which:
        n = 512
        vol = S.image(cl.CL_R, cl.CL_FLOAT, n, n, n,
                      host=synth.image_codes(synth.rng(3), cl.CL_R, cl.CL_FLOAT, n, n, n))
        out = S.buffer(n ** 3 * 4)
        smp = S.sampler(True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
        for aff in (synth.affine_stencil_3d(n), synth.affine_rotate_3d(n, 20.0)):
            A = (ctypes.c_float * 12)(*aff.tolist())
            for _ in range(3):
                cl.check(L.b2clEnqueueReadImageGrid(S.queue, vol, smp, 0, A, cl.sz3((n, n, n)), 1,
                                                    out, 0, 0, None, None))
        S.finish()
        S.release(vol, out)
    if "copy" in which or "fill" in which:
        region = (16384, 2048, 256)
        srp, ssp = 16512, 2056 * 16512
        nb = region[0] * region[1] * region[2]
        src = S.buffer(ssp * region[2])
        dst = S.buffer(nb)
        z = cl.sz3((0, 0, 0))
        if "copy" in which:
            for _ in range(3):
                cl.check(L.clEnqueueCopyBufferRect(S.queue, src, dst, z, z, cl.sz3(region), srp, ssp,
                                                   0, 0, 0, None, None))
            for _ in range(3):
                cl.check(L.clEnqueueCopyBufferRect(S.queue, src, dst, cl.sz3((3, 0, 0)), z,
                                                   cl.sz3((16384, 2048, 255)), 16387, 16387 * 2056,
                                                   0, 0, 0, None, None))
        if "fill" in which:
            pat = np.arange(16, dtype=np.uint8)
            for _ in range(3):
                cl.check(L.clEnqueueFillBuffer(S.queue, dst, pat.ctypes.data, 16, 0, nb, 0, None,
                                               None))
        S.finish()
        S.release(src, dst)
    S.close()


if __name__ == "__main__":
    main(set(sys.argv[1:]) or {"c2", "c3", "copy", "fill"})
