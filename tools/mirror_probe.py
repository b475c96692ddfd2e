"""Probe DRAM re-reads of the MIRRORED config-2 pass under ncu: the full output,
the top half only, and the REPEAT pass (run under `ncu --metrics ...`)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_kimdjjl15_b200 import build, cl, synth  # noqa: E402


def main():
    build.build()
    S = cl.Session(0)
    L = cl.lib()
    n = 4096
    img = S.image(cl.CL_RGBA, cl.CL_FLOAT, n, n,
                  host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n, n))
    out = S.buffer(n * n * 16)
    A = (ctypes.c_float * 12)(*synth.affine_translate_2d(n, n).tolist())
    mir = S.sampler(True, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR)
    rep = S.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR)
    for smp, origin, region in ((mir, (0, 0, 0), (n, n, 1)), (mir, (0, 0, 0), (n, n // 2, 1)),
                                (mir, (0, 0, 0), (n // 2, n // 2, 1)), (rep, (0, 0, 0), (n, n, 1))):
        cl.check(L.b2clEnqueueReadImageGridRegion(S.queue, img, smp, 0, A, cl.sz3(origin),
                                                  cl.sz3(region), 4, out, 0, 0, None, None))
    S.finish()
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
