"""Time the general-map reads: config-2 map (B) (30 deg rotation, 4096^2
RGBA32F, REPEAT and MIRRORED) and config-3 map (B) through the general kernel
(B2CL_GRID_KERNEL=g) or the default choice.
    python tools/time_maps.py"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_kimdjjl15_b200 import build, cl, synth  # noqa: E402


def timed(st, fn, it=20):
    for _ in range(3):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(it):
        fn()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it * 1e3


def main():
    if not os.environ.get("B2CL_LIB"):
        build.build()
    st = torch.cuda.Stream()
    S = cl.Session(0, stream=st.cuda_stream)
    L = cl.lib()
    n = 4096
    tiled = "--tiled" in sys.argv  # B2CL_MEM_TILED_IMAGE storage
    img = S.image(cl.CL_RGBA, cl.CL_FLOAT, n, n,
                  host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n, n),
                  flags=cl.CL_MEM_READ_WRITE | (cl.B2CL_MEM_TILED_IMAGE if tiled else 0))
    out = S.buffer(n * n * 16)
    A = (ctypes.c_float * 12)(*synth.affine_rotate_2d(n, n, 30.0).tolist())
    d = cl.sz3((n, n, 1))
    res = []
    for addr in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT):
        smp = S.sampler(True, addr, cl.CL_FILTER_LINEAR)
        res.append(timed(st, lambda: cl.check(L.b2clEnqueueReadImageGrid(S.queue, img, smp, 0, A, d, 4, out, 0, 0,
                                                                           None, None))))
    S.release(img, out)
    print(f"{os.path.basename(os.environ.get('B2CL_LIB', 'libb2cl.so'))}{' tiled' if tiled else ''} "
          f"[{os.environ.get('B2CL_GRID_KERNEL', 'default')}]: C2 map B REPEAT {res[0]:.1f} us, "
          f"MIRRORED {res[1]:.1f} us ({n * n / res[0] / 1e3:.0f} / {n * n / res[1] / 1e3:.0f} Gsamples/s)")


if __name__ == "__main__":
    main()
