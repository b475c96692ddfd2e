"""Time the config-3 read (512^3 R32F trilinear, stencil map) with CUDA events.

    python tools/time_c3.py [rot]   (rot: the volume-render rotation, map B)
"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_kimdjjl15_b200 import build, cl, synth  # noqa: E402


def main():
    build.build()
    st = torch.cuda.Stream()
    S = cl.Session(0, stream=st.cuda_stream)
    L = cl.lib()
    n = 512
    vol = S.image(cl.CL_R, cl.CL_FLOAT, n, n, n,
                  host=synth.image_codes(synth.rng(3), cl.CL_R, cl.CL_FLOAT, n, n, n))
    out = S.buffer(n ** 3 * 4)
    smp = S.sampler(True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    rot = len(sys.argv) > 1 and sys.argv[1] == "rot"
    A = (ctypes.c_float * 12)(*(synth.affine_rotate_3d(n, 20.0) if rot else synth.affine_stencil_3d(n)).tolist())
    d = cl.sz3((n, n, n))

    def go():
        cl.check(L.b2clEnqueueReadImageGrid(S.queue, vol, smp, 0, A, d, 1, out, 0, 0, None, None))
    for _ in range(5):
        go()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(20):
        go()
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 20
    print(f"{'rotated' if rot else 'stencil'}  {os.environ.get('B2CL_TUNE', '0')}: {ms * 1e3:.1f} us, "
          f"{n ** 3 / ms / 1e6:.1f} Gsamples/s, {2 * n ** 3 * 4 / ms / 1e6:.0f} GB/s")


if __name__ == "__main__":
    main()
