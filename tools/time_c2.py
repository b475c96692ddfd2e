"""Time the config-2 reads (4096^2 RGBA32F, LINEAR, REPEAT and MIRRORED, map (A))
with CUDA events, through b2clEnqueueReadImageGrid only (works with older
builds via B2CL_LIB for A/B runs)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_kimdjjl15_b200 import build, cl, synth  # noqa: E402


def main():
    if not os.environ.get("B2CL_LIB"):
        build.build()
    st = torch.cuda.Stream()
    S = cl.Session(0, stream=st.cuda_stream)
    L = cl.lib()
    n = 4096
    img = S.image(cl.CL_RGBA, cl.CL_FLOAT, n, n,
                  host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n, n))
    out = S.buffer(n * n * 16)
    A = (ctypes.c_float * 12)(*synth.affine_translate_2d(n, n).tolist())
    d = cl.sz3((n, n, 1))
    res = []
    for addr in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT):
        smp = S.sampler(True, addr, cl.CL_FILTER_LINEAR)

        def go():
            cl.check(L.b2clEnqueueReadImageGrid(S.queue, img, smp, 0, A, d, 4, out, 0, 0, None, None))
        for _ in range(5):
            go()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(50):
            go()
        e1.record(st)
        torch.cuda.synchronize()
        res.append(e0.elapsed_time(e1) / 50 * 1e3)
    # the bench step: REPEAT then MIRRORED back to back, no events in between
    smps = [S.sampler(True, a, cl.CL_FILTER_LINEAR)
            for a in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT)]
    outs = [out, S.buffer(n * n * 16)]

    def step():
        for k in range(2):
            cl.check(L.b2clEnqueueReadImageGrid(S.queue, img, smps[k], 0, A, d, 4, outs[k], 0, 0,
                                                None, None))
    for _ in range(5):
        step()
    e0.record(st)
    for _ in range(50):
        step()
    e1.record(st)
    torch.cuda.synchronize()
    pair = e0.elapsed_time(e1) / 50 * 1e3
    print(f"{os.path.basename(os.environ.get('B2CL_LIB', 'libb2cl.so'))}: REPEAT {res[0]:.1f} us, "
          f"MIRRORED {res[1]:.1f} us, sum {res[0] + res[1]:.1f} us, step {pair:.1f} us")


if __name__ == "__main__":
    main()
