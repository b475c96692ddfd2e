"""Config-2 step with the two reads (REPEAT, MIRRORED) on two command queues of
one context, joined by events every step, against the same step on one queue.
    python tools/time_c2_queues.py"""
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
    q2 = S.queue_for(0)
    n = 4096
    img = S.image(cl.CL_RGBA, cl.CL_FLOAT, n, n,
                  host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n, n))
    outs = [S.buffer(n * n * 16), S.buffer(n * n * 16)]
    A = (ctypes.c_float * 12)(*synth.affine_translate_2d(n, n).tolist())
    d = cl.sz3((n, n, 1))
    smps = [S.sampler(True, a, cl.CL_FILTER_LINEAR)
            for a in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT)]

    def one_queue():
        for k in range(2):
            cl.check(L.b2clEnqueueReadImageGrid(S.queue, img, smps[k], 0, A, d, 4, outs[k], 0, 0, None, None))

    def two_queues(order):
        ev = [ctypes.c_void_p(), ctypes.c_void_p()]
        # q2 waits for the previous step's work on the main queue (marker), then both run
        mk = ctypes.c_void_p()
        cl.check(L.clEnqueueMarkerWithWaitList(S.queue, 0, None, ctypes.byref(mk)))
        for k in order:
            q = S.queue if k == 0 else q2
            wl = (ctypes.c_void_p * 1)(mk) if k == 1 else None
            cl.check(L.b2clEnqueueReadImageGrid(q, img, smps[k], 0, A, d, 4, outs[k], 0, 1 if k == 1 else 0,
                                                wl, ctypes.byref(ev[k])))
        wl2 = (ctypes.c_void_p * 1)(ev[1])
        cl.check(L.clEnqueueMarkerWithWaitList(S.queue, 1, wl2, None))
        for e in ev + [mk]:
            L.clReleaseEvent(e)

    for name, fn in (("one queue", one_queue), ("two queues R,M", lambda: two_queues((0, 1))),
                     ("two queues M,R", lambda: two_queues((1, 0)))):
        for _ in range(5):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(50):
            fn()
        e1.record(st)
        torch.cuda.synchronize()
        print(f"{name}: step {e0.elapsed_time(e1) / 50 * 1e3:.1f} us")


if __name__ == "__main__":
    main()
