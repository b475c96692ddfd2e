"""Time the config-4 rect copies (8 GiB pitched, aligned and misaligned) with
CUDA events through clEnqueueCopyBufferRect (B2CL_LIB selects an A/B build)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_kimdjjl15_b200 import build, cl  # noqa: E402


def main():
    if not os.environ.get("B2CL_LIB"):
        build.build()
    st = torch.cuda.Stream()
    S = cl.Session(0, stream=st.cuda_stream)
    L = cl.lib()
    region = (16384, 2048, 256)
    srp, ssp = 16512, 2056 * 16512
    nb = region[0] * region[1] * region[2]
    src, dst = S.buffer(ssp * region[2]), S.buffer(nb)
    zero = cl.sz3((0, 0, 0))
    cases = {
        "aligned": lambda: L.clEnqueueCopyBufferRect(S.queue, src, dst, zero, zero, cl.sz3(region), srp,
                                                     ssp, 0, 0, 0, None, None),
        "misaligned": lambda: L.clEnqueueCopyBufferRect(S.queue, src, dst, cl.sz3((3, 0, 0)), zero,
                                                        cl.sz3((16384, 2048, 255)), 16387, 16387 * 2056,
                                                        0, 0, 0, None, None),
        "misaligned_both": lambda: L.clEnqueueCopyBufferRect(S.queue, src, dst, cl.sz3((3, 0, 0)),
                                                             cl.sz3((7, 0, 0)), cl.sz3((16384, 2048, 255)),
                                                             16387, 16387 * 2056, 16400, 16400 * 2048,
                                                             0, None, None),
    }
    out = []
    for name, f in cases.items():
        for _ in range(3):
            cl.check(f())
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(10):
            cl.check(f())
        e1.record(st)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        b = nb if name == "aligned" else 16384 * 2048 * 255
        out.append(f"{name} {ms:.3f} ms ({2 * b / ms / 1e6 / 6468:.3f} of HBM)")
    print(os.path.basename(os.environ.get("B2CL_LIB", "libb2cl.so")) + ": " + ", ".join(out))


if __name__ == "__main__":
    main()
