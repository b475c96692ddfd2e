"""Time the coordinate-list read (b2clEnqueueReadImageSamples, k_sample_list)
at config-2 size: a 4096^2 RGBA32F image, 16.8 M float2 coordinates, LINEAR,
normalized -- the coordinates of map (A) (the bench's translate) and map (B)
(30 degree rotation) in row-major output order, and uniform random ones.
Algorithmic bytes: 8 B coordinate + 16 B output per sample + 16 B per distinct
texel tapped (counted here on the host for the grid maps; random: all texels).
    python tools/time_list.py"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
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


def grid_coords(A, n):
    """float32 coordinates of the affine map in the kernels' operand order."""
    x = np.arange(n, dtype=np.float32)[None, :]
    y = np.arange(n, dtype=np.float32)[:, None]
    s = ((A[0] * x + A[1] * y).astype(np.float32) + np.float32(0)).astype(np.float32) + A[3]
    t = ((A[4] * x + A[5] * y).astype(np.float32) + np.float32(0)).astype(np.float32) + A[7]
    return np.stack([s.astype(np.float32), t.astype(np.float32)], -1).reshape(-1, 2)


def main():
    if not os.environ.get("B2CL_LIB"):
        build.build()
    peak = 6550.7
    st = torch.cuda.Stream()
    S = cl.Session(0, stream=st.cuda_stream)
    L = cl.lib()
    n = 4096
    img = S.image(cl.CL_RGBA, cl.CL_FLOAT, n, n,
                  host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n, n))
    out = S.buffer(n * n * 16)
    g = np.random.default_rng(5)
    cases = [("map A", grid_coords(synth.affine_translate_2d(n, n), n)),
             ("map B", grid_coords(synth.affine_rotate_2d(n, n, 30.0), n)),
             ("random", g.random((n * n, 2), dtype=np.float32))]
    for name, co in cases:
        co = np.ascontiguousarray(co, dtype=np.float32)
        cbuf = S.buffer(co.nbytes, co)
        for addr in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT):
            smp = S.sampler(True, addr, cl.CL_FILTER_LINEAR)
            us = timed(st, lambda: cl.check(L.b2clEnqueueReadImageSamples(
                S.queue, img, smp, cl.B2CL_RTYPE_FLOAT, cl.B2CL_COORD_FLOAT, cbuf, 0, n * n, out, 0, 0,
                None, None)))
            ker = cl.last_kernel()
            nbytes = co.nbytes + n * n * 16 + n * n * 16  # (every texel tapped: a bound for map A / random)
            print(f"{os.path.basename(os.environ.get('B2CL_LIB', 'libb2cl.so'))} list {name:6s} "
                  f"{'REPEAT  ' if addr == cl.CL_ADDRESS_REPEAT else 'MIRRORED'} {ker}: {us:7.1f} us "
                  f"{n * n / us / 1e3:6.1f} Gsamples/s  {nbytes / us / 1e3:7.1f} GB/s "
                  f"({nbytes / us / 1e3 / peak:.3f} of HBM at <= {nbytes / 1e6:.0f} MB)")
        S.release(cbuf)
    S.release(img, out)


if __name__ == "__main__":
    main()
