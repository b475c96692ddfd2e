#!/usr/bin/env python
"""bench.py -- headline benchmark of the b2cl hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl b2cl|reference]
    python -m torch.distributed.run --nproc-per-node N ... bench.py --gpus N ...

Workload (BASELINE.json configs[1], the config the metric is quoted on):
a 4096x4096 CL_RGBA/CL_FLOAT image, normalized coordinates, LINEAR filter.
One STEP = read_imagef over the full 4096^2 output grid under REPEAT and
again under MIRRORED_REPEAT (map (A): translate by (0.3, 0.7) px plus a half
period so the wrap seam crosses the output), i.e. two launches of the
sampling kernel, 2 x 16.8 M samples.  `value` = samples / step time in
Gsamples/s, whole job (sum over ranks; each rank owns its own image: weak
scaling, no collective on the data path).

Secondary measurements in the same JSON line (`secondary`): config 3
(512^3 R32F trilinear), config 4 (8 GiB pitched CopyBufferRect, FillBuffer,
CopyImageToBuffer) and the copy-size sweep, each with its HBM fraction.

Timing: CUDA events on the queue's stream around every launch, after W
untimed steps, barrier + synchronize on both sides, max over ranks.  The
working set (256 MiB image + 2 x 256 MiB output) exceeds the 126 MB L2, so no
flush is needed between steps.  Clocks are sampled with nvidia-smi during
the timed region.  `--impl reference` times the CPU oracle (oracle/) on the
host cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "read_imagef Gsamples/s and BufferRect copy GB/s vs HBM peak at 1/2/4/8 B200"
N2D = 4096
WORKLOAD = "C2: 4096x4096 CL_RGBA/CL_FLOAT, normalized, LINEAR, REPEAT + MIRRORED_REPEAT, map (A)"


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------------ clocks
class Clocks:
    """SM clock + throttle reasons sampled DURING the timed region: an NVML
    polling thread (5 ms) when pynvml finds the driver library, else
    `nvidia-smi -lms 100` in the background."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index: int):
        self.index = index
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.thread = self.proc = None
        self._stop = False

    def start(self):
        try:
            import threading

            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)

            def poll():
                while not self._stop:
                    self.samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                    r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                    for n, bit in self.REASONS.items():
                        if r & bit:
                            self.reasons.add(n)
                    time.sleep(0.005)
            self.thread = threading.Thread(target=poll, daemon=True)
            self.thread.start()
            time.sleep(0.01)
            return
        except Exception:
            self.thread = None
        try:
            self.file = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=self.file, stderr=subprocess.DEVNULL)
        except (OSError, FileNotFoundError):
            self.proc = None

    def stop(self):
        if self.thread is not None:
            self._stop = True
            self.thread.join(timeout=2)
            sm = self.samples
            src = "nvml 5 ms"
        elif self.proc is not None:
            time.sleep(0.15)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
            self.file.flush()
            rows = [ln.split(",") for ln in open(self.file.name).read().splitlines() if ln.strip()]
            os.unlink(self.file.name)
            sm = []
            names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
            for r in rows:
                try:
                    sm.append(float(r[0]))
                    self.max_mhz = float(r[1])
                except (ValueError, IndexError):
                    continue
                for n, v in zip(names, r[2:6]):
                    if v.strip() == "Active":
                        self.reasons.add(n)
            src = "nvidia-smi 100 ms"
        else:
            return None
        if not sm:
            return None
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": self.max_mhz, "samples": len(sm),
                "reasons": sorted(self.reasons), "source": src}


# ------------------------------------------------------------------ oracle (CPU) timing
def oracle_rate(codes, n_rows_target_s: float, threads: int):
    """Time the oracle on REPEAT + MIRRORED rows of the C2 workload.  Returns
    (Gsamples/s, rows, seconds)."""
    import oracle as orc
    from paper_conf_sc_kimdjjl15_b200 import synth
    img = orc.Image(codes, N2D, N2D, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    A = synth.affine_translate_2d(N2D, N2D)
    run = lambda r0, r1: [orc.read_grid(img, True, a, orc.FILTER_LINEAR, orc.RT_F, A,
                                        (N2D, N2D, 1), 4, yrange=(r0, r1), nthreads=threads)
                          for a in (orc.ADDRESS_REPEAT, orc.ADDRESS_MIRRORED_REPEAT)]
    t0 = time.perf_counter()
    run(0, 16)
    dt = time.perf_counter() - t0
    rows = int(max(16, 16 * n_rows_target_s / max(dt, 1e-6)))  # may exceed one full pass
    t0 = time.perf_counter()
    done = 0
    while done < rows:
        r = min(N2D, rows - done)
        run(0, r)
        done += r
    dt = time.perf_counter() - t0
    return 2 * rows * N2D / dt / 1e9, rows, dt


def _axis_taps(coef, offset, n_out, n, mode, start=0):
    """Set of texel indices along one axis that a LINEAR read of a separable
    affine map touches with a non-zero weight, for outputs start..start+n_out-1
    ([CL1.2 §8.2] in numpy float32; measurement bookkeeping only -- the bytes a
    launch must move, and the rows a shard must hold)."""
    f32 = np.float32
    x = np.arange(start, start + n_out, dtype=np.float32)
    s = (f32(coef) * x).astype(f32) + f32(offset)
    fn = f32(n)
    if mode == "repeat":
        u = ((s - np.floor(s)).astype(f32) * fn).astype(f32)
    elif mode == "clamp_to_edge":
        u = (s * fn).astype(f32)
    else:
        sp = (f32(2.0) * np.rint((f32(0.5) * s).astype(f32))).astype(f32)
        u = (np.abs((s - sp).astype(f32)) * fn).astype(f32)
    t = (u - f32(0.5)).astype(f32)
    b = np.floor(t).astype(np.int64)
    a = (t - np.floor(t)).astype(f32)
    if mode == "repeat":
        i0, i1 = np.where(b < 0, b + n, b), np.where(b + 1 > n - 1, b + 1 - n, b + 1)
    elif mode == "clamp_to_edge":
        i0, i1 = np.clip(b, 0, n - 1), np.clip(b + 1, 0, n - 1)
    else:
        i0, i1 = np.maximum(b, 0), np.minimum(b + 1, n - 1)
    return np.unique(np.concatenate([i0[a != 1], i1[a != 0]]))


def _distinct_texels_2d(A, W, H, mode, chunk=256):
    """Number of distinct texels a LINEAR read of the 2D affine map A (output
    W x H, image W x H, normalized, z = 0) touches with a non-zero tap weight,
    under REPEAT, MIRRORED_REPEAT or CLAMP_TO_EDGE ([CL1.2 §8.2] in numpy float32, one RN op
    per step as the kernels and the oracle; measurement bookkeeping only)."""
    f32 = np.float32
    seen = np.zeros((H, W), dtype=bool)
    x = np.arange(W, dtype=f32)[None, :]

    def axis(c, n):
        fn = f32(n)
        if mode == "repeat":
            u = ((c - np.floor(c)).astype(f32) * fn).astype(f32)
        elif mode == "clamp_to_edge":
            u = (c * fn).astype(f32)
        else:
            sp = (f32(2.0) * np.rint((f32(0.5) * c).astype(f32))).astype(f32)
            u = (np.abs((c - sp).astype(f32)) * fn).astype(f32)
        t = (u - f32(0.5)).astype(f32)
        b = np.floor(t).astype(np.int64)
        a = (t - np.floor(t)).astype(f32)
        if mode == "repeat":
            return np.where(b < 0, b + n, b), np.where(b + 1 > n - 1, b + 1 - n, b + 1), a
        if mode == "clamp_to_edge":
            return np.clip(b, 0, n - 1), np.clip(b + 1, 0, n - 1), a
        return np.maximum(b, 0), np.minimum(b + 1, n - 1), a

    for y0 in range(0, H, chunk):
        y = np.arange(y0, min(H, y0 + chunk), dtype=f32)[:, None]
        cs = []
        for r in range(2):
            v = (f32(A[4 * r]) * x).astype(f32) + (f32(A[4 * r + 1]) * y).astype(f32)
            v = (v.astype(f32) + (f32(A[4 * r + 2]) * f32(0.0))).astype(f32)
            cs.append((v + f32(A[4 * r + 3])).astype(f32))
        i0, i1, a = axis(cs[0], W)
        j0, j1, b = axis(cs[1], H)
        for jj, ii, m in ((j0, i0, (a != 1) & (b != 1)), (j0, i1, (a != 0) & (b != 1)),
                          (j1, i0, (a != 1) & (b != 0)), (j1, i1, (a != 0) & (b != 0))):
            seen[jj[m], ii[m]] = True
    return int(seen.sum())


def circular_interval(idx, n):
    """Smallest (begin, count) whose circular range {(begin+s) mod n} covers idx."""
    rows = np.unique(np.asarray(idx, dtype=np.int64))
    if rows.size == 1:
        return int(rows[0]), 1
    gaps = (np.roll(rows, -1) - rows) % n
    i = int(np.argmax(gaps))
    begin = int(rows[(i + 1) % rows.size])
    return begin, int((rows[i] - begin) % n + 1)


def distinct_texels_separable(A, w_out, h_out, mode):
    assert A[1] == 0 and A[4] == 0, "separable map expected"
    return (_axis_taps(A[0], A[3], w_out, N2D, mode).size *
            _axis_taps(A[5], A[7], h_out, N2D, mode).size)


def c2_codes():
    from paper_conf_sc_kimdjjl15_b200 import cl, synth
    g = synth.rng(2)  # the same seed the parity test of config 2 uses
    return synth.image_codes(g, cl.CL_RGBA, cl.CL_FLOAT, N2D, N2D, 1)


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    threads = os.cpu_count() or 1
    codes = c2_codes()
    total_budget = 60.0
    per_step = total_budget / max(1, args.steps + args.warmup)
    rate, rows, _ = oracle_rate(codes, per_step, threads)  # calibrates rows per step
    import oracle as orc
    from paper_conf_sc_kimdjjl15_b200 import synth
    img = orc.Image(codes, N2D, N2D, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    A = synth.affine_translate_2d(N2D, N2D)

    def step(i):
        done = 0
        while done < rows:
            r = min(N2D, rows - done)
            y0 = (i * 977 + done) % (N2D - r + 1)
            for a in (orc.ADDRESS_REPEAT, orc.ADDRESS_MIRRORED_REPEAT):
                orc.read_grid(img, True, a, orc.FILTER_LINEAR, orc.RT_F, A, (N2D, N2D, 1), 4,
                              yrange=(y0, y0 + r), nthreads=threads)
            done += r
    for i in range(args.warmup):
        step(i)
    t0 = time.perf_counter()
    for i in range(args.steps):
        step(args.warmup + i)
    dt = (time.perf_counter() - t0) / args.steps
    value = 2 * rows * N2D / dt / 1e9
    sample = f"{rows} rows x {N2D} columns of each pass (REPEAT, MIRRORED) per step"
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "Gsamples/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": dt * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic (seed 20151115)",
            "config": {"workload": WORKLOAD, "sample": sample},
            "cpu_baseline": {"value": value, "unit": "Gsamples/s", "cores": threads,
                             "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": "Gsamples/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ GPU arm
class Timer:
    """CUDA events on a torch stream (the queue's stream)."""

    def __init__(self, torch, stream):
        self.torch, self.stream = torch, stream

    def event(self):
        e = self.torch.cuda.Event(enable_timing=True)
        e.record(self.stream)
        return e


def run_gpu(args):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_kimdjjl15_b200 import build, cl, synth
    from paper_conf_sc_kimdjjl15_b200 import dist as bdist
    build.build()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # one GPU per rank; more ranks than GPUs only happens in the single-GPU
    # rehearsal of the multi-rank path (ranks share a device, control plane on gloo)
    ndev = torch.cuda.device_count()
    gpu = local % ndev
    shared = world > ndev
    torch.cuda.set_device(gpu)
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", gpu))
    dev = torch.device("cuda", gpu)
    red_dev = None if shared else dev  # device of the max-over-ranks tensors
    stream = torch.cuda.Stream(device=dev)
    S = cl.Session(gpu, stream=stream.cuda_stream)
    L = cl.lib()
    T = Timer(torch, stream)
    hbm_peak, peak_src = peaks()

    # ---- inputs resident in HBM before timing ----
    # N = 1: config 2 itself, one 4096^2 image.  N > 1 (config 5 style): one
    # global (4096*N) x 4096 image, row-sharded: rank r computes output rows
    # [4096 r, 4096 (r+1)) of map (A) on the GLOBAL image from shards holding
    # exactly the texel rows that band needs (one per pass: REPEAT and the
    # folded MIRRORED rows differ) -- bit-identical to a single-GPU read
    # (tests/test_gpu_shards.py), same per-GPU work as N = 1 (weak scaling).
    Hg = N2D * world
    r0 = rank * N2D
    Af = synth.affine_translate_2d(N2D, Hg)
    A = (ctypes.c_float * 12)(*Af.tolist())
    modes = ("repeat", "mirrored")
    codes = None
    shard_rows, shard_host, shard_begin = [], [], []
    if world == 1:
        codes = c2_codes()
        img = S.image(cl.CL_RGBA, cl.CL_FLOAT, N2D, N2D, host=codes)
        imgs = [img, img]
    else:
        imgs = []
        for m in modes:
            need = _axis_taps(Af[5], Af[7], N2D, Hg, m, start=r0)
            begin, count = circular_interval(need, Hg)
            rows = [(begin + s) % Hg for s in range(count)]
            shard_rows.append(count)
            shard_begin.append(begin)
            shard_host.append(synth.image_rows(cl.CL_RGBA, cl.CL_FLOAT, N2D, rows))
            imgs.append(S.image_shard(cl.CL_RGBA, cl.CL_FLOAT, N2D, Hg, 0, begin, count, 0,
                                      host=shard_host[-1]))
    nout = N2D * N2D * 16
    outs = [S.buffer(nout), S.buffer(nout)]
    smps = [S.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR),
            S.sampler(True, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR)]
    origin, region = cl.sz3((0, r0, 0)), cl.sz3((N2D, N2D, 1))

    def launch(k, images=None, queue=None, nwait=0, wait=None, ev=None):
        cl.check(L.b2clEnqueueReadImageGridRegion(queue or S.queue, (images or imgs)[k], smps[k],
                                                  cl.B2CL_RTYPE_FLOAT, A, origin, region, 4, outs[k],
                                                  0, nwait, wait, ev),
                 "read grid")

    # The step: the two reads are independent (one image, two samplers, two
    # outputs), so the program issues them on two command queues of the
    # device, as an OpenCL program would, and joins them with events: the
    # second queue starts after a marker of the first (the previous step is
    # complete) and the first queue's barrier waits for the second read.
    q_two = S.queue_for(gpu)

    def step():
        mk, e1 = ctypes.c_void_p(), ctypes.c_void_p()
        cl.check(L.clEnqueueMarkerWithWaitList(S.queue, 0, None, ctypes.byref(mk)))
        launch(1, queue=q_two, nwait=1, wait=(ctypes.c_void_p * 1)(mk), ev=ctypes.byref(e1))
        launch(0)
        cl.check(L.clEnqueueBarrierWithWaitList(S.queue, 1, (ctypes.c_void_p * 1)(e1), None))
        L.clReleaseEvent(mk)
        L.clReleaseEvent(e1)

    # ---- parity spot check of this exact launch configuration (bench as test) ----
    launch(0)
    launch(1)
    S.finish()
    parity = "skipped (oracle missing)"
    if world > 1:
        parity = ("sharded: bit-identity of shard reads to whole-image reads is tested in "
                  "tests/test_gpu_shards.py; the whole-image path is checked against the oracle")
    else:
        try:
            import oracle as orc
            oimg = orc.Image(codes, N2D, N2D, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
            worst = 0.0
            for k, a in enumerate((orc.ADDRESS_REPEAT, orc.ADDRESS_MIRRORED_REPEAT)):
                got = S.read(outs[k], nout, np.float32).reshape(N2D, N2D, 4)
                for y in (0, N2D // 2 - 1, N2D // 2, N2D - 1, 1234):
                    exp = orc.read_grid(oimg, True, a, orc.FILTER_LINEAR, orc.RT_F, Af,
                                        (N2D, N2D, 1), 4, yrange=(y, y + 1))[0, 0]
                    err = np.abs(got[y].astype(np.float64) - exp) / np.maximum(
                        np.spacing(np.abs(exp)).astype(np.float64), 1e-30)
                    ok = np.all((err <= 4) | (np.abs(got[y] - exp) <= 1e-6))
                    worst = max(worst, float(np.max(np.minimum(err, 1e9))))
                    if not ok:
                        raise SystemExit(f"bench parity check failed (pass {k}, row {y})")
            parity = f"ok (10 rows vs oracle, worst {worst:.2f} ulp)"
        except ImportError:
            pass

    # ---- warmup + timed steps ----
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    clocks = Clocks(gpu)
    clocks.start()
    # (1) the step time: K steps back to back, events only at the two ends
    # (an event between launches serialises the kernel boundary: +3.5 us each)
    n_launch0 = cl.launch_count()
    t_start = T.event()
    for _ in range(args.steps):
        step()
    t_end = T.event()
    torch.cuda.synchronize(dev)
    gpu_launches = cl.launch_count() - n_launch0
    total_ms = t_start.elapsed_time(t_end)
    # (2) each kernel's average launch duration for the roofline: K launches of
    # it back to back between two events on the launching stream
    pass_ms = []
    for k in range(2):
        a = T.event()
        for _ in range(args.steps):
            launch(k)
        b = T.event()
        torch.cuda.synchronize(dev)
        pass_ms.append(a.elapsed_time(b) / args.steps)
    clk = clocks.stop()
    ms_step = total_ms / args.steps
    if world > 1:
        ms_step = bdist.max_over_ranks(ms_step, red_dev)
    samples_step = 2 * N2D * N2D
    value = world * samples_step / (ms_step * 1e-3) / 1e9
    # algorithmic bytes per launch = distinct texels with a non-zero tap weight x 16 B
    # + 16 B output per sample; counted exactly per map on the host
    ncols = [_axis_taps(Af[0], Af[3], N2D, N2D, m).size for m in modes]
    nrows = [_axis_taps(Af[5], Af[7], N2D, Hg, m, start=r0).size for m in modes]
    alg = [ncols[k] * nrows[k] * 16 + N2D * N2D * 16 for k in range(2)]
    achieved = [alg[k] / (pass_ms[k] * 1e-3) / 1e9 for k in range(2)]
    dom = 0 if pass_ms[0] * 1.0 >= pass_ms[1] else 1  # the kernel with the larger share of the step
    traffic = None
    import glob
    profs = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*", "ncu_c2_traffic.json")))
    if profs:
        traffic = json.load(open(profs[-1])).get("dram_bytes_per_launch")

    # ---- e2e: host buffers through the C-ABI, copies inside the timed region ----
    # Every step uploads its image(s) from pinned host memory and reads both
    # outputs back to pinned host memory.  The copies are the step's bound
    # (256 MiB up, 512 MiB down over the host link per GPU), so the step is
    # pipelined the way an OpenCL program would: uploads on a second queue
    # into one of two image copies, so step s+1's upload runs while step s's
    # results come down; cross-queue order by events only (wait lists).
    e2e = None
    if not args.no_e2e:
        q_up = S.queue_for(gpu)
        hbufs = []
        for k in range(1 if world == 1 else 2):
            hrows = N2D if world == 1 else shard_rows[k]
            hbuf = torch.empty(hrows * N2D * 16, dtype=torch.uint8).pin_memory()
            src = codes if world == 1 else shard_host[k]
            hbuf.copy_(torch.from_numpy(np.ascontiguousarray(src).reshape(-1).view(np.uint8)))
            hbufs.append((hbuf, cl.sz3((N2D, hrows, 1))))
        # two device copies of the step's images (copy 0 is the resident one)
        e2e_imgs = [imgs]
        if world == 1:
            im2 = S.image(cl.CL_RGBA, cl.CL_FLOAT, N2D, N2D)
            e2e_imgs.append([im2, im2])
        else:
            e2e_imgs.append([S.image_shard(cl.CL_RGBA, cl.CL_FLOAT, N2D, Hg, 0, shard_begin[k],
                                           shard_rows[k], 0) for k in range(2)])
        host_out = [torch.empty(nout, dtype=torch.uint8).pin_memory() for _ in range(2)]
        zero3 = cl.sz3((0, 0, 0))
        done = [None, None]  # marker event of the last step that read image copy b

        def e2e_step(s, first_wait=None):
            b = s % 2
            wl = [e for e in (done[b], first_wait) if e]
            wla = (ctypes.c_void_p * 2)(*wl) if wl else None
            up = ctypes.c_void_p()
            targets = e2e_imgs[b][:1] if world == 1 else e2e_imgs[b]
            for k, (im, (hbuf, reg)) in enumerate(zip(targets, hbufs)):
                last = k == len(hbufs) - 1
                cl.check(L.clEnqueueWriteImage(q_up, im, 0, zero3, reg, 0, 0,
                                               ctypes.c_void_p(hbuf.data_ptr()), len(wl), wla,
                                               ctypes.byref(up) if last else None))
            upa = (ctypes.c_void_p * 1)(up)
            cl.check(L.clEnqueueBarrierWithWaitList(S.queue, 1, upa, None))
            L.clReleaseEvent(up)
            for k in range(2):
                launch(k, e2e_imgs[b])
                cl.check(L.clEnqueueReadBuffer(S.queue, outs[k], 0, 0, nout,
                                               ctypes.c_void_p(host_out[k].data_ptr()), 0, None, None))
            ev = ctypes.c_void_p()
            cl.check(L.clEnqueueMarkerWithWaitList(S.queue, 0, None, ctypes.byref(ev)))
            if done[b]:
                L.clReleaseEvent(done[b])
            done[b] = ev.value

        for s in range(2):
            e2e_step(s)
        S.finish()
        cl.check(L.clFinish(q_up))
        if world > 1:
            dist.barrier()
        steps_e2e = max(4, args.steps // 4)
        a = T.event()
        start = ctypes.c_void_p()  # the first upload starts after the start event
        cl.check(L.clEnqueueMarkerWithWaitList(S.queue, 0, None, ctypes.byref(start)))
        for s in range(steps_e2e):
            e2e_step(s, start.value if s == 0 else None)
        b_ev = T.event()
        torch.cuda.synchronize(dev)
        cl.check(L.clFinish(q_up))
        L.clReleaseEvent(start)
        for e in done:
            if e:
                L.clReleaseEvent(e)
        e2e_ms = a.elapsed_time(b_ev) / steps_e2e
        if world > 1:
            e2e_ms = bdist.max_over_ranks(e2e_ms, red_dev)
        # the downloaded results are this step's: spot-check one row of each pass
        for k in range(2):
            dev_row = S.read(outs[k], N2D * 16, np.uint8, offset=N2D * 16 * 777)
            assert np.array_equal(host_out[k].numpy()[N2D * 16 * 777:N2D * 16 * 778], dev_row)
        e2e = {"value": world * samples_step / (e2e_ms * 1e-3) / 1e9, "unit": "Gsamples/s",
               "ms_per_step": e2e_ms, "h2d_bytes_per_step": int(sum(h[0].numel() for h in hbufs)),
               "d2h_bytes_per_step": 2 * nout,
               "pipeline": "uploads on a second queue into two image copies, overlapping the previous "
                           "step's downloads (event-ordered)"}
        S.release(*[im for im in set(e2e_imgs[1])])
        L.clReleaseCommandQueue(q_up)

    secondary = None
    if not args.no_secondary:
        secondary = run_secondary(S, L, T, torch, dev, hbm_peak, args)
    if world > 1 and not args.no_p2p:
        secondary = secondary or {}
        secondary["p2p_ring_migrate"] = run_p2p_ring(S, L, T, torch, dev, red_dev, rank, world)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:  # the oracle baseline: N = 1 only
        try:
            threads = os.cpu_count() or 1
            rate, rows, dt = oracle_rate(codes, args.cpu_seconds, threads)
            cpu = {"value": rate, "unit": "Gsamples/s", "cores": threads, "kind": "oracle",
                   "sample": f"{rows} rows x {N2D} columns of each pass (REPEAT, MIRRORED), "
                             f"{dt:.1f} s on {threads} threads"}
        except ImportError:
            cpu = None

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "Gsamples/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (numpy default_rng seed 20151115; U[0,1) RGBA32F texels)",
            "config": {"workload": WORKLOAD, "image": "4096x4096 RGBA32F (256 MiB)",
                       "samples_per_step": samples_step, "launches_per_step": 2,
                       "timing": ("step: K steps between two events; kernel_ms: K back-to-back "
                                  "launches of that kernel between two events, right after"),
                       "step": ("REPEAT read on the queue, MIRRORED read on a second queue of "
                                "the device, joined by a marker and a barrier every step"),
                       "parallelism": ("single GPU" if world == 1 else
                                       f"row-sharded x{world}: global {Hg}x{N2D} image, "
                                       f"4096 output rows per GPU from shards of "
                                       f"{shard_rows} texel rows (REPEAT, MIRRORED)"),
                       "l2": "no flush: 768 MiB working set > 126 MB L2", "parity": parity},
            "roofline": {"bound": "hbm", "achieved": achieved[dom], "peak": hbm_peak, "unit": "GB/s",
                         "frac": achieved[dom] / hbm_peak, "traffic": traffic,
                         "kernel": ["k_sample_grid<2D RGBA32F LINEAR REPEAT>",
                                    "k_sample_grid<2D RGBA32F LINEAR MIRRORED>"][dom],
                         "kernel_ms": pass_ms[dom], "algorithmic_bytes_per_launch": alg[dom],
                         "peak_source": peak_src,
                         "per_pass": [{"mode": m, "ms": pass_ms[k], "algorithmic_bytes": alg[k],
                                       "GB/s": achieved[k], "frac": achieved[k] / hbm_peak}
                                      for k, m in enumerate(("repeat", "mirrored"))],
                         "step_frac": sum(alg) / (sum(pass_ms) * 1e-3) / 1e9 / hbm_peak},
            "cpu_baseline": cpu, "e2e": e2e, "clocks": clk, "gpu_launches": gpu_launches,
            "secondary": secondary,
        }
        print(json.dumps(line), flush=True)
    L.clReleaseCommandQueue(q_two)
    S.release(*set(imgs), *outs)
    for s in smps:
        L.clReleaseSampler(s)
    S.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_p2p_ring(S, L, T, torch, dev, red_dev, rank, world):
    """Config 5 migration, one process per GPU: every rank exports an
    IPC-exportable band buffer, opens its left neighbour's band over CUDA IPC
    and pulls it with the library's SM copy kernel (clEnqueueCopyBuffer on the
    peer mapping -> NVLink reads), all ranks concurrently (ring shift).  Band =
    32768^2 RGBA32F / G rows, capped at 2 GiB.  Reported: GB/s per GPU (the
    slowest rank) and its fraction of the 770 GB/s measured peer-copy figure
    (B200_PROFILING.md; 900 GB/s nominal)."""
    from paper_conf_sc_kimdjjl15_b200 import cl
    from paper_conf_sc_kimdjjl15_b200 import dist as bdist
    band = min((32768 * 32768 * 16) // world, 2 << 30)
    err = ctypes.c_int32()
    mine = L.clCreateBuffer(S.ctx, cl.CL_MEM_READ_WRITE | cl.B2CL_MEM_IPC_EXPORTABLE, band, None,
                            ctypes.byref(err))
    cl.check(err.value, "clCreateBuffer(IPC)")
    pat = np.array([rank & 0xFF], np.uint8)
    cl.check(L.clEnqueueFillBuffer(S.queue, mine, pat.ctypes.data, 1, 0, band, 0, None, None))
    S.finish()
    h = (ctypes.c_uint8 * 64)()
    cl.check(L.b2clGetMemIpcHandle(mine, h), "b2clGetMemIpcHandle")
    handles = bdist.exchange_bytes(bytes(h))
    left, _ = bdist.ring_neighbors(rank, world)
    hl = (ctypes.c_uint8 * 64).from_buffer_copy(handles[left])
    peer = L.b2clCreateBufferFromIpcHandle(S.ctx, S.device, hl, band, ctypes.byref(err))
    cl.check(err.value, "b2clCreateBufferFromIpcHandle")
    local = S.buffer(band)

    def pull():
        cl.check(L.clEnqueueCopyBuffer(S.queue, peer, local, 0, 0, band, 0, None, None))
    pull()
    S.finish()
    ok = bool(np.all(S.read(local, 4096) == (left & 0xFF)))  # data equality (O9) on a sample
    import torch.distributed as dist
    dist.barrier()
    ms = _time_launches(T, torch, dev, pull, 5)
    ms = bdist.max_over_ranks(ms, red_dev)
    gbs = band / (ms * 1e-3) / 1e9
    S.release(local, peer, mine)
    return {"band_bytes": band, "ms": ms, "GB/s_per_gpu": gbs, "frac_of_770": gbs / 770.0,
            "pattern": "ring shift, all ranks pull from rank-1 concurrently",
            "data_check": "ok" if ok else "MISMATCH",
            "link": ("NVLink P2P (peer GPU memory over CUDA IPC)" if red_dev is not None else
                     "same GPU (multi-rank rehearsal with ranks sharing one device: not NVLink)")}


def _time_launches(T, torch, dev, fn, iters):
    fn()
    torch.cuda.synchronize(dev)
    a = T.event()
    for _ in range(iters):
        fn()
    b = T.event()
    torch.cuda.synchronize(dev)
    return a.elapsed_time(b) / iters


def _time_graph(T, torch, dev, fn, calls, nbytes):
    """`calls` enqueues captured into one CUDA graph on the queue's stream and
    replayed 10 times on that stream between two events: per-copy ms without
    host overhead.  Returns {"unavailable": why} if capture fails."""
    try:
        torch.cuda.synchronize(dev)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=T.stream):
            for _ in range(calls):
                fn()
        with torch.cuda.stream(T.stream):
            g.replay()
            torch.cuda.synchronize(dev)
            a = T.event()
            for _ in range(10):
                g.replay()
            b = T.event()
        torch.cuda.synchronize(dev)
        ms = a.elapsed_time(b) / (10 * calls)
        return {"ms": ms, "GB/s_copied": nbytes / ms / 1e6, "copies_per_graph": calls,
                "l2_resident": 2 * nbytes < 120e6}  # replays re-read the same bytes
    except Exception as exc:  # an extra measurement, never fatal
        torch.cuda.synchronize(dev)
        return {"unavailable": str(exc).splitlines()[0][:200]}


def run_secondary(S, L, T, torch, dev, hbm_peak, args):
    from paper_conf_sc_kimdjjl15_b200 import cl, synth
    res = {}
    # config 2 map (B): 30 deg rotation about the centre, unit scale (the general
    # kernel, warps on 8 x 4 output patches); algorithmic bytes = the distinct
    # texels with a non-zero tap weight (counted on the host) x 16 B + 16 B out
    n2 = 4096
    img2 = S.image(cl.CL_RGBA, cl.CL_FLOAT, n2, n2,
                   host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n2, n2))
    out2 = S.buffer(n2 * n2 * 16)
    A2 = (ctypes.c_float * 12)(*synth.affine_rotate_2d(n2, n2, 30.0).tolist())
    d2 = cl.sz3((n2, n2, 1))
    for name, addr in (("repeat", cl.CL_ADDRESS_REPEAT), ("mirrored", cl.CL_ADDRESS_MIRRORED_REPEAT)):
        smp2 = S.sampler(True, addr, cl.CL_FILTER_LINEAR)
        ms = _time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueReadImageGrid(
            S.queue, img2, smp2, 0, A2, d2, 4, out2, 0, 0, None, None)), 10)
        e = {"Gsamples/s": n2 * n2 / ms / 1e6, "ms": ms, "map": "rotation 30 deg (B)",
             "kernel": "k_sample_grid (8x4 output patch per warp)"}
        texels = _distinct_texels_2d(synth.affine_rotate_2d(n2, n2, 30.0), n2, n2, name)
        b2 = 16 * texels + 16 * n2 * n2
        e.update({"GB/s": b2 / ms / 1e6, "hbm_frac": b2 / ms / 1e6 / hbm_peak, "algorithmic_bytes": b2,
                  "distinct_texels": texels})
        res[f"c2_map_b_{name}"] = e
        L.clReleaseSampler(smp2)
    # config 5's image on one GPU (the N = 1 point of its row-sharded scaling):
    # 32768^2 RGBA32F, 16 GiB, map (A), both samplers.  Its rows are the
    # 4096-row seeded band above copied 8 times (device copies; the texel
    # addresses, and so the traffic, are those of a 16 GiB image)
    n5 = 32768
    img5 = S.image(cl.CL_RGBA, cl.CL_FLOAT, n5, n5)
    for by in range(0, n5, n2):
        for bx in range(0, n5, n2):
            cl.check(L.clEnqueueCopyImage(S.queue, img2, img5, cl.sz3((0, 0, 0)), cl.sz3((bx, by, 0)),
                                          cl.sz3((n2, n2, 1)), 0, None, None))
    S.release(img2, out2)
    out5 = S.buffer(n5 * n5 * 16)
    A5 = (ctypes.c_float * 12)(*synth.affine_translate_2d(n5, n5).tolist())
    d5 = cl.sz3((n5, n5, 1))
    smp5 = [S.sampler(True, a, cl.CL_FILTER_LINEAR)
            for a in (cl.CL_ADDRESS_REPEAT, cl.CL_ADDRESS_MIRRORED_REPEAT)]

    def step5():
        for k in range(2):
            cl.check(L.b2clEnqueueReadImageGrid(S.queue, img5, smp5[k], 0, A5, d5, 4, out5, 0, 0, None, None))
    ms = _time_launches(T, torch, dev, step5, 3)
    res["c5_image_32768_1gpu"] = {"Gsamples/s": 2 * n5 * n5 / ms / 1e6, "ms_per_step": ms,
                                  "step": "REPEAT + MIRRORED_REPEAT reads of map (A), 2 x 1.07 G samples",
                                  "image": "32768x32768 RGBA32F (16 GiB)"}
    for smp in smp5:
        L.clReleaseSampler(smp)
    S.release(img5, out5)
    # config 3: 512^3 R32F trilinear, stencil map, CLAMP_TO_EDGE
    n3 = 512
    g = synth.rng(3)
    vol = S.image(cl.CL_R, cl.CL_FLOAT, n3, n3, n3,
                  host=synth.image_codes(g, cl.CL_R, cl.CL_FLOAT, n3, n3, n3))
    out3 = S.buffer(n3 ** 3 * 4)
    smp3 = S.sampler(True, cl.CL_ADDRESS_CLAMP_TO_EDGE, cl.CL_FILTER_LINEAR)
    A3 = (ctypes.c_float * 12)(*synth.affine_stencil_3d(n3).tolist())
    d3 = cl.sz3((n3, n3, n3))
    ms = _time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueReadImageGrid(
        S.queue, vol, smp3, 0, A3, d3, 1, out3, 0, 0, None, None)), 10)
    byt = 2 * n3 ** 3 * 4
    res["c3_trilinear_512"] = {"Gsamples/s": n3 ** 3 / ms / 1e6, "ms": ms, "GB/s": byt / ms / 1e6,
                               "hbm_frac": byt / ms / 1e6 / hbm_peak, "map": "stencil (A)",
                               "kernel": "k_sample_grid_vol (256x16 tiles, per-row cp.async.bulk ring)",
                               "algorithmic_bytes": byt}
    A3b = (ctypes.c_float * 12)(*synth.affine_rotate_3d(n3, 20.0).tolist())
    ms = _time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueReadImageGrid(
        S.queue, vol, smp3, 0, A3b, d3, 1, out3, 0, 0, None, None)), 10)
    # map (B) is a rotation about z: the texels it taps with a non-zero weight
    # are (the xy taps of one slice) x (the z taps), counted on the host
    Arot = synth.affine_rotate_3d(n3, 20.0)
    txy = _distinct_texels_2d(Arot, n3, n3, "clamp_to_edge")
    tz = _axis_taps(Arot[10], Arot[11], n3, n3, "clamp_to_edge").size
    bytr = 4 * txy * tz + 4 * n3 ** 3
    res["c3_trilinear_512_rotated"] = {"Gsamples/s": n3 ** 3 / ms / 1e6, "ms": ms, "GB/s": bytr / ms / 1e6,
                                       "hbm_frac": bytr / ms / 1e6 / hbm_peak, "algorithmic_bytes": bytr,
                                       "distinct_texels": txy * tz,
                                       "map": "volume-render rotation (B), 20 deg about z",
                                       "kernel": "k_sample_grid_volr (64x32 tiles, tensor-TMA footprint box)"}
    S.release(vol, out3)
    L.clReleaseSampler(smp3)
    # config 4: 8 GiB pitched CopyBufferRect (src padded, dst tight) and a misaligned variant
    region = (16384, 2048, 256)
    srp, ssp = 16512, 2056 * 16512
    S_bytes = region[0] * region[1] * region[2]
    src = S.buffer(ssp * region[2])
    dst = S.buffer(S_bytes)
    zero = cl.sz3((0, 0, 0))
    ms = _time_launches(T, torch, dev, lambda: cl.check(L.clEnqueueCopyBufferRect(
        S.queue, src, dst, zero, zero, cl.sz3(region), srp, ssp, 0, 0, 0, None, None)), 5)
    res["c4_copy_rect_8GiB"] = {"GB/s_copied": S_bytes / ms / 1e6, "ms": ms,
                                "hbm_frac": 2 * S_bytes / ms / 1e6 / hbm_peak}
    reg2 = (16384, 2048, 255)
    ms = _time_launches(T, torch, dev, lambda: cl.check(L.clEnqueueCopyBufferRect(
        S.queue, src, dst, cl.sz3((3, 0, 0)), zero, cl.sz3(reg2), 16387, 16387 * 2056, 0, 0, 0, None,
        None)), 5)
    b2 = reg2[0] * reg2[1] * reg2[2]
    res["c4_copy_rect_misaligned"] = {"GB/s_copied": b2 / ms / 1e6, "ms": ms,
                                      "hbm_frac": 2 * b2 / ms / 1e6 / hbm_peak}
    pat = np.arange(16, dtype=np.uint8)
    ms = _time_launches(T, torch, dev, lambda: cl.check(L.clEnqueueFillBuffer(
        S.queue, dst, pat.ctypes.data, 16, 0, S_bytes, 0, None, None)), 5)
    res["c4_fill_8GiB"] = {"GB/s": S_bytes / ms / 1e6, "ms": ms, "hbm_frac": S_bytes / ms / 1e6 / hbm_peak}
    S.release(src)
    # CopyImageToBuffer sweep 4 KiB .. 8 GiB (RGBA32F 2D images shaped to the size)
    sweep = []
    for lg in range(12, 34, 3 if not args.full_sweep else 1):
        nbytes = 1 << lg
        w = min(32768, max(1, nbytes // 16))
        h = max(1, nbytes // 16 // w)
        im = S.image(cl.CL_RGBA, cl.CL_FLOAT, w, h)
        it = 20 if nbytes < (1 << 28) else 5
        ms = _time_launches(T, torch, dev, lambda: cl.check(L.clEnqueueCopyImageToBuffer(
            S.queue, im, dst, zero, cl.sz3((w, h, 1)), 0, 0, None, None)), it)
        e = {"bytes": w * h * 16, "ms": ms, "GB/s_copied": w * h * 16 / ms / 1e6,
             "hbm_frac": 2 * w * h * 16 / ms / 1e6 / hbm_peak}
        if nbytes < (1 << 26):
            # below ~64 MiB one call is launch-bound: also time the same calls
            # captured once into a CUDA graph on the queue's stream and replayed
            # there (no Python / host enqueue cost between the copies)
            e["graph"] = _time_graph(T, torch, dev, lambda: cl.check(L.clEnqueueCopyImageToBuffer(
                S.queue, im, dst, zero, cl.sz3((w, h, 1)), 0, 0, None, None)), 20, w * h * 16)
        sweep.append(e)
        S.release(im)
    res["c4_copy_image_to_buffer_sweep"] = sweep
    S.release(dst)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="b2cl", choices=["b2cl", "reference"])
    ap.add_argument("--no-secondary", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--full-sweep", action="store_true")
    ap.add_argument("--no-p2p", action="store_true", help="skip the N>1 NVLink ring migration")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return run_reference(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
