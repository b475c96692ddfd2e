#!/usr/bin/env python
"""bench.py -- headline benchmark of the b2cl hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl b2cl|reference]
    python -m torch.distributed.run --nproc-per-node N ... bench.py --gpus N ...

N = 1 -- BASELINE.json configs[1], the config the metric is quoted on: a
4096x4096 CL_RGBA/CL_FLOAT image, normalized coordinates, LINEAR filter.  One
STEP = read_imagef over the full 4096^2 output grid under REPEAT and again
under MIRRORED_REPEAT (map (A): translate by (0.3, 0.7) px plus a half period
so the wrap seam crosses the output), i.e. two launches, 2 x 16.8 M samples.
`value` = samples / step time in Gsamples/s.

N > 1 -- BASELINE.json configs[4] (C5): ONE 32768x32768 RGBA32F image (16 GiB)
row-sharded over the N ranks (one process per GPU): rank d owns texel rows
[d H/N, (d+1) H/N) in an IPC-exportable band image; for each pass it holds a
shard of exactly the texel rows its output band [d H/N, (d+1) H/N) needs,
filled by cross-device clEnqueueCopyImage region copies from the owners' band
images (NVLink P2P, in place: no whole-object migration); a step = the
REPEAT and MIRRORED reads of its output band, bit-identical to one GPU's
(tests/test_gpu_shards.py).  Strong scaling: `value` = 2 x 32768^2 samples /
the slowest rank's step time.  Also measured: the shard fill (the P2P
exchange) and a ring migration of every owner band to its right neighbour
through clEnqueueMigrateMemObjects, against the copy engines'
(b2clEnqueueCopyBufferEngine) time for the same bytes in the same run -- the
NVLink denominator.  The C5 image on ONE GPU is the `c5_image_32768_1gpu`
secondary of the N = 1 line.

Secondary measurements in the N = 1 line (`secondary`): config 2 map (B)
(30 degree rotation), config 3 (512^3 R32F trilinear, stencil and rotated
maps), config 4 (8 GiB pitched CopyBufferRect, FillBuffer with patterns 1, 4,
16, 128 B, the 22-point CopyImageToBuffer sweep 4 KiB .. 8 GiB) and the host
cost of one enqueue measured from C (tools/enqueue_bench.c), each with its
HBM fraction.

Timing: CUDA events on the queue's stream around every launch, after W
untimed steps, barrier + synchronize on both sides, max over ranks.  The
working set (256 MiB image + 2 x 256 MiB output) exceeds the 126 MB L2, so no
flush is needed between steps.  Clocks are sampled with NVML during the timed
region.  The dominant kernel's DRAM traffic is captured by ncu in a separate
process of this run (`roofline.traffic`).  `--impl reference` times the CPU
oracle (oracle/) on the host cores on a bounded sample of the same workload.
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
_CLOCK_POLLER = r"""
import sys, time
import pynvml
idx, path = int(sys.argv[1]), sys.argv[2]
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(idx)
mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
with open(path, "w", buffering=1) as f:
    f.write(f"max,{mx},0\n")
    while True:
        f.write(f"{time.time():.6f},{pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)},"
                f"{pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)}\n")
        time.sleep(0.002)
"""


class Clocks:
    """SM clock + throttle reasons sampled DURING the timed region: NVML polled
    every 2 ms by a separate process (no GIL shared with the enqueue loop; only
    the samples stamped between start() and stop() count), else
    `nvidia-smi -lms 100` in the background."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index: int):
        self.index = index
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.poller = self.proc = None
        self.t0 = self.t1 = 0.0

    def start(self):
        self.file = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.file.close()
        try:
            import pynvml  # noqa: F401  (the poller needs it)
            self.poller = subprocess.Popen([sys.executable, "-c", _CLOCK_POLLER, str(self.index), self.file.name],
                                           stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
            deadline = time.time() + 20
            while time.time() < deadline and self.poller.poll() is None:
                if len(open(self.file.name).read().splitlines()) >= 2:
                    break
                time.sleep(0.01)
            if self.poller.poll() is not None or len(open(self.file.name).read().splitlines()) < 2:
                self.poller.kill()
                self.poller = None
        except Exception:
            self.poller = None
        if self.poller is None:
            try:
                self.proc = subprocess.Popen(
                    ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,"
                     "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                     "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                     "--format=csv,noheader,nounits", "-lms", "100"],
                    stdout=open(self.file.name, "w"), stderr=subprocess.DEVNULL)
            except (OSError, FileNotFoundError):
                self.proc = None
        self.t0 = time.time()

    def stop(self):
        self.t1 = time.time()
        if self.poller is not None:
            time.sleep(0.005)
            self.poller.terminate()
            try:
                self.poller.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.poller.kill()
            rows = [ln.split(",") for ln in open(self.file.name).read().splitlines() if ln.strip()]
            os.unlink(self.file.name)
            timed, sm = [], []
            for r in rows:
                if r[0] == "max":
                    self.max_mhz = float(r[1])
                    continue
                try:
                    timed.append((float(r[0]), float(r[1]), int(r[2])))
                except (ValueError, IndexError):
                    continue
            inside = [t for t in timed if self.t0 <= t[0] <= self.t1]
            if not inside and timed:  # (a region shorter than the poll period: the nearest sample)
                inside = [min(timed, key=lambda t: abs(t[0] - 0.5 * (self.t0 + self.t1)))]
            for _, mhz, bits in inside:
                sm.append(mhz)
                for n, bit in self.REASONS.items():
                    if bits & bit:
                        self.reasons.add(n)
            src = "nvml 2 ms (separate process)"
        elif self.proc is not None:
            time.sleep(0.15)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
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


def linear_parity(got, exp):
    """Reading A10, the tests' rule (tests/gpu_helpers.py): |g - o| <= 4 ulp(o),
    the 1e-6 absolute floor only near zero (|o| < 2^-10), NaN iff NaN.
    Returns (ok, worst error in ulps over |o| >= 2^-10)."""
    got = np.asarray(got, np.float32)
    exp = np.asarray(exp, np.float32)
    gn, en = np.isnan(got), np.isnan(exp)
    if not np.array_equal(gn, en):
        return False, float("inf")
    g, e = got[~en].astype(np.float64), exp[~en].astype(np.float64)
    err = np.abs(g - e)
    mag = np.abs(exp[~en])
    ulp = np.spacing(mag).astype(np.float64)
    near = mag < 2.0 ** -10
    bad = np.where(near, err > 1e-6, err > 4.0 * ulp)
    worst = float((err[~near] / ulp[~near]).max()) if (~near).any() else 0.0
    return not bad.any(), worst


def ncu_traffic(kernels, which, timeout=300):
    """DRAM bytes (read + write) and duration per launch of each kernel named in
    `kernels`, from ONE ncu capture of tools/prof_kernels.py `which` (a separate
    process of this run; cold cache, clocks not locked).  Returns
    {kernel: {...}} or {"unavailable": why}."""
    import csv
    import io
    import shutil
    ncu = shutil.which("ncu") or "/usr/local/cuda/bin/ncu"
    if not os.path.exists(ncu):
        return {"unavailable": "ncu not found"}
    regex = "|".join(kernels)
    cmd = [ncu, "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum",
           "--clock-control", "none", "--csv", "-k", f"regex:{regex}", "-c", str(len(kernels)),
           sys.executable, os.path.join(ROOT, "tools", "prof_kernels.py"), *which]
    try:
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT)
    except subprocess.TimeoutExpired:
        return {"unavailable": f"ncu timed out after {timeout} s"}
    rows = [ln for ln in r.stdout.splitlines() if ln.startswith('"')]
    if not rows:
        return {"unavailable": f"ncu produced no rows (rc {r.returncode}): " + (r.stderr or r.stdout)[-200:]}
    out = {}
    for rec in csv.DictReader(io.StringIO("\n".join(rows))):
        name = rec.get("Kernel Name", "")
        key = next((k for k in kernels if k in name), name)
        unit, val = rec.get("Metric Unit", ""), float(rec.get("Metric Value", "0").replace(",", ""))
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
                 "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}.get(unit, 1)
        out.setdefault(key, {})[rec.get("Metric Name", "")] = val * scale
    res = {}
    for k, m in out.items():
        rd, wr = m.get("dram__bytes_read.sum", 0.0), m.get("dram__bytes_write.sum", 0.0)
        res[k] = {"dram_read_bytes": rd, "dram_write_bytes": wr, "traffic_bytes": rd + wr,
                  "ncu_us": m.get("gpu__time_duration.sum", 0.0) * 1e6}
    return res or {"unavailable": "no matching kernel in the capture"}


def enqueue_cost():
    """Host cost of one enqueue measured from C (tools/enqueue_bench.c, compiled
    here with gcc; no Python in the loop), beside the CUDA runtime's own cost of
    launching an empty kernel on this host (tools/launch_floor.cu, nvcc): the
    difference is the library's overhead per call."""
    out = {}
    try:
        exe = os.path.join(ROOT, "build", "enqueue_bench")
        os.makedirs(os.path.dirname(exe), exist_ok=True)
        subprocess.run(["gcc", "-O2", "-o", exe, os.path.join(ROOT, "tools", "enqueue_bench.c"), "-ldl"],
                       check=True, capture_output=True)
        r = subprocess.run([exe, os.path.join(ROOT, "paper_conf_sc_kimdjjl15_b200", "libb2cl.so")],
                           capture_output=True, text=True, timeout=120, cwd=ROOT)
        out.update(json.loads(r.stdout.strip().splitlines()[-1]))
        fl = os.path.join(ROOT, "build", "launch_floor")
        subprocess.run([os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc"), "-O2", "-gencode",
                        "arch=compute_100a,code=sm_100a", "-o", fl, os.path.join(ROOT, "tools", "launch_floor.cu")],
                       check=True, capture_output=True, timeout=300)
        r = subprocess.run([fl], capture_output=True, text=True, timeout=120)
        floor = json.loads(r.stdout.strip().splitlines()[-1])
        out["cuda_launch_floor"] = floor
        # (the floor is noisy run to run: the smallest of its launch variants)
        best = min(v for k, v in floor.items() if k.startswith(("launch_us", "cuLaunchKernel_us")))
        out["library_overhead_us"] = out["copy_image_to_buffer_4KiB_us"] - best
    except Exception as exc:  # a secondary measurement, never fatal
        out["unavailable"] = str(exc)[:200]
    return out


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


def run_reference_c5(args, world):
    """The reference arm at N > 1: the oracle on a bounded sample of output rows
    of the GPU arm's workload, C5 (a 32768^2 RGBA32F image, map (A), REPEAT +
    MIRRORED).  The oracle image is a lazily zero-filled 16 GiB array in which
    only the texel rows the sampled output rows tap are written (row j = the
    seeded block row j mod 256, as on the GPU), so host memory holds only those."""
    import oracle as orc
    from paper_conf_sc_kimdjjl15_b200 import synth
    threads = os.cpu_count() or 1
    H = W = args.c5_size
    data = np.zeros((H, W, 4), np.float32)  # calloc'd: untouched pages stay unmapped
    block = synth.image_rows(0x10B5, 0x10DE, W, range(256))[0]
    img = orc.Image(data, W, H, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
    A = synth.affine_translate_2d(W, H)
    filled = set()

    def rows_for(y0, n):
        for mname in ("repeat", "mirrored"):
            for j in _axis_taps(A[5], A[7], n, H, mname, start=y0):
                if int(j) not in filled:
                    data[int(j)] = block[int(j) % 256]
                    filled.add(int(j))

    def run(y0, n):
        rows_for(y0, n)
        for a in (orc.ADDRESS_REPEAT, orc.ADDRESS_MIRRORED_REPEAT):
            orc.read_grid(img, True, a, orc.FILTER_LINEAR, orc.RT_F, A, (W, H, 1), 4, yrange=(y0, y0 + n),
                          nthreads=threads)
    t0 = time.perf_counter()
    run(0, 2)
    per_row = (time.perf_counter() - t0) / 2
    budget = 60.0 / max(1, args.steps + args.warmup)
    rows = int(max(1, min(H // 2, budget / max(per_row, 1e-6))))

    def step(i):
        run((i * 4099) % (H - rows), rows)
    for i in range(args.warmup):
        step(i)
    t0 = time.perf_counter()
    for i in range(args.steps):
        step(args.warmup + i)
    dt = (time.perf_counter() - t0) / args.steps
    value = 2 * rows * W / dt / 1e9
    sample = (f"{rows} output rows x {W} columns of each pass (REPEAT, MIRRORED) per step, from the {W}x{H} "
              f"image (only the tapped texel rows materialised)")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "Gsamples/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": dt * 1e3, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic (seed 20151115 rows, 256-row period)",
            "config": {"workload": C5_WORKLOAD, "sample": sample},
            "cpu_baseline": {"value": value, "unit": "Gsamples/s", "cores": threads, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": "Gsamples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1:  # the GPU arm's N > 1 workload is config 5
        return run_reference_c5(args, world)
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
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1:
        return run_c5(args)
    from paper_conf_sc_kimdjjl15_b200 import build, cl
    build.build()
    gpu = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(gpu)
    dev = torch.device("cuda", gpu)
    stream = torch.cuda.Stream(device=dev)
    S = cl.Session(gpu, stream=stream.cuda_stream)
    L = cl.lib()
    T = Timer(torch, stream)
    hbm_peak, peak_src = peaks()

    # ---- inputs resident in HBM before timing: config 2, one 4096^2 image ----
    from paper_conf_sc_kimdjjl15_b200 import synth
    Af = synth.affine_translate_2d(N2D, N2D)
    A = (ctypes.c_float * 12)(*Af.tolist())
    modes = ("repeat", "mirrored")
    codes = c2_codes()
    img = S.image(cl.CL_RGBA, cl.CL_FLOAT, N2D, N2D, host=codes)
    imgs = [img, img]
    nout = N2D * N2D * 16
    outs = [S.buffer(nout), S.buffer(nout)]
    smps = [S.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR),
            S.sampler(True, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR)]
    origin, region = cl.sz3((0, 0, 0)), cl.sz3((N2D, N2D, 1))

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
    # The REPEAT read is enqueued first (tools/time_c2_queues.py: 135.3 us per
    # step against 137.4 us with the MIRRORED read first; across bench
    # processes the step still varies 135-138.5 us either way).
    q_two = S.queue_for(gpu)

    def step():
        mk, e1 = ctypes.c_void_p(), ctypes.c_void_p()
        cl.check(L.clEnqueueMarkerWithWaitList(S.queue, 0, None, ctypes.byref(mk)))
        launch(0)
        launch(1, queue=q_two, nwait=1, wait=(ctypes.c_void_p * 1)(mk), ev=ctypes.byref(e1))
        cl.check(L.clEnqueueBarrierWithWaitList(S.queue, 1, (ctypes.c_void_p * 1)(e1), None))
        L.clReleaseEvent(mk)
        L.clReleaseEvent(e1)

    # ---- parity spot check of this exact launch configuration (bench as test) ----
    kernels = []
    for k in range(2):
        launch(k)
        kernels.append(cl.last_kernel())  # the kernel the library picked for this pass
    S.finish()
    parity = "skipped (oracle missing)"
    try:
        import oracle as orc
        oimg = orc.Image(codes, N2D, N2D, 1, dims=2, order=orc.RGBA, type=orc.FLOAT)
        worst, nrows = 0.0, 0
        rows = sorted({0, 1, N2D // 2 - 2, N2D // 2 - 1, N2D // 2, N2D // 2 + 1, N2D - 2, N2D - 1}
                      | set(range(97, N2D, 331)))
        for k, a in enumerate((orc.ADDRESS_REPEAT, orc.ADDRESS_MIRRORED_REPEAT)):
            got = S.read(outs[k], nout, np.float32).reshape(N2D, N2D, 4)
            for y in rows:
                exp = orc.read_grid(oimg, True, a, orc.FILTER_LINEAR, orc.RT_F, Af,
                                    (N2D, N2D, 1), 4, yrange=(y, y + 1))[0, 0]
                ok, w = linear_parity(got[y], exp)
                worst = max(worst, w)
                nrows += 1
                if not ok:
                    raise SystemExit(f"bench parity check failed (pass {k}, row {y}, {w:.2f} ulp)")
        parity = (f"ok ({nrows} full rows of both passes vs the oracle incl. the seam and edge rows; "
                  f"worst {worst:.2f} ulp, bound 4 ulp / 1e-6 below 2^-10)")
    except ImportError:
        pass

    # ---- warmup + timed steps ----
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
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
    samples_step = 2 * N2D * N2D
    value = samples_step / (ms_step * 1e-3) / 1e9
    # algorithmic bytes per launch = distinct texels with a non-zero tap weight x 16 B
    # + 16 B output per sample; counted exactly per map on the host
    ncols = [_axis_taps(Af[0], Af[3], N2D, N2D, m).size for m in modes]
    nrows_t = [_axis_taps(Af[5], Af[7], N2D, N2D, m).size for m in modes]
    alg = [ncols[k] * nrows_t[k] * 16 + N2D * N2D * 16 for k in range(2)]
    achieved = [alg[k] / (pass_ms[k] * 1e-3) / 1e9 for k in range(2)]
    dom = 0 if pass_ms[0] >= pass_ms[1] else 1  # the kernel with the larger share of the step

    e2e = None
    if not args.no_e2e:
        e2e = run_e2e_c2(S, L, T, torch, dev, gpu, codes, imgs, outs, launch, samples_step, nout, args)

    secondary = None
    if not args.no_secondary:
        secondary = run_secondary(S, L, T, torch, dev, hbm_peak, args)
    L.clReleaseCommandQueue(q_two)
    S.release(img, *outs)
    for sm in smps:
        L.clReleaseSampler(sm)
    S.close()

    # ---- DRAM traffic of both passes: ncu in a separate process of this run ----
    traffic = {"unavailable": "--no-ncu"}
    if not args.no_ncu:
        traffic = ncu_traffic(kernels, ["c2r", "c2m"])
    traffic_dom = traffic.get(kernels[dom], {}).get("traffic_bytes") if "unavailable" not in traffic else None

    cpu = None
    if not args.no_cpu:  # the oracle baseline: all host cores, and one thread
        try:
            threads = os.cpu_count() or 1
            rate, rows, dt = oracle_rate(codes, args.cpu_seconds, threads)
            rate1, rows1, dt1 = oracle_rate(codes, args.cpu_seconds / 2, 1)
            cpu = {"value": rate, "unit": "Gsamples/s", "cores": threads, "kind": "oracle",
                   "sample": f"{rows} rows x {N2D} columns of each pass (REPEAT, MIRRORED), "
                             f"{dt:.1f} s on {threads} threads",
                   "single_thread": {"value": rate1, "unit": "Gsamples/s", "cores": 1,
                                     "sample": f"{rows1} rows x {N2D} columns of each pass, {dt1:.1f} s"}}
        except ImportError:
            cpu = None

    line = {
        "metric": METRIC, "value": value, "unit": "Gsamples/s", "n_gpus": 1,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic (numpy default_rng seed 20151115; U[0,1) RGBA32F texels)",
        "config": {"workload": WORKLOAD, "image": "4096x4096 RGBA32F (256 MiB)",
                   "samples_per_step": samples_step, "launches_per_step": 2,
                   "kernels": kernels,
                   "timing": ("step: K steps between two events; kernel_ms: K back-to-back "
                              "launches of that kernel between two events, right after"),
                   "step": ("REPEAT read on the queue, MIRRORED read on a second queue of "
                            "the device, joined by a marker and a barrier every step"),
                   "parallelism": "single GPU",
                   "l2": "no flush: 768 MiB working set > 126 MB L2", "parity": parity},
        "roofline": {"bound": "hbm", "achieved": achieved[dom], "peak": hbm_peak, "unit": "GB/s",
                     "frac": achieved[dom] / hbm_peak, "traffic": traffic_dom,
                     "kernel": kernels[dom], "kernel_ms": pass_ms[dom],
                     "algorithmic_bytes_per_launch": alg[dom], "peak_source": peak_src,
                     "traffic_source": ("ncu dram__bytes_read.sum + dram__bytes_write.sum, one cold-cache "
                                        "launch captured in a separate process of this run"),
                     "per_pass": [{"mode": m, "kernel": kernels[k], "ms": pass_ms[k], "algorithmic_bytes": alg[k],
                                   "GB/s": achieved[k], "frac": achieved[k] / hbm_peak,
                                   "ncu": traffic.get(kernels[k]) if "unavailable" not in traffic else traffic}
                                  for k, m in enumerate(modes)],
                     "step_frac": sum(alg) / (sum(pass_ms) * 1e-3) / 1e9 / hbm_peak},
        "cpu_baseline": cpu, "e2e": e2e, "clocks": clk, "gpu_launches": gpu_launches,
        "secondary": secondary,
    }
    print(json.dumps(line), flush=True)
    return 0


def run_e2e_c2(S, L, T, torch, dev, gpu, codes, imgs, outs, launch, samples_step, nout, args):
    """e2e: host buffers through the C-ABI, copies inside the timed region.
    Every step uploads the image from pinned host memory and reads both outputs
    back to pinned host memory.  The copies are the step's bound (256 MiB up,
    512 MiB down over the host link), so the step is pipelined the way an
    OpenCL program would: uploads on a second queue into one of two image
    copies, so step s+1's upload runs while step s's results come down;
    cross-queue order by events only (wait lists)."""
    from paper_conf_sc_kimdjjl15_b200 import cl
    q_up = S.queue_for(gpu)
    hbuf = torch.empty(N2D * N2D * 16, dtype=torch.uint8).pin_memory()
    hbuf.copy_(torch.from_numpy(np.ascontiguousarray(codes).reshape(-1).view(np.uint8)))
    reg = cl.sz3((N2D, N2D, 1))
    im2 = S.image(cl.CL_RGBA, cl.CL_FLOAT, N2D, N2D)
    e2e_imgs = [imgs, [im2, im2]]  # two device copies of the step's image (copy 0 is the resident one)
    host_out = [torch.empty(nout, dtype=torch.uint8).pin_memory() for _ in range(2)]
    zero3 = cl.sz3((0, 0, 0))
    done = [None, None]  # marker event of the last step that read image copy b

    def e2e_step(s, first_wait=None):
        b = s % 2
        wl = [e for e in (done[b], first_wait) if e]
        wla = (ctypes.c_void_p * 2)(*wl) if wl else None
        up = ctypes.c_void_p()
        cl.check(L.clEnqueueWriteImage(q_up, e2e_imgs[b][0], 0, zero3, reg, 0, 0,
                                       ctypes.c_void_p(hbuf.data_ptr()), len(wl), wla, ctypes.byref(up)))
        cl.check(L.clEnqueueBarrierWithWaitList(S.queue, 1, (ctypes.c_void_p * 1)(up), None))
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
    # the downloaded results are this step's: spot-check one row of each pass
    for k in range(2):
        dev_row = S.read(outs[k], N2D * 16, np.uint8, offset=N2D * 16 * 777)
        assert np.array_equal(host_out[k].numpy()[N2D * 16 * 777:N2D * 16 * 778], dev_row)
    S.release(im2)
    L.clReleaseCommandQueue(q_up)
    return {"value": samples_step / (e2e_ms * 1e-3) / 1e9, "unit": "Gsamples/s",
            "ms_per_step": e2e_ms, "h2d_bytes_per_step": int(hbuf.numel()),
            "d2h_bytes_per_step": 2 * nout,
            "pipeline": "uploads on a second queue into two image copies, overlapping the previous "
                        "step's downloads (event-ordered)"}


C5 = 32768
C5_WORKLOAD = ("C5: 32768x32768 CL_RGBA/CL_FLOAT row-sharded over N GPUs (one process per GPU), "
               "normalized, LINEAR, REPEAT + MIRRORED_REPEAT, map (A)")


def _runs(rows, lo, hi):
    """Maximal runs of consecutive global rows inside [lo, hi), in order:
    (first row, end row, index in `rows` of the first row)."""
    out = []
    for i, r in enumerate(rows):
        if not (lo <= r < hi):
            continue
        if out and out[-1][1] == r and out[-1][2] + (out[-1][1] - out[-1][0]) == i:
            out[-1] = (out[-1][0], r + 1, out[-1][2])
        else:
            out.append((r, r + 1, i))
    return out


def shard_copy_plan(rows, band, world):
    """Region copies that fill a shard holding global texel rows `rows` (shard
    row t = rows[t]) from the owners' bands (rank d owns [d*band, (d+1)*band)):
    [(owner d, first row in d's band, first shard row, row count)]."""
    plan = []
    for d in range(world):
        for ga, gb, si in _runs(rows, d * band, (d + 1) * band):
            plan.append((d, ga - d * band, si, gb - ga))
    return plan


def run_c5(args):
    """BASELINE configs[4] at N > 1 (see the module docstring).  Control plane:
    gloo (barrier, max over ranks, 64-byte IPC handles); no NCCL -- nothing
    reduces on the data path."""
    import torch
    import torch.distributed as dist

    from paper_conf_sc_kimdjjl15_b200 import build, cl, synth
    from paper_conf_sc_kimdjjl15_b200 import dist as bdist
    build.build()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ndev = torch.cuda.device_count()
    gpu = local % ndev
    shared = world > ndev  # the single-GPU rehearsal: ranks share a device (IPC, not NVLink)
    torch.cuda.set_device(gpu)
    dist.init_process_group("gloo")
    dev = torch.device("cuda", gpu)
    stream = torch.cuda.Stream(device=dev)
    S = cl.Session(gpu, stream=stream.cuda_stream)
    L = cl.lib()
    T = Timer(torch, stream)
    hbm_peak, peak_src = peaks()
    err = ctypes.c_int32()
    H = W = args.c5_size
    band = H // world
    assert H % world == 0 and band % 256 == 0, "band rows: a multiple of 256"
    r0 = rank * band
    fmt = cl.ImageFormat(cl.CL_RGBA, cl.CL_FLOAT)
    gdesc = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE2D, W, H, 0, 0, 0, 0, 0, 0, None)
    bdesc = cl.ImageDesc(cl.CL_MEM_OBJECT_IMAGE2D, W, band, 0, 0, 0, 0, 0, 0, None)
    rowb = W * 16

    # ---- 1. the owned band: global texel rows [r0, r0 + band), IPC-exportable.
    # Content: global row j = seeded block row (j mod 256) (synth.image_rows): one
    # 128 MiB block uploaded, then doubled in place by clEnqueueCopyImage.
    own = L.b2clCreateImageShard(S.ctx, cl.CL_MEM_READ_WRITE | cl.B2CL_MEM_IPC_EXPORTABLE, ctypes.byref(fmt),
                                 ctypes.byref(gdesc), r0, band, 0, None, ctypes.byref(err))
    cl.check(err.value, "owned band")
    block = synth.image_rows(cl.CL_RGBA, cl.CL_FLOAT, W, range(256))
    cl.check(L.clEnqueueWriteImage(S.queue, own, 1, cl.sz3((0, 0, 0)), cl.sz3((W, 256, 1)), 0, 0,
                                   block.ctypes.data, 0, None, None))
    k = 256
    while k < band:
        n = min(k, band - k)
        cl.check(L.clEnqueueCopyImage(S.queue, own, own, cl.sz3((0, 0, 0)), cl.sz3((0, k, 0)),
                                      cl.sz3((W, n, 1)), 0, None, None))
        k += n
    S.finish()

    # ---- 2. every rank imports every other rank's band (valid copy: the owner's GPU)
    h = (ctypes.c_uint8 * 64)()
    cl.check(L.b2clGetMemIpcHandle(own, h), "b2clGetMemIpcHandle")
    handles = bdist.exchange_bytes(bytes(h))
    bands = []
    for d in range(world):
        if d == rank:
            bands.append(own)
            continue
        hd = (ctypes.c_uint8 * 64).from_buffer_copy(handles[d])
        m = L.b2clCreateImageFromIpcHandle(S.ctx, S.device, cl.CL_MEM_READ_ONLY, ctypes.byref(fmt),
                                           ctypes.byref(bdesc), hd, ctypes.byref(err))
        cl.check(err.value, f"import band {d}")
        bands.append(m)

    # ---- 3. per pass: a shard holding exactly the texel rows output band
    # [r0, r0 + band) taps, filled by region copies from the owners' bands
    Af = synth.affine_translate_2d(W, H)
    A = (ctypes.c_float * 12)(*Af.tolist())
    modes = ("repeat", "mirrored")
    shards, shard_info, copies = [], [], []
    for mname in modes:
        need = _axis_taps(Af[5], Af[7], band, H, mname, start=r0)
        begin, count = circular_interval(need, H)
        rows = [(begin + t) % H for t in range(count)]
        sh = L.b2clCreateImageShard(S.ctx, cl.CL_MEM_READ_WRITE, ctypes.byref(fmt), ctypes.byref(gdesc),
                                    begin, count, 0, None, ctypes.byref(err))
        cl.check(err.value, "shard")
        shards.append(sh)
        plan = [(bands[d], sr, dr, n, d != rank) for d, sr, dr, n in shard_copy_plan(rows, band, world)]
        shard_info.append({"begin": begin, "rows": count,
                           "rows_from_peers": int(sum(n for *_, n, peer in plan if peer)),
                           "copies": len(plan)})
        copies.append(plan)

    def fill():
        for k, plan in enumerate(copies):
            for src, sr, dr, n, _ in plan:
                cl.check(L.clEnqueueCopyImage(S.queue, src, shards[k], cl.sz3((0, sr, 0)), cl.sz3((0, dr, 0)),
                                              cl.sz3((W, n, 1)), 0, None, None), "shard fill")
    fill()
    S.finish()
    # the shards hold the right bytes (global row j = block row j mod 256): sampled rows
    for k, info in enumerate(shard_info):
        for t in sorted({0, info["rows"] // 2, info["rows"] - 1}):
            j = (info["begin"] + t) % H
            got = S.read_image(shards[k], (0, t, 0), (W, 1, 1))
            assert np.array_equal(got.view(np.float32).reshape(W, 4), block[0, j % 256]), ("shard row", k, t)
    dist.barrier()
    fill_ms = _time_launches(T, torch, dev, fill, 3)
    fill_ms = bdist.max_over_ranks(fill_ms)
    fill_bytes = sum(i["rows"] for i in shard_info) * rowb

    # ---- 4. the step: REPEAT and MIRRORED reads of the output band
    nout = W * band * 16
    outs = [S.buffer(nout), S.buffer(nout)]
    smps = [S.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR),
            S.sampler(True, cl.CL_ADDRESS_MIRRORED_REPEAT, cl.CL_FILTER_LINEAR)]
    origin, region = cl.sz3((0, r0, 0)), cl.sz3((W, band, 1))
    kernels = []

    def launch(k):
        cl.check(L.b2clEnqueueReadImageGridRegion(S.queue, shards[k], smps[k], cl.B2CL_RTYPE_FLOAT, A, origin,
                                                  region, 4, outs[k], 0, 0, None, None), "read grid")

    def step():
        launch(0)
        launch(1)

    for k in range(2):
        launch(k)
        kernels.append(cl.last_kernel())
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
    dist.barrier()
    clocks = Clocks(gpu)
    clocks.start()
    n_launch0 = cl.launch_count()
    t0 = T.event()
    for _ in range(args.steps):
        step()
    t1 = T.event()
    torch.cuda.synchronize(dev)
    gpu_launches = cl.launch_count() - n_launch0
    clk = clocks.stop()
    ms_step = bdist.max_over_ranks(t0.elapsed_time(t1) / args.steps)
    dist.barrier()
    samples_step = 2 * W * H  # all ranks
    value = samples_step / (ms_step * 1e-3) / 1e9
    ncols = [_axis_taps(Af[0], Af[3], W, W, m).size for m in modes]
    alg = [ncols[k] * shard_info[k]["rows"] * 16 + nout for k in range(2)]
    pass_ms = []
    for k in range(2):
        pass_ms.append(bdist.max_over_ranks(_time_launches(T, torch, dev, lambda k=k: launch(k), 5)))
    achieved = [alg[k] / (pass_ms[k] * 1e-3) / 1e9 for k in range(2)]
    dom = 0 if pass_ms[0] >= pass_ms[1] else 1

    # ---- 5. migration (a16): every rank migrates its LEFT neighbour's band to
    # its own GPU with clEnqueueMigrateMemObjects (one SM copy kernel pulling the
    # peer mapping over NVLink), all ranks at once (ring shift); and the same
    # peer pull of a 1 GiB buffer by the SM copy kernel and by the copy engines
    left, _ = bdist.ring_neighbors(rank, world)
    hl = (ctypes.c_uint8 * 64).from_buffer_copy(handles[left])
    mig_ms = []
    for it in range(3):
        m = L.b2clCreateImageFromIpcHandle(S.ctx, S.device, cl.CL_MEM_READ_ONLY, ctypes.byref(fmt),
                                           ctypes.byref(bdesc), hl, ctypes.byref(err))
        cl.check(err.value, "import for migration")
        torch.cuda.synchronize(dev)
        dist.barrier()
        a = T.event()
        cl.check(L.clEnqueueMigrateMemObjects(S.queue, 1, (ctypes.c_void_p * 1)(m), 0, 0, None, None))
        b = T.event()
        torch.cuda.synchronize(dev)
        mig_ms.append(a.elapsed_time(b))
        if it == 0:  # data equality (O9): a migrated row equals the owner's
            j = left * band + 5
            got = S.read_image(m, (0, 5, 0), (W, 1, 1))
            assert np.array_equal(got.view(np.float32).reshape(W, 4), block[0, j % 256])
        L.clReleaseMemObject(m)
        S.finish()  # (reaps the deferred free: the mapping closes before the next import)
    mig_ms = bdist.max_over_ranks(float(np.median(mig_ms)))
    band_bytes = band * rowb
    nb = 1 << 30
    mine = L.clCreateBuffer(S.ctx, cl.CL_MEM_READ_WRITE | cl.B2CL_MEM_IPC_EXPORTABLE, nb, None, ctypes.byref(err))
    cl.check(err.value)
    pat = np.array([rank & 0xFF], np.uint8)
    cl.check(L.clEnqueueFillBuffer(S.queue, mine, pat.ctypes.data, 1, 0, nb, 0, None, None))
    S.finish()
    hb = (ctypes.c_uint8 * 64)()
    cl.check(L.b2clGetMemIpcHandle(mine, hb))
    hbs = bdist.exchange_bytes(bytes(hb))
    peer = L.b2clCreateBufferFromIpcHandle(S.ctx, S.device, (ctypes.c_uint8 * 64).from_buffer_copy(hbs[left]), nb,
                                           ctypes.byref(err))
    cl.check(err.value)
    dst = S.buffer(nb)
    dist.barrier()
    sm_ms = bdist.max_over_ranks(_time_launches(T, torch, dev, lambda: cl.check(L.clEnqueueCopyBuffer(
        S.queue, peer, dst, 0, 0, nb, 0, None, None)), 5))
    ok_sm = bool(np.all(S.read(dst, 4096) == (left & 0xFF)))
    dist.barrier()
    ce_ms = bdist.max_over_ranks(_time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueCopyBufferEngine(
        S.queue, peer, dst, 0, 0, nb, 0, None, None)), 5))
    dist.barrier()
    link = ("same GPU (rehearsal: ranks share one device, CUDA IPC within it -- not NVLink)" if shared
            else "NVLink P2P (peer GPU memory over CUDA IPC)")
    migration = {
        "pattern": "ring shift: every rank migrates its left neighbour's band concurrently",
        "band_bytes": band_bytes, "migrate_ms": mig_ms, "migrate_GB/s_per_gpu": band_bytes / (mig_ms * 1e-3) / 1e9,
        "call": "clEnqueueMigrateMemObjects (SM copy kernel reading the peer mapping)",
        "p2p_1GiB": {"sm_kernel_ms": sm_ms, "sm_kernel_GB/s": nb / (sm_ms * 1e-3) / 1e9,
                     "copy_engine_ms": ce_ms, "copy_engine_GB/s": nb / (ce_ms * 1e-3) / 1e9,
                     "sm_vs_copy_engine": ce_ms / sm_ms, "data_check": "ok" if ok_sm else "MISMATCH"},
        "frac_of_copy_engine": (band_bytes / (mig_ms * 1e-3)) / (nb / (ce_ms * 1e-3)),
        "nominal_GB/s": 900.0, "link": link}

    # ---- 6. e2e: each step uploads the rank's band from pinned host memory, the
    # ranks meet at a (host) barrier, the shards are filled over P2P, the two
    # reads run, and both outputs come back to pinned host memory
    e2e = None
    if not args.no_e2e:
        try:
            import psutil
            need = (band_bytes + nout) * world
            room = psutil.virtual_memory().available > 2 * need
        except ImportError:
            room = True
        if room:
            hb_in = torch.empty(band_bytes, dtype=torch.uint8).pin_memory()
            blk = torch.from_numpy(block.reshape(-1).view(np.uint8))
            hb_in.view(-1, blk.numel()).copy_(blk.expand(band // 256, -1))
            hb_out = torch.empty(nout, dtype=torch.uint8).pin_memory()
            zero3, breg = cl.sz3((0, 0, 0)), cl.sz3((W, band, 1))

            def e2e_step():
                cl.check(L.clEnqueueWriteImage(S.queue, own, 1, zero3, breg, 0, 0,
                                               ctypes.c_void_p(hb_in.data_ptr()), 0, None, None))
                dist.barrier()  # every owner's band is in place before the peers read it
                fill()
                step()
                for k in range(2):
                    cl.check(L.clEnqueueReadBuffer(S.queue, outs[k], 0, 0, nout,
                                                   ctypes.c_void_p(hb_out.data_ptr()), 0, None, None))
                S.finish()
                dist.barrier()  # nobody overwrites its band while a peer may still copy from it
            e2e_step()
            ns = max(2, min(4, args.steps // 8))
            torch.cuda.synchronize(dev)
            dist.barrier()
            a = T.event()
            for _ in range(ns):
                e2e_step()
            b = T.event()
            torch.cuda.synchronize(dev)
            e2e_ms = bdist.max_over_ranks(a.elapsed_time(b) / ns)
            e2e = {"value": samples_step / (e2e_ms * 1e-3) / 1e9, "unit": "Gsamples/s", "ms_per_step": e2e_ms,
                   "h2d_bytes_per_step": band_bytes, "d2h_bytes_per_step": 2 * nout,
                   "per": "rank (each rank's own copies)",
                   "pipeline": ("upload own band (pinned) -> barrier -> P2P shard fill -> 2 reads -> "
                                "download both outputs (pinned) -> barrier")}
        else:
            e2e = {"unavailable": "not enough host memory for the pinned band and output buffers"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "Gsamples/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (numpy default_rng seed 20151115 rows; U[0,1) RGBA32F texels, 256-row period)",
            "config": {"workload": C5_WORKLOAD, "image": f"{W}x{H} RGBA32F ({W * H * 16 / 2**30:.0f} GiB)",
                       "samples_per_step": samples_step, "launches_per_step_per_rank": 2, "kernels": kernels,
                       "parallelism": (f"row-sharded x{world}: rank d owns texel rows [d*{band}, (d+1)*{band}) and "
                                       f"reads output rows [d*{band}, (d+1)*{band}) from per-pass shards "
                                       f"{[(i['begin'], i['rows']) for i in shard_info]} (rank 0)"),
                       "shards": shard_info, "l2": "no flush: working set >> 126 MB L2",
                       "parity": ("shard contents checked byte-exact on sampled rows; shard reads are "
                                  "bit-identical to whole-image reads (tests/test_gpu_shards.py), which are "
                                  "checked against the oracle (tests/test_gpu_config5.py)"),
                       "control_plane": "torch.distributed gloo (barrier, max over ranks, IPC handles)"},
            "roofline": {"bound": "hbm", "achieved": achieved[dom], "peak": hbm_peak, "unit": "GB/s",
                         "frac": achieved[dom] / hbm_peak, "traffic": None, "kernel": kernels[dom],
                         "kernel_ms": pass_ms[dom], "algorithmic_bytes_per_launch": alg[dom],
                         "peak_source": peak_src, "per": "rank (slowest)",
                         "per_pass": [{"mode": m, "kernel": kernels[k], "ms": pass_ms[k], "algorithmic_bytes": alg[k],
                                       "GB/s": achieved[k], "frac": achieved[k] / hbm_peak}
                                      for k, m in enumerate(modes)]},
            "exchange": {"shard_fill_ms": fill_ms, "shard_fill_bytes_per_rank": fill_bytes,
                         "shard_fill_GB/s_per_gpu": fill_bytes / (fill_ms * 1e-3) / 1e9,
                         "call": "clEnqueueCopyImage region copies from the owners' bands (in place, P2P)"},
            "migration": migration,
            "cpu_baseline": None, "e2e": e2e, "clocks": clk, "gpu_launches": gpu_launches,
        }
        print(json.dumps(line), flush=True)
    for o in [*outs, *shards, dst, peer, mine]:
        L.clReleaseMemObject(o)
    for d, m in enumerate(bands):
        if d != rank:
            L.clReleaseMemObject(m)
    S.finish()
    dist.barrier()
    L.clReleaseMemObject(own)
    for sm in smps:
        L.clReleaseSampler(sm)
    S.close()
    dist.destroy_process_group()
    return 0


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
             "kernel": cl.last_kernel()}
        texels = _distinct_texels_2d(synth.affine_rotate_2d(n2, n2, 30.0), n2, n2, name)
        b2 = 16 * texels + 16 * n2 * n2
        e.update({"GB/s": b2 / ms / 1e6, "hbm_frac": b2 / ms / 1e6 / hbm_peak, "algorithmic_bytes": b2,
                  "distinct_texels": texels})
        res[f"c2_map_b_{name}"] = e
        L.clReleaseSampler(smp2)
    # the coordinate-list form of the built-in (b2clEnqueueReadImageSamples,
    # k_sample_list: a float2 per sample, the way a translated kernel passes
    # arbitrary coordinates) on config 2's image: the coordinates of map (A)
    # and map (B) in output order, precomputed and resident; algorithmic bytes
    # = 8 B coordinate + 16 B output per sample + 16 B per distinct texel
    f32 = np.float32
    xs = np.arange(n2, dtype=f32)[None, :]
    ys = np.arange(n2, dtype=f32)[:, None]
    for mname, Al in (("a", synth.affine_translate_2d(n2, n2)), ("b", synth.affine_rotate_2d(n2, n2, 30.0))):
        cs = ((Al[0] * xs).astype(f32) + (Al[1] * ys).astype(f32)).astype(f32) + Al[3]
        ct = ((Al[4] * xs).astype(f32) + (Al[5] * ys).astype(f32)).astype(f32) + Al[7]
        co = np.ascontiguousarray(np.stack([cs.astype(f32), ct.astype(f32)], -1).reshape(-1, 2))
        del cs, ct
        cbuf = S.buffer(co.nbytes, co)
        del co
        for name, addr in (("repeat", cl.CL_ADDRESS_REPEAT), ("mirrored", cl.CL_ADDRESS_MIRRORED_REPEAT)):
            smpl = S.sampler(True, addr, cl.CL_FILTER_LINEAR)
            ms = _time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueReadImageSamples(
                S.queue, img2, smpl, cl.B2CL_RTYPE_FLOAT, cl.B2CL_COORD_FLOAT, cbuf, 0, n2 * n2, out2, 0, 0,
                None, None)), 10)
            texels = (distinct_texels_separable(Al, n2, n2, name) if mname == "a"
                      else res[f"c2_map_b_{name}"]["distinct_texels"])
            bl = 24 * n2 * n2 + 16 * texels
            res[f"c2_list_map_{mname}_{name}"] = {
                "Gsamples/s": n2 * n2 / ms / 1e6, "ms": ms, "kernel": cl.last_kernel(),
                "coords": "float2 list (map A translate)" if mname == "a" else "float2 list (map B, 30 deg)",
                "GB/s": bl / ms / 1e6, "hbm_frac": bl / ms / 1e6 / hbm_peak, "algorithmic_bytes": bl,
                "distinct_texels": texels}
            L.clReleaseSampler(smpl)
        S.release(cbuf)
    # the same rotated read from TILED storage (B2CL_MEM_TILED_IMAGE, 8 x 8-texel
    # 1 KiB tiles; the one-thread-per-sample kernel), against that kernel on the
    # pitched image: does block-linear storage help the rotated gathers?
    imgt = S.image(cl.CL_RGBA, cl.CL_FLOAT, n2, n2, host=synth.image_codes(synth.rng(2), cl.CL_RGBA, cl.CL_FLOAT, n2, n2),
                   flags=cl.CL_MEM_READ_WRITE | cl.B2CL_MEM_TILED_IMAGE)
    smp2 = S.sampler(True, cl.CL_ADDRESS_REPEAT, cl.CL_FILTER_LINEAR)
    ms_t = _time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueReadImageGrid(
        S.queue, imgt, smp2, 0, A2, d2, 4, out2, 0, 0, None, None)), 10)
    kt = cl.last_kernel()
    b2 = res["c2_map_b_repeat"]["algorithmic_bytes"]
    res["c2_map_b_repeat_tiled_storage"] = {"Gsamples/s": n2 * n2 / ms_t / 1e6, "ms": ms_t, "kernel": kt,
                                            "hbm_frac": b2 / ms_t / 1e6 / hbm_peak,
                                            "storage": "B2CL_MEM_TILED_IMAGE (1 KiB tiles of 8 x 8 texels)"}
    S.release(imgt)
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
                               "kernel": cl.last_kernel(), "algorithmic_bytes": byt}
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
                                       "kernel": cl.last_kernel()}
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
    ms_ce = _time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueCopyBufferRectEngine(
        S.queue, src, dst, zero, zero, cl.sz3(region), srp, ssp, 0, 0, 0, None, None)), 5)
    res["c4_copy_rect_8GiB"] = {"GB/s_copied": S_bytes / ms / 1e6, "ms": ms,
                                "hbm_frac": 2 * S_bytes / ms / 1e6 / hbm_peak, "kernel": cl.last_kernel(),
                                "copy_engine_reference": {"call": "b2clEnqueueCopyBufferRectEngine (cudaMemcpy3DAsync)",
                                                          "ms": ms_ce, "GB/s_copied": S_bytes / ms_ce / 1e6,
                                                          "kernel_vs_engine": ms_ce / ms}}
    reg2 = (16384, 2048, 255)
    ms = _time_launches(T, torch, dev, lambda: cl.check(L.clEnqueueCopyBufferRect(
        S.queue, src, dst, cl.sz3((3, 0, 0)), zero, cl.sz3(reg2), 16387, 16387 * 2056, 0, 0, 0, None,
        None)), 5)
    b2 = reg2[0] * reg2[1] * reg2[2]
    res["c4_copy_rect_misaligned"] = {"GB/s_copied": b2 / ms / 1e6, "ms": ms,
                                      "hbm_frac": 2 * b2 / ms / 1e6 / hbm_peak}
    fills = []
    for ps in (1, 4, 16, 128):  # FillBuffer patterns
        pat = np.arange(ps, dtype=np.uint8)
        ms = _time_launches(T, torch, dev, lambda: cl.check(L.clEnqueueFillBuffer(
            S.queue, dst, pat.ctypes.data, ps, 0, S_bytes, 0, None, None)), 5)
        fills.append({"pattern_bytes": ps, "GB/s": S_bytes / ms / 1e6, "ms": ms,
                      "hbm_frac": S_bytes / ms / 1e6 / hbm_peak})
    pat4 = np.arange(4, dtype=np.uint8)
    ms_ce = _time_launches(T, torch, dev, lambda: cl.check(L.b2clEnqueueFillBufferEngine(
        S.queue, dst, pat4.ctypes.data, 4, 0, S_bytes, 0, None, None)), 5)
    fills.append({"pattern_bytes": 4, "reference": "b2clEnqueueFillBufferEngine (cuMemsetD32Async)",
                  "GB/s": S_bytes / ms_ce / 1e6, "ms": ms_ce, "hbm_frac": S_bytes / ms_ce / 1e6 / hbm_peak})
    res["c4_fill_8GiB"] = fills
    S.release(src)
    # CopyImageToBuffer sweep 4 KiB .. 8 GiB (RGBA32F 2D images shaped to the size)
    sweep = []
    for lg in range(12, 34, 1 if not args.short_sweep else 3):  # 22 sizes: 4 KiB .. 8 GiB
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
    # host cost of one enqueue, measured from C (no Python / ctypes in the loop)
    res["host_enqueue_us"] = enqueue_cost()
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
    ap.add_argument("--short-sweep", action="store_true", help="8 of the 22 C4 sweep sizes")
    ap.add_argument("--no-ncu", action="store_true", help="skip the in-run ncu traffic capture")
    ap.add_argument("--c5-size", type=int, default=C5, help="N > 1: the sharded image's side (C5: 32768)")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return run_reference(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
