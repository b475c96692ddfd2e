"""Summarise ncu outputs brought back from the GPU box into profiles/.

    python tools/ncu_summary.py launches <launches.csv> <out.md>
    python tools/ncu_summary.py full <prof.ncu-rep> <out.md> [--traffic-json out.json --kernel REGEX]

`launches`: per-kernel count, mean device time (ncu gpu__time_duration.sum,
cold-cache and serialised: compare shares, not absolutes) and share of the
total.  `full`: the key counters of each profiled launch (DRAM bytes, L2 hit
rate, throughput percentages, registers, instruction counts).
"""
import collections
import csv
import io
import json
import re
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "l1tex__t_sector_hit_rate.pct", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed.sum", "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__occupancy_limit_registers", "sm__cycles_elapsed.avg.per_second",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard",
    "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
    "l1tex__t_requests_pipe_lsu_mem_local_op_ld.sum",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
]


def launches(path, out):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.OrderedDict()
    unit = None
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        unit = r[ui]
        agg.setdefault(r[ki], []).append(float(r[vi].replace(",", "")))
    scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "msecond": 1e3, "ms": 1e3}.get(unit, 1.0)
    total = sum(sum(v) for v in agg.values())
    lines = ["| kernel | launches | mean us | share of all launches |", "|---|---|---|---|"]
    for k, v in agg.items():
        lines.append(f"| `{k[:100]}` | {len(v)} | {sum(v) / len(v) * scale:.1f} | "
                     f"{sum(v) / total * 100:.1f}% |")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


def full(path, out, traffic_json=None, kernel=None):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    h, units = r[0], r[1]
    lines = []
    per_kernel = collections.defaultdict(list)
    for row in r[2:]:
        name = row[h.index("Kernel Name")]
        lines.append(f"### `{name[:120]}`")
        lines.append("| metric | value | unit |")
        lines.append("|---|---|---|")
        for k in KEYS:
            if k in h:
                lines.append(f"| {k} | {row[h.index(k)]} | {units[h.index(k)]} |")
        lines.append("")
        if kernel is None or re.search(kernel, name):
            rd = float(row[h.index("dram__bytes_read.sum")].replace(",", ""))
            wr = float(row[h.index("dram__bytes_write.sum")].replace(",", ""))
            u = units[h.index("dram__bytes_read.sum")]
            mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            per_kernel[name].append((rd + wr) * mult)
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))
    if traffic_json and per_kernel:
        name, vals = next(iter(per_kernel.items()))
        json.dump({"kernel": name, "dram_bytes_per_launch": sum(vals) / len(vals),
                   "launches_profiled": len(vals), "source": path}, open(traffic_json, "w"), indent=1)


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        tj = sys.argv[sys.argv.index("--traffic-json") + 1] if "--traffic-json" in sys.argv else None
        kn = sys.argv[sys.argv.index("--kernel") + 1] if "--kernel" in sys.argv else None
        full(sys.argv[2], sys.argv[3], tj, kn)
