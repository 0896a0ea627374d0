#!/usr/bin/env python
"""Summarise ncu artefacts into profiles/ (tracked).

  python profiles/summarize.py full <report.ncu-rep> <out.md> [alg_bytes_per_launch]
  python profiles/summarize.py launches <launches.csv> <out.md>
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed.sum.per_cycle_active",
    "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic", "launch__block_size",
    "launch__grid_size", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__maximum_warps_per_active_cycle_pct",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "lts__t_bytes.sum", "lts__t_sector_hit_rate.pct",
    "sass__inst_executed_local_loads", "sass__inst_executed_local_stores",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_selected_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_sleeping_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_membar_per_issue_active.ratio",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
]


def full(rep, out, alg_bytes=None):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    lines = [f"# ncu --set full summary: `{rep}`", ""]
    data = {}
    for r in rows[2:]:
        name = r[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        lines += [f"## {name[:120]}", "", "| metric | unit | value |", "|---|---|---|"]
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                lines.append(f"| {k} | {units[i]} | {r[i]} |")
                data[k] = (units[i], r[i])
        lines.append("")
    if alg_bytes and "dram__bytes_read.sum" in data:
        def to_bytes(u, v):
            v = float(v.replace(",", ""))
            return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)
        tr = to_bytes(*data["dram__bytes_read.sum"]) + to_bytes(*data["dram__bytes_write.sum"])
        lines += [f"traffic (dram read+write) per launch: {tr:.4e} B; algorithmic: {float(alg_bytes):.4e} B; "
                  f"ratio {tr / float(alg_bytes):.3f}", ""]
        print(json.dumps({"dram_bytes_per_launch": tr, "alg_bytes_per_launch": float(alg_bytes)}))
    open(out, "w").write("\n".join(lines))


def launches(path, out):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    recs = rows[start + 1:]
    ki, mi, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    lines = [f"# ncu launch list (gpu__time_duration.sum, --clock-control none): `{path}`", "",
             "Cold-cache, serialised replays: compare shares, not absolutes.", "",
             "| # | kernel | duration | unit |", "|---|---|---|---|"]
    tot = {}
    for j, r in enumerate(recs):
        if len(r) <= max(ki, vi) or r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki].split("(")[0]
        v = float(r[vi].replace(",", ""))
        lines.append(f"| {j} | {name[:90]} | {v} | {r[ui]} |")
        tot[name] = tot.get(name, 0.0) + v
    s = sum(tot.values())
    lines += ["", "| kernel | total | share |", "|---|---|---|"]
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        lines.append(f"| {k[:90]} | {v:.1f} | {v / s:.3f} |")
    open(out, "w").write("\n".join(lines) + "\n")


if __name__ == "__main__":
    if sys.argv[1] == "full":
        full(sys.argv[2], sys.argv[3], sys.argv[4] if len(sys.argv) > 4 else None)
    else:
        launches(sys.argv[2], sys.argv[3])
