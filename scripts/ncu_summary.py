#!/usr/bin/env python
"""Summarise ncu output for profiles/: the per-kernel launch list (share of
the step) and the key counters of one `--set full` capture of the counting
kernel.  Usage:

    python scripts/ncu_summary.py --launches gpurun_out/launches.csv \
        --report gpurun_out/prof_count.ncu-rep --wa <warp-accesses of that launch> \
        --out profiles/<name>
"""
from __future__ import annotations

import argparse
import collections
import csv
import io
import json
import subprocess

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_uniform.avg.pct_of_peak_sustained_active",
    "sm__cycles_elapsed.avg.per_second", "smsp__average_warp_latency_per_inst_issued.ratio",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__sass_thread_inst_executed_op_integer_pred_on.sum",
]


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) >= 15 and r[0] != "ID"]
    tot = collections.OrderedDict()
    for r in rows:
        name = r[4].split("(")[0].replace("void ", "")
        v = float(r[14])
        t = tot.setdefault(name, [0.0, 0])
        t[0] += v
        t[1] += 1
    T = sum(v[0] for v in tot.values())
    return [{"kernel": k, "launches": c, "total_ms": v / 1e6, "share": v / T}
            for k, (v, c) in sorted(tot.items(), key=lambda x: -x[1][0])]


def report(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = {}
    for i, h in enumerate(hdr):
        if h in KEYS:
            try:
                d[h] = float(vals[i].replace(",", ""))
            except ValueError:
                d[h] = vals[i]
            d[h + ".unit"] = units[i]
    return d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--report")
    ap.add_argument("--wa", type=float, default=0.0, help="warp-accesses analysed by the captured launch")
    ap.add_argument("--out", required=True)
    a = ap.parse_args()
    res = {}
    if a.launches:
        res["launch_list"] = launches(a.launches)
    if a.report:
        r = report(a.report)
        res["count_kernel_full"] = r
        rd = r.get("dram__bytes_read.sum", 0.0)
        wr = r.get("dram__bytes_write.sum", 0.0)
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        rd *= scale.get(r.get("dram__bytes_read.sum.unit", "byte"), 1)
        wr *= scale.get(r.get("dram__bytes_write.sum.unit", "byte"), 1)
        res["dram_bytes_per_launch"] = rd + wr
        if a.wa:
            ins = r.get("smsp__inst_executed.sum", 0.0)
            res["warp_instructions_per_wa"] = ins / a.wa
            res["wa_in_capture"] = a.wa
    with open(a.out + ".json", "w") as f:
        json.dump(res, f, indent=1)
    lines = [f"# ncu summary: {a.out}", ""]
    if "launch_list" in res:
        lines += ["| kernel | launches | total ms | share |", "|---|---|---|---|"]
        lines += [f"| {x['kernel']} | {x['launches']} | {x['total_ms']:.3f} | {100 * x['share']:.2f}% |"
                  for x in res["launch_list"]]
        lines.append("")
    if "count_kernel_full" in res:
        lines += ["| counter (count kernel, --set full) | value |", "|---|---|"]
        for k in KEYS:
            if k in res["count_kernel_full"]:
                lines.append(f"| {k} | {res['count_kernel_full'][k]} {res['count_kernel_full'].get(k + '.unit', '')} |")
        lines.append(f"| dram bytes per launch (read + write) | {res['dram_bytes_per_launch']:.4g} |")
        if "warp_instructions_per_wa" in res:
            lines.append(f"| warp instructions per warp-access | {res['warp_instructions_per_wa']:.2f} |")
    with open(a.out + ".md", "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
