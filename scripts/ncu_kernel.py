#!/usr/bin/env python
"""Key counters + top source lines of every kernel in an ncu --set full report."""
import csv, io, subprocess, sys
rep = sys.argv[1]
M = ("gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__registers_per_thread,"
     "sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,"
     "smsp__inst_executed.sum,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,"
     "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active,"
     "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,"
     "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio,"
     "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio,"
     "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio,"
     "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio,"
     "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio,"
     "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio,"
     "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio,"
     "smsp__thread_inst_executed_per_inst_executed.ratio,dram__throughput.avg.pct_of_peak_sustained_elapsed")
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", M], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
for r in rows[2:]:
    print('----', r[h.index('Kernel Name')][:60])
    for i, k in enumerate(h):
        if '__' in k:
            print(f"   {k:80s} {r[i]}")
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
agg, fn = [], None
for r in csv.reader(io.StringIO(out)):
    if len(r) >= 2 and r[0] == 'File Path':
        fn = r[1].split('/')[-1]
    if len(r) > 8 and r[2] == '-' and r[0].isdigit():
        agg.append((int(r[4]), int(r[7]) if r[7].isdigit() else 0, fn, int(r[0]), r[1][:90]))
tot = sum(a[0] for a in agg) or 1
ti = sum(a[1] for a in agg) or 1
print('samples', tot, 'inst', ti)
for a in sorted(agg, reverse=True)[:top]:
    print(f"{a[0] / tot * 100:5.1f}% {a[1] / ti * 100:5.1f}%i {a[2]}:{a[3]} {a[4]}")
