#!/usr/bin/env python
"""Per-kernel counters of an ncu --set full capture of whole bench steps ->
profiles/ncu_kernels.json (read by bench.py for roofline.traffic and the ncu
context of each region).  The last launch of each kernel name is kept (the
last captured step).

    python scripts/ncu_kernels.py gpurun_out/prof_step.ncu-rep profiles/ncu_kernels.json "<what was captured>"
"""
import csv
import io
import json
import subprocess
import sys

M = {
    "gpu__time_duration.sum": "time_ms",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "smsp__inst_executed.sum": "warp_instructions",
    "smsp__thread_inst_executed_per_inst_executed.ratio": "threads_per_instruction",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active": "alu_pipe_pct",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active": "fma_pipe_pct",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active": "alu_cycles_pct",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active": "fma_cycles_pct",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active": "fp64_cycles_pct",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "sm__warps_active.avg.per_cycle_active": "warps_active_per_cycle",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active": "fp64_pipe_pct",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active": "lsu_pipe_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio": "stall_long_scoreboard",
}
UNIT = {"msecond": 1.0, "ms": 1.0, "usecond": 1e-3, "us": 1e-3, "nsecond": 1e-6, "ns": 1e-6,
        "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def main():
    rep, out, what = sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else ""
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--print-units", "base", "--metrics", ",".join(M)],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    h, units = rows[0], rows[1]
    kernels = {}
    for r in rows[2:]:
        name = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").split("<")[0].replace("sel::", "")
        d = {}
        for k, short in M.items():
            if k not in h:
                continue
            i = h.index(k)
            try:
                v = float(r[i].replace(",", ""))
            except ValueError:
                continue
            u = units[i]
            if short == "time_ms":
                v *= {"second": 1e3, "s": 1e3, "msecond": 1.0, "ms": 1.0, "usecond": 1e-3, "us": 1e-3,
                      "nsecond": 1e-6, "ns": 1e-6}.get(u, 1.0)
            elif short.startswith("dram_") and short != "dram_throughput_pct":
                v *= UNIT.get(u, 1.0)
            d[short] = v
        d["dram_bytes"] = d.get("dram_read", 0.0) + d.get("dram_write", 0.0)
        kernels[name] = d                      # last launch of this name wins
    json.dump({"source": what or rep, "kernels": kernels}, open(out, "w"), indent=1)
    for k, d in kernels.items():
        print(f"{k:18s} {d.get('time_ms', 0):8.3f} ms  dram {d['dram_bytes'] / 1e9:7.3f} GB  issue "
              f"{d.get('issue_active_pct', 0):5.1f}%  thr/inst {d.get('threads_per_instruction', 0):5.1f}")


if __name__ == "__main__":
    main()
