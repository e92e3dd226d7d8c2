# per variant (VARIANTS="name:-DFOO=1;..."): build libsel, time it with bench.py, and one ncu pass over the
# kernels matching NCUK (default k_model_fused) of the last bench step: duration, executed instructions,
# issue activity, occupancy, DRAM bytes, local-memory traffic, stall reasons
mkdir -p gpurun_out
python __graft_entry__.py
NCUK=${NCUK:-k_model_fused}
IFS=';' read -ra VS <<< "$VARIANTS"
for v in "${VS[@]}"; do
  name="${v%%:*}"; defs="${v#*:}"
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared $defs \
     -o /tmp/libsel_$name.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu
  for rep in 1 2; do
    SEL_LIBSEL=/tmp/libsel_$name.so timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-next \
       > gpurun_out/bench_${name}_$rep.json 2>> gpurun_out/variants.err
  done
  SEL_LIBSEL=/tmp/libsel_$name.so timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum,smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio,smsp__average_warp_latency_issue_stalled_short_scoreboard.ratio,smsp__average_warp_latency_issue_stalled_wait.ratio,smsp__average_warp_latency_issue_stalled_math_pipe_throttle.ratio,smsp__average_warp_latency_issue_stalled_no_instruction.ratio,smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio,smsp__inst_executed_pipe_fp64.sum \
      --clock-control none -k "regex:$NCUK" -s 1 -c 2 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-next \
      > gpurun_out/ncu_${name}.csv 2>> gpurun_out/variants.err
  python - "$name" <<'PY'
import json, sys, glob, csv, io, os
name = sys.argv[1]
for f in sorted(glob.glob(f"gpurun_out/bench_{name}_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(name, f[-6:], "ms/step %.3f" % d["ms_per_step"], " ".join("%s %.3f" % (k, v) for k, v in d["kernel_ms"].items()))
    except Exception as e:
        print(name, f, "failed", e)
txt = open(f"gpurun_out/ncu_{name}.csv").read()
i = txt.find('"ID"')
rows = list(csv.reader(io.StringIO(txt[i:]))) if i >= 0 else []
if rows:
    h = rows[0]
    for r in rows[1:]:
        print("   ", r[h.index("ID")], r[h.index("Kernel Name")][:20], r[h.index("Metric Name")], r[h.index("Metric Value")])
PY
done
