# build variants of libsel (VARIANTS="name:-DFOO=1 -DBAR=2;name2:...") and time each with bench.py;
# NCUK=regex also records executed instructions / duration / spills of those kernels per variant
mkdir -p gpurun_out
python __graft_entry__.py
IFS=';' read -ra VS <<< "$VARIANTS"
for v in "${VS[@]}"; do
  name="${v%%:*}"; defs="${v#*:}"
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared $defs \
     -o /tmp/libsel_$name.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu
  for rep in 1 2; do
    SEL_LIBSEL=/tmp/libsel_$name.so timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-next \
       > gpurun_out/bench_${name}_$rep.json 2>> gpurun_out/variants.err
  done
  if [ -n "$NCUK" ]; then
    SEL_LIBSEL=/tmp/libsel_$name.so timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum \
      --clock-control none -k "regex:$NCUK" -s 2 -c 4 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-next \
      > gpurun_out/ncu_${name}.csv 2>> gpurun_out/variants.err
  fi
  python - "$name" <<'PY'
import json, sys, glob, csv, io, os
name = sys.argv[1]
for f in sorted(glob.glob(f"gpurun_out/bench_{name}_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        rr = d["roofline_by_region"]
        print(name, f[-6:], "ms/step %.3f" % d["ms_per_step"], " ".join("%s %.3f" % (k, v["ms_per_launch"]) for k, v in rr.items()))
    except Exception as e:
        print(name, f, "failed", e)
p = f"gpurun_out/ncu_{name}.csv"
if os.path.exists(p):
    txt = open(p).read()
    i = txt.find('"ID"')
    rows = list(csv.reader(io.StringIO(txt[i:]))) if i >= 0 else []
    if rows:
        h = rows[0]
        for r in rows[1:]:
            print("   ", r[h.index("Kernel Name")][:24], r[h.index("Metric Name")], r[h.index("Metric Value")])
PY
done
