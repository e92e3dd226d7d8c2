# ncu --set full (with source) of one kernel (TOPK regex) in a bench step, summarised on the box
mkdir -p gpurun_out
python __graft_entry__.py
TOPK=${TOPK:-k_model_tile}
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$TOPK" -s ${SKIP:-1} -c 1 -o gpurun_out/prof_top \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next ${BENCH_ARGS:-} > gpurun_out/ncu_top.log 2>&1
ncu -i gpurun_out/prof_top.ncu-rep --page details --csv > gpurun_out/top_details.csv 2>&1
ncu -i gpurun_out/prof_top.ncu-rep --page source --csv --print-source sass > gpurun_out/top_source_sass.csv 2>&1
ls -la gpurun_out; tail -3 gpurun_out/ncu_top.log
