# full round measurement: build, GPU tests, full bench line, reference arm, launch list, ncu --set full of every
# kernel of a bench step (summarised on the box: the full report exceeds what gpurun copies back), + a
# source-level capture of the top kernel
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1500 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/tests.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2>> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_launch_bench.json 2>&1
rm -f /tmp/prof_step.ncu-rep                 # /tmp survives on a reused box: never read a stale capture
timeout 1800 ncu --set full -f --clock-control none \
    -k 'regex:k_(classes|insert|rank|scan|assign|finalize|problem|mark|drop|plan|lane|queue|count|model)' -o /tmp/prof_step \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_full.log 2>&1
python scripts/ncu_kernels.py /tmp/prof_step.ncu-rep gpurun_out/ncu_kernels.json \
    "ncu --set full --clock-control none, every kernel of bench.py --steps 1 --warmup 1 (c5, 10^8 candidates), last step" > gpurun_out/ncu_kernels.txt 2>&1
TOPK=${TOPK:-k_model_fused}
timeout 900 ncu --set full -f --clock-control none --import-source on -k "regex:$TOPK" -s 1 -c 1 -o gpurun_out/prof_top \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_top.log 2>&1
ncu -i gpurun_out/prof_top.ncu-rep --page details > gpurun_out/top_details.txt 2>&1
tail -3 gpurun_out/tests.log; head -c 600 gpurun_out/bench.json; echo; tail -3 gpurun_out/bench.err; cat gpurun_out/ncu_kernels.txt; ls -la gpurun_out
