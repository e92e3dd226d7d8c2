# one GPU call: build, bench (default + variants), ncu launch list, ncu full capture of the count kernel
mkdir -p gpurun_out
python __graft_entry__.py
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --steps 3 --warmup 3 --flags 1 --no-e2e --no-cpu-baseline > gpurun_out/bench_nodedup.json 2>> gpurun_out/bench.err
timeout 600 python bench.py --steps 3 --warmup 3 --flags 2 --no-e2e --no-cpu-baseline > gpurun_out/bench_match.json 2>> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_bench.json 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 -o gpurun_out/prof_count \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
cat gpurun_out/bench.json gpurun_out/bench_nodedup.json gpurun_out/bench_match.json; tail -5 gpurun_out/bench.err
