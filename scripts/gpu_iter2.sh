# iteration: build, GPU tests, short bench, launch list (share per kernel)
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_launch_bench.json 2>&1
if [ -n "$NCU_K" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$NCU_K" -s ${NCU_S:-3} -c ${NCU_C:-1} -o gpurun_out/prof_iter \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_full.log 2>&1
fi
tail -3 gpurun_out/tests.log; cat gpurun_out/bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value',d['value']/1e9,'G ms',d['ms_per_step'], 'count_ms', d['roofline']['count_ms_per_launch'])"; tail -3 gpurun_out/bench.err
