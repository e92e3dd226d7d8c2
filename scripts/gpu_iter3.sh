# iteration: build, selected GPU tests first (TESTS), full GPU suite, short bench, launch list
mkdir -p gpurun_out
python __graft_entry__.py
if [ -n "$TESTS" ]; then timeout 600 python -m pytest $TESTS -x -q > gpurun_out/tests_sel.log 2>&1; tail -15 gpurun_out/tests_sel.log; fi
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_launch_bench.json 2>&1
tail -3 gpurun_out/tests.log
python -c "import json; d=json.loads(open('gpurun_out/bench.json').read()); print('G/s', round(d['value']/1e9,3), 'ms', round(d['ms_per_step'],3), {k: round(v['ms_per_launch'],3) for k, v in d['roofline_by_region'].items()})"
tail -3 gpurun_out/bench.err
