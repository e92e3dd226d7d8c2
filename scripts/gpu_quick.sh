# quick check: build, GPU tests (TESTSEL = pytest -k expression), bench (no ncu)
mkdir -p gpurun_out
python __graft_entry__.py
if [ -n "$TESTSEL" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -k "$TESTSEL" --durations=10 > gpurun_out/tests.log 2>&1
else
  timeout 1500 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/tests.log 2>&1
fi
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench.json 2> gpurun_out/bench.err
if [ -n "$LAUNCHES" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_launch_bench.json 2>&1
fi
tail -40 gpurun_out/tests.log; head -c 1500 gpurun_out/bench.json; tail -3 gpurun_out/bench.err
