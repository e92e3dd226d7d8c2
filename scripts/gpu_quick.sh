# quick check: build, selected GPU tests (TESTSEL = pytest -k expression), bench (no ncu)
mkdir -p gpurun_out
python __graft_entry__.py
if [ -n "$TESTSEL" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q -k "$TESTSEL" 2>&1 | tail -15 > gpurun_out/tests.log
else
  timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/tests.log
fi
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench.json 2> gpurun_out/bench.err
if [ -n "$NCU_SLICE" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${NCU_K:-k_queue} -s 1 -c 1 -o gpurun_out/prof_count \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next --candidates $NCU_SLICE > gpurun_out/ncu_full.log 2>&1
fi
cat gpurun_out/tests.log gpurun_out/bench.json; tail -3 gpurun_out/bench.err
