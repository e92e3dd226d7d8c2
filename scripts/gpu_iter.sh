# quick iteration: build, gpu tests, bench, ncu full capture of the count kernel on a 2e7-candidate slice
mkdir -p gpurun_out
python __graft_entry__.py
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/tests.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 -o gpurun_out/prof_count \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --candidates 20000000 > gpurun_out/ncu_full.log 2>&1
cat gpurun_out/tests.log gpurun_out/bench.json; tail -3 gpurun_out/bench.err
