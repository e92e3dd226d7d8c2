# full round measurement: build, GPU tests, full bench line, launch list, ncu --set full of every kernel of the bench steps
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/tests.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_launch_bench.json 2>&1
timeout 1800 ncu --set full --clock-control none --import-source on \
    -k 'regex:k_(classes|insert|rank|scan|assign|finalize|problem|plan|lane|queue|count|model)' -o gpurun_out/prof_step \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/tests.log; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err; tail -2 gpurun_out/ncu_full.log
