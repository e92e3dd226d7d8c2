# ncu launch list of one full bench step (+ warm-up): per-kernel durations
mkdir -p gpurun_out
python __graft_entry__.py
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next ${BENCH_ARGS:-} > gpurun_out/ncu_launch_bench.json 2>&1
python scripts/ncu_summary.py --launches gpurun_out/launches.csv --out gpurun_out/launches_summary | head -30
