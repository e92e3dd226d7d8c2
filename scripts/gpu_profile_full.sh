# full-size profiles of the bench configuration (c5, 10^8 candidates) + torchrun world-size-1 check
mkdir -p gpurun_out
python __graft_entry__.py
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus 1 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/torchrun1.json 2> gpurun_out/torchrun1.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_launch_bench.json 2>&1
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:k_count -s 3 -c 1 -o gpurun_out/prof_count_full \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_full.log 2>&1
cat gpurun_out/torchrun1.json; tail -3 gpurun_out/torchrun1.err; tail -2 gpurun_out/ncu_full.log
