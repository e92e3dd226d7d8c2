# gpu tests + default bench + config-4 bench (1 rank, and 2 ranks sharing the GPU over gloo)
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/tests.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c4.json 2>> gpurun_out/bench.err
SEL_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29533 bench.py --config 4 --gpus 2 --steps 3 --warmup 3 > gpurun_out/bench_c4_2r.json 2>> gpurun_out/bench.err
cat gpurun_out/tests.log gpurun_out/bench.json gpurun_out/bench_c4.json gpurun_out/bench_c4_2r.json; tail -3 gpurun_out/bench.err
