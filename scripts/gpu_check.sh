mkdir -p gpurun_out
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
nproc
python __graft_entry__.py smoke 2>&1 | tail -20
timeout 1200 python -m pytest tests -m gpu -x -q --durations=10 2>&1 | tail -40
