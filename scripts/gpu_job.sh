set -x
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1500 python -m pytest tests -m gpu -q -x --durations=5 > gpurun_out/tests.log 2>&1
tail -3 gpurun_out/tests.log
VARIANTS="items:;items0:-DSEL_LANE_BLOCK_PERIOD=0" bash scripts/gpu_variants.sh
