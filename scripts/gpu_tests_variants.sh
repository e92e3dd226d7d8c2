set -x
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1500 python -m pytest tests -m gpu -q -x --durations=5 > gpurun_out/tests.log 2>&1
tail -3 gpurun_out/tests.log
VARIANTS=${VARIANTS:-"cur:"} bash scripts/gpu_variants.sh
for f in gpurun_out/bench_*.json; do python -c "
import json; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['kernel_ms'].items()})"; done
