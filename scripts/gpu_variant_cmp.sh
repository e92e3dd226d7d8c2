mkdir -p gpurun_out
python __graft_entry__.py
timeout 900 python -m pytest tests -m gpu -x -q -k "c5 or c2 or c1_gemm or random_tiny or invalid or slot_overflow or deterministic" 2>&1 | tail -3 > gpurun_out/tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-next > gpurun_out/bench.json 2> gpurun_out/bench.err
nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared $VARIANT_FLAGS \
     -o /tmp/libsel_variant.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu
SEL_LIBSEL=/tmp/libsel_variant.so timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench_variant.json 2>> gpurun_out/bench.err
bash scripts/gpu_launches.sh > /dev/null 2>&1
cat gpurun_out/tests.log; python -c "
import json
for f in ['gpurun_out/bench.json','gpurun_out/bench_variant.json']:
    d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, d['ms_per_step'], d['value']/1e9, d['roofline']['count_ms_per_launch'], d.get('e2e'))
"; cat gpurun_out/launches_summary.md | head -14
