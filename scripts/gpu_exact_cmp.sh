# model kernel: exact re-evaluation as a noinline call (SEL_MODEL_EXACT_CALL) x min blocks/SM; full GPU tests on the default build
mkdir -p gpurun_out
python __graft_entry__.py
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/tests_ec.log 2>&1
for cfg in "0 4" "1 4" "1 5" "1 6"; do set -- $cfg
  nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared -DSEL_MODEL_EXACT_CALL=$1 -DSEL_MODEL_MIN_BLOCKS=$2 \
     -o /tmp/libsel_ec$1_mb$2.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu &
done
wait
for r in 1 2; do for cfg in ec0_mb4 ec1_mb4 ec1_mb5 ec1_mb6; do
  SEL_LIBSEL=/tmp/libsel_$cfg.so timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench_${cfg}_$r.json 2>> gpurun_out/bench_ec.err
done; done
tail -2 gpurun_out/tests_ec.log
python -c "
import json
for r in (1,2):
  for v in ('ec0_mb4','ec1_mb4','ec1_mb5','ec1_mb6'):
    d=json.loads(open(f'gpurun_out/bench_{v}_{r}.json').read().strip().splitlines()[-1]); rb=d['roofline_by_region']
    print(r, v, round(d['ms_per_step'],4), round(d['value']/1e9,3), 'model', round(rb['model']['ms_per_launch'],4))
"
