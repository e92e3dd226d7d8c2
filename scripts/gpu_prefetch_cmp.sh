# model-kernel L2 prefetch variants (SEL_MODEL_PREFETCH 0/1/2), bench c5 twice each, interleaved
mkdir -p gpurun_out
python __graft_entry__.py
for v in 0 1 2; do
  nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared -DSEL_MODEL_PREFETCH=$v \
     -o /tmp/libsel_p$v.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu &
done
wait
for r in 1 2; do for v in 0 1 2; do
  SEL_LIBSEL=/tmp/libsel_p$v.so timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench_p${v}_$r.json 2>> gpurun_out/bench_p.err
done; done
python -c "
import json
for r in (1,2):
  for v in (0,1,2):
    d=json.loads(open(f'gpurun_out/bench_p{v}_{r}.json').read().strip().splitlines()[-1]); rb=d['roofline_by_region']
    print(r, v, round(d['ms_per_step'],4), round(d['value']/1e9,3), 'model', round(rb['model']['ms_per_launch'],4), 'count', round(rb['count']['ms_per_launch'],4))
"
