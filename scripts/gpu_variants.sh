# bench the default build and compile-time variants of the counting kernel (VARIANTS="flags1;flags2;...")
mkdir -p gpurun_out
python __graft_entry__.py
timeout 600 python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench_default.json 2> gpurun_out/bench.err
i=0
IFS=';' read -ra VS <<< "$VARIANTS"
for v in "${VS[@]}"; do
  i=$((i+1))
  nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared $v \
     -o /tmp/libsel_v$i.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu
  SEL_LIBSEL=/tmp/libsel_v$i.so timeout 600 python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench_v$i.json 2>> gpurun_out/bench.err
  echo "variant $i: $v"
done
for f in gpurun_out/bench_default.json gpurun_out/bench_v*.json; do python -c "
import json,sys; d=json.load(open('$f')); print('$f', round(d['value']/1e6,2), 'M evals/s frac', round(d['roofline']['frac'],3))"; done
tail -3 gpurun_out/bench.err
