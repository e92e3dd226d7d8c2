# build, GPU tests, bench default + variants given as VARIANTS="name1:-DFOO=1 name2:-DBAR=2" (launch list of default)
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_launch_bench.json 2>&1
for v in $VARIANTS; do
  name=${v%%:*}; flags=$(echo ${v#*:} | tr ',' ' ')
  nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared $flags \
     -o /tmp/libsel_$name.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu
  SEL_LIBSEL=/tmp/libsel_$name.so timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-next > gpurun_out/bench_$name.json 2>> gpurun_out/bench.err
done
tail -3 gpurun_out/tests.log
for f in gpurun_out/bench*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', 'G/s', round(d['value']/1e9,3), 'ms', round(d['ms_per_step'],3), {k: round(v['ms_per_launch'],3) for k, v in d['roofline_by_region'].items()})"; done
tail -3 gpurun_out/bench.err
