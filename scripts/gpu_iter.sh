# quick iteration: build, gpu tests, bench, optional variant bench, ncu full capture on a 2e7-candidate slice
mkdir -p gpurun_out
python __graft_entry__.py
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/tests.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
if [ -n "$VARIANT_FLAGS" ]; then
  nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared $VARIANT_FLAGS \
     -o /tmp/libsel_variant.so paper_conf_ipps_chikinaat19_b200/csrc/{sel_api,sel_plan,sel_count,sel_model,sel_next,int_peak}.cu
  SEL_LIBSEL=/tmp/libsel_variant.so timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_variant.json 2>> gpurun_out/bench.err
fi
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 -o gpurun_out/prof_count \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --candidates 20000000 > gpurun_out/ncu_full.log 2>&1
cat gpurun_out/tests.log gpurun_out/bench.json gpurun_out/bench_variant.json 2>/dev/null; tail -3 gpurun_out/bench.err
