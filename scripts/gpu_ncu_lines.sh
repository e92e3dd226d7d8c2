# source-level ncu captures of several kernels (KERNELS="k_a k_b"), one report each, summarised by CUDA line
mkdir -p gpurun_out
python __graft_entry__.py
for K in ${KERNELS:-k_lane_problems}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$K" -s 1 -c 1 -o gpurun_out/prof_$K \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next > gpurun_out/ncu_$K.log 2>&1
done
ls gpurun_out
