# ncu --set full capture of one launch of the kernels matching $KREGEX in the bench configuration
mkdir -p gpurun_out
python __graft_entry__.py
for K in $KREGEX; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 -o gpurun_out/prof_$K \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-next ${BENCH_ARGS:-} > gpurun_out/ncu_$K.log 2>&1
done
ls gpurun_out
