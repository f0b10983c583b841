#!/bin/bash
# ncu: pre-partition pass kernels at 2^30 per side; k_skewjoin on cfg1.  Plus the pkfk30 bench line.
mkdir -p gpurun_out
timeout 600 python bench.py --workload pkfk30 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_pkfk30.json 2> gpurun_out/bench_pkfk30.err; echo "bench30 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_split_count_tiles|k_split_scatter_tiles" -s 4 -c 2 \
    -o gpurun_out/prof_prepass python bench.py --workload pkfk30 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_prepass.log 2>&1
echo "ncu prepass rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_skewjoin" -s 2 -c 1 \
    -o gpurun_out/prof_skew python bench.py --workload cfg1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_skew.log 2>&1
echo "ncu skew rc=$?"
