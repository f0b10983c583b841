#!/bin/bash
# Round profile: launch list of a 2-step bench (cold, serialised) + one ncu --set full capture of
# the top kernels.  Usage: gpu_profile_round.sh TAG
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/launches_${TAG}.out 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_scatter|k_nmjoin_ring|k_hist2d" -s 4 -c 4 \
    -o gpurun_out/prof_${TAG} python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_${TAG}.log 2>&1
echo "ncu rc=$?"
