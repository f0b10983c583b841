#!/bin/bash
# ncu full capture of the top kernels of the cfg2 bench.  Usage: gpu_ncu.sh TAG [regex]
TAG=${1:-r}
RE=${2:-"k_scatter|k_nmjoin|k_hist2d"}
SKIP=${3:-6}
CNT=${4:-4}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$RE" -s $SKIP -c $CNT \
    -o gpurun_out/prof_${TAG} python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --workload ${WL:-cfg2} --mode ${MODE:-count} > gpurun_out/ncu_${TAG}.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_${TAG}.log
