#!/bin/bash
# ncu --set full of the cfg2 kernels (source-level), + launch list.  Usage: gpu_ncu_cfg2.sh TAG
TAG=${1:-r02}
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sweep > /dev/null 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_scatter|k_nmjoin|k_hist2d" -s 5 -c 4 \
    -o gpurun_out/prof_${TAG} python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_${TAG}.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_${TAG}.log
