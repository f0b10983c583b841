#!/bin/bash
# Pre-partition kernels: live bench at 2^30, launch list of the split kernels, one full capture.
mkdir -p gpurun_out
timeout 600 python bench.py --workload pkfk30 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/sweep_pkfk30.json 2> gpurun_out/sweep_pkfk30.err
echo "pkfk30 rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/sweep_pkfk30.json')); print('value',d['value'],'ms',d['ms_per_step']); print(d['phases_ms'])" 2>&1 | tail -3
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_split --csv \
  --log-file gpurun_out/prepass_launches.csv python bench.py --workload pkfk30 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
echo "ncu list rc=$?"; grep -c k_split gpurun_out/prepass_launches.csv
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_split_scatter -c 1 -o gpurun_out/prepass_scatter \
  python bench.py --workload pkfk30 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
echo "ncu full rc=$?"
