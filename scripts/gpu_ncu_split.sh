#!/bin/bash
# Source-level ncu of detect + split at theta = 1.0 (input side, 2^27 per side).
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_split|k_detect_smem" -s 6 -c 2 \
    -o gpurun_out/prof_split10 python bench.py --workload zipf10 --input-side --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_split10.log 2>&1
echo "ncu rc=$?"; tail -1 gpurun_out/ncu_split10.log
