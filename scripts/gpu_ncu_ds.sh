#!/bin/bash
# ncu of detect / split at theta = 1.5 and 1.0 (2^27 per side, input side only).
mkdir -p gpurun_out
for w in zipf15 zipf10; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_detect_smem|k_split" -s 2 -c 2 \
    -o gpurun_out/prof_ds_$w python bench.py --workload $w --input-side --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_ds_$w.log 2>&1
echo "ncu $w rc=$?"; tail -2 gpurun_out/ncu_ds_$w.log
done
