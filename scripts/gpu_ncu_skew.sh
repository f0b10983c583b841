#!/bin/bash
# ncu of the input side at theta = 1.5 / 1.0 (2^27 per side): scatter passes, histogram, detect, split.
mkdir -p gpurun_out
for w in zipf15 zipf10; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_scatter|k_hist2d|k_detect|k_split" -s 12 -c 6 \
    -o gpurun_out/prof_$w python bench.py --workload $w --input-side --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_$w.log 2>&1
echo "ncu $w rc=$?"; tail -3 gpurun_out/ncu_$w.log
done
