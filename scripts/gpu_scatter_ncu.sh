#!/bin/bash
# ncu of pass-2 scatter, TMA-store vs sector-store variants
mkdir -p gpurun_out
for c in 0 1; do
GSH_SCATTER_CFG=$c timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_scatter" -s 3 -c 1 \
    -o gpurun_out/prof_scab$c python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_scab$c.log 2>&1
echo "ncu $c rc=$?"
done
