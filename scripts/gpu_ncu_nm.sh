#!/bin/bash
mkdir -p gpurun_out
for t in 2 3; do
GSH_BENCH_CFG="{\"nm_table\": $t}" timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/bench_nm$t.json 2>&1
GSH_BENCH_CFG="{\"nm_table\": $t}" timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_nmjoin" -s 2 -c 1 \
    -o gpurun_out/prof_nm$t python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_nm$t.log 2>&1
echo "t=$t rc=$?"
done
