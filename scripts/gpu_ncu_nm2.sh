#!/bin/bash
# Source-level ncu of the NM ring: cfg2 (chained table) and theta = 0.5 (CSR, duplicated keys).
mkdir -p gpurun_out
for w in cfg2 zipf05; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_nmjoin_ring" -s 3 -c 1 \
    -o gpurun_out/prof_nm_$w python bench.py --workload $w --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_nm_$w.log 2>&1
echo "ncu $w rc=$?"; tail -1 gpurun_out/ncu_nm_$w.log
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-sweep > gpurun_out/e2e_check.json 2>/dev/null; echo "bench rc=$?"
python -c "import json; d=json.loads(open('gpurun_out/e2e_check.json').read().strip().splitlines()[-1]); print(d['e2e'])"
