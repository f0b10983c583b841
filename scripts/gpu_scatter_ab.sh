#!/bin/bash
# A/B of the scatter write-out: TMA bulk stores (default) vs per-tuple sector stores (cfg 1).
mkdir -p gpurun_out
for c in 0 1; do
  GSH_SCATTER_CFG=$c timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/scab_$c.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/scab_$c.json')); p=d['phases_ms']; print('cfg $c', 'p1', round(p['ms_pass1'],3), 'p2', round(p['ms_pass2'],3), 'total', round(d['ms_per_step'],3))"
done
