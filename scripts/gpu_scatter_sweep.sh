#!/bin/bash
for c in 0 1 2 3; do
  GSH_SCATTER_CFG=$c timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/sweep_$c.json 2>&1
  python -c "import json; d=json.load(open('gpurun_out/sweep_$c.json')); p=d['phases_ms']; print('cfg $c pass1 %.3f pass2 %.3f total %.3f' % (p['ms_pass1'], p['ms_pass2'], d['ms_per_step']))" 2>&1 | tail -1
done
