#!/bin/bash
for d in 0 1 2 4 5 3; do
  echo "dbg $d"
  GSH_SCATTER_DEBUG=$d timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/dbg_$d.json 2>gpurun_out/dbg_$d.err
  python -c "import json; d=json.load(open('gpurun_out/dbg_$d.json')); p=d['phases_ms']; print('  pass1 %.3f pass2 %.3f' % (p['ms_pass1'], p['ms_pass2']))" 2>&1 | tail -1
done
