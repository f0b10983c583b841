#!/bin/bash
# A/B of the NM table on skewed workloads: auto (CSR when any partition is large) vs forced chained.
for w in ${WL:-zipf05 cfg1 zipf075}; do
  for t in 0 2; do
    GSH_BENCH_CFG="{\"nm_table\": $t}" timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/nmab_${w}_$t.json 2>gpurun_out/nmab_${w}_$t.err
    python -c "
import json; d=json.load(open('gpurun_out/nmab_${w}_$t.json')); p=d['phases_ms']; s=d['stats']
print('$w nm_table=$t', 'ms %.3f' % d['ms_per_step'], 'nm %.3f' % p['ms_nmjoin'], 'table', s['nm_table'], 'count', s['count'])" 2>&1 | tail -1
  done
done
