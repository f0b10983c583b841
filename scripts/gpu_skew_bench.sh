#!/bin/bash
for w in ${WL:-cfg1 zipf05 zipf075 zipf10s zipf15s graph}; do
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --mode ${MODE:-count} > gpurun_out/skew_$w.json 2>gpurun_out/skew_$w.err
  python -c "
import json; d=json.load(open('gpurun_out/skew_$w.json')); p=d['phases_ms']; s=d['stats']
print('$w', 'ms %.3f' % d['ms_per_step'], 'in/s %.3g out/s %.3g' % (d['value'], d['output_tuples_per_s']), {k: round(v,3) for k,v in p.items()}, 'heavy', s['n_heavy'], 'large', s['n_large'], 'skew_pairs %.3g' % s['skew_pairs'], 'written', s.get('written'), 'ovf', s.get('overflow'))" 2>&1 | tail -2
done
