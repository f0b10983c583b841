#!/bin/bash
# End-of-round-2 workload sweep (one line per workload).
mkdir -p gpurun_out
for w in cfg1 zipf05 zipf075 graph pkfkzipf pkfk28 pkfk29 pkfk30 zipf07_29; do
  timeout 900 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/fsweep_$w.json 2> gpurun_out/fsweep_$w.err
  echo "$w rc=$? $(python -c "import json;d=json.loads(open('gpurun_out/fsweep_$w.json').read().strip().splitlines()[-1]);print(round(d['ms_per_step'],3),'ms',f\"{d['value']:.3e}\",'in/s',f\"{d['output_tuples_per_s']:.3e}\",'out/s',{k:round(v,2) for k,v in d['phases_ms'].items() if v})" 2>/dev/null)"
done
