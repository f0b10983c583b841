#!/bin/bash
# bench under several gsh_config overrides (experiments)
i=0
for c in '{}' '{"pass_bits":[8,7],"capacity":8192}' '{"pass_bits":[8,6],"capacity":8192}' '{"pass_bits":[7,7],"capacity":8192}'; do
  GSH_BENCH_CFG="$c" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cfg_$i.json 2>gpurun_out/cfg_$i.err
  python -c "import json; d=json.load(open('gpurun_out/cfg_$i.json')); p=d['phases_ms']; print('$c', 'hist %.3f p1 %.3f p2 %.3f nm %.3f total %.3f' % (p['ms_hist'], p['ms_pass1'], p['ms_pass2'], p['ms_nmjoin'], d['ms_per_step']))" 2>&1 | tail -1
  i=$((i+1))
done
