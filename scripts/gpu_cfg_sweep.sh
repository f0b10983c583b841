#!/bin/bash
# bench under several gsh_config overrides (experiments): CFGS env = list of json configs
i=0
for c in ${CFGS:-'{}'}; do
  GSH_BENCH_CFG="$c" timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e ${BARGS} > gpurun_out/cfg_$i.json 2>gpurun_out/cfg_$i.err
  python -c "import json; d=json.load(open('gpurun_out/cfg_$i.json')); p=d['phases_ms']; print('$c', 'hist %.3f p1 %.3f p2 %.3f det %.3f spl %.3f nm %.3f sk %.3f total %.3f' % (p['ms_hist'], p['ms_pass1'], p['ms_pass2'], p['ms_detect'], p['ms_split'], p['ms_nmjoin'], p['ms_skewjoin'], d['ms_per_step']))" 2>&1 | tail -1
  i=$((i+1))
done
