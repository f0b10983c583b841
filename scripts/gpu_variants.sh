#!/bin/bash
# Experiments only: bench each built variant (build/var_*/libgsh.so) and the default library.
# Usage: gpu_variants.sh [names...]
mkdir -p gpurun_out
names=${@:-$(ls build | grep '^var_' | sed 's/^var_//')}
for n in base $names; do
  if [ $n = base ]; then lib=""; else lib=build/var_$n/libgsh.so; fi
  GSH_LIB=$lib timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/var_$n.json 2> gpurun_out/var_$n.err
  python -c "
import json; d=json.load(open('gpurun_out/var_$n.json')); p=d['phases_ms']
print('%-10s hist %.3f p1 %.3f p2 %.3f nm %.3f total %.3f step %.3f' % ('$n', p['ms_hist'], p['ms_pass1'], p['ms_pass2'], p['ms_nmjoin'], p['ms_total'], d['ms_per_step']))" 2>&1 | tail -1
done
