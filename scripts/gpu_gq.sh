#!/bin/bash
# NM group queue A/B (build/var_gq64, var_gq128) vs default: NM parity subset per variant, benches.
mkdir -p gpurun_out
for v in gq64 gq128; do
  GSH_LIB=$PWD/build/var_$v/libgsh.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ladder or nm_table or invariant or edge" > gpurun_out/gq_$v.log 2>&1; echo "$v pytest rc=$?"; tail -1 gpurun_out/gq_$v.log
done
for v in base gq64 gq128; do
  if [ $v = base ]; then unset GSH_LIB; else export GSH_LIB=$PWD/build/var_$v/libgsh.so; fi
  for w in zipf05 zipf075 cfg1 cfg2; do
    timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/gq_${v}_$w.json 2>/dev/null
    echo "$v $w: $(python -c "import json;d=json.loads(open('gpurun_out/gq_${v}_$w.json').read().strip().splitlines()[-1]);p=d['phases_ms'];print(round(d['ms_per_step'],3),'NM',round(p['ms_nmjoin'],3),d['count'])" 2>/dev/null)"
  done
done
