#!/bin/bash
# A/B of scatter tile / occupancy variants (build/var_*): parity subset, cfg2 and theta=1.5 input side.
mkdir -p gpurun_out
for v in base i12m3 i8m4 i12m3b; do
  if [ $v = base ]; then unset GSH_LIB; else export GSH_LIB=$PWD/build/var_$v/libgsh.so; fi
  timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "partition_phase or ladder" > gpurun_out/occ_$v.log 2>&1; echo "$v pytest rc=$?"
  for r in 1 2; do
    timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/occ_$v.json 2>/dev/null
    echo "$v cfg2: $(python scripts/show_bench.py gpurun_out/occ_$v.json 2>/dev/null | sed -n 2p)"
  done
  timeout 300 python bench.py --workload zipf15 --input-side --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/occ15_$v.json 2>/dev/null
  echo "$v zipf15: $(python scripts/show_bench.py gpurun_out/occ15_$v.json 2>/dev/null | sed -n 2p)"
done
