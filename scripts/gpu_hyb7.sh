#!/bin/bash
# Hybrid histogram with predicated batched counts and two-slot lookups; cfg2 default line.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_hybrid.py -q -x > gpurun_out/pytest_hyb7.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_hyb7.log
for w in zipf10 zipf15; do
  for h in "" "--hybrid"; do
  timeout 300 python bench.py --workload $w --input-side $h --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb7_$w$h.json 2>/dev/null
  echo "$w $h: $(python scripts/show_bench.py gpurun_out/hyb7_$w$h.json 2>/dev/null | sed -n 2p)"
  done
done
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb7_cfg2.json 2>/dev/null
echo "cfg2: $(python scripts/show_bench.py gpurun_out/hyb7_cfg2.json 2>/dev/null | head -2)"
