#!/bin/bash
# Hybrid sample without singleton flushes: hybrid tests, hybrid under the sharded driver, sweep.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_hybrid.py tests/test_gpu_sharded_native.py -q -x -k "hybrid" > gpurun_out/pytest_hyb6.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_hyb6.log
for w in zipf05 cfg2; do
  timeout 300 python bench.py --workload $w --hybrid --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb6_$w.json 2>/dev/null
  echo "$w --hybrid: $(python scripts/show_bench.py gpurun_out/hyb6_$w.json 2>/dev/null | sed -n 2p)"
done
for w in zipf10 zipf15; do
  timeout 300 python bench.py --workload $w --input-side --hybrid --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb6_$w.json 2>/dev/null
  echo "$w --hybrid: $(python scripts/show_bench.py gpurun_out/hyb6_$w.json 2>/dev/null | sed -n 2p)"
done
