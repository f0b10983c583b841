#!/bin/bash
# Hybrid share gate: hybrid tests, sharded hybrid, full-size hybrid, sweep arms.
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_hybrid.py tests/test_gpu_sharded_native.py tests/test_gpu_fullsize.py -q -x -k "hybrid or theta075" > gpurun_out/hyb8_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/hyb8_pytest.log
for w in zipf10 zipf15; do
  timeout 300 python bench.py --workload $w --input-side --hybrid --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb8_$w.json 2>/dev/null
  echo "$w --hybrid: $(python scripts/show_bench.py gpurun_out/hyb8_$w.json 2>/dev/null | sed -n 2p | cut -c1-240)"
done
for w in cfg1 zipf05; do
  timeout 300 python bench.py --workload $w --hybrid --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb8_$w.json 2>/dev/null
  echo "$w --hybrid: $(python scripts/show_bench.py gpurun_out/hyb8_$w.json 2>/dev/null | sed -n 2p | cut -c1-240)"
done
