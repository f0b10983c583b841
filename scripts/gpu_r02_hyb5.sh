#!/bin/bash
# Hybrid pass 1 with a per-unit ballot-ranked reference key; tests + input-side points + full joins.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_hybrid.py -q -x --durations=3 > gpurun_out/pytest_hyb5.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_hyb5.log
tail -3 gpurun_out/pytest_hyb5.log
for w in zipf10 zipf15; do
  for h in "" "--hybrid"; do
  timeout 300 python bench.py --workload $w --input-side $h --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb5_${w}${h}.json 2> gpurun_out/hyb5_${w}${h}.err
  echo "$w $h rc=$?"; python scripts/show_bench.py gpurun_out/hyb5_${w}${h}.json 2>/dev/null | sed -n 2p
  done
done
for w in zipf075 cfg1 graph; do
  for h in "" "--hybrid"; do
  timeout 300 python bench.py --workload $w $h --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb5_${w}${h}.json 2> gpurun_out/hyb5_${w}${h}.err
  echo "$w $h rc=$?"; python scripts/show_bench.py gpurun_out/hyb5_${w}${h}.json 2>/dev/null | sed -n 2p
  done
done
