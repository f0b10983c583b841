#!/bin/bash
# Round 2: hybrid partition (NEXT-1) with u32 lookup tables + aggregated counts, Gbase-style join
# with one barrier per COUNT round; GPU tests, bench points, Table I sweep, scatter write-out A/B.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_hybrid.py tests/test_gpu_gbase.py -q --durations=5 > gpurun_out/pytest_hyb.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_hyb.log
tail -8 gpurun_out/pytest_hyb.log
for w in zipf10 zipf15; do
  for h in "" "--hybrid"; do
    timeout 300 python bench.py --workload $w --input-side $h --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb_${w}${h}.json 2> gpurun_out/hyb_${w}${h}.err
    echo "$w $h rc=$?"; python scripts/show_bench.py gpurun_out/hyb_${w}${h}.json 2>/dev/null | head -2
  done
done
for w in zipf05 zipf075 cfg2; do
  for h in "" "--hybrid"; do
    timeout 300 python bench.py --workload $w $h --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb_${w}${h}.json 2> gpurun_out/hyb_${w}${h}.err
    echo "$w $h rc=$?"; python scripts/show_bench.py gpurun_out/hyb_${w}${h}.json 2>/dev/null | head -2
  done
done
timeout 900 python bench.py --gbase-sweep > gpurun_out/gbase_sweep.json 2> gpurun_out/gbase_sweep.err; echo "gbase sweep rc=$?"
tail -9 gpurun_out/gbase_sweep.err | cut -c1-400
bash scripts/gpu_wob_ab.sh
