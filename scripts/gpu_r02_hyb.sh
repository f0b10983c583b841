#!/bin/bash
# Round 2: hybrid partition (NEXT-1) + Gbase-style comparison (NEXT-4): GPU tests, quick bench
# points, the Table I sweep, and memcheck over the new kernels.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_hybrid.py tests/test_gpu_gbase.py -x -q --durations=10 > gpurun_out/pytest_hyb.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_hyb.log
tail -15 gpurun_out/pytest_hyb.log
for w in zipf10 zipf15; do
  for h in "" "--hybrid"; do
    timeout 300 python bench.py --workload $w --input-side $h --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb_${w}${h}.json 2> gpurun_out/hyb_${w}${h}.err
    echo "$w $h rc=$?"; python scripts/show_bench.py gpurun_out/hyb_${w}${h}.json 2>/dev/null | head -5
  done
done
for w in zipf05 zipf075 cfg2; do
  for h in "" "--hybrid"; do
    timeout 300 python bench.py --workload $w $h --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb_${w}${h}.json 2> gpurun_out/hyb_${w}${h}.err
    echo "$w $h rc=$?"
  done
done
timeout 900 python bench.py --gbase-sweep > gpurun_out/gbase_sweep.json 2> gpurun_out/gbase_sweep.err; echo "gbase sweep rc=$?"
tail -12 gpurun_out/gbase_sweep.err
SAN_TOOL=memcheck timeout 1500 compute-sanitizer --tool memcheck --print-limit 50 python scripts/sanitize_ladder.py > gpurun_out/sanitize_memcheck_r02b.log 2>&1; echo "memcheck rc=$?"; tail -4 gpurun_out/sanitize_memcheck_r02b.log
