#!/bin/bash
# Hybrid pass 1 with static (key, unit) offsets: tests, input-side points, ncu of the hybrid kernels.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_hybrid.py -q -x --durations=3 > gpurun_out/pytest_hyb4.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_hyb4.log
tail -4 gpurun_out/pytest_hyb4.log
for w in zipf10 zipf15; do
  timeout 300 python bench.py --workload $w --input-side --hybrid --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb4_${w}.json 2> gpurun_out/hyb4_${w}.err
  echo "$w --hybrid rc=$?"; python scripts/show_bench.py gpurun_out/hyb4_${w}.json 2>/dev/null | sed -n 2p
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_scatter|k_hist2d" -s 9 -c 3 \
    -o gpurun_out/prof_hyb_zipf10 python bench.py --workload zipf10 --input-side --hybrid --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_hyb.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_hyb.log
