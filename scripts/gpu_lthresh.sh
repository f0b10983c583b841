#!/bin/bash
# Experiment: large-partition threshold L and skew threshold T_h at theta = 0.5 (NM-join bound by keys
# duplicated below the skew threshold) and their cost on uniform cfg2; plus the generator pin test.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "histogram or partition_phase or ladder or prepass_unaligned" > gpurun_out/hist_pytest.log 2>&1; echo "hist-batch pytest rc=$?"; tail -1 gpurun_out/hist_pytest.log
timeout 600 python -m pytest tests/test_gpu_datagen.py -q > gpurun_out/gen_pytest.log 2>&1; echo "gen pytest rc=$?"; tail -1 gpurun_out/gen_pytest.log
for c in '{}' '{"nm_table": 2}' '{"large_threshold": 2300}' '{"large_threshold": 2200}' '{"large_threshold": 2120}' '{"large_threshold": 2120, "heavy_threshold": 32}' '{"large_threshold": 2200, "heavy_threshold": 32}'; do
  for w in zipf05 cfg2; do
    GSH_BENCH_CFG="$c" timeout 300 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/lt.json 2>/dev/null
    echo "$w $c: $(python scripts/show_bench.py gpurun_out/lt.json 2>/dev/null | sed -n 2p)"
  done
done
