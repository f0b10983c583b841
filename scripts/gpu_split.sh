#!/bin/bash
# Split with the compact skewed-key table: parity subset (bounds-checked build and release), input side.
mkdir -p gpurun_out
GSH_LIB=$PWD/build/var_bounds/libgsh.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_decompose.py -q -x -k "ladder or materialize or detection or invariant or edge or decompose_ladder or sampled" > gpurun_out/split_bounds.log 2>&1; echo "bounds pytest rc=$?"; tail -1 gpurun_out/split_bounds.log
timeout 900 python -m pytest tests/test_gpu_hybrid.py tests/test_gpu_fullsize.py -q -x -k "not next3 and not pkfk_large" > gpurun_out/split_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/split_pytest.log
for w in zipf10 zipf15; do
  timeout 300 python bench.py --workload $w --input-side --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/split_$w.json 2>/dev/null
  echo "$w: $(python scripts/show_bench.py gpurun_out/split_$w.json 2>/dev/null | sed -n 2,3p | cut -c1-250)"
done
for w in zipf05 zipf075 cfg1 cfg2; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/split_$w.json 2>/dev/null
  echo "$w: $(python scripts/show_bench.py gpurun_out/split_$w.json 2>/dev/null | sed -n 2p | cut -c1-250)"
done
