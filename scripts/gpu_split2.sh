#!/bin/bash
# Split reserving only claimed slots: parity subset, input-side points, ncu of detect + split.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_decompose.py tests/test_gpu_hybrid.py -q -x -k "ladder or materialize or detection or invariant or edge or decompose_ladder or sampled or hybrid" > gpurun_out/split2_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/split2_pytest.log
for w in zipf10 zipf15 zipf075; do
  f=""; [ $w != zipf075 ] && f="--input-side"
  timeout 300 python bench.py --workload $w $f --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/split2_$w.json 2>/dev/null
  echo "$w: $(python scripts/show_bench.py gpurun_out/split2_$w.json 2>/dev/null | sed -n 2p | cut -c1-250)"
done
bash scripts/gpu_ncu_split.sh
