#!/bin/bash
# Round 2: hybrid partition with batched first probes; hybrid GPU tests; input-side and full bench
# points with and without --hybrid; full-size output runs (cfg4 graph 2^28 edges COUNT, cfg3
# theta = 1.0 MATERIALIZE with the 2^30-pair buffer).
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_hybrid.py -q -x --durations=3 > gpurun_out/pytest_hyb3.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_hyb3.log
tail -6 gpurun_out/pytest_hyb3.log
for w in zipf10 zipf15; do
  for h in "" "--hybrid"; do
    timeout 300 python bench.py --workload $w --input-side $h --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb3_${w}${h}.json 2> gpurun_out/hyb3_${w}${h}.err
    echo "$w $h rc=$?"; python scripts/show_bench.py gpurun_out/hyb3_${w}${h}.json 2>/dev/null | sed -n 2p
  done
done
for w in zipf05 cfg2; do
  timeout 300 python bench.py --workload $w --hybrid --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/hyb3_${w}--hybrid.json 2> gpurun_out/hyb3_${w}--hybrid.err
  echo "$w --hybrid rc=$?"; python scripts/show_bench.py gpurun_out/hyb3_${w}--hybrid.json 2>/dev/null | sed -n 2p
done
timeout 900 python bench.py --workload graph28 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/full_graph28.json 2> gpurun_out/full_graph28.err; echo "graph28 rc=$?"
timeout 900 python bench.py --workload zipf10 --mode materialize --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/full_zipf10_mat.json 2> gpurun_out/full_zipf10_mat.err; echo "zipf10 mat rc=$?"
for f in full_graph28 full_zipf10_mat; do python scripts/show_bench.py gpurun_out/$f.json 2>/dev/null | head -2; done
