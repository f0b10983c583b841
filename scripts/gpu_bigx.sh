#!/bin/bash
# CSR probe: warp-walked long candidate lists, threshold A/B (theta 0.5 / 0.75 NM, cfg2) + parity.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "nm_table_modes or materialize or ladder or sampled" > gpurun_out/bigx_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/bigx_pytest.log
for v in base bigoff bigx8 bigx64; do
  if [ $v = base ]; then unset GSH_LIB; else export GSH_LIB=$PWD/build/var_$v/libgsh.so; fi
  for w in zipf05 zipf075 cfg2; do
    timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/bigx_${v}_${w}.json 2>/dev/null
    echo "$v $w: $(python scripts/show_bench.py gpurun_out/bigx_${v}_${w}.json 2>/dev/null | sed -n 2p | cut -c1-220)"
  done
done
timeout 600 python bench.py --workload zipf05 --mode materialize --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/bigx_mat.json 2>/dev/null
echo "base zipf05 mat: $(python scripts/show_bench.py gpurun_out/bigx_mat.json 2>/dev/null | sed -n 2p | cut -c1-220)"
