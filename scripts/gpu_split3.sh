#!/bin/bash
# Split item size A/B: 2048-tuple items / 256 threads (default) vs 4096 / 512 (build/var_split512).
mkdir -p gpurun_out
GSH_LIB=$PWD/build/var_split512/libgsh.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ladder or materialize or detection or invariant or edge or sampled" > gpurun_out/split3_pytest.log 2>&1; echo "512 pytest rc=$?"; tail -1 gpurun_out/split3_pytest.log
for v in base split512; do
  if [ $v = base ]; then unset GSH_LIB; else export GSH_LIB=$PWD/build/var_$v/libgsh.so; fi
  for w in zipf10 zipf15; do
    timeout 300 python bench.py --workload $w --input-side --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/split3_${v}_$w.json 2>/dev/null
    echo "$v $w: $(python scripts/show_bench.py gpurun_out/split3_${v}_$w.json 2>/dev/null | sed -n 2p | cut -c1-230)"
  done
done
