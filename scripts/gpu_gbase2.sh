#!/bin/bash
# Bucket-chained Gbase: tests (bounds-checked build first), sweep.
mkdir -p gpurun_out
GSH_LIB=$PWD/build/var_bounds/libgsh.so timeout 900 python -m pytest tests/test_gpu_gbase.py -q -x > gpurun_out/gbase2_bounds.log 2>&1; echo "bounds pytest rc=$?"; tail -3 gpurun_out/gbase2_bounds.log
timeout 900 python -m pytest tests/test_gpu_gbase.py -q -x > gpurun_out/gbase2_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/gbase2_pytest.log
timeout 1200 python bench.py --gbase-sweep > gpurun_out/gbase_sweep2.json 2> gpurun_out/gbase_sweep2.err; echo "gbase sweep rc=$?"
tail -9 gpurun_out/gbase_sweep2.err | cut -c1-330
