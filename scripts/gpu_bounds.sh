#!/bin/bash
# Bounds-checked build (GSH_CHECK_BOUNDS: computed indices asserted in-kernel; compute-sanitizer is
# closed on the GPU pool) over the sanitizer ladder and the hybrid / Gbase suites.
mkdir -p gpurun_out
export GSH_LIB=$PWD/build/var_bounds/libgsh.so
SAN_TOOL=bounds timeout 900 python scripts/sanitize_ladder.py > gpurun_out/bounds_ladder.log 2>&1; echo "ladder rc=$?"; tail -3 gpurun_out/bounds_ladder.log
timeout 1200 python -m pytest tests/test_gpu_hybrid.py tests/test_gpu_gbase.py tests/test_gpu_parity.py -q -x -k "not prepass_exact and not nm_table_modes" > gpurun_out/bounds_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/bounds_pytest.log
