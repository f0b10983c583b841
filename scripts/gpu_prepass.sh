#!/bin/bash
# Pre-partition pass: parity (forced bits + 2^30 full size), then the 2^28 / 2^30 scale points and cfg2.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "prepass or pkfk_large" > gpurun_out/pytest_prepass.log 2>&1
echo "pytest rc=$?"; tail -3 gpurun_out/pytest_prepass.log
for w in ${WL:-pkfk30}; do
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/sweep_$w.json 2> gpurun_out/sweep_$w.err
  echo "$w rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/sweep_$w.json')); print('value',d['value'],'ms',d['ms_per_step']); print(d['phases_ms']); print(d['roofline'])" 2>&1 | tail -3
done
GSH_BENCH_CFG='{"prepass_bits": 3}' timeout 600 python bench.py --workload pkfk30 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/sweep_pkfk30_p3.json 2> gpurun_out/sweep_pkfk30_p3.err
echo "pkfk30 p3 rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/sweep_pkfk30_p3.json')); print('value',d['value'],'ms',d['ms_per_step']); print(d['phases_ms'])" 2>&1 | tail -3
