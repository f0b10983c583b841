#!/bin/bash
# parity tests + bench (no ncu).  Usage: gpu_quick.sh TAG [pytest -k expr]
TAG=${1:-q}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q ${2:+-k "$2"} > gpurun_out/pytest_${TAG}.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_${TAG}.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/bench_${TAG}.json')); print('value',d['value'],'ms',d['ms_per_step']); print(d['phases_ms']); print(d['roofline'])" 2>&1 | tail -5
tail -3 gpurun_out/bench_${TAG}.err
