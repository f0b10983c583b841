#!/bin/bash
# Multi-GPU path on the one-GPU box: sharded GPU tests + bench with fake ranks + the default bench.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sharded.py -x -q --durations=8 > gpurun_out/pytest_sharded.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_sharded.log
tail -25 gpurun_out/pytest_sharded.log
timeout 300 python bench.py --fake-ranks 4 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_fake4.json 2> gpurun_out/bench_fake4.err; echo "fake4 rc=$?"
timeout 300 python bench.py --fake-ranks 4 --workload pkfkzipf --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_fake4_pz.json 2> gpurun_out/bench_fake4_pz.err; echo "fake4pz rc=$?"
timeout 300 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r02a.json 2> gpurun_out/bench_r02a.err; echo "bench rc=$?"
tail -3 gpurun_out/*.err
