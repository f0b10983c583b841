#!/bin/bash
# Launch list of the sharded step (world of one over NCCL) and the one-GPU step, + a short native test subset.
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_sharded_native.py tests/test_gpu_sharded.py -x -q -k "agreement or native or route or p2p or local_world" > gpurun_out/pytest_np.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_np.log
timeout 300 python bench.py --sharded --steps 5 --warmup 3 --no-e2e > gpurun_out/bench_nccl1_b.json 2> gpurun_out/bench_nccl1_b.err; echo "nccl1 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_sharded1.csv python bench.py --sharded --steps 1 --warmup 3 --no-e2e > /dev/null 2>&1; echo "ncu rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_route_scatter -c 1 -o gpurun_out/route_full -f python bench.py --sharded --steps 1 --warmup 3 --no-e2e > /dev/null 2>&1; echo "ncu full rc=$?"
