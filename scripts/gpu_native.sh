#!/bin/bash
# Native multi-GPU driver on the one-GPU box: GPU tests + bench in its sharded modes.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sharded_native.py tests/test_gpu_sharded.py -x -q --durations=8 > gpurun_out/pytest_native.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_native.log
tail -15 gpurun_out/pytest_native.log
for ex in p2p a2a; do
  timeout 300 python bench.py --fake-ranks 4 --exchange $ex --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_nfake4_$ex.json 2> gpurun_out/bench_nfake4_$ex.err; echo "nfake4 $ex rc=$?"
done
timeout 300 python bench.py --fake-ranks 4 --driver python --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_pfake4.json 2> gpurun_out/bench_pfake4.err; echo "pfake4 rc=$?"
for ex in p2p a2a; do
  timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --sharded --exchange $ex --steps 5 --warmup 3 > gpurun_out/bench_nccl1_$ex.json 2> gpurun_out/bench_nccl1_$ex.err; echo "nccl1 $ex rc=$?"
done
timeout 300 python bench.py --sharded --workload zipf10 --steps 3 --warmup 3 --no-e2e > gpurun_out/bench_nccl1_z10.json 2> gpurun_out/bench_nccl1_z10.err; echo "nccl1 z10 rc=$?"
tail -3 gpurun_out/bench_n*.err gpurun_out/bench_p*.err
