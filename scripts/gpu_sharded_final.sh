#!/bin/bash
# Multi-GPU code path on one GPU (final code): the native sharded driver over an in-process world of
# G logical ranks (--fake-ranks) and over an NCCL world of one (--sharded).  Code-path timings only.
mkdir -p gpurun_out
for args in "--fake-ranks 8 --exchange p2p" "--fake-ranks 8 --exchange a2a" "--fake-ranks 4 --exchange p2p --workload zipf10s" "--sharded --exchange a2a"; do
  tag=$(echo $args | tr ' ' '_' | tr -d '-')
  timeout 600 python bench.py $args --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/sh_$tag.json 2> gpurun_out/sh_$tag.err
  echo "$args rc=$?"
done
