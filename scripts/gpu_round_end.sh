#!/bin/bash
# Round-end measurements: ncu launch list + full captures (cfg2), the default bench line, the
# reference (oracle) arm, and the workload sweep (Zipf theta points, graph, scale points).
mkdir -p gpurun_out
bash scripts/gpu_profile_round.sh ${1:-r01}
timeout 600 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$?"
for w in cfg1 zipf05 zipf075 zipf10s zipf15s graph pkfk28 pkfk30; do
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/sweep_$w.json 2> gpurun_out/sweep_$w.err
  echo "$w rc=$?"
done
