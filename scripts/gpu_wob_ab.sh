#!/bin/bash
# A/B of the scatter write-out: per staged position (cfg 0, default) vs per bucket run (cfg 2:
# both passes, cfg 3: pass 2 only); parity subset under cfg 2 first.
mkdir -p gpurun_out
GSH_SCATTER_CFG=2 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "partition_phase or ladder or materialize_pairs or edge or unaligned" > gpurun_out/wob_pytest.log 2>&1; echo "wob pytest rc=$?"; tail -2 gpurun_out/wob_pytest.log
for rep in 1 2; do
for c in 0 2 3; do
  GSH_SCATTER_CFG=$c timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/wob_cfg$c.json 2>/dev/null
  echo "cfg $c:"; python scripts/show_bench.py gpurun_out/wob_cfg$c.json | head -2
done
done
for c in 0 2; do
  GSH_SCATTER_CFG=$c timeout 300 python bench.py --workload zipf15 --input-side --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > gpurun_out/wob15_cfg$c.json 2>/dev/null
  echo "zipf15 cfg $c:"; python scripts/show_bench.py gpurun_out/wob15_cfg$c.json | sed -n 2p
done
