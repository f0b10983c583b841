#!/bin/bash
# NM ring experiments: full / stream-only / build-only timings of the cfg2 bench; phase clocks.
mkdir -p gpurun_out
for m in 0 1 2; do
  GSH_RING_DEBUG=$m timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ringdbg_$m.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/ringdbg_$m.json')); print('mode $m nm ms', d['phases_ms']['ms_nmjoin'])"
done
GSH_RING_DEBUG=3 timeout 300 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 >/dev/null | grep "ring clocks" | tail -2
