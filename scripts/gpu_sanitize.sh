#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over the ladder (logs -> gpurun_out/).
mkdir -p gpurun_out
for t in memcheck racecheck synccheck; do
  SAN_TOOL=$t timeout 2400 compute-sanitizer --tool $t --print-limit 50 python scripts/sanitize_ladder.py > gpurun_out/sanitize_$t.log 2>&1
  echo "$t rc=$?"; tail -4 gpurun_out/sanitize_$t.log
done
