#!/bin/bash
# End-of-round ncu: launch list + one --set full capture of each cfg2 kernel (final code).
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_r02end.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/launches_r02end.out 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_scatter|k_nmjoin_ring|k_hist2d" -s 12 -c 4 \
    -o gpurun_out/prof_r02end python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_r02end.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_r02end.log
