#!/bin/bash
# Round-2 end check: smoke, full GPU suite, default bench line (theta sweep with the hybrid arm),
# reference arm, launch list of the cfg2 step, ncu full of the Gbase-style join.
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/final_smoke.log
tail -2 gpurun_out/final_smoke.log
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/final_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/final_pytest_gpu.log
tail -4 gpurun_out/final_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err; echo "bench rc=$?"
python scripts/show_bench.py gpurun_out/final_bench.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_bench_ref.json 2> gpurun_out/final_bench_ref.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/final_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/final_launches.out 2>&1
echo "launches rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gbase_join -c 1 \
    -o gpurun_out/prof_gbase python scripts/gbase_once.py 0.5 > gpurun_out/ncu_gbase.log 2>&1
echo "ncu gbase rc=$?"; tail -2 gpurun_out/ncu_gbase.log
