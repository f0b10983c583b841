#!/bin/bash
# Full GPU suite + smoke + default bench line.
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/suite_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/suite_smoke.log
tail -2 gpurun_out/suite_smoke.log
timeout 2700 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/suite_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/suite_pytest.log
tail -14 gpurun_out/suite_pytest.log
timeout 900 python bench.py > gpurun_out/suite_bench.json 2> gpurun_out/suite_bench.err; echo "bench rc=$?"
python scripts/show_bench.py gpurun_out/suite_bench.json | head -3
