#!/bin/bash
# Gbase bucket size A/B (4096 default vs 2048): tests + Table I sweep.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_gbase.py -q -x > gpurun_out/gbase3_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/gbase3_pytest.log
timeout 1200 python bench.py --gbase-sweep > gpurun_out/gbase_sweep3.json 2> gpurun_out/gbase_sweep3.err; echo "sweep 4096 rc=$?"
GSH_LIB=$PWD/build/var_gb2048/libgsh.so timeout 1200 python bench.py --gbase-sweep > gpurun_out/gbase_sweep3b.json 2> gpurun_out/gbase_sweep3b.err; echo "sweep 2048 rc=$?"
python - <<'PY'
import json
for f in ("gpurun_out/gbase_sweep3.json", "gpurun_out/gbase_sweep3b.json"):
    d = json.loads(open(f).read().strip().splitlines()[-1])
    print(f, [(p["theta"], round(p["gbase"]["partition_ms"], 2), round(p["gbase"]["join_ms"], 1)) for p in d["points"] if p["gbase"]])
PY
