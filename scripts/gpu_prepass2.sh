#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "prepass or pkfk_large or materialize" > gpurun_out/pytest_prepass.log 2>&1
echo "pytest rc=$?"; tail -3 gpurun_out/pytest_prepass.log
bash scripts/gpu_prepass_ncu.sh
python - <<'PY'
import csv, collections
rows=list(csv.reader(open('gpurun_out/prepass_launches.csv')))
for i,r in enumerate(rows):
    if 'Kernel Name' in r: hdr=r; st=i+1; break
ki,mi,vi,ii=(hdr.index(x) for x in ('Kernel Name','Metric Name','Metric Value','ID'))
d=collections.defaultdict(dict)
for r in rows[st:]: d[(int(r[ii]),r[ki][:28])][r[mi]]=r[vi]
for k,v in sorted(d.items())[:8]: print(k, v)
PY
