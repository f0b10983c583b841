#!/usr/bin/env python
"""Per-CUDA-source-line metrics of one kernel from an ncu report (cuda,sass source view):
instructions executed, thread utilisation and warp-stall samples, top lines first.

usage: python scripts/ncu_lines.py REPORT KERNEL_REGEX [N]
"""
import csv
import subprocess
import sys

rep, kre = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "-k",
                      f"regex:{kre}", "--launch-count", "1"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
agg = {}
cur_file, cur = None, None
hdr = None
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if not hdr or len(r) < len(hdr):
        continue
    if r[0]:  # a CUDA source line
        cur = (cur_file, int(r[0]), r[1][:90])
        continue
    if cur is None:
        continue
    d = dict(zip(hdr[2:], r[2:]))
    def g(k):
        try:
            return float(d.get(k, "0") or 0)
        except ValueError:
            return 0.0
    a = agg.setdefault(cur, [0.0, 0.0, 0.0])
    a[0] += g("Instructions Executed")
    a[1] += g("Thread Instructions Executed")
    a[2] += g("Warp Stall Sampling (All Samples)")
ti = sum(v[0] for v in agg.values()) or 1
ts = sum(v[2] for v in agg.values()) or 1
print(f"total warp-instr {ti:.3g}  stall samples {ts:.0f}")
for key, v in sorted(agg.items(), key=lambda kv: -(kv[1][2] / ts + kv[1][0] / ti))[:top]:
    f, ln, src = key
    print(f"{f}:{ln:<5d} instr {100 * v[0] / ti:5.1f}%  thr/inst {v[1] / max(v[0], 1):5.1f}  stall {100 * v[2] / ts:5.1f}%  {src}")
