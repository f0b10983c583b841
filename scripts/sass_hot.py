#!/usr/bin/env python
"""Hot SASS of one kernel in an ncu report: stall samples and executed instructions aggregated by
opcode, plus the top instructions.  usage: sass_hot.py REPORT KERNEL_REGEX [N]"""
import csv
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "-k", f"regex:{kern}", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(txt.splitlines()))
hdr = rows[1]
col = {h: i for i, h in enumerate(hdr)}
S, E = "Warp Stall Sampling (All Samples)", "Instructions Executed"


def f(x):
    try:
        return float(x)
    except ValueError:
        return None


data = [r for r in rows[2:] if len(r) == len(hdr) and f(r[col[S]]) is not None]
ts = sum(f(r[col[S]]) for r in data)
te = sum(f(r[col[E]]) or 0 for r in data)
print(f"{len(data)} SASS lines, {ts:.0f} stall samples, {te:.3g} warp instructions executed")
agg = {}
for r in data:
    t = r[1].strip().split()
    if not t:
        continue
    op = (t[1] if t[0].startswith("@") else t[0]).split(".")[0]
    a = agg.setdefault(op, [0.0, 0.0])
    a[0] += f(r[col[S]])
    a[1] += f(r[col[E]]) or 0
print("opcode      stall%   inst%")
for k, (s, e) in sorted(agg.items(), key=lambda x: -x[1][0])[:18]:
    print(f"{k:10s} {s / ts * 100:6.1f} {e / te * 100:7.1f}")
data.sort(key=lambda r: -f(r[col[S]]))
for r in data[:top]:
    print(f"{f(r[col[S]]) / ts * 100:5.1f}% exec {f(r[col[E]]) or 0:10.0f}  {r[0][-5:]}  {r[1].strip()[:90]}")
