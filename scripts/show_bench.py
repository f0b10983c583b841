#!/usr/bin/env python
"""Print the key numbers of a bench.py JSON line (gpurun_out/bench_TAG.json)."""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(f"value {d['value'] / 1e9:.2f} G tuples/s  {d['ms_per_step']:.3f} ms/step  roofline {d['roofline']['kernel']} "
      f"{d['roofline']['frac']:.3f}")
print("phases", {k: round(v, 3) for k, v in d["phases_ms"].items()})
print("fractions", {k: round(v, 3) for k, v in (d.get("pass_fractions") or {}).items() if v})
for p in (d.get("theta_sweep") or {}).get("points", []):
    print(f"  theta {p['theta']}: " + " ".join(f"{k}={v:.3f}" for k, v in p.items() if k.endswith("_frac") and v),
          {k: round(v, 3) for k, v in p["phases_ms"].items() if v})
for p in (d.get("theta_sweep") or {}).get("dense", []):
    print(f"  dense theta {p['theta']} n {p['n_per_side']}: {p['skew_pairs_per_s'] / 1e12:.3f} Tpairs/s")
if d.get("sharded"):
    print("sharded", d["sharded"])
