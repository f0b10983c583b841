"""profiles/<tag>_sweep.md from gpurun_out/sweep_*.json (scripts/gpu_round_end.sh)."""
import glob
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
order = ["cfg2", "pkfk28", "pkfk30", "zipf05", "zipf075", "cfg1", "zipf10s", "zipf15s", "graph"]
rows = {}
for f in glob.glob(os.path.join(ROOT, "gpurun_out", "sweep_*.json")) + [os.path.join(ROOT, "gpurun_out", "bench_full.json")]:
    try:
        d = json.load(open(f))
    except Exception:
        continue
    w = os.path.basename(f)[6:-5] if "sweep_" in f else "cfg2"
    rows[w] = d
out = [f"# {tag}: workload sweep (one B200, COUNT, `bench.py --workload W --steps 3 --warmup 3`; cfg2 = the default bench line)",
       "",
       "Input tuples/s = (|R|+|S|) / step; output tuples/s = join count / step.  Phases in ms (CUDA events).",
       "",
       "| workload | input tuples/s | output tuples/s | ms/step | hist | pass 1 | pass 2 | detect | split | NM | skew | heavy keys | large parts |",
       "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
for w in order + sorted(set(rows) - set(order)):
    if w not in rows:
        continue
    d = rows[w]
    p = d["phases_ms"]
    s = d["stats"]
    out.append(f"| {d['config']['workload']} | {d['value']:.3g} | {d['output_tuples_per_s']:.3g} | {d['ms_per_step']:.3f} | "
               f"{p['ms_hist']:.3f} | {p['ms_pass1']:.3f} | {p['ms_pass2']:.3f} | {p['ms_detect']:.3f} | {p['ms_split']:.3f} | "
               f"{p['ms_nmjoin']:.3f} | {p['ms_skewjoin']:.3f} | {s['n_heavy']} | {s['n_large']} |")
mat = sorted(glob.glob(os.path.join(ROOT, "gpurun_out", "sweepmat_*.json")))
if mat:
    out += ["", "MATERIALIZE (`--mode materialize --out-cap 2^30`: pairs written to an 8 GiB device buffer; the NM-join"
                " counts each item's matches, reserves one output range, then emits)", "",
            "| workload | input tuples/s | output tuples/s | ms/step | NM | skew | written | overflow |", "|---|---|---|---|---|---|---|---|"]
    for f in mat:
        try:
            d = json.load(open(f))
        except Exception:
            continue
        p, s_ = d["phases_ms"], d["stats"]
        out.append(f"| {d['config']['workload'].replace('COUNT', 'MATERIALIZE')} | {d['value']:.3g} | {d['output_tuples_per_s']:.3g} | {d['ms_per_step']:.3f} | "
                   f"{p['ms_nmjoin']:.3f} | {p['ms_skewjoin']:.3f} | {s_['written']} | {s_['overflow']} |")
open(os.path.join(ROOT, "profiles", f"{tag}_sweep.md"), "w").write("\n".join(out) + "\n")
print("\n".join(out))
