#!/usr/bin/env python
"""Summarise a round's GPU profiles into profiles/ (tracked):

  profiles/<tag>_launches.md   per-kernel share of the step from the ncu launch list
                               (gpu__time_duration, cold-cache and serialised: compare SHARES)
  profiles/<tag>_ncu_full.md   one --set full capture per top kernel: time, DRAM bytes,
                               throughputs, occupancy, top stall reasons
  profiles/ncu_traffic.json    DRAM traffic per launch of the roofline kernels, read by bench.py

usage: python scripts/summarize_profiles.py TAG [workload]
"""
import collections
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1]
workload = sys.argv[2] if len(sys.argv) > 2 else "cfg2"
out_dir = os.path.join(ROOT, "profiles")
os.makedirs(out_dir, exist_ok=True)


def short(name):
    n = name.split("(")[0].replace("void ", "").replace("gsh::", "")
    return n.split("<")[0] if n.startswith("k_") else n[:40]


# ------------------------------------------------------------------ launch list
lrows = [r for r in csv.reader(open(os.path.join(ROOT, "gpurun_out", f"launches_{tag}.csv"))) if r]
hdr = next(r for r in lrows if "Kernel Name" in r and "Metric Name" in r)
per = collections.OrderedDict()
for r in lrows:
    if len(r) != len(hdr) or r is hdr or r[0] == "ID":
        continue
    d = dict(zip(hdr, r))
    per.setdefault(d["ID"], {"name": d["Kernel Name"]})[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
launches = list(per.values())
ours = [x for x in launches if "gsh::" in x["name"] or short(x["name"]).startswith("k_")]
agg = collections.OrderedDict()
for x in ours:
    k = short(x["name"])
    a = agg.setdefault(k, {"n": 0, "ns": 0.0, "rd": 0.0, "wr": 0.0})
    a["n"] += 1
    a["ns"] += x.get("gpu__time_duration.sum", 0.0)
    a["rd"] += x.get("dram__bytes_read.sum", 0.0)
    a["wr"] += x.get("dram__bytes_write.sum", 0.0)
tot = sum(a["ns"] for a in agg.values()) or 1.0
lines = [f"# {tag}: launch list of `python bench.py --steps 2 --warmup 1` ({workload})", "",
         "ncu `--metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none`.",
         "Per-launch times are cold-cache and serialised (ncu replays): compare the SHARE of the step,",
         "not absolute times.  All launches of the run (warm-up + timed) are aggregated.", "",
         "| kernel | launches | share of GSH kernel time | mean µs/launch | mean DRAM read MB | mean DRAM write MB |",
         "|---|---|---|---|---|---|"]
for k, a in sorted(agg.items(), key=lambda kv: -kv[1]["ns"]):
    lines.append(f"| {k} | {a['n']} | {100 * a['ns'] / tot:.1f} % | {a['ns'] / a['n'] / 1e3:.1f} | "
                 f"{a['rd'] / a['n'] / 1e6:.1f} | {a['wr'] / a['n'] / 1e6:.1f} |")
lines.append("")
lines.append(f"Kernels of other libraries in the run (data generation by torch): "
             f"{len(launches) - len(ours)} launches, not part of the timed join.")
open(os.path.join(out_dir, f"{tag}_launches.md"), "w").write("\n".join(lines) + "\n")

# traffic per roofline kernel: from the --set full capture below (one capture per kernel, the
# contract's definition); the launch-list DRAM columns are a fallback when present
traffic = {}
scat = [x for x in ours if short(x["name"]) == "k_scatter"]
for i, key in ((0, "ms_pass1"), (1, "ms_pass2")):
    xs = scat[i::2]
    v = sum(x.get("dram__bytes_read.sum", 0) + x.get("dram__bytes_write.sum", 0) for x in xs) / max(len(xs), 1)
    if v:
        traffic[key] = v
for kname, key in (("k_nmjoin_ring", "ms_nmjoin"), ("k_hist2d", "ms_hist")):
    xs = [x for x in ours if short(x["name"]) == kname]
    v = sum(x.get("dram__bytes_read.sum", 0) + x.get("dram__bytes_write.sum", 0) for x in xs) / max(len(xs), 1)
    if v:
        traffic[key] = v

# ------------------------------------------------------------------ full capture
rep = os.path.join(ROOT, "gpurun_out", f"prof_{tag}.ncu-rep")
if os.path.exists(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    h, units = rows[0], rows[1]
    col = {x: i for i, x in enumerate(h)}
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
            "launch__grid_size", "launch__block_size", "launch__occupancy_limit_shared_mem",
            "launch__occupancy_limit_registers", "smsp__thread_inst_executed_per_inst_executed.ratio",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum"]
    out = [f"# {tag}: ncu --set full (one capture per kernel, `--clock-control none`, {workload})", ""]
    for r in rows[2:]:
        out.append(f"## {short(r[col['Kernel Name']])} (launch id {r[col['ID']]})")
        out.append("")
        for k in keys:
            if k in col:
                out.append(f"- {k}: {r[col[k]]} {units[col[k]]}")
        st = []
        for k, i in col.items():
            if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
                try:
                    st.append((float(r[i].replace(",", "")), k.split("stalled_")[1]))
                except ValueError:
                    pass
        s = sum(v for v, _ in st) or 1
        out.append("- top stalls: " + ", ".join(f"{n} {100 * v / s:.0f}%" for v, n in sorted(st, reverse=True)[:6]))
        pipes = []
        for k, i in col.items():
            if k.startswith("sm__inst_executed_pipe_") and k.endswith(".avg.pct_of_peak_sustained_active"):
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                if v > 5:
                    pipes.append((v, k.split("pipe_")[1].split(".")[0]))
        out.append("- busiest pipes: " + ", ".join(f"{n} {v:.0f}%" for v, n in sorted(pipes, reverse=True)[:5]))
        out.append("")
    open(os.path.join(out_dir, f"{tag}_ncu_full.md"), "w").write("\n".join(out) + "\n")
    nscat = 0
    for r in rows[2:]:
        k = short(r[col["Kernel Name"]])
        b = float(r[col["dram__bytes_read.sum"]].replace(",", "")) * (1e9 if units[col["dram__bytes_read.sum"]] == "Gbyte" else 1e6 if units[col["dram__bytes_read.sum"]] == "Mbyte" else 1) + \
            float(r[col["dram__bytes_write.sum"]].replace(",", "")) * (1e9 if units[col["dram__bytes_write.sum"]] == "Gbyte" else 1e6 if units[col["dram__bytes_write.sum"]] == "Mbyte" else 1)
        if k == "k_scatter":
            traffic["ms_pass1" if nscat % 2 == 0 else "ms_pass2"] = b
            nscat += 1
        elif k == "k_nmjoin_ring":
            traffic["ms_nmjoin"] = b
        elif k == "k_hist2d":
            traffic["ms_hist"] = b
tpath = os.path.join(out_dir, "ncu_traffic.json")
tj = json.load(open(tpath)) if os.path.exists(tpath) else {}
if traffic:
    tj[workload] = {k: v / 1e9 for k, v in traffic.items()}
    tj["_unit"] = "GB per launch (dram__bytes_read.sum + dram__bytes_write.sum)"
    tj["_source"] = f"profiles/{tag}_ncu_full.md (ncu --set full) / {tag}_launches.md"
json.dump(tj, open(tpath, "w"), indent=1)
print("wrote", [f for f in os.listdir(out_dir) if f.startswith(tag)], "traffic", tj.get(workload))
