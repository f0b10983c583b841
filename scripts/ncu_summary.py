#!/usr/bin/env python
"""Summarise an ncu report (raw page) for the GSH kernels: time, DRAM bytes, throughput, top stalls."""
import csv
import subprocess
import sys

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
hdr, units = rows[0], rows[1]
col = {h: i for i, h in enumerate(hdr)}
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_shared_mem", "launch__occupancy_limit_registers", "launch__grid_size",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", "lts__t_bytes.sum",
        "smsp__thread_inst_executed_per_inst_executed.ratio"]
for r in rows[2:]:
    print("=" * 8, r[col["Kernel Name"]][:60])
    for k in KEYS:
        if k in col:
            print(f"  {k:62s} {r[col[k]]:>14s} {units[col[k]]}")
    st = []
    for h, i in col.items():
        if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued"):
            try:
                st.append((float(r[i].replace(",", "")), h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            except ValueError:
                pass
    tot = sum(v for v, _ in st) or 1
    print("  stalls:", ", ".join(f"{n} {100 * v / tot:.0f}%" for v, n in sorted(st, reverse=True)[:6]))
    pipes = []
    for h, i in col.items():
        if h.startswith("sm__inst_executed_pipe_") and h.endswith(".avg.pct_of_peak_sustained_active"):
            try:
                v = float(r[i].replace(",", ""))
            except ValueError:
                continue
            if v > 5:
                pipes.append((v, h.split("sm__inst_executed_pipe_")[1].split(".")[0]))
    print("  pipes:", ", ".join(f"{n} {v:.0f}%" for v, n in sorted(pipes, reverse=True)[:6]))
