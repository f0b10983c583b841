#!/usr/bin/env python
"""Benchmark of the B200 GSH join (BASELINE.json metric: join input tuples/s, plus output tuples/s
and % of HBM roofline).

Default workload = BASELINE.json configs[1] (cfg2): |R| = |S| = 2^27 uniform keys, 1:1 PK-FK,
COUNT mode, one B200.  A step = one full gsh_join (histogram, two partition passes, classify,
[detect, split,] NM-join, [skewed join]) over device-resident inputs.  Inputs (2 GiB) exceed
the 126 MB L2, so no flush is needed between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl gsh|reference] [--workload cfg2|cfg1|zipf]
  N > 1: launched by torch.distributed.run; hash-sharded join over NCCL (weak scaling: each rank
  holds a cfg2-sized shard).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

MEASURED_PEAKS = os.path.join(ROOT, "MEASURED_PEAKS.json")
PROFILE_SUMMARY = os.path.join(ROOT, "profiles", "ncu_traffic.json")
FALLBACK_HBM_GBS = 6650.0  # /opt/skills/guides/B200_PROFILING.md fallback
DEVSTATE_BYTES = 152        # sizeof(gsh::DevState): D2H'd twice per step (classify + final)

WORKLOADS = {
    # name: (kind, n per side (per rank), theta, description)
    "cfg2": ("pkfk", 1 << 27, 0.0, "cfg2: |R|=|S|=2^27 uniform keys, 1:1 PK-FK (theta=0), COUNT"),
    "cfg1": ("zipf", 1 << 20, 1.0, "cfg1: |R|=|S|=2^20 Zipf theta=1.0 both sides, COUNT"),
    "zipf05": ("zipf", 1 << 27, 0.5, "cfg3 point: |R|=|S|=2^27 Zipf theta=0.5 both sides, COUNT"),
    "zipf075": ("zipf", 1 << 27, 0.75, "cfg3 point: |R|=|S|=2^27 Zipf theta=0.75 both sides, COUNT"),
    "zipf10s": ("zipf", 1 << 24, 1.0, "cfg3-shaped (scaled): |R|=|S|=2^24 Zipf theta=1.0 both sides, COUNT"),
    "zipf15s": ("zipf", 1 << 22, 1.5, "cfg3-shaped (scaled): |R|=|S|=2^22 Zipf theta=1.5 both sides, COUNT"),
    "graph": ("graph", 1 << 26, 0.909, "cfg4-shaped (scaled): 2^26-edge power-law graph self-join (dst, src), COUNT"),
    "pkfk28": ("pkfk", 1 << 28, 0.0, "scale point: |R|=|S|=2^28 uniform 1:1 PK-FK (cfg5's per-GPU share at G=8), COUNT"),
    "pkfk29": ("pkfk", 1 << 29, 0.0, "scale point: |R|=|S|=2^29 uniform 1:1 PK-FK (4x cfg2; 2^30 input tuples), COUNT"),
    "pkfk30": ("pkfk", 1 << 30, 0.0, "scale point: |R|=|S|=2^30 uniform 1:1 PK-FK (8x cfg2; 2^31 input tuples), COUNT"),
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gsh", choices=["gsh", "reference"])
    ap.add_argument("--workload", default="cfg2", choices=sorted(WORKLOADS))
    ap.add_argument("--seed", type=int, default=0x6A5)
    ap.add_argument("--mode", default="count", choices=["count", "materialize"])
    ap.add_argument("--detect", default="exact", choices=["exact", "sampled"],
                    help="skew detection: exact counts (default) or the paper's 1%% sample + top-3 (L107, L112)")
    ap.add_argument("--out-cap", type=int, default=1 << 30, help="MATERIALIZE output capacity (pairs)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    return ap.parse_args()


def hbm_peak():
    try:
        d = json.load(open(MEASURED_PEAKS))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


_SAMPLER_SRC = r"""
import json, sys, time
import pynvml
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(int(sys.argv[1]))
bits = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40, "sw_power_cap": 0x4}
print(json.dumps({"max": pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)}), flush=True)
rows = []
import select
while True:
    r, _, _ = select.select([sys.stdin], [], [], 0.02)
    if r:
        break
    try:
        sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
        e = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
        rows.append((sm, [k for k, b in bits.items() if e & b]))
    except Exception:
        pass
print(json.dumps({"rows": rows}), flush=True)
"""


class ClockSampler:
    """SM clocks + throttle reasons sampled every 20 ms during the timed region, by NVML in a
    separate process (a sampler thread here would contend for the GIL with the launch loop and
    open gaps between steps); falls back to `nvidia-smi -lms 100`."""

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.max_mhz = None
        self.mode = None

    def __enter__(self):
        try:
            import pynvml  # noqa: F401  (the sampler process needs it)
            self.proc = subprocess.Popen([sys.executable, "-c", _SAMPLER_SRC, str(self.index)], stdin=subprocess.PIPE,
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.max_mhz = json.loads(self.proc.stdout.readline())["max"]   # sampler is running
            self.mode = "nvml"
        except Exception:
            self.proc = None
            self.mode = "smi"
            q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
            try:
                self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                              "--format=csv,noheader,nounits", "-lms", "100"],
                                             stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            except Exception:
                self.proc = None
        return self

    def __exit__(self, *a):
        if not self.proc:
            return
        try:
            if self.mode == "nvml":
                out, _ = self.proc.communicate(input="stop\n", timeout=10)
                for line in out.splitlines():
                    if line.startswith("{"):
                        d = json.loads(line)
                        if "rows" in d:
                            self.rows = [(float(r[0]), list(r[1])) for r in d["rows"]]
            else:
                time.sleep(0.15)
                self.proc.terminate()
                out, _ = self.proc.communicate(timeout=5)
                names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
                for line in out.splitlines():
                    p = [x.strip() for x in line.split(",")]
                    if len(p) == 6 and p[0].replace(".", "").isdigit():
                        self.max_mhz = float(p[1])
                        self.rows.append((float(p[0]), [names[i] for i in range(4) if p[2 + i].lower() == "active"]))
        except Exception:
            self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unsampled"], "samples": 0}
        sm = [r[0] for r in self.rows]
        reasons = sorted({x for r in self.rows for x in r[1]})
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": self.max_mhz, "reasons": reasons,
                "samples": len(self.rows), "source": self.mode}


def make_data(kind, n, theta, seed, device, rank=0):
    import datagen
    return datagen.make_workload(kind, n, theta, seed=seed + 7919 * rank, device=device)


def cpu_baseline(kind, n, theta, seed, budget_s=12.0):
    """The oracle (oracle/, plain C hash join, threaded probe) on a bounded sample of the workload."""
    import numpy as np

    import datagen
    import oracle
    ns = min(n, 1 << 23)
    rk, rp, sk, sp = datagen.make_workload(kind, ns, theta, seed=seed)
    a = [t.numpy().view(np.uint32) for t in (rk, rp, sk, sp)]
    threads = os.cpu_count() or 1
    t0 = time.perf_counter()
    reps = 0
    while True:
        oracle.join(*a, nthreads=threads)
        reps += 1
        if time.perf_counter() - t0 >= budget_s or reps >= 500:
            break
    dt = time.perf_counter() - t0
    return {"value": 2 * ns * reps / dt, "unit": "input tuples/s", "cores": threads, "kind": "oracle",
            "sample": f"{kind} |R|=|S|={ns} theta={theta}, {reps} joins in {dt:.1f}s (hash build 1 thread, probe "
                      f"{threads} threads)"}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle as the reference arm (no upstream code exists; PAPER.md
    only).  Rank 0 only."""
    kind, n, theta, desc = WORKLOADS[args.workload]
    if rank != 0:
        return
    import numpy as np

    import datagen
    import oracle
    ns = min(n, 1 << 21)
    rk, rp, sk, sp = datagen.make_workload(kind, ns, theta, seed=args.seed)
    a = [t.numpy().view(np.uint32) for t in (rk, rp, sk, sp)]
    threads = os.cpu_count() or 1
    for _ in range(args.warmup):
        oracle.join(*a, nthreads=threads)
    t0 = time.perf_counter()
    cnt = 0
    for _ in range(args.steps):
        cnt, _, _ = oracle.join(*a, nthreads=threads)
    dt = time.perf_counter() - t0
    v = 2 * ns * args.steps / dt
    print(json.dumps({
        "impl": "reference", "metric": "join input tuples/s", "value": v, "unit": "input tuples/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": desc, "sample_n_per_side": ns},
        "cpu_baseline": {"value": v, "unit": "input tuples/s", "cores": threads, "kind": "oracle",
                         "sample": f"{kind} |R|=|S|={ns} theta={theta} per step"},
        "e2e": {"value": v, "unit": "input tuples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "output_tuples_per_step": cnt}))


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    import paper_conf_icde_caic24_b200 as gsh

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    kind, n, theta, desc = WORKLOADS[args.workload]
    if args.mode == "materialize":
        desc = desc.replace("COUNT", "MATERIALIZE")
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    rk, rp, sk, sp = make_data(kind, n, theta, args.seed, dev, rank)
    torch.cuda.synchronize()
    extra = json.loads(os.environ.get("GSH_BENCH_CFG", "{}"))  # experiments only
    if args.detect == "sampled":
        extra["detect_mode"] = 1
    # per-phase CUDA events stay on inside the timed region (the roofline's kernel time is
    # measured live there); they cost ~30 us of host time per call, included in the step time
    cfg = gsh.make_config(timing=True, **extra)
    if world > 1:
        from paper_conf_icde_caic24_b200 import sharded

        def step():
            return sharded.join_sharded(rk, rp, sk, sp, config=cfg)
    else:
        ws = torch.empty(gsh.workspace_bytes(n, n, cfg), dtype=torch.uint8, device=dev)
        out = torch.empty((args.out_cap, 2), dtype=torch.int32, device=dev) if args.mode == "materialize" else None

        def step():
            return gsh.join(rk, rp, sk, sp, mode=args.mode, out=out, config=cfg, workspace=ws)

    for _ in range(max(3, args.warmup)):
        r = step()
    stream = torch.cuda.current_stream()
    phases = {}
    launches = 0
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        e0.record(stream)
        for _ in range(args.steps):
            r = step()
            for k, v in r.stats.items():
                if k.startswith("ms_"):
                    phases[k] = phases.get(k, 0.0) + v
            launches += r.stats.get("launches", 0)
        e1.record(stream)
        torch.cuda.synchronize()
    if dist:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    if dist:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    total_in = 2 * n * world * args.steps
    value = total_in / (ms / 1e3)
    out_per_s = r.count * args.steps / (ms / 1e3)
    phases = {k: v / args.steps for k, v in phases.items()}

    # roofline of the dominant kernel: the phase with the largest share of the step
    peak, peak_src = hbm_peak()
    clocks = clk.summary()
    n_tot = 2 * n
    st = r.stats
    heavy_t = st.get("heavy_tuples_r", 0) + st.get("heavy_tuples_s", 0)
    # algorithmic bytes per launch: hist 4 B, each pass 16 B, NM 8 B per normal tuple
    # (+ the pre-partition pass beyond 2^28 per side: 4 B count + 16 B split per tuple; with it the
    # phase figures below are summed over the 2^prepass_bits sub-joins)
    algo = {"ms_hist": 4 * n_tot, "ms_pass1": 16 * n_tot, "ms_pass2": 16 * n_tot, "ms_nmjoin": 8 * (n_tot - heavy_t),
            "ms_prepass": 20 * n_tot}
    kernels = {"ms_prepass": "k_split_count + k_split_scatter", "ms_pass1": "k_scatter (pass 1)", "ms_pass2": "k_scatter (pass 2)", "ms_nmjoin": "k_nmjoin_ring",
               "ms_hist": "k_hist2d", "ms_skewjoin": "k_skewjoin"}
    dom = max(list(algo) + ["ms_skewjoin"], key=lambda k: phases.get(k, 0.0))
    traffic = None
    try:
        prof = json.load(open(PROFILE_SUMMARY))
        traffic = prof.get(args.workload, {}).get(dom)
    except Exception:
        pass
    if dom == "ms_skewjoin":
        # ALU roofline of the dense skewed-key tiles: the inner loop's SASS issues
        # 7.0 ALU-pipe ops per pair (LOP3 3.25, SHF 2.25, IADD3 1.5; the IMADs go to the FMA pipe,
        # which ncu shows at ~1/3 of its issue rate), and the ALU pipe retires 64 lanes/clk/SM ->
        # 64 / 7.0 = 9.14 pairs/clk/SM x 148 SMs x max SM clock
        mhz = clocks.get("sm_max_mhz") or 1965.0
        alu_peak = (64 / 7.0) * 148 * mhz * 1e6 / 1e9
        achieved = st.get("skew_pairs", 0) / (phases[dom] / 1e3) / 1e9 if phases.get(dom) else None
        roofline = {"bound": "alu", "kernel": kernels[dom], "achieved": achieved, "peak": alu_peak,
                    "peak_source": "derived: 64 ALU lanes/clk/SM / 7.0 ALU ops per pair x 148 SMs x max SM clock",
                    "unit": "Gpairs/s", "frac": (achieved / alu_peak) if achieved else None, "traffic": traffic,
                    "algorithmic_pairs_per_launch": st.get("skew_pairs", 0)}
    else:
        achieved = algo[dom] / (phases[dom] / 1e3) / 1e9 if phases.get(dom) else None
        roofline = {"bound": "hbm", "kernel": kernels[dom], "achieved": achieved, "peak": peak,
                    "peak_source": peak_src, "unit": "GB/s", "frac": (achieved / peak) if achieved else None,
                    "traffic": traffic, "algorithmic_bytes_per_launch": algo[dom]}

    # end-to-end through the public API with host buffers (H2D inside the timed region)
    e2e = None
    if not args.no_e2e and world == 1:
        hk = [t.cpu().pin_memory() for t in (rk, rp, sk, sp)]
        ws_h = torch.empty(gsh._lib.load().gsh_host_workspace_bytes(n, n, 0, 0, None), dtype=torch.uint8, device=dev)
        for _ in range(2):
            gsh.join_host(*hk, workspace=ws_h)
        ke = max(2, min(args.steps, 5))
        torch.cuda.synchronize()
        h0 = torch.cuda.Event(enable_timing=True)
        h1 = torch.cuda.Event(enable_timing=True)
        h0.record(stream)
        for _ in range(ke):
            rr = gsh.join_host(*hk, workspace=ws_h)
        h1.record(stream)
        torch.cuda.synchronize()
        ems = h0.elapsed_time(h1)
        assert rr.count == r.count and rr.checksum == r.checksum
        e2e = {"value": 2 * n * ke / (ems / 1e3), "unit": "input tuples/s", "h2d_bytes_per_step": 16 * n,
               "d2h_bytes_per_step": 2 * DEVSTATE_BYTES, "steps": ke, "ms_per_step": ems / ke,
               "api": "gsh_join_host (pinned host buffers)"}
        del ws_h, hk

    base = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        base = cpu_baseline(kind, n, theta, args.seed)

    if rank == 0:
        line = {
            "metric": "join input tuples/s", "value": value, "unit": "input tuples/s", "n_gpus": world,
            "steps": args.steps, "warmup": max(3, args.warmup), "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (datagen, seeded)",
            "config": {"workload": desc, "n_r": n * world, "n_s": n * world, "mode": args.mode, "detect": args.detect,
                       "parallelism": f"hash-sharded x{world}" if world > 1 else "single GPU",
                       "l2": "inputs 2 GiB per GPU > 126 MB L2: no flush needed", "seed": args.seed},
            "output_tuples_per_s": out_per_s, "count": r.count, "checksum": f"{r.checksum:#018x}",
            "phases_ms": phases, "roofline": roofline, "clocks": clocks, "e2e": e2e,
            "gpu_launches": launches, "cpu_baseline": base,
            "stats": {k: v for k, v in r.stats.items() if not k.startswith("ms_")},
        }
        print(json.dumps(line))
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
