#!/usr/bin/env python
"""Benchmark of the B200 GSH join (BASELINE.json metric: join input tuples/s, plus output tuples/s
and % of HBM roofline).

Default workload = BASELINE.json configs[1] (cfg2): |R| = |S| = 2^27 uniform keys, 1:1 PK-FK,
COUNT mode, one B200.  A step = one full gsh_join (histogram, two partition passes, classify,
[detect, split,] NM-join, [skewed join]) over device-resident inputs.  Inputs (2 GiB) exceed
the 126 MB L2, so no flush is needed between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl gsh|reference] [--workload cfg2|cfg1|zipf]
  N > 1: one process per GPU under torch.distributed.run (started here when WORLD_SIZE is unset);
  hash-sharded join: gsh_join_sharded (the native driver in libgsh) over an NCCL communicator,
  the route kernel storing straight into the peers' receive buffers (--exchange p2p, default) or
  NCCL all-to-all (--exchange a2a); --driver python runs sharded.join_sharded instead.  Weak
  scaling: each rank holds a shard of the workload's per-GPU size, so the job joins N x that size.
  --fake-ranks G: the same sharded step for G logical ranks sharing ONE GPU (threads, the
  library's local world): exercises the multi-GPU code path on a one-GPU box; never the headline.
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
DEVSTATE_BYTES = 568        # sizeof(gsh::DevState): D2H'd twice per step (classify + final)

WORKLOADS = {
    # name: (kind, n per side (per rank), theta, description)
    "cfg2": ("pkfk", 1 << 27, 0.0, "cfg2: |R|=|S|=2^27 uniform keys, 1:1 PK-FK (theta=0), COUNT"),
    "cfg1": ("zipf", 1 << 20, 1.0, "cfg1: |R|=|S|=2^20 Zipf theta=1.0 both sides, COUNT"),
    "zipf05": ("zipf", 1 << 27, 0.5, "cfg3 point: |R|=|S|=2^27 Zipf theta=0.5 both sides, COUNT"),
    "zipf075": ("zipf", 1 << 27, 0.75, "cfg3 point: |R|=|S|=2^27 Zipf theta=0.75 both sides, COUNT"),
    "zipf10": ("zipf", 1 << 27, 1.0, "cfg3 point: |R|=|S|=2^27 Zipf theta=1.0 both sides (use --input-side), COUNT"),
    "zipf15": ("zipf", 1 << 27, 1.5, "cfg3 point: |R|=|S|=2^27 Zipf theta=1.5 both sides (use --input-side), COUNT"),
    "zipf10s": ("zipf", 1 << 24, 1.0, "cfg3-shaped (scaled): |R|=|S|=2^24 Zipf theta=1.0 both sides, COUNT"),
    "zipf15s": ("zipf", 1 << 22, 1.5, "cfg3-shaped (scaled): |R|=|S|=2^22 Zipf theta=1.5 both sides, COUNT"),
    "graph": ("graph", 1 << 26, 0.909, "cfg4-shaped (scaled): 2^26-edge power-law graph self-join (dst, src), COUNT"),
    "graph28": ("graph", 1 << 28, 0.909, "cfg4: 2^28-edge power-law graph self-join (dst, src), V = 2^24, COUNT (~8.6e13 pairs)"),
    "pkfk28": ("pkfk", 1 << 28, 0.0, "scale point: |R|=|S|=2^28 uniform 1:1 PK-FK (cfg5's per-GPU share at G=8), COUNT"),
    "pkfk29": ("pkfk", 1 << 29, 0.0, "scale point: |R|=|S|=2^29 uniform 1:1 PK-FK (4x cfg2; 2^30 input tuples), COUNT"),
    "pkfk30": ("pkfk", 1 << 30, 0.0, "scale point: |R|=|S|=2^30 uniform 1:1 PK-FK (8x cfg2; 2^31 input tuples), COUNT"),
    "zipf07_29": ("zipf", 1 << 29, 0.7, "NEXT-3 (PAPER.md L170: 560M x 560M, theta=0.7) on one B200: |R|=|S|=2^29 Zipf theta=0.7 both sides, COUNT"),
    "pkfkzipf": ("pkfk_zipf", 1 << 27, 1.0, "skewed-FK PK-FK: |R|=|S|=2^27, R unique, S Zipf theta=1.0 over R's rows, COUNT"),
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
    ap.add_argument("--gbase-sweep", action="store_true",
                    help="GSH vs the Gbase-style join (NEXT-4) at the paper's Table I size (2^25 per side), one JSON line")
    ap.add_argument("--hybrid", action="store_true",
                    help="CSH's hybrid partition (gsh_config.hybrid, SURVEY NEXT-1): sampled skewed keys routed in pass 1")
    ap.add_argument("--out-cap", type=int, default=1 << 30, help="MATERIALIZE output capacity (pairs)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sweep", action="store_true", help="skip the theta_sweep sub-object (N=1 only)")
    ap.add_argument("--input-side", action="store_true",
                    help="time only the input side (partition, detect, split): gsh_config.input_side_only")
    ap.add_argument("--exchange", default="p2p", choices=["a2a", "p2p"],
                    help="multi-GPU exchange: the route kernel's direct peer stores (p2p) or NCCL all_to_all (a2a)")
    ap.add_argument("--sharded", action="store_true",
                    help="run the hash-sharded step over NCCL even with one GPU (world of one)")
    ap.add_argument("--driver", default="native", choices=["native", "python"],
                    help="multi-GPU protocol: gsh_join_sharded inside libgsh (native) or sharded.join_sharded")
    ap.add_argument("--fake-ranks", type=int, default=0,
                    help="run the sharded step for G logical ranks on one GPU (code-path check, not a headline)")
    return ap.parse_args()


def maybe_relaunch(args):
    """--gpus N > 1 without a torch.distributed environment: re-exec this script under
    torch.distributed.run with one process per GPU (the driver's own launch line)."""
    world = int(os.environ.get("WORLD_SIZE", "0"))
    if args.gpus > 1 and world == 0:
        import socket
        sk = socket.socket()
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
        sk.close()
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
        sys.exit(subprocess.call(cmd))
    if world and args.gpus != world and args.impl != "reference":
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")


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


def cpu_baseline(kind, n, theta, seed, rk=None, rp=None, sk=None, sp=None, gpu=None, budget_s=12.0):
    """The oracle (oracle/, plain C hash join, threaded probe) on the bench's own arrays (copied
    device -> host) when the whole join fits the budget (count and checksum must then equal the
    GPU result); otherwise on a bounded regenerated sample of the workload."""
    import numpy as np

    import datagen
    import oracle
    threads = os.cpu_count() or 1
    est_pairs = 2 * n if kind in ("pkfk", "pkfk_zipf") else None
    if rk is not None and est_pairs is not None and n <= (1 << 27):
        a = [t.cpu().numpy().view(np.uint32) for t in (rk, rp, sk, sp)]
        t0 = time.perf_counter()
        cnt, chk, _ = oracle.join(*a, nthreads=threads)
        dt = time.perf_counter() - t0
        if gpu is not None:
            assert (cnt, chk) == (gpu.count, gpu.checksum), "oracle and GPU disagree on the bench arrays"
        return {"value": 2 * n / dt, "unit": "input tuples/s", "cores": threads, "kind": "oracle",
                "sample": f"the bench's own arrays ({kind} |R|=|S|={n}, copied D2H), one join in {dt:.1f}s "
                          f"(hash build 1 thread, probe {threads} threads); count and checksum equal the GPU's",
                "matches_gpu": gpu is not None}
    ns = min(n, 1 << 23)
    rk, rp, sk, sp = datagen.make_workload(kind, ns, theta, seed=seed)
    a = [t.numpy().view(np.uint32) for t in (rk, rp, sk, sp)]
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


def pass_fractions(ph, st, n_tot):
    """HBM fraction of every input-side pass (algorithmic bytes) of one join."""
    peak, _ = hbm_peak()
    large = st.get("large_tuples", None)
    out = {}
    for k, b in (("ms_hist", 4 * n_tot), ("ms_pass1", 16 * n_tot), ("ms_pass2", 16 * n_tot)):
        ms = ph.get(k) or 0.0
        out[k.replace("ms_", "") + "_frac"] = (b / (ms * 1e6)) / peak if ms > 0 else None
    if large:
        for k, b in (("ms_detect", 8 * large), ("ms_split", 16 * large)):
            ms = ph.get(k) or 0.0
            out[k.replace("ms_", "") + "_frac"] = (b / (ms * 1e6)) / peak if ms > 0 else None
    return out


SWEEP = [  # (theta, n per side, input side only): BASELINE configs[2] points at full size
    (0.5, 1 << 27, False), (0.75, 1 << 27, False), (1.0, 1 << 27, True), (1.5, 1 << 27, True)]
DENSE = [(1.0, 1 << 24), (1.5, 1 << 22)]   # skewed-key phase at the largest sizes that finish in ~1-2 s


def theta_sweep(gsh, dev, seed, steps=3):
    """configs[2]: |R|=|S|=2^27 both-sides Zipf at theta in {0.5, 0.75, 1.0, 1.5}: per-phase ms and the
    HBM fraction of every input-side pass (theta >= 1.0: input side only -- the output is 8e13 to
    3e15 pairs), plus the skewed-key phase's pairs/s at the largest sizes that finish in seconds."""
    import datagen
    out = {"points": [], "dense": []}

    def timed(rk, rp, sk, sp, cfg, ws):
        r = gsh.join(rk, rp, sk, sp, config=cfg, workspace=ws)
        ph = {}
        for _ in range(steps):
            r = gsh.join(rk, rp, sk, sp, config=cfg, workspace=ws)
            for k, v in r.stats.items():
                if k.startswith("ms_"):
                    ph[k] = ph.get(k, 0.0) + v / steps
        return r, ph

    for theta, n, inp in SWEEP:
        rk, rp, sk, sp = datagen.make_workload("zipf", n, theta, seed=seed, device=dev)
        cfg = gsh.make_config(timing=True, input_side_only=inp)
        ws = torch.empty(gsh.workspace_bytes(n, n, gsh.make_config(hybrid=True)), dtype=torch.uint8, device=dev)
        r, ph = timed(rk, rp, sk, sp, cfg, ws)
        st = dict(r.stats)
        pt = {"theta": theta, "n_per_side": n, "input_side_only": inp, "phases_ms": ph,
              "n_large": st["n_large"], "n_heavy": st["n_heavy"],
              "heavy_tuples": st["heavy_tuples_r"] + st["heavy_tuples_s"], "skew_pairs": st["skew_pairs"]}
        pt.update(pass_fractions(ph, st, 2 * n))
        if not inp:
            pt["count"] = r.count
            pt["input_tuples_per_s"] = 2 * n / (ph["ms_total"] / 1e3)
            pt["output_tuples_per_s"] = r.count / (ph["ms_total"] / 1e3)
        # the same point with CSH's hybrid partition (NEXT-1): sampled keys skip pass 2, detect, split
        rh, phh = timed(rk, rp, sk, sp, gsh.make_config(timing=True, input_side_only=inp, hybrid=True), ws)
        assert inp or (rh.count, rh.checksum) == (r.count, r.checksum), "hybrid result differs"
        pt["hybrid"] = {"phases_ms": phh, "n_hybrid": rh.stats["n_hybrid"], "n_heavy": rh.stats["n_heavy"],
                        "n_large": rh.stats["n_large"], "large_tuples": rh.stats["large_tuples"]}
        out["points"].append(pt)
        del rk, rp, sk, sp, ws
    for theta, n in DENSE:
        rk, rp, sk, sp = datagen.make_workload("zipf", n, theta, seed=seed, device=dev)
        cfg = gsh.make_config(timing=True)
        r = gsh.join(rk, rp, sk, sp, config=cfg)
        st = r.stats
        out["dense"].append({"theta": theta, "n_per_side": n, "count": r.count, "ms_total": st["ms_total"],
                             "ms_skewjoin": st["ms_skewjoin"], "skew_pairs": st["skew_pairs"],
                             "skew_pairs_per_s": st["skew_pairs"] / (st["ms_skewjoin"] / 1e3),
                             "output_tuples_per_s": r.count / (st["ms_total"] / 1e3)})
        del rk, rp, sk, sp
    torch.cuda.empty_cache()
    return out


GBASE_THETAS = [0.0, 0.25, 0.5, 0.6, 0.7, 0.8, 0.9, 1.0]


def gbase_sweep(gsh, dev, seed, n=1 << 25, budget_s=8.0):
    """PAPER.md Table I (L157-L160) re-measured on this GPU: |R| = |S| = 2^25 (the paper's 32M) Zipf
    tuples, both sides, COUNT.  GSH (and its hybrid variant) vs the Gbase-style comparison join
    (gsh_join_gbase) per theta: partition ms and join ms as the paper splits them, the same count /
    checksum required of both.  Gbase is skipped at a theta once its previous point exceeded
    budget_s (its join time grows ~10x per 0.1 of theta, L158)."""
    import datagen
    out = []
    gb_last = 0.0
    cfg = gsh.make_config(timing=True)
    cfgh = gsh.make_config(timing=True, hybrid=True)
    ws = torch.empty(max(gsh.workspace_bytes(n, n, cfgh), gsh.gbase_workspace_bytes(n, n, cfg)), dtype=torch.uint8,
                     device=dev)

    def run(impl, c, reps):
        r = gsh.join(rk, rp, sk, sp, config=c, workspace=ws, impl=impl)
        ph = {}
        for _ in range(reps):
            r = gsh.join(rk, rp, sk, sp, config=c, workspace=ws, impl=impl)
            for k, v in r.stats.items():
                if k.startswith("ms_"):
                    ph[k] = ph.get(k, 0.0) + v / reps
        return r, ph

    for theta in GBASE_THETAS:
        rk, rp, sk, sp = datagen.make_workload("zipf", n, theta, seed=seed, device=dev)
        r, ph = run("gsh", cfg, 3 if theta < 0.9 else 1)
        part = ph["ms_hist"] + ph["ms_pass1"] + ph["ms_pass2"]
        pt = {"theta": theta, "n_per_side": n, "count": r.count,
              "gsh": {"partition_ms": part, "all_other_ms": ph["ms_total"] - part, "total_ms": ph["ms_total"],
                      "n_heavy": r.stats["n_heavy"]}}
        rh, phh = run("gsh", cfgh, 3 if theta < 0.9 else 1)
        assert (rh.count, rh.checksum) == (r.count, r.checksum), "hybrid result differs"
        pt["gsh_hybrid"] = {"total_ms": phh["ms_total"], "n_hybrid": rh.stats["n_hybrid"]}
        if gb_last <= budget_s:
            g, pg = run("gbase", cfg, 1 if theta >= 0.6 else 3)
            assert (g.count, g.checksum) == (r.count, r.checksum), "Gbase result differs"
            gpart = pg["ms_pass1"] + pg["ms_pass2"]
            pt["gbase"] = {"partition_ms": gpart, "join_ms": pg["ms_nmjoin"], "total_ms": pg["ms_total"]}
            pt["speedup_gsh_over_gbase"] = pg["ms_total"] / ph["ms_total"]
            gb_last = pg["ms_total"] / 1e3
        else:
            pt["gbase"] = None
        out.append(pt)
        print(json.dumps(pt), file=sys.stderr, flush=True)
        del rk, rp, sk, sp
    return out


def flatten(r, world):
    """(phases_ms, launches, join stats) of one step's result: the single-GPU gsh_join stats, or for
    the sharded step its protocol phases plus the routed normal shard's per-kernel phases."""
    st = r.stats
    if world == 1 and "join_normal" not in st:
        return {k: v for k, v in st.items() if k.startswith("ms_")}, st.get("launches", 0), st
    jn = st.get("join_normal") or st.get("normal") or {}   # python driver / native driver
    jh = st.get("join_heavy") or st.get("heavy") or {}
    ph = {k: v for k, v in st.items() if k.startswith("ms_")}
    for k, v in jn.items():
        if k.startswith("ms_") and k != "ms_total":
            ph[k] = v
    for k, v in jh.items():
        if k.startswith("ms_") and k != "ms_total":
            ph["heavy_" + k] = v
    return ph, st.get("launches", 0), dict(jn, n_local=st.get("normal_r", 0) + st.get("normal_s", 0))


def roofline_of(phases, st, n_tot, clocks, workload):
    """Roofline of the dominant kernel (the phase with the largest share of the step)."""
    peak, peak_src = hbm_peak()
    heavy_t = st.get("heavy_tuples_r", 0) + st.get("heavy_tuples_s", 0)
    # algorithmic bytes per launch: hist 4 B, each pass 16 B, NM 8 B per normal tuple
    # (+ the pre-partition pass beyond 2^28 per side: 4 B count + 16 B split per tuple; with it the
    # phase figures below are summed over the 2^prepass_bits sub-joins)
    algo = {"ms_hist": 4 * n_tot, "ms_pass1": 16 * n_tot, "ms_pass2": 16 * n_tot, "ms_nmjoin": 8 * (n_tot - heavy_t),
            "ms_prepass": 20 * n_tot}
    kernels = {"ms_prepass": "k_split_count + k_split_scatter", "ms_pass1": "k_scatter (pass 1)",
               "ms_pass2": "k_scatter (pass 2)", "ms_nmjoin": "k_nmjoin_ring", "ms_hist": "k_hist2d",
               "ms_skewjoin": "k_skewjoin"}
    dom = max(list(algo) + ["ms_skewjoin"], key=lambda k: phases.get(k, 0.0))
    traffic = None
    try:
        traffic = json.load(open(PROFILE_SUMMARY)).get(workload, {}).get(dom)
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
        return {"bound": "alu", "kernel": kernels[dom], "achieved": achieved, "peak": alu_peak,
                "peak_source": "derived: 64 ALU lanes/clk/SM / 7.0 ALU ops per pair x 148 SMs x max SM clock",
                "unit": "Gpairs/s", "frac": (achieved / alu_peak) if achieved else None, "traffic": traffic,
                "algorithmic_pairs_per_launch": st.get("skew_pairs", 0)}
    achieved = algo[dom] / (phases[dom] / 1e3) / 1e9 if phases.get(dom) else None
    return {"bound": "hbm", "kernel": kernels[dom], "achieved": achieved, "peak": peak, "peak_source": peak_src,
            "unit": "GB/s", "frac": (achieved / peak) if achieved else None, "traffic": traffic,
            "algorithmic_bytes_per_launch": algo[dom]}


def sharded_summary(phases, st, world, one_gpu=False):
    """Multi-GPU step: protocol phase times and the exchange's bytes against NVLink 5
    (900 GB/s per direction per GPU).  one_gpu (--fake-ranks): the "exchange" is device copies inside
    one GPU's HBM, so no NVLink fraction is reported."""
    keys = ("ms_agree", "ms_route", "ms_exchange", "ms_broadcast", "ms_join_normal", "ms_join_heavy", "ms_reduce")
    out = {k: phases.get(k) for k in keys}
    xb = st.get("exchange_send_bytes", st.get("exchange_bytes", 0))
    bb = st.get("broadcast_recv_bytes", st.get("broadcast_bytes", 0))
    for name, nb in (("exchange", xb), ("broadcast", bb)):
        ms = phases.get(f"ms_{name}") or 0.0
        gbs = nb / (ms * 1e6) if ms > 0 else None
        out[f"{name}_bytes_per_rank"] = nb
        out[f"{name}_GBps"] = gbs
        out[f"{name}_nvlink_frac"] = gbs / 900.0 if gbs and not one_gpu else None
    out["nvlink_peak_GBps"] = None if one_gpu else 900.0
    if one_gpu:
        out["note"] = "logical ranks on one GPU: exchanges are local HBM copies (code-path timing, not NVLink)"
    out["world"] = world
    return out


def main():
    args = parse()
    maybe_relaunch(args)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    import paper_conf_icde_caic24_b200 as gsh
    from paper_conf_icde_caic24_b200 import sharded

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if args.gbase_sweep:
        pts = gbase_sweep(gsh, dev, args.seed)
        print(json.dumps({"metric": "GSH vs Gbase-style join, PAPER.md Table I shape (ms per join)",
                          "config": {"workload": "|R|=|S|=2^25 Zipf both sides, COUNT, 1 B200"},
                          "impl": "gsh+gbase", "points": pts}))
        return
    kind, n, theta, desc = WORKLOADS[args.workload]
    if args.mode == "materialize":
        desc = desc.replace("COUNT", "MATERIALIZE")
    dist = None
    nccl_world = world > 1 or args.sharded
    if nccl_world:
        import torch.distributed as dist
        for k, v in (("MASTER_ADDR", "127.0.0.1"), ("MASTER_PORT", "29541"), ("RANK", "0"), ("WORLD_SIZE", "1")):
            os.environ.setdefault(k, v)
        dist.init_process_group("nccl", device_id=dev)
    extra = json.loads(os.environ.get("GSH_BENCH_CFG", "{}"))  # experiments only
    if args.detect == "sampled":
        extra["detect_mode"] = 1
    if args.hybrid:
        extra["hybrid"] = True
    # per-phase CUDA events stay on inside the timed region (the roofline's kernel time is
    # measured live there); they cost ~30 us of host time per call, included in the step time
    if args.input_side:
        extra["input_side_only"] = True
    cfg = gsh.make_config(timing=True, **extra)
    fake = args.fake_ranks if world == 1 else 0   # 1 = the sharded protocol with one rank
    native = args.driver == "native"
    if fake >= 1:
        # G logical ranks on this one GPU: each holds a 1/G positional shard of ONE workload
        full = make_data(kind, n, theta, args.seed, dev, 0)
        shards = [tuple(t[g * n // fake:(g + 1) * n // fake] for t in full) for g in range(fake)]
        rk, rp, sk, sp = full
        runner = sharded.LocalNativeRunner(fake, dev) if native else None

        def step():
            if native:
                t0 = time.perf_counter()
                rs = runner.run(shards, config=cfg, exchange=args.exchange)
                rs[0].stats["wall_s"] = time.perf_counter() - t0
            else:
                rs = sharded.run_local(fake, shards, config=cfg, exchange=args.exchange)
            rs[0].stats["launches"] = sum(x.stats.get("launches", 0) for x in rs)
            return rs[0]
    elif nccl_world:
        rk, rp, sk, sp = make_data(kind, n, theta, args.seed, dev, rank)
        drv = sharded.ShardedJoin(sharded.nccl_comm(device=dev), dev) if native else None

        def step():
            if native:
                return drv.join(rk, rp, sk, sp, config=cfg, exchange=args.exchange)
            return sharded.join_sharded(rk, rp, sk, sp, config=cfg, exchange=args.exchange)
    else:
        rk, rp, sk, sp = make_data(kind, n, theta, args.seed, dev, rank)
        ws = torch.empty(gsh.workspace_bytes(n, n, cfg), dtype=torch.uint8, device=dev)
        out = torch.empty((args.out_cap, 2), dtype=torch.int32, device=dev) if args.mode == "materialize" else None

        def step():
            return gsh.join(rk, rp, sk, sp, mode=args.mode, out=out, config=cfg, workspace=ws)
    torch.cuda.synchronize()
    multi = nccl_world or fake >= 1

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
            ph, nl, _ = flatten(r, 2 if multi else 1)
            for k, v in ph.items():
                phases[k] = phases.get(k, 0.0) + v
            launches += nl
        e1.record(stream)
        torch.cuda.synchronize()
    if dist:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    if fake >= 1:   # run_local synchronises every rank's stream; its wall clock bounds the step
        ms = max(ms, 1e3 * r.stats["wall_s"] * args.steps)
    if dist:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    total_in = 2 * n * (world if not fake else 1) * args.steps
    value = total_in / (ms / 1e3)
    out_per_s = r.count * args.steps / (ms / 1e3)
    phases = {k: v / args.steps for k, v in phases.items()}
    clocks = clk.summary()
    _, _, jst = flatten(r, 2 if multi else 1)
    n_tot = jst.get("n_local", 2 * n)
    roofline = roofline_of(phases, jst, n_tot, clocks, args.workload if not multi else None)

    # end-to-end through the public API with host buffers (H2D inside the timed region)
    e2e = None
    if not args.no_e2e and not fake:
        hk = [t.cpu().pin_memory() for t in (rk, rp, sk, sp)]
        ke = max(2, min(args.steps, 5))
        if not multi:
            ws_h = torch.empty(gsh._lib.load().gsh_host_workspace_bytes(n, n, 0, 0, None), dtype=torch.uint8,
                               device=dev)

            def estep():
                return gsh.join_host(*hk, workspace=ws_h)
            api, d2h = "gsh_join_host (pinned host buffers)", 2 * DEVSTATE_BYTES
        else:
            def estep():
                d = [h.to(dev, non_blocking=True) for h in hk]
                if native:
                    return drv.join(*d, config=cfg, exchange=args.exchange)
                return sharded.join_sharded(*d, config=cfg, exchange=args.exchange)
            api, d2h = ("H2D of the rank's pinned shard + " +
                        ("gsh_join_sharded" if native else "sharded.join_sharded")), 16
        for _ in range(2):
            estep()
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        h0 = torch.cuda.Event(enable_timing=True)
        h1 = torch.cuda.Event(enable_timing=True)
        h0.record(stream)
        for _ in range(ke):
            rr = estep()
        h1.record(stream)
        torch.cuda.synchronize()
        ems = h0.elapsed_time(h1)
        if dist:
            t = torch.tensor([ems], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        assert rr.count == r.count and rr.checksum == r.checksum
        e2e = {"value": 2 * n * world * ke / (ems / 1e3), "unit": "input tuples/s", "h2d_bytes_per_step": 16 * n,
               "d2h_bytes_per_step": d2h, "steps": ke, "ms_per_step": ems / ke, "api": api}
        # the bound of this number: the same bytes as plain pinned-memory H2D copies (PCIe), timed alike
        dst = [torch.empty_like(h, device=dev) for h in hk]
        for _ in range(2):
            for dd, hh in zip(dst, hk):
                dd.copy_(hh, non_blocking=True)
        torch.cuda.synchronize()
        h0.record(stream)
        for _ in range(ke):
            for dd, hh in zip(dst, hk):
                dd.copy_(hh, non_blocking=True)
        h1.record(stream)
        torch.cuda.synchronize()
        cms = h0.elapsed_time(h1) / ke
        e2e["h2d_copy"] = {"ms_per_step": cms, "gbs": 16 * n / (cms * 1e6),
                           "e2e_frac": cms / (ems / ke)}   # share of the e2e step that is the bare copy
        del hk, dst

    sweep = None
    if not multi and not args.no_sweep and args.workload == "cfg2" and args.mode == "count":
        del rk, rp, sk, sp, ws
        torch.cuda.empty_cache()
        sweep = theta_sweep(gsh, dev, args.seed)
        rk, rp, sk, sp = make_data(kind, n, theta, args.seed, dev, rank)

    base = None
    if rank == 0 and not multi and not args.no_cpu_baseline:
        base = cpu_baseline(kind, n, theta, args.seed, rk, rp, sk, sp, r)

    if rank == 0:
        line = {
            "metric": "join input tuples/s", "value": value, "unit": "input tuples/s", "n_gpus": world,
            "steps": args.steps, "warmup": max(3, args.warmup), "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (datagen, seeded)",
            "config": {"workload": desc, "n_r": n * world, "n_s": n * world, "mode": args.mode, "detect": args.detect,
                       "exchange": args.exchange if multi else None,
                       "driver": (("gsh_join_sharded" if native else "sharded.join_sharded") if multi else None),
                       "parallelism": (f"hash-sharded x{world} (NCCL)" if nccl_world else
                                       f"{fake} logical ranks on one GPU (code-path check)" if fake >= 1 else
                                       "single GPU"),
                       "l2": "inputs 2 GiB per GPU > 126 MB L2: no flush needed" if n >= (1 << 24) else
                             "inputs smaller than L2 (launch-bound workload)", "seed": args.seed},
            "output_tuples_per_s": out_per_s, "count": r.count, "checksum": f"{r.checksum:#018x}",
            "phases_ms": phases, "roofline": roofline, "clocks": clocks, "e2e": e2e,
            "gpu_launches": launches, "cpu_baseline": base,
            "stats": {k: v for k, v in r.stats.items() if not k.startswith("ms_") and not isinstance(v, dict)},
        }
        if multi:
            line["sharded"] = sharded_summary(phases, r.stats, fake or world, one_gpu=fake >= 1)
        if sweep is not None:
            line["theta_sweep"] = sweep
        line["pass_fractions"] = pass_fractions(phases, jst, n_tot)
        print(json.dumps(line))
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
