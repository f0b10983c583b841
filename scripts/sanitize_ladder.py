#!/usr/bin/env python
"""Workload ladder for compute-sanitizer (memcheck / racecheck / synccheck): every GSH phase and
both NM tables, COUNT and MATERIALIZE, the pre-partition pass, and the sharded path at G = 2 on
one GPU, at n <= 2^18 per side -- each result checked against the oracle.

  compute-sanitizer --tool racecheck python scripts/sanitize_ladder.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icde_caic24_b200 as gsh  # noqa: E402
from paper_conf_icde_caic24_b200 import sharded  # noqa: E402

CASES = [  # kind, n, theta, config
    ("pkfk", 1 << 16, 0.0, {}),
    ("pkfk", (1 << 16) + 77, 0.0, {"nm_table": 1}),
    ("uniform", 5000, 0.0, {}),
    ("zipf", 1 << 16, 0.5, {}),
    ("zipf", 1 << 17, 1.0, {}),
    ("zipf", 1 << 15, 1.5, {}),
    ("zipf", 1 << 16, 1.0, {"detect_mode": 1}),
    ("zipf", 1 << 15, 1.0, {"force_all_heavy": True}),
    ("graph", 1 << 16, 0.909, {}),
    ("zipf", 1 << 16, 1.0, {"prepass_bits": 2}),
    ("pkfk_zipf", 1 << 16, 1.0, {"heavy_detail": True}),
    ("zipf", 1 << 17, 1.0, {"hybrid": True, "hybrid_share": 1}),
    ("zipf", 1 << 15, 1.5, {"hybrid": True, "hybrid_stride": 1, "hybrid_share": 1}),
    ("pkfk_zipf", 1 << 16, 1.0, {"hybrid": True, "hybrid_share": 1}),
    ("zipf", (1 << 15) + 3, 1.0, {"impl": "gbase"}),
    ("graph", 1 << 15, 0.909, {"impl": "gbase"}),
]


def u(t):
    return t.cpu().numpy().view(np.uint32)


def main():
    dev = torch.device("cuda", 0)
    tool = os.environ.get("SAN_TOOL", "?")
    for kind, n, theta, kw in CASES:
        kw = dict(kw)
        impl = kw.pop("impl", "gsh")
        rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=3)
        on, oc, _ = oracle.join(u(rk), u(rp), u(sk), u(sp))
        d = [t.to(dev) for t in (rk, rp, sk, sp)]
        cfg = gsh.make_config(**kw)
        r = gsh.join(*d, config=cfg, impl=impl)
        assert (r.count, r.checksum) == (on, oc), (kind, n, theta, kw)
        if on <= (1 << 22) and not kw.get("heavy_detail"):
            m = gsh.join(*d, mode="materialize", out_capacity=on, config=gsh.make_config(**kw), impl=impl)
            assert (m.count, m.checksum, m.written) == (on, oc, on)
        print(f"[{tool}] ok {impl} {kind} n={n} theta={theta} {kw} count={on}", flush=True)
    full = [t.to(dev) for t in datagen.make_workload("zipf", 1 << 15, 1.0, seed=5)]
    on, oc, _ = oracle.join(*(u(t) for t in full))
    shards = [tuple(t[g * (1 << 14):(g + 1) * (1 << 14)] for t in full) for g in range(2)]
    res = sharded.run_local(2, shards)
    assert all((x.count, x.checksum) == (on, oc) for x in res)
    print(f"[{tool}] ok sharded G=2 count={on}", flush=True)
    torch.cuda.synchronize()
    print(f"[{tool}] ladder done", flush=True)


if __name__ == "__main__":
    main()
