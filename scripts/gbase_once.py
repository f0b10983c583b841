#!/usr/bin/env python
"""One Gbase-style join (gsh_join_gbase) at PAPER.md Table I's shape for an ncu capture:
|R| = |S| = 2^25 Zipf(theta) both sides, COUNT.  Usage: gbase_once.py [theta]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icde_caic24_b200 as gsh  # noqa: E402

theta = float(sys.argv[1]) if len(sys.argv) > 1 else 0.5
d = datagen.make_workload("zipf", 1 << 25, theta, seed=0x6A5, device="cuda")
r = gsh.join(*d, impl="gbase", config=gsh.make_config(timing=True))
torch.cuda.synchronize()
print(f"gbase theta={theta} count={r.count} ms_total={r.stats['ms_total']:.3f} join={r.stats['ms_nmjoin']:.3f}")
