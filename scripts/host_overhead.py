"""Experiments only: where the per-call gap between ms_total (first to last kernel) and the
step time comes from.  Times N back-to-back calls through (a) gsh.join, (b) a pre-marshalled
ctypes call of gsh_join, with CUDA events around the loop and perf_counter per call."""
import ctypes
import sys
import time

import torch

sys.path.insert(0, ".")
import datagen  # noqa: E402
import paper_conf_icde_caic24_b200 as gsh  # noqa: E402
from paper_conf_icde_caic24_b200 import _lib  # noqa: E402

n = 1 << 27
dev = torch.device("cuda", 0)
rk, rp, sk, sp = datagen.make_workload("pkfk", n, 0.0, 0x6A5, dev)
for timing in (True, False):
    cfg = gsh.make_config(timing=timing)
    ws = torch.empty(gsh.workspace_bytes(n, n, cfg), dtype=torch.uint8, device=dev)
    for _ in range(3):
        r = gsh.join(rk, rp, sk, sp, config=cfg, workspace=ws)
    torch.cuda.synchronize()
    N = 20
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    t0 = time.perf_counter()
    for _ in range(N):
        r = gsh.join(rk, rp, sk, sp, config=cfg, workspace=ws)
    t1 = time.perf_counter()
    e1.record()
    torch.cuda.synchronize()
    print(f"timing={timing} gsh.join: events {e0.elapsed_time(e1) / N:.4f} ms/call, wall {(t1 - t0) / N * 1e3:.4f}",
          f"ms_total {r.stats.get('ms_total', 0):.4f}")
    lib = _lib.load()
    R = _lib.GshRelation(rk.data_ptr(), rp.data_ptr(), n)
    S = _lib.GshRelation(sk.data_ptr(), sp.data_ptr(), n)
    res = _lib.GshResult()
    stream = torch.cuda.current_stream().cuda_stream
    args = (ctypes.byref(R), ctypes.byref(S), _lib.GSH_OUT_COUNT, None, ws.data_ptr(), ws.numel(), ctypes.byref(cfg),
            stream, ctypes.byref(res))
    e0.record()
    t0 = time.perf_counter()
    for _ in range(N):
        lib.gsh_join(*args)
    t1 = time.perf_counter()
    e1.record()
    torch.cuda.synchronize()
    print(f"timing={timing} raw ctypes: events {e0.elapsed_time(e1) / N:.4f} ms/call, wall {(t1 - t0) / N * 1e3:.4f}",
          f"ms_total {res.ms_total:.4f}")
