"""GPU check of the multi-GPU driver's production data path (sharded.CudaOps: libgsh.so route /
count / candidate kernels + gsh_join) under torch.distributed NCCL.  This run has one GPU, so the
world is a single rank (route bits 0): every kernel and collective call of join_sharded runs for
real on the device; the multi-rank exchange itself is covered by tests/test_sharded_cpu.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import datagen
import oracle

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(port, kind, n, theta, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        from paper_conf_icde_caic24_b200 import make_config, sharded
        cfg = make_config(large_threshold=512, heavy_threshold=64)
        rk, rp, sk, sp = (t.cuda() for t in datagen.make_workload(kind, n, theta, seed=23))
        heavy, params = sharded.agree_heavy(rk, rp, sk, sp, config=cfg)
        res = sharded.join_sharded(rk, rp, sk, sp, config=cfg)
        q.put((res.count, res.checksum, sorted(heavy.cpu().numpy().view(np.uint32).tolist()), params))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("kind,n,theta", [("zipf", 1 << 16, 1.0), ("pkfk", 1 << 15, 0.0), ("graph", 1 << 16, 0.909)])
def test_sharded_single_rank_nccl(kind, n, theta):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_worker, args=(_free_port(), kind, n, theta, q))
    p.start()
    cnt, chk, heavy, params = q.get(timeout=300)
    p.join(timeout=60)
    assert p.exitcode == 0
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=23)
    u = lambda t: t.numpy().view(np.uint32)  # noqa: E731
    on, oc, _ = oracle.join(u(rk), u(rp), u(sk), u(sp))
    assert (cnt, chk) == (on, oc)
    B, L, Th, _, _ = params
    oh, _, _ = oracle.heavy_rule(u(rk), u(sk), B, L, Th)
    assert heavy == oh.tolist()
    if theta >= 1.0:
        assert len(heavy) > 0
