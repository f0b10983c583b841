"""Multi-GPU protocol (paper_conf_icde_caic24_b200.sharded) exercised on CPU with
torch.distributed gloo, world_size 2 and 4.  The per-rank kernels are replaced by a test double
built on the oracle (tests only); the collectives, skew agreement, routing bookkeeping and the
final reduction are the production host code.  The global result must equal the single-process
oracle bit-exactly and the agreed skewed set must equal oracle.heavy_rule on the whole input."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import datagen
import oracle


def _u32(t):
    return t.numpy().view(np.uint32)


class OracleOps:
    """CPU test double of sharded.CudaOps (same contract, oracle arithmetic)."""

    def radix_histogram(self, keys, hi, nbits):
        return torch.from_numpy(oracle.radix_histogram(_u32(keys), hi, nbits))

    def local_candidates(self, rk, rp, sk, sp, B, large_u8, tau):
        large = large_u8.numpy().astype(bool)
        out = []
        counts = []
        for k in (rk, sk):
            h = oracle.fmix32(_u32(k))
            d = oracle.radix_digits(_u32(k), 0, B)
            u, c = np.unique(h[large[d]], return_counts=True)
            counts.append(dict(zip(u.tolist(), c.tolist())))
        keys = set(counts[0]) | set(counts[1])
        for x in keys:
            if max(counts[0].get(x, 0), counts[1].get(x, 0)) >= tau:
                out.append(x)
        return torch.tensor(sorted(out), dtype=torch.int64)

    def count_keys(self, keys, q32):
        h = oracle.fmix32(_u32(keys))
        q = q32.numpy().view(np.uint32)
        u, c = np.unique(h, return_counts=True)
        m = dict(zip(u.tolist(), c.tolist()))
        return torch.tensor([m.get(int(x), 0) for x in q], dtype=torch.int64)

    def route(self, keys, pays, rb, heavy32):
        G = 1 << rb
        h = oracle.fmix32(_u32(keys)).astype(np.int64)
        hv = set(heavy32.numpy().view(np.uint32).tolist())
        dest = (h >> (32 - rb)) if rb else np.zeros_like(h)
        isheavy = np.array([int(x) in hv for x in h.tolist()], dtype=bool) if hv else np.zeros(h.shape, bool)
        dest = np.where(isheavy, G, dest)
        order = np.argsort(dest, kind="stable")
        counts = np.bincount(dest, minlength=G + 1).tolist()
        return keys[torch.from_numpy(order)], pays[torch.from_numpy(order)], counts

    def join(self, rk, rp, sk, sp, config):
        n, c, _ = oracle.join(_u32(rk), _u32(rp), _u32(sk), _u32(sp), nthreads=1)
        return n, c, {}


def _worker(rank, world, port, kind, n, theta, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icde_caic24_b200 import make_config, sharded
        cfg = make_config(large_threshold=512, heavy_threshold=64)
        rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=17)
        lo_r, hi_r = rank * rk.numel() // world, (rank + 1) * rk.numel() // world
        lo_s, hi_s = rank * sk.numel() // world, (rank + 1) * sk.numel() // world
        heavy, params = sharded.agree_heavy(rk[lo_r:hi_r], rp[lo_r:hi_r], sk[lo_s:hi_s], sp[lo_s:hi_s],
                                            config=cfg, ops=OracleOps())
        res = sharded.join_sharded(rk[lo_r:hi_r], rp[lo_r:hi_r], sk[lo_s:hi_s], sp[lo_s:hi_s], config=cfg,
                                   ops=OracleOps())
        q.put((rank, res.count, res.checksum, sorted(heavy.numpy().view(np.uint32).tolist()), params,
               res.stats["heavy_r_recv"]))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world,kind,n,theta", [(2, "zipf", 1 << 14, 1.0), (2, "pkfk", 1 << 13, 0.0),
                                                (4, "zipf", 1 << 14, 1.25), (2, "graph", 1 << 14, 0.909)])
def test_sharded_matches_oracle(world, kind, n, theta):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, n, theta, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=17)
    on, oc, _ = oracle.join(_u32(rk), _u32(rp), _u32(sk), _u32(sp))
    heavy_sets = {tuple(o[3]) for o in out}
    assert len(heavy_sets) == 1  # all ranks agree
    B, L, Th, _, _ = out[0][4]
    oh, _, _ = oracle.heavy_rule(_u32(rk), _u32(sk), B, L, Th)
    assert list(heavy_sets.pop()) == oh.tolist()
    for o in out:
        assert (o[1], o[2]) == (on, oc)
    if theta >= 1.0:
        assert len(oh) > 0 and out[0][5] > 0  # skewed R really broadcast
