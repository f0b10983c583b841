"""Multi-GPU protocol (paper_conf_icde_caic24_b200.sharded) exercised on CPU:
torch.distributed gloo at world_size 2 and 4 (one process per rank), and the in-process
LocalWorld communicator (threads) at world 2, 4 and 8.  The per-rank libgsh kernels are replaced by
a test double built on the oracle (tests only); the collectives, skew agreement, routing
bookkeeping (buffer layout, own-segment placement, split sizes) and the final reduction are the
production host code.  The global result must equal the single-process oracle bit-exactly and the
agreed skewed set must equal oracle.heavy_rule on the whole input."""
import os
import socket
import time

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import datagen
import oracle


def _u32(t):
    return t.numpy().view(np.uint32)


def _i32(a):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(a, dtype=np.uint32)).view(np.int32))


class OracleOps:
    """CPU test double of sharded.CudaOps (same contract, oracle arithmetic)."""

    def __init__(self):
        self.t = []

    def tensor(self, vals, dtype=torch.int64):
        return torch.tensor(vals, dtype=dtype)

    def empty(self, n):
        return torch.zeros(int(n), dtype=torch.int32)

    def mark(self, name):
        self.t.append((name, time.perf_counter()))

    def phase_ms(self):
        return {f"ms_{n}": 1e3 * (b - a) for (_, a), (n, b) in zip(self.t, self.t[1:])}

    def histogram(self, rk, sk, P):
        B = int(P.part_bits)
        return torch.from_numpy(np.concatenate([oracle.radix_histogram(_u32(rk), 0, B),
                                                oracle.radix_histogram(_u32(sk), 0, B)]))

    def candidates(self, state, rk, rp, sk, sp, P, hist):
        B, L = int(P.part_bits), int(P.large_threshold)
        h = hist.numpy().reshape(2, -1)
        large = (h[0] > 0) & (h[1] > 0) & ((h[0] > L) | (h[1] > L)) & (not P.force_all_normal)
        counts = []
        for k in (rk, sk):
            hk = oracle.fmix32(_u32(k))
            d = oracle.radix_digits(_u32(k), 0, B)
            u, c = np.unique(hk[large[d]], return_counts=True)
            counts.append(dict(zip(u.tolist(), c.tolist())))
        state["local"] = counts
        keys = sorted(set(counts[0]) | set(counts[1]))
        tau = int(P.cand_threshold)
        out = [x for x in keys if max(counts[0].get(x, 0), counts[1].get(x, 0)) >= tau]
        return _i32(out), False

    def agree(self, state, gathered, sizes, stride):
        g = gathered.numpy().view(np.uint32)
        seen, uni = set(), []
        for r, n in enumerate(sizes):
            for x in g[r * stride: r * stride + n].tolist():
                if x not in seen:
                    seen.add(x)
                    uni.append(x)
        c = state["local"]
        cnt = [v for x in uni for v in (c[0].get(x, 0), c[1].get(x, 0))]
        return _i32(uni), torch.tensor(cnt, dtype=torch.int64)

    def select(self, state, uni, cnt, P):
        c = cnt.numpy().reshape(-1, 2)
        u = uni.numpy().view(np.uint32)
        heavy = [int(x) for x, (a, b) in zip(u.tolist(), c.tolist()) if max(a, b) >= int(P.heavy_threshold)]
        state["set"] = set(heavy)
        return _i32(heavy)

    def _dest(self, state, keys, rb):
        G = 1 << rb
        h = oracle.fmix32(_u32(keys)).astype(np.int64)
        dest = (h >> (32 - rb)) if rb else np.zeros_like(h)
        hv = state["set"]
        if hv:
            dest = np.where(np.isin(h, np.array(sorted(hv), dtype=np.int64)), G, dest)
        return dest

    def route_count(self, state, keys, rb):
        return np.bincount(self._dest(state, keys, rb), minlength=(1 << rb) + 1).tolist()

    def route_scatter(self, state, keys, pays, rb, dst, heavy_copies=1):
        dest = self._dest(state, keys, rb)
        G = 1 << rb
        for d, (kb, pb, off) in enumerate(dst):
            sel = torch.from_numpy(np.nonzero(dest == min(d, G))[0])   # d >= G: copies of the skewed tuples
            n = sel.numel()
            if n:
                kb[off: off + n] = keys[sel]
                pb[off: off + n] = pays[sel]

    def join(self, rk, rp, sk, sp, config, out=None):
        n, c, pairs = oracle.join(_u32(rk), _u32(rp), _u32(sk), _u32(sp), nthreads=1,
                                  materialize=out is not None)
        w = 0
        if out is not None:
            w = min(n, out.shape[0])
            out[:w] = torch.from_numpy(pairs[:w].view(np.int32))
        return n, c, w, {}


def _shard(t, rank, world):
    lo, hi = rank * t.numel() // world, (rank + 1) * t.numel() // world
    return t[lo:hi]


def _expect(kind, n, theta, seed, cfg_kw):
    from paper_conf_icde_caic24_b200 import make_config, sharded
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=seed)
    on, oc, _ = oracle.join(_u32(rk), _u32(rp), _u32(sk), _u32(sp))
    P = sharded.shard_plan(rk.numel(), sk.numel(), 1, make_config(**cfg_kw))
    oh, _, _ = oracle.heavy_rule(_u32(rk), _u32(sk), int(P.part_bits), int(P.large_threshold),
                                 int(P.heavy_threshold))
    return (rk, rp, sk, sp), on, oc, oh


def _worker(rank, world, port, kind, n, theta, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icde_caic24_b200 import make_config, sharded
        cfg = make_config(large_threshold=512, heavy_threshold=64)
        full = datagen.make_workload(kind, n, theta, seed=17)
        rk, rp, sk, sp = (_shard(t, rank, world) for t in full)
        res = sharded.join_sharded(rk, rp, sk, sp, config=cfg, ops=OracleOps())
        q.put((rank, res.count, res.checksum, res.stats["n_heavy_global"], res.stats["heavy_r"],
               res.stats["normal_r"], res.stats["normal_s"], res.stats["heavy_s"]))
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
def test_sharded_gloo_matches_oracle(world, kind, n, theta):
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
    (rk, _, sk, _), on, oc, oh = _expect(kind, n, theta, 17, dict(large_threshold=512, heavy_threshold=64))
    for o in out:
        assert (o[1], o[2]) == (on, oc)
        assert o[3] == len(oh)
    # every tuple lands exactly once: normal tuples routed, skewed S local, skewed R everywhere
    assert sum(o[6] for o in out) + sum(o[7] for o in out) == sk.numel()
    heavy_r = {o[4] for o in out}
    assert len(heavy_r) == 1   # all-gathered: the same skewed R on every rank
    assert sum(o[5] for o in out) + heavy_r.pop() == rk.numel()
    if theta >= 1.0:
        assert len(oh) > 0 and out[0][4] > 0


@pytest.mark.parametrize("exchange", ["a2a", "p2p"])
@pytest.mark.parametrize("world,kind,n,theta,mode", [(2, "zipf", 1 << 13, 1.0, "count"),
                                                     (4, "zipf", 1 << 13, 1.5, "count"),
                                                     (8, "graph", 1 << 13, 0.909, "count"),
                                                     (4, "zipf", 1 << 12, 0.75, "materialize"),
                                                     (8, "uniform", 1 << 12, 0.0, "count")])
def test_sharded_localworld_cpu(world, kind, n, theta, mode, exchange):
    """The LocalWorld communicator (threads, the one-GPU harness's exchange) on CPU tensors."""
    import threading

    from paper_conf_icde_caic24_b200 import make_config, sharded
    kw = dict(large_threshold=256, heavy_threshold=32)
    (rk, rp, sk, sp), on, oc, oh = _expect(kind, n, theta, 5, kw)
    cfg = make_config(**kw)
    lw = sharded.LocalWorld(world)
    res = [None] * world
    cap = on + 16

    def worker(g):
        out = torch.zeros((cap, 2), dtype=torch.int32) if mode == "materialize" else None
        res[g] = sharded.join_sharded(*(_shard(t, g, world) for t in (rk, rp, sk, sp)), config=cfg, ops=OracleOps(),
                                      comm=lw.comm(g), mode=mode, out=out, exchange=exchange)

    th = [threading.Thread(target=worker, args=(g,)) for g in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    for r in res:
        assert (r.count, r.checksum) == (on, oc)
        assert r.stats["n_heavy_global"] == len(oh)
    if mode == "materialize":
        got = np.concatenate([r.pairs.numpy().view(np.uint32) for r in res])
        _, _, want = oracle.join_sorted_pairs(_u32(rk), _u32(rp), _u32(sk), _u32(sp))
        got = got[np.lexsort((got[:, 1], got[:, 0]))]
        assert np.array_equal(got, want)


def test_shard_plan_matches_single_gpu_rule():
    """gsh_shard_plan (host-only) gives the single-GPU (B, L, T_h) of the global sizes."""
    from paper_conf_icde_caic24_b200 import make_config, sharded, workspace_bytes  # noqa: F401
    for n in (1 << 10, 1 << 20, 1 << 27, 1 << 31):
        P = sharded.shard_plan(n, n // 2, 8)
        B = 0
        while B < 16 and (n >> B) > 2048:
            B += 1
        assert P.part_bits == B and P.route_bits == 3 and P.world == 8
        mean = n / (1 << B)
        assert P.large_threshold == max(64, int(mean + 8 * max(mean, 1.0) ** 0.5) + 1)
        assert P.heavy_threshold == 64 and P.cand_threshold == 8
    P = sharded.shard_plan(1000, 1000, 4, make_config(heavy_threshold=10, large_threshold=77, pass_bits=(3, 2)))
    assert (P.part_bits, P.large_threshold, P.heavy_threshold, P.cand_threshold) == (5, 77, 10, 3)
    with pytest.raises(Exception):
        sharded.shard_plan(10, 10, 3)
