"""GPU checks of the multi-GPU path through the C-ABI:

* the routing kernels (gsh_route_count / gsh_route_scatter) at route_bits 1, 2, 3 against the
  oracle's destinations and per-destination multisets;
* the skew-agreement kernels (gsh_shard_histogram / _candidates / _agree / _select /
  gsh_heavy_set_build) against the oracle's counts and rules;
* the whole sharded join with the real kernels for G = 2, 4 (and 8) logical ranks sharing the one
  GPU (sharded.run_local: threads + device-copy exchange), against the oracle on the
  whole input -- including a skewed-FK PK-FK join whose skewed keys are locally small (the
  round-1 defect: heavy tuples joined under the routed shard's route_bits);
* gsh_join's check of the route_bits assertion;
* a single-rank NCCL process group (the torch.distributed path with world size 1).
"""
import ctypes
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import datagen
import oracle

pytestmark = pytest.mark.gpu


def _u32(t):
    return t.cpu().numpy().view(np.uint32)


def _i32(a, dev):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(a, dtype=np.uint32)).view(np.int32)).to(dev)


def _shard(t, g, G):
    lo, hi = g * t.numel() // G, (g + 1) * t.numel() // G
    return t[lo:hi]


def _heavy_set(hk_u32, dev):
    from paper_conf_icde_caic24_b200 import load
    lib = load()
    hk = _i32(hk_u32, dev)
    nb = int(lib.gsh_heavy_set_bytes(len(hk_u32)))
    buf = torch.empty(max(nb, 256), dtype=torch.uint8, device=dev)
    st = lib.gsh_heavy_set_build(hk.data_ptr() if len(hk_u32) else None, len(hk_u32), buf.data_ptr(), nb,
                                 torch.cuda.current_stream().cuda_stream)
    assert st == 0
    return buf, nb


@pytest.mark.parametrize("rb", [0, 1, 2, 3])
@pytest.mark.parametrize("n_heavy", [0, 5, 3000])
def test_route_kernels_vs_oracle(rb, n_heavy):
    from paper_conf_icde_caic24_b200 import load
    lib = load()
    dev = torch.device("cuda", 0)
    rk, rp, _, _ = datagen.make_workload("zipf", 200_003, 0.9, seed=31)
    keys = _u32(rk)
    h = oracle.fmix32(keys)
    uniq = np.unique(h)
    heavy = uniq[np.random.default_rng(rb).permutation(uniq.size)[:n_heavy]]
    G = 1 << rb
    want = np.where(np.isin(h, heavy), G, (h.astype(np.int64) >> (32 - rb)) if rb else 0).astype(np.int64)
    setbuf, nb = _heavy_set(heavy, dev)
    dk, dp = rk.to(dev), rp.to(dev)
    cnt = torch.empty(G + 1, dtype=torch.int64, device=dev)
    s = torch.cuda.current_stream().cuda_stream
    assert lib.gsh_route_count(dk.data_ptr(), dk.numel(), rb, setbuf.data_ptr() if nb else None, nb,
                               cnt.data_ptr(), s) == 0
    counts = cnt.cpu().numpy()
    assert counts.tolist() == np.bincount(want, minlength=G + 1).tolist()
    # one output buffer per destination, padded so a write past a run would be caught
    outs = [(torch.full((int(c) + 64,), -7, dtype=torch.int32, device=dev),
             torch.full((int(c) + 64,), -7, dtype=torch.int32, device=dev)) for c in counts]
    ptrs = []
    for k, p in outs:
        ptrs += [k.data_ptr() + 4 * 32, p.data_ptr() + 4 * 32]
    d_dst = torch.tensor(ptrs, dtype=torch.int64, device=dev)
    cur = torch.empty(G + 1, dtype=torch.int64, device=dev)
    assert lib.gsh_route_scatter(dk.data_ptr(), dp.data_ptr(), dk.numel(), rb, setbuf.data_ptr() if nb else None,
                                 nb, d_dst.data_ptr(), 1, cur.data_ptr(), s) == 0
    torch.cuda.synchronize()
    pays = _u32(rp)
    for d, (k, p) in enumerate(outs):
        c = int(counts[d])
        kk, pp = _u32(k), _u32(p)
        assert (kk[:32] == np.uint32(0xFFFFFFF9)).all() and (kk[32 + c:] == np.uint32(0xFFFFFFF9)).all()
        got = np.stack([kk[32:32 + c], pp[32:32 + c]], 1)
        sel = want == d
        exp = np.stack([keys[sel], pays[sel]], 1)
        got = got[np.lexsort((got[:, 1], got[:, 0]))]
        exp = exp[np.lexsort((exp[:, 1], exp[:, 0]))]
        assert np.array_equal(got, exp), d


@pytest.mark.parametrize("kind,n,theta", [("zipf", 1 << 17, 1.0), ("graph", 1 << 17, 0.909),
                                          ("pkfk_zipf", 1 << 17, 1.1)])
def test_agreement_kernels_vs_oracle(kind, n, theta):
    """gsh_shard_* on one rank's data: histogram == bincount; candidates == keys of large
    partitions with local count >= tau; agree == first-occurrence union + exact counts; select ==
    stable compaction of max >= T_h."""
    from paper_conf_icde_caic24_b200 import make_config, sharded
    dev = torch.device("cuda", 0)
    rk, rp, sk, sp = (t.to(dev) for t in datagen.make_workload(kind, n, theta, seed=9))
    cfg = make_config(large_threshold=300, heavy_threshold=40)
    P = sharded.shard_plan(rk.numel(), sk.numel(), 4, cfg)
    ops = sharded.CudaOps(dev)
    B, L = int(P.part_bits), int(P.large_threshold)
    hist = ops.histogram(rk, sk, P)
    kr, ks = _u32(rk), _u32(sk)
    hr = oracle.radix_histogram(kr, 0, B)
    hs = oracle.radix_histogram(ks, 0, B)
    assert np.array_equal(hist.cpu().numpy(), np.concatenate([hr, hs]))
    state = {}
    cand, ovf = ops.candidates(state, rk, rp, sk, sp, P, hist)
    assert not ovf
    large = (hr > 0) & (hs > 0) & ((hr > L) | (hs > L))
    cnts = []
    for k in (kr, ks):
        hh = oracle.fmix32(k)
        u, c = np.unique(hh[large[oracle.radix_digits(k, 0, B)]], return_counts=True)
        cnts.append(dict(zip(u.tolist(), c.tolist())))
    tau = int(P.cand_threshold)
    exp = sorted(x for x in set(cnts[0]) | set(cnts[1]) if max(cnts[0].get(x, 0), cnts[1].get(x, 0)) >= tau)
    assert sorted(_u32(cand).tolist()) == exp and len(exp) > 0
    # a fake 3-rank gather: this rank's candidates, a shuffled copy with extra keys, an empty rank
    c = _u32(cand)
    extra = np.array([1, 2, 3, exp[0]], dtype=np.uint32)
    segs = [c, np.concatenate([extra, c[::-1]]), np.zeros(0, np.uint32)]
    stride = max(s.size for s in segs)
    buf = np.zeros(3 * stride, np.uint32)
    for g, sg in enumerate(segs):
        buf[g * stride: g * stride + sg.size] = sg
    uni, cnt = ops.agree(state, _i32(buf, dev), [s.size for s in segs], stride)
    first, seen = [], set()
    for g, sg in enumerate(segs):
        for x in sg.tolist():
            if x not in seen:
                seen.add(x)
                first.append(x)
    assert _u32(uni).tolist() == first
    cc = cnt.cpu().numpy().reshape(-1, 2)
    assert cc.tolist() == [[cnts[0].get(x, 0), cnts[1].get(x, 0)] for x in first]
    heavy = ops.select(state, uni, cnt, P)
    th = int(P.heavy_threshold)
    assert _u32(heavy).tolist() == [x for x, (a, b) in zip(first, cc.tolist()) if max(a, b) >= th]


_CASES = [
    # (world, kind, n, theta, config)
    (2, "zipf", 1 << 18, 1.0, {}),
    (4, "zipf", 1 << 18, 1.25, dict(large_threshold=512)),
    (4, "pkfk", 1 << 18, 0.0, {}),
    (2, "graph", 1 << 18, 0.909, {}),
    (4, "uniform", 1 << 18, 0.0, {}),
    (8, "zipf", 1 << 17, 0.75, {}),
    # skewed-FK PK-FK: R unique, S Zipf over R's rows -> skewed keys whose local counts are small
    # (the round-1 defect: they were joined under the normal shard's route_bits with the chained
    # NM table, which compares only h's low 16 bits)
    (4, "pkfk_zipf", 1 << 18, 1.0, dict(heavy_threshold=64)),
    (8, "pkfk_zipf", 1 << 18, 0.8, dict(heavy_threshold=16, large_threshold=64)),
]


@pytest.mark.parametrize("world,kind,n,theta,kw", _CASES)
def test_sharded_local_world_vs_oracle(world, kind, n, theta, kw):
    from paper_conf_icde_caic24_b200 import make_config, sharded
    dev = torch.device("cuda", 0)
    full = datagen.make_workload(kind, n, theta, seed=23)
    on, oc, _ = oracle.join(*(t.numpy().view(np.uint32) for t in full))
    cfg = make_config(**kw)
    shards = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
    res = sharded.run_local(world, shards, config=cfg)
    P = sharded.shard_plan(n, n, world, cfg)
    oh, _, _ = oracle.heavy_rule(full[0].numpy().view(np.uint32), full[2].numpy().view(np.uint32),
                                 int(P.part_bits), int(P.large_threshold), int(P.heavy_threshold))
    for r in res:
        assert (r.count, r.checksum) == (on, oc), (r.stats, on, oc)
        assert r.stats["n_heavy_global"] == len(oh)
        assert not r.stats["candidate_table_overflow"]
    # every S tuple on exactly one rank (normal routed + skewed local); skewed R on every rank
    assert sum(r.stats["normal_s"] + r.stats["heavy_s"] for r in res) == n
    assert len({r.stats["heavy_r"] for r in res}) == 1
    assert sum(r.stats["normal_r"] for r in res) + res[0].stats["heavy_r"] == n
    if kind in ("zipf", "pkfk_zipf") and theta >= 1.0:
        assert len(oh) > 0 and res[0].stats["heavy_r"] > 0
    if kind == "pkfk_zipf":
        assert on == n and sum(r.stats["count_heavy"] for r in res) > 0


def test_sharded_local_world_materialize():
    from paper_conf_icde_caic24_b200 import sharded
    dev = torch.device("cuda", 0)
    world, n = 4, 1 << 16
    full = datagen.make_workload("zipf", n, 0.9, seed=4)
    on, oc, want = oracle.join_sorted_pairs(*(t.numpy().view(np.uint32) for t in full))
    shards = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
    res = sharded.run_local(world, shards, mode="materialize", out_capacity=on)
    got = np.concatenate([r.pairs.cpu().numpy().view(np.uint32) for r in res])
    assert sum(r.written for r in res) == on and all(not r.overflow for r in res)
    got = got[np.lexsort((got[:, 1], got[:, 0]))]
    assert np.array_equal(got, want)
    for r in res:
        assert (r.count, r.checksum) == (on, oc)


def test_join_rejects_false_route_bits_assertion():
    """gsh_config.route_bits asserts that every tuple shares the top route_bits of h; gsh_join
    verifies it in the histogram pass and refuses (GSH_ERR_INVALID) instead of trusting it."""
    from paper_conf_icde_caic24_b200 import GshError, join, make_config
    dev = torch.device("cuda", 0)
    rk, rp, sk, sp = (t.to(dev) for t in datagen.make_workload("pkfk", 1 << 16, 0.0, seed=2))
    with pytest.raises(GshError, match="route_bits"):
        join(rk, rp, sk, sp, config=make_config(route_bits=2))
    # the same call on a shard whose tuples do share the bits is accepted and exact
    h = oracle.fmix32(_u32(rk))
    sel = torch.from_numpy(np.nonzero((h >> 30) == 1)[0]).to(dev)
    hs = oracle.fmix32(_u32(sk))
    sels = torch.from_numpy(np.nonzero((hs >> 30) == 1)[0]).to(dev)
    r = join(rk[sel], rp[sel], sk[sels], sp[sels], config=make_config(route_bits=2))
    on, oc, _ = oracle.join(_u32(rk[sel]), _u32(rp[sel]), _u32(sk[sels]), _u32(sp[sels]))
    assert (r.count, r.checksum) == (on, oc)


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
        res = sharded.join_sharded(rk, rp, sk, sp, config=cfg)
        q.put((res.count, res.checksum, res.stats["n_heavy_global"]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("kind,n,theta", [("zipf", 1 << 16, 1.0), ("pkfk", 1 << 15, 0.0)])
def test_sharded_single_rank_nccl(kind, n, theta):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_worker, args=(_free_port(), kind, n, theta, q))
    p.start()
    cnt, chk, nh = q.get(timeout=300)
    p.join(timeout=60)
    assert p.exitcode == 0
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=23)
    on, oc, _ = oracle.join(_u32(rk), _u32(rp), _u32(sk), _u32(sp))
    assert (cnt, chk) == (on, oc)
    if theta >= 1.0:
        assert nh > 0


@pytest.mark.parametrize("world,kind,n,theta,kw", [
    (2, "zipf", 1 << 18, 1.0, {}),
    (4, "pkfk_zipf", 1 << 18, 1.0, dict(heavy_threshold=64)),
    (8, "graph", 1 << 17, 0.909, {}),
    (4, "uniform", 1 << 18, 0.0, {}),
])
def test_sharded_p2p_local_world_vs_oracle(world, kind, n, theta, kw):
    """exchange="p2p": the route kernel stores every tuple straight into its destination rank's
    receive buffer (skewed R into every rank's), so the scatter IS the exchange -- here the G
    logical ranks' buffers share the one GPU.  Twice in a row: the second call reuses the buffers."""
    from paper_conf_icde_caic24_b200 import make_config, sharded
    dev = torch.device("cuda", 0)
    full = datagen.make_workload(kind, n, theta, seed=41)
    on, oc, _ = oracle.join(*(t.numpy().view(np.uint32) for t in full))
    cfg = make_config(**kw)
    shards = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
    for _ in range(2):
        res = sharded.run_local(world, shards, config=cfg, exchange="p2p")
        for r in res:
            assert (r.count, r.checksum) == (on, oc), r.stats
            assert r.stats["exchange"] == "p2p"
        assert sum(r.stats["normal_s"] + r.stats["heavy_s"] for r in res) == n


def _p2p_worker(rank, world, port, kind, n, theta, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icde_caic24_b200 import sharded
        full = datagen.make_workload(kind, n, theta, seed=43)
        rk, rp, sk, sp = (_shard(t, rank, world).cuda() for t in full)
        out = []
        for _ in range(2):
            r = sharded.join_sharded(rk, rp, sk, sp, exchange="p2p")
            out.append((r.count, r.checksum))
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_sharded_p2p_two_processes_ipc():
    """The peer-store exchange across PROCESSES: two ranks on the one GPU, receive buffers shared
    through CUDA IPC (gsh_ipc_handle / gsh_ipc_open -- the same calls that map a peer GPU's memory
    over NVLink), host-side collectives on gloo.  Exact vs the oracle, and again on reused buffers."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    world, kind, n, theta = 2, "zipf", 1 << 17, 1.0
    procs = [ctx.Process(target=_p2p_worker, args=(r, world, port, kind, n, theta, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    full = datagen.make_workload(kind, n, theta, seed=43)
    on, oc, _ = oracle.join(*(t.numpy().view(np.uint32) for t in full))
    for _, res in out:
        assert res == [(on, oc), (on, oc)]
