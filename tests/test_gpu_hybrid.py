"""CSH's hybrid partition on the GPU (gsh_config.hybrid; §IV-A,
L100): keys sampled before partitioning are counted exactly by the histogram pass and their R and
S tuples go straight from pass 1 into R_k / S_k.  Which keys are chosen changes performance only,
so every result must equal the oracle's bit-exactly (count, checksum, sorted pairs), and the
decomposition (P5) must show the chosen keys with their exact counts."""
import numpy as np
import pytest
import torch

import datagen
import oracle
import paper_conf_icde_caic24_b200 as gsh

pytestmark = pytest.mark.gpu
DEV = "cuda"
M64 = (1 << 64) - 1


def _np(t):
    return t.cpu().numpy().view(np.uint32)


def _dev(*ts):
    return [t.to(DEV) for t in ts]


def _sorted_pairs(p):
    a = p.cpu().numpy().view(np.uint32).reshape(-1, 2)
    return a[np.lexsort((a[:, 1], a[:, 0]))]


# hybrid_share=1: engage whenever the sample chose keys (the default 1/2 gate would keep GSH's passes
# on several of these inputs); the gate itself: test_hybrid_share_gate
HYB = dict(hybrid=True, timing=True, hybrid_share=1)

# skewed: the sample must choose keys (True), must not (False: chance triples of a skew-free input
# hold < 1/64 of the sample), or either (None: theta = 0.5, little mass in the top keys)
LADDER = [("uniform", 100_000, 0.0, False), ("pkfk", (1 << 18) + 5, 0.0, False),
          ("zipf", 1 << 18, 0.5, None), ("zipf", (1 << 18) + 7, 0.75, True), ("zipf", 1 << 20, 1.0, True),
          ("zipf", 1 << 16, 1.25, True), ("zipf", 1 << 17, 1.5, True), ("graph", 1 << 18, 0.909, True),
          ("pkfk_zipf", 1 << 18, 1.0, True), ("zipf", 5_000, 1.0, True)]


@pytest.mark.parametrize("kind,n,theta,skewed", LADDER)
def test_hybrid_count_checksum_ladder(kind, n, theta, skewed):
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=13)
    on, oc, _ = oracle.join(_np(rk), _np(rp), _np(sk), _np(sp))
    r = gsh.join(*_dev(rk, rp, sk, sp), config=gsh.make_config(**HYB))
    assert (r.count, r.checksum) == (on, oc)
    st = r.stats
    assert st["n_hybrid"] <= min(st["n_heavy"], 512)
    if skewed:
        assert st["n_hybrid"] > 0 and st["ms_sample"] > 0
    elif skewed is False:
        assert st["n_hybrid"] == 0


@pytest.mark.parametrize("kind,n,theta", [("zipf", 40_000, 1.0), ("zipf", (1 << 16) + 1, 0.75),
                                          ("zipf", 20_000, 1.5), ("graph", 1 << 16, 0.909),
                                          ("pkfk_zipf", 1 << 17, 1.25)])
def test_hybrid_materialize_pairs_exact(kind, n, theta):
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=5)
    on, oc, op = oracle.join_sorted_pairs(_np(rk), _np(rp), _np(sk), _np(sp))
    r = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=on + 10, config=gsh.make_config(**HYB))
    assert (r.count, r.checksum, r.written, r.overflow) == (on, oc, on, False)
    assert r.stats["n_hybrid"] > 0
    assert np.array_equal(_sorted_pairs(r.pairs), op)


@pytest.mark.parametrize("kind,n,theta", [("zipf", 1 << 20, 1.0), ("zipf", 1 << 18, 1.5), ("graph", 1 << 19, 0.909)])
def test_hybrid_decomposition_exact_counts(kind, n, theta):
    """P5 with the hybrid keys: the first n_hybrid skewed keys carry exact per-side counts (the
    histogram pass's), the parts add up, the NM share is the oracle join without every skewed key,
    and C_k equals brute force for the keys whose product is small enough."""
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=17)
    r, det = gsh.join_detail(*_dev(rk, rp, sk, sp), config=gsh.make_config(hybrid=True, heavy_detail=True, hybrid_share=1))
    st = r.stats
    nh = st["n_hybrid"]
    assert 0 < nh <= det["h"].numel() == st["n_heavy"]
    hk = det["h"].numpy().astype(np.uint32)
    cr, cs, ck = det["cnt_r"].numpy(), det["cnt_s"].numpy(), det["checksum"]
    assert r.count == st["normal_count"] + int(np.sum(cr * cs))
    assert r.checksum == (st["normal_checksum"] + sum(ck)) & M64
    kr, ks, pr_all, ps_all = _np(rk), _np(sk), _np(rp), _np(sp)
    hr, hs_ = oracle.fmix32(kr), oracle.fmix32(ks)
    assert np.unique(hk).size == hk.size   # a key is skewed once (hybrid or detected, not both)
    for i in range(hk.size):
        assert (int(np.sum(hr == hk[i])), int(np.sum(hs_ == hk[i]))) == (cr[i], cs[i]), i
    heavy_r, heavy_s = np.isin(hr, hk), np.isin(hs_, hk)
    on, oc, _ = oracle.join(kr[~heavy_r], pr_all[~heavy_r], ks[~heavy_s], ps_all[~heavy_s])
    assert (st["normal_count"], st["normal_checksum"]) == (on, oc)
    rng = np.random.default_rng(3)
    small = np.nonzero(cr.astype(np.float64) * cs <= 3e6)[0]
    for i in rng.choice(small, size=min(6, small.size), replace=False):
        pr, ps = pr_all[hr == hk[i]], ps_all[hs_ == hk[i]]
        aa, bb = np.repeat(pr, ps.size), np.tile(ps, pr.size)
        assert int(np.sum(oracle.pair_hash(aa, bb), dtype=np.uint64)) == ck[i], i


@pytest.mark.parametrize("cfg", [dict(hybrid_stride=1, hybrid_min=1), dict(hybrid_stride=1),
                                 dict(hybrid_stride=7, hybrid_min=2), dict(hybrid_stride=100000),
                                 dict(detect_mode=1), dict(prepass_bits=2), dict(capacity=256),
                                 dict(nm_table=2), dict(pass_bits=(3, 2)), dict(heavy_threshold=100000),
                                 dict(force_all_normal=True), dict(force_all_heavy=True)])
def test_hybrid_invariant_under_config(cfg):
    """Metamorphic (P4): sample rate, threshold, the 512-key cap (stride 1, min 1: every key is a
    candidate), the other detection, pre-partition pass, fanout and table choices change
    performance only."""
    rk, rp, sk, sp = datagen.zipf_pair(1 << 16, (1 << 16) + 9, 1.0, seed=21)
    on, oc, op = oracle.join_sorted_pairs(_np(rk), _np(rp), _np(sk), _np(sp))
    d = _dev(rk, rp, sk, sp)
    c = gsh.make_config(hybrid=True, hybrid_share=1, **cfg)
    r = gsh.join(*d, config=c)
    assert (r.count, r.checksum) == (on, oc)
    if cfg.get("hybrid_min") == 1:
        assert r.stats["n_hybrid"] <= 512
    m = gsh.join(*d, mode="materialize", out_capacity=on, config=c)
    assert (m.count, m.checksum, m.written) == (on, oc, on)
    assert np.array_equal(_sorted_pairs(m.pairs), op)


def test_hybrid_edge_cases():
    z = torch.zeros
    cases = [
        # one giant key on both sides (every sample hits it)
        (z(3000, dtype=torch.int32), torch.arange(3000, dtype=torch.int32),
         z(2000, dtype=torch.int32), torch.arange(2000, dtype=torch.int32)),
        # the giant key only in S (R unique: PK-FK), all-ones key (h = fmix32(~0) != the table's empty mark)
        (torch.arange(-5, 5000, dtype=torch.int32), torch.arange(5005, dtype=torch.int32),
         torch.full((50000,), -1, dtype=torch.int32), torch.arange(50000, dtype=torch.int32)),
        # a giant key whose h = fmix32(0x331da083) = 0xffffffff, the lookup table's empty mark: never
        # routed by the hybrid pass (detected after partitioning instead), still joined
        (torch.cat([torch.full((4000,), 0x331da083, dtype=torch.int32), torch.arange(100, dtype=torch.int32)]),
         torch.arange(4100, dtype=torch.int32),
         torch.cat([torch.full((3000,), 0x331da083, dtype=torch.int32), torch.arange(50, 150, dtype=torch.int32)]),
         torch.arange(3100, dtype=torch.int32)),
        # fewer tuples than the sample stride, empty side
        (torch.tensor([7, 7, 7], dtype=torch.int32), torch.arange(3, dtype=torch.int32),
         torch.tensor([7], dtype=torch.int32), torch.arange(1, dtype=torch.int32)),
        (z(0, dtype=torch.int32), z(0, dtype=torch.int32), z(100, dtype=torch.int32),
         torch.arange(100, dtype=torch.int32)),
    ]
    for rk, rp, sk, sp in cases:
        on, oc, op = oracle.join_sorted_pairs(_np(rk), _np(rp), _np(sk), _np(sp))
        for stride in (0, 1):
            c = gsh.make_config(hybrid=True, hybrid_stride=stride, hybrid_share=1)
            r = gsh.join(*_dev(rk, rp, sk, sp), config=c)
            assert (r.count, r.checksum) == (on, oc)
            m = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=on, config=c)
            assert m.written == on and np.array_equal(_sorted_pairs(m.pairs), op)


def test_hybrid_unaligned_views_and_routing_bits():
    """Unaligned SoA views take pass 1's scalar (non-TMA) path; a shard that shares the top 2 bits
    of h runs under route_bits = 2 (the multi-GPU local join's configuration)."""
    rk, rp, sk, sp = datagen.zipf_pair(90_001, 70_003, 1.0, seed=3)
    d = _dev(rk, rp, sk, sp)
    on, oc, _ = oracle.join(_np(rk[1:]), _np(rp[1:]), _np(sk[3:]), _np(sp[2:-1]))
    r = gsh.join(d[0][1:], d[1][1:], d[2][3:], d[3][2:-1], config=gsh.make_config(hybrid=True, hybrid_share=1))
    assert (r.count, r.checksum) == (on, oc) and r.stats["n_hybrid"] > 0
    kr = (oracle.fmix32(_np(rk)) >> 30) == 1
    ks = (oracle.fmix32(_np(sk)) >> 30) == 1
    sh = [t[torch.from_numpy(m)] for t, m in ((rk, kr), (rp, kr), (sk, ks), (sp, ks))]
    on2, oc2, _ = oracle.join(*(_np(t) for t in sh))
    r2 = gsh.join(*_dev(*sh), config=gsh.make_config(hybrid=True, route_bits=2, hybrid_share=1))
    assert (r2.count, r2.checksum) == (on2, oc2)


def test_hybrid_repeatable():
    rk, rp, sk, sp = _dev(*datagen.zipf_pair(1 << 18, 1 << 18, 1.25, seed=2))
    c = gsh.make_config(hybrid=True, hybrid_share=1)
    a = gsh.join(rk, rp, sk, sp, config=c)
    b = gsh.join(rk, rp, sk, sp, config=c)
    assert (a.count, a.checksum, a.stats["n_heavy"]) == (b.count, b.checksum, b.stats["n_heavy"])


def test_hybrid_share_gate():
    """gsh_config.hybrid_share: the hybrid passes run only when the chosen keys hold at least that share
    of the sample.  Zipf 1.5 (the top keys hold ~90 % of the input) passes the default 1/2; theta 0.75 does
    not (GSH's passes run, the same result); any sampled skew passes 1/256."""
    for theta, engaged_default in ((1.5, True), (0.75, False)):
        rk, rp, sk, sp = _dev(*datagen.zipf_pair(1 << 18, 1 << 18, theta, seed=4))
        on, oc, _ = oracle.join(*(_np(t) for t in (rk, rp, sk, sp)))
        r = gsh.join(rk, rp, sk, sp, config=gsh.make_config(hybrid=True))
        assert (r.count, r.checksum) == (on, oc)
        assert (r.stats["n_hybrid"] > 0) == engaged_default, (theta, r.stats["n_hybrid"])
        r1 = gsh.join(rk, rp, sk, sp, config=gsh.make_config(hybrid=True, hybrid_share=1))
        assert (r1.count, r1.checksum) == (on, oc) and r1.stats["n_hybrid"] > 0
        r2 = gsh.join(rk, rp, sk, sp, config=gsh.make_config(hybrid=True, hybrid_share=256))
        assert (r2.count, r2.checksum) == (on, oc) and r2.stats["n_hybrid"] == 0
