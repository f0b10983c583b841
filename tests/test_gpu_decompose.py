"""decomposition of the giant COUNT joins (cfg3 theta = 1.0 at 2^27 per side,
the power-law graph at 2^28 edges), whose outputs (~8e13 pairs) no oracle can enumerate.

gsh_config.heavy_detail + gsh_heavy_detail split the result into the NM-join's share and one term
per skewed key k (cnt_R(k), cnt_S(k), C_k = sum of pair_hash over R_k x S_k).  Checked against
values that never come from the CUDA path:
  * the split adds up: count = normal + sum cnt_R cnt_S, checksum = normal + sum C_k (mod 2^64);
  * cnt_R(k), cnt_S(k) equal exact histograms of the inputs (numpy over the generator's arrays);
  * the normal share equals the oracle's join of the inputs with every skewed key removed;
  * C_k equals brute force (oracle pair_hash over the outer product of the key's payloads) for a
    random sample of skewed keys with |R_k| |S_k| <= 2e7; at the ladder size (2^20) for all of them.
The very largest keys' C_k at full size stay parity-unpinned by the oracle: they are the same
kernel as the ladder's fully checked keys, and the total checksum is the sum of the pinned parts."""
import os

import numpy as np
import pytest
import torch

import datagen
import oracle
import paper_conf_icde_caic24_b200 as gsh

pytestmark = pytest.mark.gpu
M64 = (1 << 64) - 1


def _u32(t):
    return t.cpu().numpy().view(np.uint32)


def _key_counts(h_all, hs_sorted):
    idx = np.searchsorted(hs_sorted, h_all)
    idx = np.minimum(idx, hs_sorted.size - 1)
    hit = hs_sorted[idx] == h_all
    return np.bincount(idx[hit], minlength=hs_sorted.size), hit


def _brute_ck(pr, ps):
    """sum over R_k x S_k of pair_hash(pr, ps) mod 2^64 (oracle pair_hash, numpy)."""
    tot = 0
    step = max(1, (1 << 22) // max(ps.size, 1))
    for a in range(0, pr.size, step):
        blk = pr[a:a + step]
        aa = np.repeat(blk, ps.size)
        bb = np.tile(ps, blk.size)
        tot += int(np.sum(oracle.pair_hash(aa, bb), dtype=np.uint64))
    return tot & M64


def _check(kind, n, theta, seed, sample_all=False, max_pairs=2e7, n_sample=8):
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=seed, device="cuda")
    r, det = gsh.join_detail(rk, rp, sk, sp)
    st = r.stats
    hk = det["h"].numpy().astype(np.uint32)
    cr = det["cnt_r"].numpy()
    cs = det["cnt_s"].numpy()
    ck = det["checksum"]
    assert hk.size == st["n_heavy"] > 0
    # (1) the parts add up
    assert r.count == st["normal_count"] + int(np.sum(cr * cs))
    assert r.checksum == (st["normal_checksum"] + sum(ck)) & M64
    # (2) per-key counts = exact histograms of the inputs
    kr, ks, pr_all, ps_all = _u32(rk), _u32(sk), _u32(rp), _u32(sp)
    hr, hs_ = oracle.fmix32(kr), oracle.fmix32(ks)
    order = np.argsort(hk)
    hsort = hk[order]
    cnt_r, hit_r = _key_counts(hr, hsort)
    cnt_s, hit_s = _key_counts(hs_, hsort)
    assert np.array_equal(cnt_r, cr[order]) and np.array_equal(cnt_s, cs[order])
    # (3) the NM share = the oracle join of everything but the skewed keys
    on, oc, _ = oracle.join(kr[~hit_r], pr_all[~hit_r], ks[~hit_s], ps_all[~hit_s])
    assert (st["normal_count"], st["normal_checksum"]) == (on, oc)
    # (4) C_k by brute force
    rng = np.random.default_rng(seed)
    idxs = np.arange(hk.size)
    small = idxs[(cr.astype(np.float64) * cs) <= max_pairs]
    pick = small if sample_all else rng.choice(small, size=min(n_sample, small.size), replace=False)
    assert pick.size > 0
    for i in pick:
        pr = pr_all[hr == hk[i]]
        ps = ps_all[hs_ == hk[i]]
        assert _brute_ck(pr, ps) == ck[i], i
    return st


def test_decompose_ladder_all_keys():
    """2^20 per side, theta = 1.0 (cfg1 shape): every skewed key's C_k by brute force."""
    _check("zipf", 1 << 20, 1.0, seed=11, sample_all=True, max_pairs=1e9)


def test_decompose_cfg3_theta1_fullsize():
    """cfg3 at theta = 1.0, |R| = |S| = 2^27 (~8e13 output pairs)."""
    st = _check("zipf", 1 << 27, 1.0, seed=0x6A5)
    assert st["n_large"] > 1000


def test_decompose_graph():
    """cfg4: power-law graph self-join, 2^28 edges, V = 2^24 (~8.6e13 two-hop paths) with
    GSH_FULLSIZE_DECOMP=1 (7 min: profiles/r02_decompose.md); 2^27 edges, V = 2^23 by default."""
    logn = 28 if os.environ.get("GSH_FULLSIZE_DECOMP") == "1" else 27
    _check("graph", 1 << logn, 0.909, seed=0x6A5)
