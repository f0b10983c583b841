"""Parity at BASELINE.json's full sizes, in bench.py's launch configuration (default config).

The oracle cannot enumerate these joins in seconds, so the checks are properties that fix the
result exactly:
  * cfg2 (|R| = |S| = 2^27, 1:1 PK-FK): every S row matches exactly the R row whose key it copied,
    so count = n_S and checksum = sum_j pair_hash(row_R(j), j) -- computed with the oracle's
    pair_hash over the generator's own row map (no CUDA-path value involved);
  * MATERIALIZE at full size: written == count, every written pair is a real match (payload =
    row id, so R.key[a] == S.key[b]), no pair repeats, and the oracle's checksum over the written
    pairs equals the returned checksum -- together these prove the pair multiset is M;
  * Zipf (both sides skewed) at 2^24: count equals the closed form sum_k cnt_R(k) * cnt_S(k) from
    exact key histograms (np.unique), and (count, checksum) are identical under configurations
    that route the work through different phases (invariance, P4).
"""
import numpy as np
import pytest
import torch

import datagen
import oracle
import paper_conf_icde_caic24_b200 as gsh

pytestmark = pytest.mark.gpu

N2 = 1 << 27


@pytest.fixture(scope="module")
def cfg2():
    rk, rp, sk, sp = datagen.pkfk_pair(N2, N2, seed=0x6A5, device="cuda")
    return rk, rp, sk, sp


def _pkfk_expected(n_r, n_s, seed):
    """Row of R copied by each S row (the generator's own draw, recomputed on the CPU)."""
    idx = datagen.rand_u63(seed, 1, n_s) % n_r
    return idx.numpy().astype(np.uint32)


def test_cfg2_count_checksum_fullsize(cfg2):
    rk, rp, sk, sp = cfg2
    r = gsh.join(rk, rp, sk, sp)
    assert r.count == N2
    rows = _pkfk_expected(N2, N2, 0x6A5)
    expect = 0
    step = 1 << 24
    for b in range(0, N2, step):
        expect += int(np.sum(oracle.pair_hash(rows[b:b + step], np.arange(b, min(b + step, N2), dtype=np.uint32)),
                             dtype=np.uint64))
    assert r.checksum == expect & ((1 << 64) - 1)
    assert r.stats["n_large"] == 0  # uniform keys never trigger detection


@pytest.mark.parametrize("logn", [28, 30])
def test_pkfk_large_count_checksum(logn):
    """2x and 8x the bench size.  |R| = |S| = 2^28: partitions average 4096 tuples per side, so
    about half of them exceed the CSR staging limit and stream through the chained table's
    larger one (kRingMaxRChain); 2^30: the pre-partition pass splits both sides by 2 hash bits
    into four 2^28 sub-problems (gsh_config.prepass_bits auto).  count = n_S and the closed-form checksum
    (oracle pair_hash over the generator's row map, computed in chunks on the CPU) must hold."""
    n = 1 << logn
    if torch.cuda.get_device_properties(0).total_memory < (96 << 30):
        pytest.skip("needs a GPU with >= 96 GB")
    rk, rp, sk, sp = datagen.pkfk_pair(n, n, seed=0x6A5, device="cuda")
    torch.cuda.synchronize()
    r = gsh.join(rk, rp, sk, sp)
    del rk, rp, sk, sp
    torch.cuda.empty_cache()
    assert r.count == n
    expect = 0
    step = 1 << 24
    base = datagen.gen._stream_base(0x6A5, 1)
    for b in range(0, n, step):
        idx = torch.arange(b, b + step, dtype=torch.int64) + base
        rows = (datagen.gen._srl(datagen.gen.splitmix64(idx), 1) % n).numpy().astype(np.uint32)
        expect += int(np.sum(oracle.pair_hash(rows, np.arange(b, b + step, dtype=np.uint32)), dtype=np.uint64))
    assert r.checksum == expect & ((1 << 64) - 1)
    assert r.stats["n_large"] == 0
    assert r.stats["prepass_bits"] == (2 if logn == 30 else 0)


def test_cfg2_materialize_fullsize(cfg2):
    rk, rp, sk, sp = cfg2
    r = gsh.join(rk, rp, sk, sp, mode="materialize", out_capacity=N2 + 16)
    assert (r.count, r.written, r.overflow) == (N2, N2, False)
    p = r.pairs.long() & 0xFFFFFFFF
    a, b = p[:, 0], p[:, 1]
    assert bool((rk[a] == sk[b]).all())                       # every pair matches (payload = rid)
    packed = (a << 32) | b
    assert torch.unique(packed).numel() == N2                 # no pair repeats
    pc = r.pairs.cpu().numpy().view(np.uint32)
    chk = 0
    for s in range(0, N2, 1 << 24):
        chk += int(np.sum(oracle.pair_hash(pc[s:s + (1 << 24), 0], pc[s:s + (1 << 24), 1]), dtype=np.uint64))
    assert chk & ((1 << 64) - 1) == r.checksum


def _closed_form(rk, sk):
    ur, cr = np.unique(rk.cpu().numpy().view(np.uint32), return_counts=True)
    us, cs = np.unique(sk.cpu().numpy().view(np.uint32), return_counts=True)
    _, ir, is_ = np.intersect1d(ur, us, assume_unique=True, return_indices=True)
    return int(np.sum(cr[ir].astype(np.int64) * cs[is_].astype(np.int64)))


@pytest.mark.parametrize("theta", [0.75, 1.0])
def test_zipf_2e24_closed_form_and_invariance(theta):
    n = 1 << 24 if theta < 1.0 else 1 << 22
    rk, rp, sk, sp = datagen.zipf_pair(n, n, theta, seed=31, device="cuda")
    r = gsh.join(rk, rp, sk, sp)
    assert r.count == _closed_form(rk, sk)
    assert r.stats["n_heavy"] > 0
    # every skewed key's |R_k| |S_k| goes through the dense phase; the same pairs through the
    # NM-join (no detection) must give the identical checksum
    r2 = gsh.join(rk, rp, sk, sp, config=gsh.make_config(force_all_normal=True))
    assert (r2.count, r2.checksum) == (r.count, r.checksum)
    r3 = gsh.join(rk, rp, sk, sp, config=gsh.make_config(large_threshold=1, heavy_threshold=2))
    assert (r3.count, r3.checksum) == (r.count, r.checksum)


@pytest.mark.parametrize("theta", [0.25, 0.5])
def test_cfg3_materialize_fullsize(theta):
    """cfg3 at its full size (|R| = |S| = 2^27, both sides Zipf theta, N = n) in MATERIALIZE mode
    (SURVEY §8(c) P3): count equals the closed form from exact key histograms, written == count,
    every written pair is a real match (payload = row id), no pair repeats, and the oracle's
    checksum over the written pairs equals the returned one -- together the pair multiset is M."""
    n = N2
    rk, rp, sk, sp = datagen.zipf_pair(n, n, theta, seed=0x6A5, device="cuda")
    expect = _closed_form(rk, sk)
    r = gsh.join(rk, rp, sk, sp, mode="materialize", out_capacity=expect + 16)
    assert (r.count, r.written, r.overflow) == (expect, expect, False)
    p = r.pairs.long() & 0xFFFFFFFF
    a, b = p[:, 0], p[:, 1]
    assert bool((rk[a] == sk[b]).all())
    assert torch.unique((a << 32) | b).numel() == expect
    del p, a, b
    pc = r.pairs.cpu().numpy().view(np.uint32)
    chk = 0
    for s in range(0, expect, 1 << 24):
        chk += int(np.sum(oracle.pair_hash(pc[s:s + (1 << 24), 0], pc[s:s + (1 << 24), 1]), dtype=np.uint64))
    assert chk & ((1 << 64) - 1) == r.checksum
    if theta == 0.5:
        assert r.stats["n_heavy"] > 0    # the skewed-key phase wrote part of the pairs


def test_cfg3_theta075_count_fullsize():
    """cfg3 at theta = 0.75, full size (2.6e11 pairs: COUNT only): count equals the closed form, and
    the checksum is identical when every pair goes through the NM-join instead (no detection)."""
    n = N2
    rk, rp, sk, sp = datagen.zipf_pair(n, n, 0.75, seed=0x6A5, device="cuda")
    r = gsh.join(rk, rp, sk, sp)
    assert r.count == _closed_form(rk, sk)
    assert r.stats["n_heavy"] > 0 and r.stats["n_large"] > 0
    r2 = gsh.join(rk, rp, sk, sp, config=gsh.make_config(force_all_normal=True))
    assert (r2.count, r2.checksum) == (r.count, r.checksum)
    # CSH's hybrid partition (NEXT-1) at full size: the same pairs (at this theta the keys sampled
    # twice by a CTA hold ~0.5 % of the input, under the 1/64 gate, so the GSH passes run; the
    # engaged hybrid passes at full size: test_hybrid_fullsize_input_side)
    r3 = gsh.join(rk, rp, sk, sp, config=gsh.make_config(hybrid=True))
    assert (r3.count, r3.checksum) == (r.count, r.checksum)


@pytest.mark.parametrize("theta", [1.0, 1.5])
def test_hybrid_fullsize_input_side(theta):
    """The hybrid partition at 2^27 per side, theta = 1.0 / 1.5 (8e13 / 3e15 pairs: input side only,
    the per-key counts are pinned by the P5 hook at the ladder size, tests/test_gpu_hybrid.py): the
    sampled keys plus the keys detected after partitioning must still send (nearly) all of the output
    to the dense skewed-key phase, as GSH's detection alone does."""
    n = N2
    rk, rp, sk, sp = datagen.zipf_pair(n, n, theta, seed=0x6A5, device="cuda")
    r = gsh.join(rk, rp, sk, sp, config=gsh.make_config(hybrid=True, input_side_only=True, hybrid_share=1))
    st = r.stats
    assert st["n_hybrid"] > 0
    g = gsh.join(rk, rp, sk, sp, config=gsh.make_config(input_side_only=True))
    assert st["skew_pairs"] > 0.99 * g.stats["skew_pairs"]
    assert st["heavy_tuples_r"] <= n and st["heavy_tuples_s"] <= n


def _closed_form_gpu(rk, sk):
    """sum_k cnt_R(k) cnt_S(k) from exact key histograms (torch.unique on the device: a library
    sort, independent of the join's kernels)."""
    ur, cr = torch.unique(rk.long() & 0xFFFFFFFF, return_counts=True)
    us, cs = torch.unique(sk.long() & 0xFFFFFFFF, return_counts=True)
    pos = torch.searchsorted(us, ur).clamp(max=us.numel() - 1)
    hit = us[pos] == ur
    return int((cr[hit] * cs[pos[hit]]).sum().item())


def test_next3_theta07_2e29():
    """the paper's large-input experiment (§V-B: 560 million
    tuples per side, Zipf theta = 0.7) scaled to one B200: |R| = |S| = 2^29 (537M), both sides
    Zipf theta = 0.7 with N = n.  Beyond 2^28 per side the pre-partition pass runs (auto 1 bit).
    count = the closed form from exact histograms; the checksum is identical when the input is
    split into 8 sub-problems instead (prepass_bits = 3): the same pairs through a different
    decomposition."""
    if torch.cuda.get_device_properties(0).total_memory < (96 << 30):
        pytest.skip("needs a GPU with >= 96 GB")
    n = 1 << 29
    rk, rp, sk, sp = datagen.zipf_pair(n, n, 0.7, seed=0x6A5, device="cuda")
    expect = _closed_form_gpu(rk, sk)
    torch.cuda.empty_cache()
    r = gsh.join(rk, rp, sk, sp)
    assert r.count == expect
    assert r.stats["prepass_bits"] == 1 and r.stats["n_heavy"] > 0
    r2 = gsh.join(rk, rp, sk, sp, config=gsh.make_config(prepass_bits=3))
    assert (r2.count, r2.checksum) == (r.count, r.checksum)
