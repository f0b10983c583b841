"""Generator pins: the synthetic workloads are shaped like the paper's (§V-A)."""
import math

import numpy as np
import pytest
import torch

import datagen
import oracle


def test_splitmix64_reference_value():
    # splitmix64 with state 0: first output of the reference generator is 0xe220a8397b1dcdaf
    v = int(datagen.splitmix64(torch.tensor([0], dtype=torch.int64)).item()) & ((1 << 64) - 1)
    assert v == 0xE220A8397B1DCDAF


def test_splitmix64_matches_numpy_uint64():
    x = torch.arange(-5000, 5000, dtype=torch.int64) * 0x1234567
    got = datagen.splitmix64(x).numpy().view(np.uint64)
    z = x.numpy().view(np.uint64) + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    z = z ^ (z >> np.uint64(31))
    assert np.array_equal(got, z)


def test_rank_to_key_is_injective():
    r = torch.arange(1 << 20, dtype=torch.int64)
    k = datagen.rank_to_key(r, 7)
    assert int(k.min()) >= 0 and int(k.max()) < (1 << 32)
    assert torch.unique(k).numel() == r.numel()


def test_zipf_top_key_count_matches_paper_L59():
    """PAPER.md §III: at zipf 1.0 with 32 million tuples 'the most popular join key is
    shared by about 1.79 million tuples in each input table'.  With N = n = 32e6,
    E = n / H_n = 1,791,868 (sigma ~ 1.3K).  Count draws below the first cut point."""
    n = 32_000_000
    T = datagen.zipf_thresholds(n, 1.0)
    u = datagen.rand_u63(0, 0, n)
    top = int((u < int(T[0])).sum())
    H = math.fsum(1.0 / k for k in range(1, 200001)) + math.log(n / 200000.5)  # H_n
    expect = n / H
    sigma = math.sqrt(n * (1 / H) * (1 - 1 / H))
    assert abs(expect - 1_791_868) < 50
    assert abs(top - expect) < 5 * sigma
    assert abs(top - 1.79e6) / 1.79e6 < 0.01


@pytest.mark.slow
def test_no_large_partition_below_theta_0_4_paper_L166():
    """PAPER.md §V-B: 'When the zipf factor is 0-0.4, none of the partitions is larger
    than the shared memory'.  32M tuples, fanout 2^14 (mean ~1953), capacity C = 2 * mean
    (the large-partition threshold reading): no partition of either side
    exceeds C at theta = 0.4; at theta = 0.5 some do (the top key alone is ~2.8K)."""
    n = 32_000_000
    bits = 14
    cap = 2 * n // (1 << bits)
    for theta, expect_large in [(0.4, False), (0.5, True)]:
        rk, _, sk, _ = datagen.zipf_pair(n, n, theta, seed=3)
        mx = 0
        for k in (rk, sk):
            hist = oracle.radix_histogram(k.numpy().view(np.uint32), 0, bits)
            mx = max(mx, int(hist.max()))
        assert (mx > cap) == expect_large, (theta, mx, cap)


def test_zipf_thresholds_monotone_and_uniform_exact():
    T = datagen.zipf_thresholds(1000, 0.0)
    assert T.size == 999 and np.all(np.diff(T) > 0)
    assert int(T[499]) == (500 << 63) // 1000
    for th in (0.25, 1.0, 1.5):
        T = datagen.zipf_thresholds(1 << 16, th)
        assert np.all(np.diff(T) >= 0) and int(T[-1]) < (1 << 63)
        # first interval length ~ p_1 = 1 / H_{N,theta}
        H = np.sum(np.arange(1, (1 << 16) + 1, dtype=np.float64) ** -th)
        assert abs(int(T[0]) / 2.0 ** 63 - 1 / H) < 1e-12


def test_pkfk_shape():
    rk, rp, sk, sp = datagen.pkfk_pair(1 << 16, 3 << 15, seed=1)
    assert torch.unique(rk).numel() == rk.numel()
    assert bool(torch.isin(sk, rk).all())
    assert torch.equal(rp, torch.arange(rk.numel(), dtype=torch.int32))


def test_zipf_shares_interval_array_and_keys():
    rk, _, sk, _ = datagen.zipf_pair(1 << 16, 1 << 16, 1.0, seed=2)
    # same rank->key map and intervals: the two top keys coincide
    vr, cr = torch.unique(rk, return_counts=True)
    vs, cs = torch.unique(sk, return_counts=True)
    assert int(vr[cr.argmax()]) == int(vs[cs.argmax()])
    assert not torch.equal(rk, sk)  # independent streams


def test_graph_shape():
    dst, eid, src, eid2 = datagen.graph_pair(1 << 16, 1 << 12, seed=4)
    assert torch.equal(eid, eid2)
    v, c = torch.unique(src, return_counts=True)
    assert v.numel() <= 1 << 12 and int(c.max()) > 16 * 8  # hubs: max degree >> mean
