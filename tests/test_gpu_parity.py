"""GPU parity of the CUDA path (through the C-ABI) against the CPU oracle, element by element,
on seeded synthetic inputs shaped like the paper's workloads (DESIGN.md §4 recipe).

Integer-only method -> the bar is bit-exact: count, checksum, and the sorted pair multiset."""
import numpy as np
import pytest
import torch

import datagen
import oracle
import paper_conf_icde_caic24_b200 as gsh

pytestmark = pytest.mark.gpu
DEV = "cuda"


def _np(t):
    return t.cpu().numpy().view(np.uint32)


def _dev(*ts):
    return [t.to(DEV) for t in ts]


def _oracle(rk, rp, sk, sp, pairs=False):
    if pairs:
        return oracle.join_sorted_pairs(_np(rk), _np(rp), _np(sk), _np(sp))
    n, c, _ = oracle.join(_np(rk), _np(rp), _np(sk), _np(sp))
    return n, c, None


def _sorted_pairs(p):
    a = p.cpu().numpy().view(np.uint32).reshape(-1, 2)
    return a[np.lexsort((a[:, 1], a[:, 0]))]


# ---------------------------------------------------------------------- single phases
@pytest.mark.parametrize("n", [0, 1, 5, 1000, (1 << 16) + 3])
def test_hash_keys_bit_exact(n):
    k = torch.randint(-(1 << 31), (1 << 31) - 1, (n,), dtype=torch.int32)
    if n >= 2:
        k[0] = 0
        k[1] = -1
    got = gsh.hash_keys(k.to(DEV))
    assert np.array_equal(_np(got), oracle.fmix32(_np(k)))


@pytest.mark.parametrize("hi,nb", [(0, 0), (0, 8), (0, 16), (3, 5), (8, 8)])
def test_radix_histogram_bit_exact(hi, nb):
    rk, _, _, _ = datagen.zipf_pair(200_003, 10, 1.0, seed=1)
    got = gsh.radix_histogram(rk.to(DEV), hi, nb).cpu().numpy()
    assert np.array_equal(got, oracle.radix_histogram(_np(rk), hi, nb))


@pytest.mark.parametrize("kind,n,theta", [("uniform", 100_000, 0.0), ("zipf", 300_001, 1.0),
                                          ("zipf", 1 << 18, 1.5), ("pkfk", 50_000, 0.0), ("uniform", 5, 0.0)])
def test_partition_phase(kind, n, theta):
    """Histogram + scan + pass-1 + pass-2 scatter: offsets equal the oracle's
    exclusive scan of the digit histogram, every partition holds exactly the tuples whose
    digits select it, and each side is a permutation of (fmix32(key), payload)."""
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=7)
    part_r, part_s, off_r, off_s, (b1, b2) = gsh.partition(*_dev(rk, rp, sk, sp))
    B = b1 + b2
    for keys, pays, part, off in ((rk, rp, part_r, off_r), (sk, sp, part_s, off_s)):
        hist = oracle.radix_histogram(_np(keys), 0, B)
        assert np.array_equal(off.cpu().numpy(), np.concatenate([[0], np.cumsum(hist)]))
        pr = part.cpu().numpy().view(np.uint32)
        digits = (pr[:, 0].astype(np.int64) >> (32 - B)) if B else np.zeros(pr.shape[0], np.int64)
        expect_digit = np.repeat(np.arange(1 << B), hist)
        assert np.array_equal(digits, expect_digit)
        # permutation of (h, payload)
        h = oracle.fmix32(_np(keys))
        a = np.stack([h, _np(pays)], 1)
        assert np.array_equal(a[np.lexsort((a[:, 1], a[:, 0]))], pr[np.lexsort((pr[:, 1], pr[:, 0]))])


def _keys_in_bins(bins, hi, nbits):
    """One key per requested partition digit (bits below the top `hi` of fmix32), found by scan."""
    cand = np.arange(1, 1 << 22, dtype=np.uint32)
    d = (oracle.fmix32(cand) << np.uint32(hi)) >> np.uint32(32 - nbits)
    return [int(cand[np.nonzero(d == b)[0][0]]) for b in bins]


@pytest.mark.parametrize("route_bits", [0, 1])
def test_partition_histogram_u16_wraps(route_bits):
    """2^16 partitions use packed u16 counters per histogram slice: digits that
    receive >= 2^16 keys of one slice wrap, both halves of one counter word wrap, and a low-half
    carry can wrap the high half -- offsets must still equal the oracle's exact scan.  Slices are
    the pass-1 units (~one per scatter CTA, whole 16K-key chunks): at n = 2^24 + 2^21 per side
    a slice holds 8 chunks = 2^17 keys, so 2^17 copies of one digit wrap its u16 twice."""
    pass_bits, B = (8, 8), 16
    ka, kb, kc = _keys_in_bins([0x1234, 0x1235, 0x7777], route_bits, B)   # ka, kb share a counter word
    n = (1 << 24) + (1 << 21) + 77
    g = np.random.default_rng(5)
    keys = g.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    keys[: 1 << 18] = ka                                   # two whole slices of one (even) digit
    keys[(1 << 18):(1 << 18) + (1 << 17):2] = ka           # a slice split evenly between the two
    keys[(1 << 18) + 1:(1 << 18) + (1 << 17):2] = kb       # halves of one word: both wrap, with carries
    pos = g.permutation(np.arange((1 << 19), n))
    keys[pos[:300_000]] = ka
    keys[pos[300_000:560_000]] = kb
    keys[pos[560_000:626_000]] = kc
    # precondition: with the library's unit sizing (api.cu plan_build) some slice holds >= 2^16
    # keys of one digit, so the wrap accounting really runs
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    nch = -(-n // 16384)
    uc = min(64, max(1, -(-(2 * nch) // (2 * sms))))
    dig = (oracle.fmix32(keys) << np.uint32(route_bits)) >> np.uint32(32 - B)
    per_slice = [np.bincount(dig[u:u + uc * 16384], minlength=1 << B).max() for u in range(0, n, uc * 16384)]
    assert max(per_slice) >= 1 << 16
    rk = torch.from_numpy(keys.view(np.int32).copy())
    rp = torch.arange(n, dtype=torch.int32)
    sk, sp = rk.flip(0).contiguous(), rp.clone()
    cfg = gsh.make_config(pass_bits=pass_bits, route_bits=route_bits)
    part_r, part_s, off_r, off_s, bits = gsh.partition(*_dev(rk, rp, sk, sp), config=cfg)
    assert bits == pass_bits
    for k, off in ((rk, off_r), (sk, off_s)):
        hist = oracle.radix_histogram(_np(k), route_bits, B)
        assert np.array_equal(off.cpu().numpy(), np.concatenate([[0], np.cumsum(hist)]))
    if route_bits == 0:  # the whole join over the same wrapped histogram
        sk2 = torch.tensor(np.array([ka, kb, kc, ka, 12345, kb, 7], dtype=np.uint32).view(np.int32))
        sp2 = torch.arange(7, dtype=torch.int32)
        r = gsh.join(*_dev(rk, rp, sk2, sp2), config=cfg)
        assert (r.count, r.checksum) == _oracle(rk, rp, sk2, sp2)[:2]


@pytest.mark.parametrize("theta,n,cfg", [(1.0, 1 << 18, {}), (1.5, 1 << 17, {}), (0.75, 1 << 18, {}),
                                         (1.0, 1 << 16, {"large_threshold": 512, "heavy_threshold": 16}),
                                         (0.5, 1 << 17, {"large_threshold": 256, "heavy_threshold": 4}),
                                         (1.0, 1 << 18, {"capacity": 256})])
def test_skew_detection_matches_exact_rule(theta, n, cfg):
    """Skewed keys (PAPER.md L107/L112 with exact counts, DESIGN.md §3 R3/R4) equal the oracle's
    heavy_rule on the same partition bits, large-partition threshold and key threshold."""
    rk, rp, sk, sp = datagen.zipf_pair(n, n, theta, seed=3)
    config = gsh.make_config(**cfg)
    h, cr, cs, st = gsh.detect(*_dev(rk, rp, sk, sp), config=config)
    B = st["pass_bits"][0] + st["pass_bits"][1]
    oh, ocr, ocs = oracle.heavy_rule(_np(rk), _np(sk), B, st["large_threshold"], st["heavy_threshold"])
    assert st["detect_overflow"] == 0
    assert np.array_equal(h.numpy().astype(np.uint32), oh)
    assert np.array_equal(cr.numpy(), ocr) and np.array_equal(cs.numpy(), ocs)
    if theta >= 1.0:
        assert len(oh) > 0


# ------------------------------------------------------------------- full join parity
LADDER = [
    ("uniform", 0, 0.0), ("uniform", 1, 0.0), ("uniform", 7, 0.0), ("uniform", 1000, 0.0),
    ("pkfk", (1 << 14) + 3, 0.0), ("uniform", 1 << 18, 0.0), ("pkfk", 1 << 20, 0.0),
    ("zipf", (1 << 14) + 3, 0.5), ("zipf", 1 << 18, 0.5), ("zipf", 1 << 18, 0.75),
    ("zipf", (1 << 14) + 3, 1.0), ("zipf", 1 << 18, 1.0), ("zipf", 1 << 20, 1.0),
    ("zipf", 1 << 16, 1.25), ("zipf", 1 << 17, 1.5), ("graph", 1 << 18, 0.909),
]


@pytest.mark.parametrize("kind,n,theta", LADDER)
def test_join_count_checksum_ladder(kind, n, theta):
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=11)
    r = gsh.join(*_dev(rk, rp, sk, sp))
    on, oc, _ = _oracle(rk, rp, sk, sp)
    assert (r.count, r.checksum) == (on, oc)
    assert r.stats["count"] == r.count


@pytest.mark.parametrize("kind,n,theta", [("uniform", 1000, 0.0), ("pkfk", 100_003, 0.0), ("zipf", 40_000, 1.0),
                                          ("zipf", 1 << 16, 0.75), ("zipf", 20_000, 1.5), ("graph", 1 << 16, 0.909)])
def test_join_materialize_pairs_exact(kind, n, theta):
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=5)
    on, oc, op = _oracle(rk, rp, sk, sp, pairs=True)
    r = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=on + 10)
    assert (r.count, r.checksum, r.written, r.overflow) == (on, oc, on, False)
    assert np.array_equal(_sorted_pairs(r.pairs), op)


def test_join_materialize_overflow_subset():
    rk, rp, sk, sp = datagen.zipf_pair(30_000, 30_000, 1.0, seed=8)
    on, oc, op = _oracle(rk, rp, sk, sp, pairs=True)
    cap = on // 3
    r = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=cap)
    assert (r.count, r.checksum, r.written, r.overflow) == (on, oc, cap, True)
    got = _sorted_pairs(r.pairs)
    # every written pair is a real match (payload = rid): R.key[a] == S.key[b]; no duplicates beyond M
    rkn, skn = _np(rk), _np(sk)
    assert np.all(rkn[got[:, 0]] == skn[got[:, 1]])
    assert np.unique(got, axis=0).shape[0] == got.shape[0]  # payloads are rids -> pairs unique


@pytest.mark.parametrize("cfg", [{"force_all_normal": True}, {"force_all_heavy": True}, {"capacity": 256},
                                 {"capacity": 8192}, {"pass_bits": (3, 2)}, {"pass_bits": (8, 8)},
                                 {"pass_bits": (0, 0)}, {"heavy_threshold": 2}, {"capacity": 128, "heavy_threshold": 1000000},
                                 {"large_threshold": 1}, {"large_threshold": 100000}, {"heavy_threshold": 100000}])
def test_join_invariant_under_config(cfg):
    """Skew classification, fanout and capacity change performance only:
    results must be identical under every configuration (metamorphic pin P4)."""
    rk, rp, sk, sp = datagen.zipf_pair(1 << 15, 1 << 15, 1.0, seed=21)
    on, oc, _ = _oracle(rk, rp, sk, sp)
    r = gsh.join(*_dev(rk, rp, sk, sp), config=gsh.make_config(**cfg))
    assert (r.count, r.checksum) == (on, oc)


@pytest.mark.parametrize("bits", [1, 3, 8])
@pytest.mark.parametrize("kind,n,theta", [("pkfk", (1 << 18) + 7, 0.0), ("zipf", 1 << 17, 1.0),
                                          ("graph", 1 << 16, 0.909), ("uniform", 1000, 0.0)])
def test_join_prepass_exact(kind, n, theta, bits):
    """Pre-partition pass (gsh_config.prepass_bits; auto beyond 2^28 tuples per side): splitting R
    and S by hash bits and joining the sub-problems changes performance only -- COUNT and
    MATERIALIZE equal the oracle's, pairs as a multiset, also with routing bits above it."""
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=29)
    on, oc, op = _oracle(rk, rp, sk, sp, pairs=True)
    d = _dev(rk, rp, sk, sp)
    r = gsh.join(*d, config=gsh.make_config(prepass_bits=bits, timing=True))
    assert (r.count, r.checksum) == (on, oc)
    assert r.stats["prepass_bits"] == bits and r.stats["ms_prepass"] > 0
    m = gsh.join(*d, mode="materialize", out_capacity=on + 3, config=gsh.make_config(prepass_bits=bits))
    assert (m.count, m.checksum, m.written, m.overflow) == (on, oc, on, False)
    assert np.array_equal(_sorted_pairs(m.pairs), op)
    # below routing bits: a shard whose tuples all share the top 2 bits of h (route_bits asserts it)
    u = lambda t: t.numpy().view(np.uint32)  # noqa: E731
    kr = (oracle.fmix32(u(rk)) >> 30) == 2
    ks = (oracle.fmix32(u(sk)) >> 30) == 2
    sh = [t[torch.from_numpy(m_)] for t, m_ in ((rk, kr), (rp, kr), (sk, ks), (sp, ks))]
    on2, oc2, op2 = _oracle(*sh, pairs=True)
    m2 = gsh.join(*_dev(*sh), mode="materialize", out_capacity=on2 + 3,
                  config=gsh.make_config(prepass_bits=bits, route_bits=2))
    assert (m2.count, m2.checksum, m2.written, m2.overflow) == (on2, oc2, on2, False)
    assert np.array_equal(_sorted_pairs(m2.pairs), op2)


@pytest.mark.parametrize("bits", [2, 3])
def test_join_prepass_unaligned_views(bits):
    """The split kernels take 16-byte vector loads only when both input pointers are aligned;
    sliced views take the scalar path and must give the same result."""
    rk, rp, sk, sp = _dev(*datagen.zipf_pair(70_001, 90_003, 1.0, seed=3))
    on, oc, _ = _oracle(rk[1:], rp[1:], sk[3:], sp[2:-1])
    r = gsh.join(rk[1:], rp[1:], sk[3:], sp[2:-1], config=gsh.make_config(prepass_bits=bits))
    assert (r.count, r.checksum) == (on, oc)


def test_join_prepass_overflow_subset():
    rk, rp, sk, sp = datagen.zipf_pair(30_000, 30_000, 1.0, seed=8)
    on, oc, _ = _oracle(rk, rp, sk, sp)
    cap = on // 3
    r = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=cap, config=gsh.make_config(prepass_bits=2))
    assert (r.count, r.checksum, r.written, r.overflow) == (on, oc, cap, True)
    got = _sorted_pairs(r.pairs)
    assert np.all(_np(rk)[got[:, 0]] == _np(sk)[got[:, 1]])
    assert np.unique(got, axis=0).shape[0] == got.shape[0]


def test_join_edge_cases():
    # all keys equal (one giant skewed key), extremes of the key range, no matches, empty sides
    z = torch.zeros
    cases = []
    cases.append((z(3000, dtype=torch.int32), torch.arange(3000, dtype=torch.int32),
                  z(2000, dtype=torch.int32), torch.arange(2000, dtype=torch.int32)))
    cases.append((torch.full((5000,), -1, dtype=torch.int32), torch.arange(5000, dtype=torch.int32),
                  torch.tensor([-1, 0, 5, -1], dtype=torch.int32), torch.arange(4, dtype=torch.int32)))
    cases.append((torch.arange(0, 10000, 2, dtype=torch.int32), torch.arange(5000, dtype=torch.int32),
                  torch.arange(1, 10001, 2, dtype=torch.int32), torch.arange(5000, dtype=torch.int32)))
    cases.append((z(0, dtype=torch.int32), z(0, dtype=torch.int32), torch.arange(10, dtype=torch.int32),
                  torch.arange(10, dtype=torch.int32)))
    cases.append((torch.arange(10, dtype=torch.int32), torch.arange(10, dtype=torch.int32), z(0, dtype=torch.int32),
                  z(0, dtype=torch.int32)))
    # duplicate payloads (pair multiset)
    cases.append((torch.tensor([1, 1, 2, 2], dtype=torch.int32), torch.tensor([7, 7, 7, 7], dtype=torch.int32),
                  torch.tensor([1, 2, 2], dtype=torch.int32), torch.tensor([9, 9, 9], dtype=torch.int32)))
    for rk, rp, sk, sp in cases:
        on, oc, op = _oracle(rk, rp, sk, sp, pairs=True)
        r = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=on + 1)
        assert (r.count, r.checksum, r.written) == (on, oc, on)
        assert np.array_equal(_sorted_pairs(r.pairs), op)


def test_join_unaligned_views():
    """Input pointers need not be 16-byte aligned (sliced views)."""
    rk, rp, sk, sp = datagen.zipf_pair(50_001, 50_003, 1.0, seed=2)
    rk, rp, sk, sp = _dev(rk, rp, sk, sp)
    r = gsh.join(rk[1:], rp[1:], sk[3:], sp[3:])
    on, oc, _ = _oracle(rk[1:], rp[1:], sk[3:], sp[3:])
    assert (r.count, r.checksum) == (on, oc)


def test_join_host_end_to_end():
    rk, rp, sk, sp = datagen.zipf_pair(70_000, 60_000, 1.0, seed=4)
    on, oc, op = _oracle(rk, rp, sk, sp, pairs=True)
    r = gsh.join_host(rk.pin_memory(), rp.pin_memory(), sk.pin_memory(), sp.pin_memory(), mode="materialize",
                      out_capacity=on)
    assert (r.count, r.checksum, r.written) == (on, oc, on)
    assert np.array_equal(_sorted_pairs(r.pairs), op)
    r2 = gsh.join_host(rk, rp, sk, sp)
    assert (r2.count, r2.checksum) == (on, oc)


def test_repeatable_bit_exact():
    rk, rp, sk, sp = _dev(*datagen.zipf_pair(1 << 18, 1 << 18, 1.25, seed=9))
    a = gsh.join(rk, rp, sk, sp)
    b = gsh.join(rk, rp, sk, sp)
    assert (a.count, a.checksum) == (b.count, b.checksum)


@pytest.mark.parametrize("kind,n,theta", [("pkfk", 1 << 19, 0.0), ("uniform", (1 << 20) + 5, 0.0),
                                          ("zipf", 1 << 18, 0.5), ("zipf", 1 << 17, 1.0), ("graph", 1 << 17, 0.909)])
@pytest.mark.parametrize("table", [1, 2])
def test_join_nm_table_modes(kind, n, theta, table):
    """The NM-join's shared-memory table -- bucketized CSR or the chained table of
    (link in the top 16 bits of h, which the 2^16 partition digits fix) -- changes performance
    only: COUNT and MATERIALIZE results equal the oracle's under both, including chains of
    duplicated keys (Zipf, graph)."""
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=17)
    on, oc, op = _oracle(rk, rp, sk, sp, pairs=True)
    d = _dev(rk, rp, sk, sp)
    cfg = gsh.make_config(pass_bits=(8, 8), nm_table=table)
    r = gsh.join(*d, config=cfg)
    assert (r.count, r.checksum) == (on, oc)
    assert r.stats["nm_table"] == table
    m = gsh.join(*d, mode="materialize", out_capacity=on, config=cfg)
    assert (m.count, m.checksum, m.written) == (on, oc, on)
    assert np.array_equal(_sorted_pairs(m.pairs), op)


@pytest.mark.parametrize("theta,n", [(1.0, 1 << 18), (1.5, 1 << 17), (0.75, 1 << 18)])
def test_sampled_detection_properties(theta, n):
    """Paper-literal detection: a 1 % sample of each
    large partition in a linear-probing table, its top-3 keys skewed.  Pins: every chosen key
    lies in a large partition, at most k per partition, its counts in H are the EXACT counts
    (np.unique), and the input's most frequent key -- which dominates its partition's sample --
    is chosen."""
    rk, rp, sk, sp = datagen.zipf_pair(n, n, theta, seed=3)
    h, cr, cs, st = gsh.detect(*_dev(rk, rp, sk, sp), config=gsh.make_config(detect_mode=1))
    B = st["pass_bits"][0] + st["pass_bits"][1]
    L = st["large_threshold"]
    rkn, skn = _np(rk), _np(sk)
    szr = np.bincount(oracle.radix_digits(rkn, 0, B), minlength=1 << B)
    szs = np.bincount(oracle.radix_digits(skn, 0, B), minlength=1 << B)
    large = ((szr > L) | (szs > L)) & (szr > 0) & (szs > 0)
    hh = h.numpy().astype(np.uint32)
    assert len(hh) > 0
    parts = (hh.astype(np.int64) >> (32 - B)) if B else np.zeros(len(hh), np.int64)
    assert large[parts].all()
    assert np.bincount(parts).max() <= 3
    for side_h, got in ((oracle.fmix32(rkn), cr.numpy()), (oracle.fmix32(skn), cs.numpy())):
        u, c = np.unique(side_h, return_counts=True)
        idx = np.searchsorted(u, hh)
        exact = np.where((idx < len(u)) & (u[np.minimum(idx, len(u) - 1)] == hh), c[np.minimum(idx, len(u) - 1)], 0)
        assert np.array_equal(got, exact)
    u, c = np.unique(oracle.fmix32(rkn), return_counts=True)
    assert u[c.argmax()] in set(hh.tolist())


@pytest.mark.parametrize("kind,n,theta,nmat", [("zipf", 1 << 18, 1.0, 40_000), ("zipf", 1 << 17, 1.5, 20_000),
                                               ("zipf", 1 << 18, 0.75, 1 << 16), ("graph", 1 << 17, 0.909, 1 << 16)])
def test_join_sampled_detection_exact(kind, n, theta, nmat):
    """Which keys are treated as skewed changes performance only: with the sampled top-k
    detection (normal remainders larger than C take the chunked NM-join) the join equals the
    oracle bit-exactly: COUNT at n, MATERIALIZE at nmat (output size ~ n^2 sum p_k^2)."""
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=23)
    on, oc, _ = _oracle(rk, rp, sk, sp)
    cfg = gsh.make_config(detect_mode=1)
    r = gsh.join(*_dev(rk, rp, sk, sp), config=cfg)
    assert (r.count, r.checksum) == (on, oc)
    assert r.stats["n_heavy"] > 0
    rk, rp, sk, sp = datagen.make_workload(kind, nmat, theta, seed=23)
    on, oc, op = _oracle(rk, rp, sk, sp, pairs=True)
    d = _dev(rk, rp, sk, sp)
    m = gsh.join(*d, mode="materialize", out_capacity=on, config=cfg)
    assert (m.count, m.checksum, m.written) == (on, oc, on)
    assert np.array_equal(_sorted_pairs(m.pairs), op)

