"""Pins for the CPU oracle (oracle/): each oracle function checked against something
other than itself -- published hash vectors, inverses, brute force, closed forms,
invariants, and the SURVEY §8(c) independent golden cases.  CPU only."""
import json
import os

import numpy as np
import pytest

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "survey_tiny_cases.json")
M64 = (1 << 64) - 1
M32 = (1 << 32) - 1


# ----------------------------------------------------------------------- fmix32 pins
def _rotl32(x, r):
    return ((x << r) | (x >> (32 - r))) & M32


def murmur3_x86_32(data: bytes, seed: int) -> int:
    """Full MurmurHash3_x86_32 (Appleby); the finalizer is the oracle's fmix32."""
    c1, c2 = 0xCC9E2D51, 0x1B873593
    h = seed & M32
    n = len(data)
    nblocks = n // 4
    for i in range(nblocks):
        k = int.from_bytes(data[4 * i: 4 * i + 4], "little")
        k = (k * c1) & M32
        k = _rotl32(k, 15)
        k = (k * c2) & M32
        h ^= k
        h = _rotl32(h, 13)
        h = (h * 5 + 0xE6546B64) & M32
    tail = data[4 * nblocks:]
    k = 0
    if len(tail) >= 3:
        k ^= tail[2] << 16
    if len(tail) >= 2:
        k ^= tail[1] << 8
    if len(tail) >= 1:
        k ^= tail[0]
        k = (k * c1) & M32
        k = _rotl32(k, 15)
        k = (k * c2) & M32
        h ^= k
    h ^= n
    return int(oracle.fmix32(np.array([h], dtype=np.uint32))[0])


# Published SMHasher / reference test vectors for MurmurHash3_x86_32.
SMHASHER_X86_32 = [
    (b"", 0, 0x00000000),
    (b"", 1, 0x514E28B7),
    (b"", 0xFFFFFFFF, 0x81F16F39),
    (b"\xff\xff\xff\xff", 0, 0x76293B50),
    (b"\x21\x43\x65\x87", 0, 0xF55B516B),
    (b"\x21\x43\x65\x87", 0x5082EDEE, 0x2362F9DE),
    (b"\x21\x43\x65", 0, 0x7E4A8634),
    (b"\x21\x43", 0, 0xA0F7B07A),
    (b"\x21", 0, 0x72661CF4),
    (b"\x00\x00\x00\x00", 0, 0x2362F9DE),
    (b"\x00\x00\x00", 0, 0x85F0B427),
    (b"\x00\x00", 0, 0x30F4C306),
    (b"\x00", 0, 0x514E28B7),
    (b"Hello, world!", 0x9747B28C, 0x24884CBA),
    (b"aaaa", 0x9747B28C, 0x5A97808A),
    (b"The quick brown fox jumps over the lazy dog", 0x9747B28C, 0x2FA826CD),
]


@pytest.mark.parametrize("data,seed,expect", SMHASHER_X86_32)
def test_fmix32_smhasher_vectors(data, seed, expect):
    assert murmur3_x86_32(data, seed) == expect


def test_fmix32_c_matches_numpy_and_is_bijective_sample():
    rng = np.random.default_rng(1)
    x = rng.integers(0, 1 << 32, size=1 << 16, dtype=np.uint64).astype(np.uint32)
    x = np.concatenate([x, np.array([0, 1, M32, 0x80000000], dtype=np.uint32)])
    lib = oracle.oracle._load()
    c_out = np.array([lib.oracle_fmix32_scalar(int(v)) for v in x[:512]], dtype=np.uint32)
    assert np.array_equal(c_out, oracle.fmix32(x[:512]))
    # bijection on u32: distinct inputs -> distinct outputs (sample)
    u = np.unique(x)
    assert np.unique(oracle.fmix32(u)).size == u.size


# ----------------------------------------------------------------------- fmix64 pins
def _inv_fmix64(y: int) -> int:
    """Inverse of MurmurHash3 fmix64 built from modular inverses of its multipliers:
    x ^= x >> 33 is an involution (33 >= 32), multiplication by an odd c is inverted by
    pow(c, -1, 2^64)."""
    i1 = pow(0xFF51AFD7ED558CCD, -1, 1 << 64)
    i2 = pow(0xC4CEB9FE1A85EC53, -1, 1 << 64)
    y ^= y >> 33
    y = (y * i2) & M64
    y ^= y >> 33
    y = (y * i1) & M64
    y ^= y >> 33
    return y


def test_fmix64_inverse_roundtrip():
    rng = np.random.default_rng(2)
    xs = rng.integers(0, 1 << 63, size=4096, dtype=np.int64).astype(np.uint64) * np.uint64(2) + np.uint64(1)
    xs = np.concatenate([xs, np.array([0, 1, M64, 1 << 63], dtype=np.uint64)])
    ys = oracle.fmix64(xs)
    for x, y in zip(xs.tolist(), ys.tolist()):
        assert _inv_fmix64(int(y)) == int(x)
    assert int(oracle.fmix64(np.array([0], dtype=np.uint64))[0]) == 0


def _rotl64(x, r):
    return ((x << r) | (x >> (64 - r))) & M64


def murmur3_x64_128(data: bytes, seed: int):
    """Full MurmurHash3_x64_128; finalizer = oracle.fmix64."""
    c1, c2 = 0x87C37B91114253D5, 0x4CF5AD432745937F
    h1 = h2 = seed & M64
    n = len(data)
    nblocks = n // 16
    for i in range(nblocks):
        k1 = int.from_bytes(data[16 * i: 16 * i + 8], "little")
        k2 = int.from_bytes(data[16 * i + 8: 16 * i + 16], "little")
        k1 = (k1 * c1) & M64; k1 = _rotl64(k1, 31); k1 = (k1 * c2) & M64; h1 ^= k1
        h1 = _rotl64(h1, 27); h1 = (h1 + h2) & M64; h1 = (h1 * 5 + 0x52DCE729) & M64
        k2 = (k2 * c2) & M64; k2 = _rotl64(k2, 33); k2 = (k2 * c1) & M64; h2 ^= k2
        h2 = _rotl64(h2, 31); h2 = (h2 + h1) & M64; h2 = (h2 * 5 + 0x38495AB5) & M64
    tail = data[16 * nblocks:]
    k1 = k2 = 0
    for i in range(len(tail) - 1, 7, -1):
        k2 ^= tail[i] << (8 * (i - 8))
    if len(tail) > 8:
        k2 = (k2 * c2) & M64; k2 = _rotl64(k2, 33); k2 = (k2 * c1) & M64; h2 ^= k2
    for i in range(min(len(tail), 8) - 1, -1, -1):
        k1 ^= tail[i] << (8 * i)
    if len(tail) > 0:
        k1 = (k1 * c1) & M64; k1 = _rotl64(k1, 31); k1 = (k1 * c2) & M64; h1 ^= k1
    h1 ^= n; h2 ^= n
    h1 = (h1 + h2) & M64; h2 = (h2 + h1) & M64
    f = lambda v: int(oracle.fmix64(np.array([v], dtype=np.uint64))[0])  # noqa: E731
    h1 = f(h1); h2 = f(h2)
    h1 = (h1 + h2) & M64; h2 = (h2 + h1) & M64
    return h1, h2


def test_fmix64_via_murmur3_x64_128_vector():
    # Reference vector: MurmurHash3_x64_128("The quick brown fox jumps over the lazy dog", 0)
    # = 6c1b07bc7bbc4be3 47939ac4a93c437a (little-endian bytes) -> h1, h2 below.
    h1, h2 = murmur3_x64_128(b"The quick brown fox jumps over the lazy dog", 0)
    assert (h1, h2) == (0xE34BBC7BBC071B6C, 0x7A433CA9C49A9347)
    assert murmur3_x64_128(b"", 0) == (0, 0)


# -------------------------------------------------------------------- pair_hash pins
def test_pair_hash_operand_order_and_salt():
    """inverse(pair_hash(a,b)) ^ SALT must give (a << 32 | b): a transposed operand,
    dropped salt or wrong packing fails."""
    rng = np.random.default_rng(3)
    a = rng.integers(0, 1 << 32, size=2000, dtype=np.uint64).astype(np.uint32)
    b = rng.integers(0, 1 << 32, size=2000, dtype=np.uint64).astype(np.uint32)
    h = oracle.pair_hash(a, b)
    for ai, bi, hi in zip(a.tolist(), b.tolist(), h.tolist()):
        assert _inv_fmix64(int(hi)) ^ 0x9E3779B97F4A7C15 == (ai << 32) | bi
    lib = oracle.oracle._load()
    for ai, bi, hi in list(zip(a.tolist(), b.tolist(), h.tolist()))[:200]:
        assert lib.oracle_pair_hash_scalar(ai, bi) == hi
    # non-symmetric
    assert int(oracle.pair_hash([1], [2])[0]) != int(oracle.pair_hash([2], [1])[0])


def test_survey_vectors():
    g = json.load(open(GOLDEN))
    for k, v in g["fmix32"].items():
        assert int(oracle.fmix32(np.array([int(k)], dtype=np.uint32))[0]) == int(v, 16)
    for a, b, v in g["pair_hash"]:
        assert int(oracle.pair_hash([a], [b])[0]) == int(v, 16)


# ------------------------------------------------------------------------- join pins
def brute_join(rk, rp, sk, sp):
    """Nested-loop definition of M (count, checksum, sorted pairs) -- numpy broadcast."""
    rk = np.asarray(rk, dtype=np.uint32); sk = np.asarray(sk, dtype=np.uint32)
    rp = np.asarray(rp, dtype=np.uint32); sp = np.asarray(sp, dtype=np.uint32)
    eq = rk[:, None] == sk[None, :]
    i, j = np.nonzero(eq)
    a, b = rp[i], sp[j]
    chk = 0
    if a.size:
        chk = int(np.sum(oracle.pair_hash(a, b), dtype=np.uint64))
    pairs = np.stack([a, b], axis=1) if a.size else np.zeros((0, 2), dtype=np.uint32)
    order = np.lexsort((pairs[:, 1], pairs[:, 0])) if a.size else np.zeros(0, dtype=np.int64)
    return int(a.size), chk, pairs[order]


def _rand_rel(rng, n, domain, special=True):
    k = rng.integers(0, domain, size=n, dtype=np.uint64).astype(np.uint32)
    if special and n >= 4:
        k[rng.integers(0, n)] = 0
        k[rng.integers(0, n)] = M32
    p = rng.integers(0, 1 << 32, size=n, dtype=np.uint64).astype(np.uint32)
    return k, p


@pytest.mark.parametrize("nr,ns,domain", [(0, 0, 5), (0, 10, 5), (10, 0, 5), (1, 1, 1), (17, 33, 3),
                                          (300, 200, 50), (1000, 1500, 10), (999, 1001, 997),
                                          (512, 4096, 1 << 32)])
def test_join_matches_brute_force(nr, ns, domain):
    rng = np.random.default_rng(nr * 7 + ns)
    rk, rp = _rand_rel(rng, nr, domain)
    sk, sp = _rand_rel(rng, ns, domain)
    # map the small domain onto spread u32 keys, keep 0 / 0xFFFFFFFF specials
    n, chk, pairs = oracle.join_sorted_pairs(rk, rp, sk, sp)
    bn, bchk, bpairs = brute_join(rk, rp, sk, sp)
    assert (n, chk) == (bn, bchk)
    assert np.array_equal(pairs, bpairs)
    for t in (1, 3, 8):
        assert oracle.join(rk, rp, sk, sp, nthreads=t)[:2] == (bn, bchk)


def test_join_golden_survey_cases():
    g = json.load(open(GOLDEN))
    t = g["tiny"]
    R = np.array(t["R"], dtype=np.uint64).astype(np.uint32)
    S = np.array(t["S"], dtype=np.uint64).astype(np.uint32)
    n, chk, pairs = oracle.join_sorted_pairs(R[:, 0], R[:, 1], S[:, 0], S[:, 1])
    assert n == t["count"] and chk == int(t["checksum"], 16)
    assert pairs.tolist() == t["pairs"]
    a = g["all_equal"]
    n, chk, _ = oracle.join(np.full(a["nR"], a["key"], np.uint32), np.arange(a["nR"], dtype=np.uint32),
                            np.full(a["nS"], a["key"], np.uint32), np.arange(a["nS"], dtype=np.uint32))
    assert n == a["count"] and chk == int(a["checksum"], 16)
    # the cross product's checksum, enumerated explicitly in Python
    s = 0
    for i in range(a["nR"]):
        s += int(np.sum(oracle.pair_hash(np.full(a["nS"], i, np.uint32), np.arange(a["nS"], dtype=np.uint32)),
                        dtype=np.uint64))
    assert s & M64 == chk


def closed_form_count(rk, sk):
    """count = sum_k cnt_R(k) * cnt_S(k) from exact histograms (np.unique)."""
    ur, cr = np.unique(np.asarray(rk, dtype=np.uint32), return_counts=True)
    us, cs = np.unique(np.asarray(sk, dtype=np.uint32), return_counts=True)
    common, ir, is_ = np.intersect1d(ur, us, assume_unique=True, return_indices=True)
    return int(np.sum(cr[ir].astype(np.int64) * cs[is_].astype(np.int64)))


@pytest.mark.parametrize("theta", [0.0, 0.5, 1.0, 1.5])
def test_join_count_closed_form_zipf(theta):
    import datagen
    rk, rp, sk, sp = datagen.zipf_pair(1 << 15, 1 << 15, theta, seed=11)
    n, chk, _ = oracle.join(rk.numpy(), rp.numpy(), sk.numpy(), sp.numpy())
    assert n == closed_form_count(rk.numpy().view(np.uint32), sk.numpy().view(np.uint32))


def test_join_pkfk_count_and_checksum_closed_form():
    """PK-FK: each S row j matches exactly the R row whose key it copied, so
    M = {(rowR(j), j)} and checksum = sum_j pair_hash(rowR(j), j)."""
    import datagen
    rk, rp, sk, sp = datagen.pkfk_pair(1 << 14, 3 * (1 << 13) + 5, seed=5)
    rku = rk.numpy().view(np.uint32); sku = sk.numpy().view(np.uint32)
    pos = {int(k): i for i, k in enumerate(rku.tolist())}
    rowr = np.array([pos[int(k)] for k in sku.tolist()], dtype=np.uint32)
    expect = int(np.sum(oracle.pair_hash(rowr, np.arange(sku.size, dtype=np.uint32)), dtype=np.uint64))
    n, chk, _ = oracle.join(rku, rp.numpy(), sku, sp.numpy())
    assert n == sku.size and chk == expect


def test_join_metamorphic_invariances():
    rng = np.random.default_rng(9)
    rk, rp = _rand_rel(rng, 5000, 300)
    sk, sp = _rand_rel(rng, 7000, 300)
    base = oracle.join(rk, rp, sk, sp)[:2]
    # row permutation of R and of S (payload travels with its key)
    pr = rng.permutation(rk.size); ps = rng.permutation(sk.size)
    assert oracle.join(rk[pr], rp[pr], sk[ps], sp[ps])[:2] == base
    # additivity over R chunks (count and checksum add mod 2^64)
    c0 = oracle.join(rk[:1234], rp[:1234], sk, sp)[:2]
    c1 = oracle.join(rk[1234:], rp[1234:], sk, sp)[:2]
    assert ((c0[0] + c1[0]), (c0[1] + c1[1]) & M64) == base
    # R <-> S swap: same count, pairs swapped
    n1, _, p1 = oracle.join_sorted_pairs(rk, rp, sk, sp)
    n2, _, p2 = oracle.join_sorted_pairs(sk, sp, rk, rp)
    assert n1 == n2
    sw = p2[:, ::-1]
    sw = sw[np.lexsort((sw[:, 1], sw[:, 0]))]
    assert np.array_equal(sw, p1)


# ------------------------------------------------------------- step-reference pins
def test_radix_histogram_loop_and_composition():
    rng = np.random.default_rng(4)
    k = rng.integers(0, 1 << 32, size=3000, dtype=np.uint64).astype(np.uint32)
    h = oracle.fmix32(k)
    for hi, nb in [(0, 0), (0, 3), (0, 8), (2, 5), (8, 8)]:
        hist = oracle.radix_histogram(k, hi, nb)
        assert hist.size == 1 << nb and int(hist.sum()) == k.size
        loop = [0] * (1 << nb)
        for hv in h.tolist():
            bits = format(hv, "032b")[hi: hi + nb]  # MSB-first bit string
            loop[int(bits, 2) if nb else 0] += 1
        assert hist.tolist() == loop
    # pass composition: (d1 << b2) | d2 == digit over b1 + b2 bits
    d1 = oracle.radix_digits(k, 0, 7); d2 = oracle.radix_digits(k, 7, 6)
    assert np.array_equal((d1 << 6) | d2, oracle.radix_digits(k, 0, 13))


def test_heavy_rule_bruteforce():
    rng = np.random.default_rng(12)
    for trial in range(6):
        # skewed small relations
        rk = np.concatenate([rng.integers(0, 40, 300), np.full(rng.integers(0, 200), 7),
                             np.full(50, 3)]).astype(np.uint32)
        sk = np.concatenate([rng.integers(0, 40, 260), np.full(rng.integers(0, 90), 7),
                             np.full(rng.integers(0, 120), 11)]).astype(np.uint32)
        pb, cap, thr = 3, 40 + trial, 20
        hk, cr, cs = oracle.heavy_rule(rk, sk, pb, cap, thr)
        # dictionary brute force
        part = lambda key: int(oracle.fmix32(np.array([key], np.uint32))[0]) >> (32 - pb)  # noqa: E731
        szr = {}; szs = {}; cntr = {}; cnts = {}
        for x in rk.tolist():
            szr[part(x)] = szr.get(part(x), 0) + 1; cntr[x] = cntr.get(x, 0) + 1
        for x in sk.tolist():
            szs[part(x)] = szs.get(part(x), 0) + 1; cnts[x] = cnts.get(x, 0) + 1
        expect = []
        for x in set(cntr) | set(cnts):
            p = part(x)
            if (szr.get(p, 0) > cap or szs.get(p, 0) > cap) and szr.get(p, 0) > 0 and szs.get(p, 0) > 0:
                if max(cntr.get(x, 0), cnts.get(x, 0)) >= thr:
                    h = int(oracle.fmix32(np.array([x], np.uint32))[0])
                    expect.append((h, cntr.get(x, 0), cnts.get(x, 0)))
        expect.sort()
        got = list(zip(hk.tolist(), cr.tolist(), cs.tolist()))
        assert got == expect


def test_heavy_rule_empty_side_partition():
    """DESIGN.md R5: a partition holding many R tuples but no S tuple is not large (it yields no
    result tuple), so its keys are never skewed; the same key with one matching S tuple is."""
    pb = 4
    part = lambda a: (oracle.fmix32(np.asarray(a, np.uint32)) >> np.uint32(32 - pb)).astype(np.int64)  # noqa: E731
    cand = np.arange(1, 5000, dtype=np.uint32)
    pc = part(cand)
    k_big = int(cand[0])
    others = cand[pc != pc[0]][:200]          # S keys from other partitions only
    rk = np.concatenate([np.full(500, k_big), others]).astype(np.uint32)
    sk = others.copy()
    hk, _, _ = oracle.heavy_rule(rk, sk, pb, 100, 50)
    assert k_big not in set(oracle.fmix32(np.asarray(hk, np.uint32)).tolist()) and hk.size == 0
    sk2 = np.concatenate([sk, [k_big]]).astype(np.uint32)   # one S tuple: the partition becomes large
    hk2, cr2, cs2 = oracle.heavy_rule(rk, sk2, pb, 100, 50)
    h_big = int(oracle.fmix32(np.array([k_big], np.uint32))[0])
    assert hk2.tolist() == [h_big] and cr2.tolist() == [500] and cs2.tolist() == [1]
