"""Counter-based, device-independent generators (see datagen/__init__.py for the recipe).

All arithmetic is int64 torch ops with explicit masking, so the CPU and CUDA outputs are
bit-identical for the same (seed, stream, index).
"""
from __future__ import annotations

import numpy as np
import torch

_M32 = (1 << 32) - 1


def _c64(v: int) -> int:
    """Reinterpret an unsigned 64-bit constant as a signed int64 python int."""
    return v - (1 << 64) if v >= (1 << 63) else v


_GOLD = _c64(0x9E3779B97F4A7C15)
_SM1 = _c64(0xBF58476D1CE4E5B9)
_SM2 = _c64(0x94D049BB133111EB)


def _srl(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of an int64 tensor viewed as u64."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """splitmix64 output function (Steele, Lea, Flood 2014) on int64 tensors (wrapping)."""
    z = x + _GOLD
    z = (z ^ _srl(z, 30)) * _SM1
    z = (z ^ _srl(z, 27)) * _SM2
    return z ^ _srl(z, 31)


def _stream_base(seed: int, stream: int) -> int:
    t = torch.tensor([_c64(((seed & ((1 << 64) - 1)) * 0x100000001B3 ^ (stream * 0x51ED27)) & ((1 << 64) - 1))],
                     dtype=torch.int64)
    return int(splitmix64(t).item())


def rand_u63(seed: int, stream: int, n: int, device="cpu", offset: int = 0) -> torch.Tensor:
    """n uniform 63-bit integers (int64, >= 0) from counter (seed, stream, offset + i)."""
    base = _stream_base(seed, stream)
    idx = torch.arange(offset, offset + n, dtype=torch.int64, device=device)
    return _srl(splitmix64(idx + base), 1)


def _to_i32(x: torch.Tensor) -> torch.Tensor:
    """int64 values in [0, 2^32) -> int32 tensor with the same 32-bit pattern."""
    return (x - ((x >> 31) & 1) * (1 << 32)).to(torch.int32)


def rank_to_key(rank: torch.Tensor, seed: int) -> torch.Tensor:
    """Seeded bijection rank -> u32 key ("randomly assign a unique key to each interval",
    PAPER.md L132).  (x + s) mod 2^32 followed by the lowbias32 permutation
    (xorshift-multiply, both steps invertible on u32).  Returns int64 in [0, 2^32)."""
    s = _stream_base(seed, 2) & _M32
    x = (rank.to(torch.int64) + s) & _M32
    x = x ^ (x >> 16)
    x = (x * 0x7FEB352D) & _M32
    x = x ^ (x >> 15)
    x = (x * 0x846CA68B) & _M32
    x = x ^ (x >> 16)
    return x


def zipf_thresholds(N: int, theta: float) -> np.ndarray:
    """Cut points of the Zipf 'interval array' as 63-bit fixed point.

    Returns int64 array T of length N-1 with T[k] = floor(CDF(k+1) * 2^63), CDF over ranks
    1..N with p_k ∝ k^-theta.  A sample u in [0, 2^63) maps to rank index
    searchsorted(T, u, right) in [0, N).  theta = 0 is exact integer arithmetic; theta > 0
    sums k^-theta in float64 blocks of 1024 with an extended-precision block prefix.
    """
    if N < 1:
        raise ValueError("N must be >= 1")
    if N == 1:
        return np.zeros(0, dtype=np.int64)
    if theta == 0.0:
        q, r = divmod(1 << 63, N)
        k1 = np.arange(1, N, dtype=np.uint64)
        t = k1 * np.uint64(q) + (k1 * np.uint64(r)) // np.uint64(N)
        return t.astype(np.int64)
    B = 1024
    nb = (N + B - 1) // B
    k = np.arange(1, nb * B + 1, dtype=np.float64)
    w = np.power(k, -float(theta))
    w[N:] = 0.0
    w = w.reshape(nb, B)
    inblock = np.cumsum(w, axis=1)
    bsum = inblock[:, -1].astype(np.longdouble)
    bprefix = np.concatenate([[np.longdouble(0)], np.cumsum(bsum)[:-1]])
    total = np.sum(bsum)
    cdf = (bprefix[:, None] + inblock.astype(np.longdouble)).reshape(-1)[: N - 1] / total
    t = np.floor(cdf * np.longdouble(2.0) ** 63)
    t = np.minimum(t, np.longdouble(2.0) ** 63 - 1)
    return t.astype(np.int64)


def zipf_keys(n: int, T: torch.Tensor, key_seed: int, seed: int, stream: int, device="cpu") -> torch.Tensor:
    """n Zipf keys: search a uniform 63-bit draw in the interval array,
    map the rank to its unique key.  Returns int32 (u32 bit pattern)."""
    u = rand_u63(seed, stream, n, device)
    if T.numel() == 0:
        rank = torch.zeros(n, dtype=torch.int64, device=device)
    else:
        rank = torch.searchsorted(T.to(device), u, right=True)
    return _to_i32(rank_to_key(rank, key_seed))


def _payloads(n: int, device) -> torch.Tensor:
    return torch.arange(n, dtype=torch.int64, device=device).to(torch.int32)


def zipf_relation(n: int, theta: float, N: int | None = None, seed: int = 0, stream: int = 0,
                  device="cpu", T: torch.Tensor | None = None):
    N = n if N is None else N
    if T is None:
        T = torch.from_numpy(zipf_thresholds(max(N, 1), theta))
    return zipf_keys(n, T, seed, seed, stream, device), _payloads(n, device)


def zipf_pair(n_r: int, n_s: int, theta: float, N: int | None = None, seed: int = 0, device="cpu"):
    """Both-sides-skewed Zipf workload: R and S share the interval array and key map
    (PAPER.md L139), independent streams R = 0, S = 1.  Domain N = max(n_r, n_s) default."""
    N = max(n_r, n_s, 1) if N is None else N
    T = torch.from_numpy(zipf_thresholds(N, theta)).to(device)
    rk = zipf_keys(n_r, T, seed, seed, 0, device)
    sk = zipf_keys(n_s, T, seed, seed, 1, device)
    return rk, _payloads(n_r, device), sk, _payloads(n_s, device)


def uniform_pair(n_r: int, n_s: int, seed: int = 0, device="cpu"):
    """theta = 0: uniform with replacement over N = max(n_r, n_s) keys."""
    return zipf_pair(n_r, n_s, 0.0, None, seed, device)


def pkfk_pair(n_r: int, n_s: int, seed: int = 0, device="cpu"):
    """1:1 PK-FK (SURVEY reading #6): R = n_r distinct keys in random order, each S key is
    R.key[uniform row], so count == n_s exactly."""
    rk64 = rank_to_key(torch.arange(n_r, dtype=torch.int64, device=device), seed)
    if n_r == 0:
        sk64 = torch.zeros(0, dtype=torch.int64, device=device)
        n_s = 0
    else:
        idx = rand_u63(seed, 1, n_s, device) % n_r
        sk64 = rk64[idx]
    return _to_i32(rk64), _payloads(n_r, device), _to_i32(sk64), _payloads(n_s, device)


def pkfk_zipf_pair(n_r: int, n_s: int, theta: float, seed: int = 0, device="cpu"):
    """Skewed-FK PK-FK: R = n_r distinct keys (row r holds key map(r)); each S row references R row
    rank ~ Zipf(theta) over the n_r rows (the interval array of PAPER.md L139), so R is unique and
    S is skewed: count == n_s exactly, cnt_R = 1 for every key."""
    T = torch.from_numpy(zipf_thresholds(max(n_r, 1), theta)).to(device)
    rk = _to_i32(rank_to_key(torch.arange(n_r, dtype=torch.int64, device=device), seed))
    sk = zipf_keys(n_s, T, seed, seed, 1, device) if n_r else torch.zeros(0, dtype=torch.int32, device=device)
    return rk, _payloads(n_r, device), sk, _payloads(sk.numel(), device)


def graph_pair(n_edges: int, n_vertices: int, theta: float = 1.0 / (2.1 - 1.0), seed: int = 0,
               device="cpu"):
    """Power-law graph edge self-join (SURVEY reading #18; PAPER.md L13 motivation).
    Vertex ranks ~ Zipf(theta = 1/(gamma-1)) over V vertices; src and dst iid from the same
    rank -> vertex map.  R = (dst, eid), S = (src, eid): the join enumerates 2-hop paths."""
    T = torch.from_numpy(zipf_thresholds(max(n_vertices, 1), theta)).to(device)
    src = zipf_keys(n_edges, T, seed, seed, 0, device)
    dst = zipf_keys(n_edges, T, seed, seed, 1, device)
    eid = _payloads(n_edges, device)
    return dst, eid, src, eid.clone()


def make_workload(kind: str, n: int, theta: float = 0.0, seed: int = 0, device="cpu", n_s: int | None = None):
    """Convenience dispatcher used by tests / bench: kind in {zipf, uniform, pkfk, pkfk_zipf, graph}."""
    n_s = n if n_s is None else n_s
    if kind == "zipf":
        return zipf_pair(n, n_s, theta, None, seed, device)
    if kind == "uniform":
        return uniform_pair(n, n_s, seed, device)
    if kind == "pkfk":
        return pkfk_pair(n, n_s, seed, device)
    if kind == "pkfk_zipf":
        return pkfk_zipf_pair(n, n_s, theta, seed, device)
    if kind == "graph":
        v = max(1, n // 16)
        return graph_pair(n, v, theta if theta else 1.0 / 1.1, seed, device)
    raise ValueError(kind)
