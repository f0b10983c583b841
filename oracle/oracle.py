"""Oracle functions (TEST INFRASTRUCTURE ONLY -- see oracle/__init__.py).

numpy step references + a ctypes front end for the plain C join in join_oracle.c.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "join_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

# pair_hash salt; removes the fixed point pair_hash(0,0) = fmix64(0) = 0.
SALT = np.uint64(0x9E3779B97F4A7C15)

_M32 = np.uint32(0xFFFFFFFF)


def lib_path() -> str:
    return _LIB


def build(force: bool = False) -> str:
    """Compile join_oracle.c with gcc (plain C, -O2, pthreads)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-pthread", _SRC, "-o", _LIB]
        )
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        u64 = ctypes.c_uint64
        p32 = ctypes.POINTER(ctypes.c_uint32)
        p64 = ctypes.POINTER(ctypes.c_uint64)
        lib.oracle_join.argtypes = [p32, p32, u64, p32, p32, u64, ctypes.c_int, p64, p64, p32, u64]
        lib.oracle_join.restype = ctypes.c_int
        lib.oracle_fmix32_scalar.argtypes = [ctypes.c_uint32]
        lib.oracle_fmix32_scalar.restype = ctypes.c_uint32
        lib.oracle_fmix64_scalar.argtypes = [u64]
        lib.oracle_fmix64_scalar.restype = u64
        lib.oracle_pair_hash_scalar.argtypes = [ctypes.c_uint32, ctypes.c_uint32]
        lib.oracle_pair_hash_scalar.restype = u64
        lib.oracle_fmix32_array.argtypes = [p32, p32, u64]
        lib.oracle_pair_hash_array.argtypes = [p32, p32, p64, u64]
        _lib = lib
    return _lib


def _u32(a) -> np.ndarray:
    a = np.asarray(a)
    if a.dtype == np.int32:
        a = a.view(np.uint32)
    return np.ascontiguousarray(a, dtype=np.uint32)


def _p32(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


# --------------------------------------------------------------------------- hashes
def fmix32(x) -> np.ndarray:
    """MurmurHash3 32-bit finalizer (SURVEY.md §8 notation h = fmix32(key); reading #7:
    partition digits are taken from h, most significant first).  numpy uint32, wraps."""
    h = _u32(x).copy()
    h ^= h >> np.uint32(16)
    h *= np.uint32(0x85EBCA6B)
    h ^= h >> np.uint32(13)
    h *= np.uint32(0xC2B2AE35)
    h ^= h >> np.uint32(16)
    return h


def fmix64(x) -> np.ndarray:
    """MurmurHash3 64-bit finalizer."""
    k = np.ascontiguousarray(x, dtype=np.uint64).copy()
    k ^= k >> np.uint64(33)
    k *= np.uint64(0xFF51AFD7ED558CCD)
    k ^= k >> np.uint64(33)
    k *= np.uint64(0xC4CEB9FE1A85EC53)
    k ^= k >> np.uint64(33)
    return k


def pair_hash(a, b) -> np.ndarray:
    """SURVEY.md §8(c) reading #2: pair_hash(a,b) = fmix64(((u64)a << 32 | b) ^ SALT).
    a = payload_R, b = payload_S (reading #1: a result tuple is (payload_R, payload_S))."""
    a64 = _u32(a).astype(np.uint64)
    b64 = _u32(b).astype(np.uint64)
    with np.errstate(over="ignore"):
        return fmix64(((a64 << np.uint64(32)) | b64) ^ SALT)


# ----------------------------------------------------------------------------- join
def join(rk, rp, sk, sp, materialize: bool = False, nthreads: int | None = None,
         pairs_cap: int | None = None):
    """The equi-join by definition (§III, §IV-B):
    M = {(payload_R[i], payload_S[j]) : key_R[i] == key_S[j]}.

    Returns (count, checksum, pairs) where pairs is an (count, 2) uint32 array in the
    C oracle's chunk order (or None when materialize is False).
    """
    lib = _load()
    rk, rp, sk, sp = _u32(rk), _u32(rp), _u32(sk), _u32(sp)
    assert rk.shape == rp.shape and sk.shape == sp.shape
    nr, ns = rk.size, sk.size
    if nthreads is None:
        nthreads = max(1, os.cpu_count() or 1)
    cnt = ctypes.c_uint64(0)
    chk = ctypes.c_uint64(0)
    if not materialize:
        rc = lib.oracle_join(_p32(rk), _p32(rp), nr, _p32(sk), _p32(sp), ns, nthreads,
                             ctypes.byref(cnt), ctypes.byref(chk), None, 0)
        if rc != 0:
            raise MemoryError("oracle_join failed")
        return int(cnt.value), int(chk.value), None
    # materialise: count first so the pair buffer is exact
    rc = lib.oracle_join(_p32(rk), _p32(rp), nr, _p32(sk), _p32(sp), ns, nthreads,
                         ctypes.byref(cnt), ctypes.byref(chk), None, 0)
    if rc != 0:
        raise MemoryError("oracle_join failed")
    n = int(cnt.value)
    if pairs_cap is not None and n > pairs_cap:
        raise ValueError(f"join produces {n} pairs > pairs_cap {pairs_cap}")
    pairs = np.empty((max(n, 1), 2), dtype=np.uint32)
    rc = lib.oracle_join(_p32(rk), _p32(rp), nr, _p32(sk), _p32(sp), ns, nthreads,
                         ctypes.byref(cnt), ctypes.byref(chk), _p32(pairs), n)
    if rc != 0:
        raise MemoryError("oracle_join failed")
    return n, int(chk.value), pairs[:n]


def join_sorted_pairs(rk, rp, sk, sp):
    """Join result M as a lexicographically sorted (count, 2) array (SURVEY §8(c):
    'pairs = M sorted lexicographically')."""
    n, chk, pairs = join(rk, rp, sk, sp, materialize=True)
    order = np.lexsort((pairs[:, 1], pairs[:, 0]))
    return n, chk, pairs[order]


# ------------------------------------------------------------------ step references
def radix_digits(keys, hi_bits: int, nbits: int) -> np.ndarray:
    """Radix digit of each key for a partition pass (§IV-B(1) L106 'partitions
    input tables into shared memory sized partitions ... two passes'; SURVEY reading #7:
    digits of h = fmix32(key), most significant first).  The digit is bits
    [32 - hi_bits - nbits, 32 - hi_bits) of h, where hi_bits are the bits consumed by
    earlier levels (multi-GPU route bits, then pass 1)."""
    h = fmix32(keys)
    if nbits == 0:
        return np.zeros(h.shape, dtype=np.int64)
    shift = 32 - hi_bits - nbits
    return ((h >> np.uint32(shift)) & np.uint32((1 << nbits) - 1)).astype(np.int64)


def radix_histogram(keys, hi_bits: int, nbits: int) -> np.ndarray:
    """'count' step of count-then-partition (§IV-B(1)): number of tuples
    per partition digit.  Returns int64 array of 2**nbits counts."""
    d = radix_digits(keys, hi_bits, nbits)
    return np.bincount(d, minlength=1 << nbits).astype(np.int64)


def heavy_rule(rk, sk, part_bits: int, large_threshold: int, threshold: int, route_bits: int = 0):
    """Skew detection after partitioning (§IV-B(2)), with the
    readings of DESIGN.md §3 (exact counts replace the 1 % sample, north star):

      partition p = top `part_bits` bits of h below `route_bits` (final partitions);
      large(p)  <=>  (|R_p| > L  or  |S_p| > L)  and  |R_p| > 0  and  |S_p| > 0
                     L = large_threshold   (L107 threshold; R5: a partition with an
                     empty side produces no result tuple, so it is never treated as large)
      heavy(k)  <=>  k lies in a large partition and
                     max(cnt_R(k), cnt_S(k)) >= threshold            (L112 'top-k')

    Returns (h, cnt_R, cnt_S) uint32/int64 arrays of heavy keys sorted by h, where
    h = fmix32(key) identifies the key (fmix32 is a bijection).
    """
    hr = fmix32(rk)
    hs = fmix32(sk)
    pr = radix_digits(rk, route_bits, part_bits)
    ps = radix_digits(sk, route_bits, part_bits)
    nparts = 1 << part_bits
    szr = np.bincount(pr, minlength=nparts)
    szs = np.bincount(ps, minlength=nparts)
    large = ((szr > large_threshold) | (szs > large_threshold)) & (szr > 0) & (szs > 0)
    ur, cr = np.unique(hr[large[pr]], return_counts=True)
    us, cs = np.unique(hs[large[ps]], return_counts=True)
    allk = np.union1d(ur, us).astype(np.uint32)
    cnt_r = np.zeros(allk.size, dtype=np.int64)
    cnt_s = np.zeros(allk.size, dtype=np.int64)
    cnt_r[np.searchsorted(allk, ur)] = cr
    cnt_s[np.searchsorted(allk, us)] = cs
    sel = np.maximum(cnt_r, cnt_s) >= threshold
    return allk[sel], cnt_r[sel], cnt_s[sel]
