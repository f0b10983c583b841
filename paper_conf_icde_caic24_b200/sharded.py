"""Multi-GPU GSH: hash sharding over one node with torch.distributed (NCCL over NVLink/NVSwitch).

SURVEY.md §8(e) / row a11 (a north-star addition; the paper runs on one A100):

  1. positional shards: rank g holds rows of R and S (any split);
  2. skew agreement: global partition histogram (all_reduce) -> globally large partitions
     (the single-GPU rule of PAPER.md L107 on global sizes); each rank proposes the keys of
     large partitions whose LOCAL count reaches ceil(T_h / G) (pigeonhole: any key with global
     count >= T_h reaches it on some rank); all_gather + sorted union; exact local counts of the
     union, all_reduce -> the global skewed set H = {k : max(cnt_R, cnt_S) >= T_h}, identical on
     every rank and equal to the single-GPU rule on the whole input;
  3. normal tuples: routed to rank top_log2(G)_bits(fmix32(key)) with all_to_all_single (split
     sizes exchanged first);
  4. skewed keys: S_k stays local, R_k is broadcast to every rank, so no GPU receives a skewed
     key's full S (only |R_k| x |S_k,local| work per rank);
  5. local GSH join of (received normal R + all skewed R) x (received normal S + local skewed S);
  6. all_reduce(sum) of (count, checksum) mod 2^64 == the single-GPU result bit-exactly.

Every data-path step is a libgsh.so kernel (route_count / route_scatter / count_keys /
local_candidates / gsh_join); torch.distributed only moves bytes.  The `ops` hook exists so the
host-side protocol can be exercised on CPU with gloo and a test double (tests/ only).
"""
from __future__ import annotations

import ctypes
import math

import torch
import torch.distributed as dist

from . import _lib
from .join import _check_dev, _rel, _stream_handle, join, make_config
from ._lib import check, load

M64 = (1 << 64) - 1


def _cfg_params(n_global: int, config) -> tuple[int, int, int]:
    """(B, L, T_h) exactly as plan_build() derives them (api.cu) for n = max side size:
    radix bits, large-partition threshold, skewed-key threshold."""
    if config is not None and config.pass_bits[0] >= 0 and config.pass_bits[1] >= 0:
        B = int(config.pass_bits[0]) + int(config.pass_bits[1])
    else:
        B = 0
        while B < 16 and (n_global >> B) > 2048:
            B += 1
    F = 1 << B
    if config is not None and config.large_threshold:
        L = int(config.large_threshold)
    else:
        mean = float(n_global) / float(F)
        L = max(64, int(mean + 8.0 * math.sqrt(max(mean, 1.0))) + 1)
    Th = int(config.heavy_threshold) if (config is not None and config.heavy_threshold) else 64
    return B, L, Th


class CudaOps:
    """The production data path: every call is a libgsh.so kernel launch."""

    def radix_histogram(self, keys, hi_bits, nbits):
        from .join import radix_histogram
        return radix_histogram(keys, hi_bits, nbits)

    def local_candidates(self, rk, rp, sk, sp, part_bits, large_u8, threshold):
        lib = load()
        R, S = _rel(rk, rp, "R"), _rel(sk, sp, "S")
        nb = lib.gsh_candidates_workspace_bytes(R.n, S.n)
        ws = torch.empty(int(nb), dtype=torch.uint8, device=rk.device)
        cap = max(1, (R.n + S.n) // max(threshold, 1) + 1)
        out = torch.empty(cap, dtype=torch.int32, device=rk.device)
        n = ctypes.c_uint64(0)
        check(lib.gsh_local_candidates(ctypes.byref(R), ctypes.byref(S), 0, part_bits, large_u8.data_ptr(), threshold,
                                       ws.data_ptr(), ws.numel(), _stream_handle(None), out.data_ptr(), cap,
                                       ctypes.byref(n)), "gsh_local_candidates")
        return out[: n.value].to(torch.int64) & 0xFFFFFFFF

    def count_keys(self, keys, q_sorted_i32):
        lib = load()
        counts = torch.zeros(q_sorted_i32.numel(), dtype=torch.int64, device=keys.device)
        if keys.numel() and q_sorted_i32.numel():
            check(lib.gsh_count_keys(keys.data_ptr(), keys.numel(), q_sorted_i32.data_ptr(), q_sorted_i32.numel(),
                                     counts.data_ptr(), _stream_handle(None)), "gsh_count_keys")
        return counts

    def route(self, keys, pays, route_bits, heavy_sorted_i32):
        lib = load()
        G = 1 << route_bits
        dev = keys.device
        counts = torch.zeros(G + 1, dtype=torch.int64, device=dev)
        hp = heavy_sorted_i32.data_ptr() if heavy_sorted_i32.numel() else None
        check(lib.gsh_route_count(keys.data_ptr() if keys.numel() else None, keys.numel(), route_bits, hp,
                                  heavy_sorted_i32.numel(), counts.data_ptr(), _stream_handle(None)), "route_count")
        host_counts = counts.cpu().tolist()
        offs = [0]
        for c in host_counts:
            offs.append(offs[-1] + c)
        off_t = torch.tensor(offs, dtype=torch.int64, device=dev)
        cur = torch.zeros(G + 1, dtype=torch.int64, device=dev)
        ok = torch.empty(max(keys.numel(), 1), dtype=torch.int32, device=dev)
        op = torch.empty(max(keys.numel(), 1), dtype=torch.int32, device=dev)
        if keys.numel():
            check(lib.gsh_route_scatter(keys.data_ptr(), pays.data_ptr(), keys.numel(), route_bits, hp,
                                        heavy_sorted_i32.numel(), off_t.data_ptr(), cur.data_ptr(), ok.data_ptr(),
                                        op.data_ptr(), _stream_handle(None)), "route_scatter")
        return ok[: keys.numel()], op[: keys.numel()], host_counts

    def join(self, rk, rp, sk, sp, config):
        r = join(rk, rp, sk, sp, config=config)
        return r.count, r.checksum, r.stats


def _to_i32_sorted(h64: torch.Tensor) -> torch.Tensor:
    """u32 values held in int64, sorted ascending -> same bit patterns as int32 (kernels compare
    as unsigned)."""
    h = torch.sort(h64).values
    return torch.where(h >= (1 << 31), h - (1 << 32), h).to(torch.int32)


def _allgather_var(t: torch.Tensor, group) -> torch.Tensor:
    """all_gather of a variable-length 1-D int64 tensor -> concatenation over ranks."""
    G = dist.get_world_size(group)
    n = torch.tensor([t.numel()], dtype=torch.int64, device=t.device)
    sizes = [torch.zeros_like(n) for _ in range(G)]
    dist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    m = max(sizes) if sizes else 0
    pad = torch.zeros(max(m, 1), dtype=t.dtype, device=t.device)
    pad[: t.numel()] = t
    bufs = [torch.empty_like(pad) for _ in range(G)]
    dist.all_gather(bufs, pad, group=group)
    return torch.cat([b[:s] for b, s in zip(bufs, sizes)])


def agree_heavy(rk, rp, sk, sp, config=None, group=None, ops=None):
    """Steps 1-2: the globally agreed skewed-key set (sorted hashes as int32) + global parameters."""
    ops = ops or CudaOps()
    dev = rk.device
    n = torch.tensor([rk.numel(), sk.numel()], dtype=torch.int64, device=dev)
    dist.all_reduce(n, group=group)
    n_r, n_s = int(n[0]), int(n[1])
    B, L, Th = _cfg_params(max(n_r, n_s), config)
    hr = ops.radix_histogram(rk, 0, B)
    hs = ops.radix_histogram(sk, 0, B)
    h = torch.stack([hr, hs])
    dist.all_reduce(h, group=group)
    large = ((h[0] > L) | (h[1] > L)) & (h[0] > 0) & (h[1] > 0)
    if config is not None and config.force_all_normal:
        large[:] = False
    G = dist.get_world_size(group)
    empty = torch.zeros(0, dtype=torch.int32, device=dev)
    if not bool(large.any()):
        return empty, (B, L, Th, n_r, n_s)
    tau = max(1, -(-Th // G))
    cand = ops.local_candidates(rk, rp, sk, sp, B, large.to(torch.uint8), tau)
    allc = _allgather_var(cand, group)
    q = torch.unique(allc)  # sorted int64 u32 values
    if q.numel() == 0:
        return empty, (B, L, Th, n_r, n_s)
    q32 = _to_i32_sorted(q)
    cnt = torch.stack([ops.count_keys(rk, q32), ops.count_keys(sk, q32)])
    dist.all_reduce(cnt, group=group)
    heavy = q[torch.maximum(cnt[0], cnt[1]) >= Th]
    return _to_i32_sorted(heavy), (B, L, Th, n_r, n_s)


def _exchange_normal(keys, pays, counts, G, group):
    """all_to_all of the destination-grouped normal tuples (first G groups)."""
    dev = keys.device
    send = torch.tensor(counts[:G], dtype=torch.int64, device=dev)
    recv = torch.empty_like(send)
    dist.all_to_all_single(recv, send, group=group)
    in_splits = [int(c) for c in counts[:G]]
    out_splits = [int(c) for c in recv.cpu().tolist()]
    tot_in = sum(in_splits)
    tot_out = sum(out_splits)
    ok = torch.empty(tot_out, dtype=torch.int32, device=dev)
    op = torch.empty(tot_out, dtype=torch.int32, device=dev)
    dist.all_to_all_single(ok, keys[:tot_in].contiguous(), out_splits, in_splits, group=group)
    dist.all_to_all_single(op, pays[:tot_in].contiguous(), out_splits, in_splits, group=group)
    return ok, op


def _broadcast_heavy_r(hk, hp, group):
    """Every rank receives every rank's skewed R tuples (exact-size broadcasts, no padding)."""
    G = dist.get_world_size(group)
    dev = hk.device
    n = torch.tensor([hk.numel()], dtype=torch.int64, device=dev)
    sizes = [torch.zeros_like(n) for _ in range(G)]
    dist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    me = dist.get_rank(group)
    tot = sum(sizes)
    ok = torch.empty(tot, dtype=torch.int32, device=dev)
    op = torch.empty(tot, dtype=torch.int32, device=dev)
    off = 0
    for g, s in enumerate(sizes):
        if s:
            if g == me:
                ok[off: off + s].copy_(hk)
                op[off: off + s].copy_(hp)
            src = dist.get_global_rank(group, g) if group is not None else g
            dist.broadcast(ok[off: off + s], src=src, group=group)
            dist.broadcast(op[off: off + s], src=src, group=group)
        off += s
    return ok, op


def join_sharded(rk, rp, sk, sp, config=None, group=None, ops=None):
    """Hash-sharded GSH join of this rank's shards; returns a JoinResult-like object whose
    count/checksum are GLOBAL (identical on all ranks)."""
    from .join import JoinResult
    ops = ops or CudaOps()
    if isinstance(ops, CudaOps):
        rk, rp = _check_dev(rk, "r_keys"), _check_dev(rp, "r_payloads")
        sk, sp = _check_dev(sk, "s_keys"), _check_dev(sp, "s_payloads")
    G = dist.get_world_size(group)
    if G & (G - 1):
        raise ValueError("world size must be a power of two (route bits)")
    rb = G.bit_length() - 1
    heavy, (B, L, Th, n_r, n_s) = agree_heavy(rk, rp, sk, sp, config, group, ops)
    rks, rps, rc = ops.route(rk, rp, rb, heavy)
    sks, sps, sc = ops.route(sk, sp, rb, heavy)
    rk_n, rp_n = _exchange_normal(rks, rps, rc, G, group)
    sk_n, sp_n = _exchange_normal(sks, sps, sc, G, group)
    nr_h = rc[G]
    ns_h = sc[G]
    r_off = sum(rc[:G])
    s_off = sum(sc[:G])
    rk_h, rp_h = _broadcast_heavy_r(rks[r_off: r_off + nr_h], rps[r_off: r_off + nr_h], group)
    # local inputs: normal received + skewed (R: all ranks', S: local)
    lrk = torch.cat([rk_n, rk_h])
    lrp = torch.cat([rp_n, rp_h])
    lsk = torch.cat([sk_n, sks[s_off: s_off + ns_h]])
    lsp = torch.cat([sp_n, sps[s_off: s_off + ns_h]])
    lcfg = make_config() if config is None else _copy_cfg(config)
    lcfg.route_bits = rb
    cnt, chk, stats = ops.join(lrk, lrp, lsk, lsp, lcfg)
    dev = rk.device
    t = torch.tensor([cnt, chk - (1 << 64) if chk >= (1 << 63) else chk], dtype=torch.int64, device=dev)
    dist.all_reduce(t, group=group)
    gc = int(t[0]) & M64
    gk = int(t[1]) & M64
    stats = dict(stats)
    stats.update({"n_heavy_global": int(heavy.numel()), "local_r": int(lrk.numel()), "local_s": int(lsk.numel()),
                  "heavy_r_recv": int(rk_h.numel()), "route_bits": rb})
    return JoinResult(count=gc, checksum=gk, stats=stats)


def _copy_cfg(c):
    n = _lib.GshConfig()
    ctypes.memmove(ctypes.byref(n), ctypes.byref(c), ctypes.sizeof(c))
    return n
