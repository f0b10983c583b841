"""Multi-GPU GSH: hash sharding over one node (a north-star addition --
the paper runs on one A100).

One process per GPU (torch.distributed, NCCL over NVLink/NVSwitch), or G logical ranks sharing one
GPU in one process (`LocalWorld`, the one-GPU test harness of SURVEY §4(i)).  Per rank:

  1. agreement (gsh_shard_*): global partition histogram (all_reduce) -> globally large
     partitions (L107) -> local candidates with local max(cnt_R, cnt_S) >= ceil(T_h / G)
     -> all_gather -> union in first-occurrence order + exact local counts -> all_reduce ->
     skewed keys max(cnt_R, cnt_S) >= T_h (L112): the single-GPU rule on the whole input, the
     same list on every rank;
  2. routing (gsh_route_*): a normal tuple goes to rank top_log2(G)_bits(fmix32(key)); a tuple of
     a skewed key stays on this rank (S) or is broadcast (R), so no GPU receives a skewed key's
     full S.  The route kernel writes every tuple straight into its final buffer: this rank's own
     normal tuples into the receive buffer, its skewed R tuples into the all-gathered R_H buffer,
     the rest into the send buffer of the all-to-all;
  3. exchange: all_to_all of the normal tuples, all-gather of the skewed R tuples;
  4. two local GSH joins (gsh_join): the received normal shard (every tuple's top route bits of h
     equal this rank's id, which gsh_config.route_bits asserts), and all ranks' R_H x local S_H
     with route_bits = 0 (skewed keys carry arbitrary top bits);
  5. all_reduce(sum) of (count, checksum) mod 2^64: the single-GPU result bit-exactly.

Every data-path step is a libgsh.so kernel; PyTorch provides device memory, streams and the
process group.  `ops` / `comm` are hooks so the host protocol runs on CPU with gloo and an oracle
test double (tests/ only).
"""
from __future__ import annotations

import ctypes
import threading
import time

import torch
import torch.distributed as dist

from . import _lib
from ._lib import GshShardParams, check, load
from .join import JoinResult, _check_dev, _rel, _stream_handle, join, make_config

M64 = (1 << 64) - 1
NVLINK_GBS = 900.0   # NVLink 5 per GPU per direction (B200_PROFILING.md)


# --------------------------------------------------------------------------- communicators
class TorchComm:
    """Collectives of the protocol over a torch.distributed process group (NCCL on GPUs, gloo on
    CPU).  Integer tensors only; sizes travel as int64 tensors on the data's device."""

    def __init__(self, group=None, device=None):
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.device = device
        # gloo moves host tensors: device tensors travel through host copies (control-size data;
        # the bulk exchange of the p2p mode never goes through a collective)
        self.host_only = dist.get_backend(group) == "gloo"
        self.ctl = torch.device("cpu") if self.host_only else device

    def _src(self, g: int) -> int:
        return dist.get_global_rank(self.group, g) if self.group is not None else g

    def all_reduce_(self, t: torch.Tensor) -> None:
        if self.host_only and t.is_cuda:
            h = t.cpu()
            dist.all_reduce(h, group=self.group)
            t.copy_(h)
        else:
            dist.all_reduce(t, group=self.group)

    def all_gather_sizes(self, n: int) -> list[int]:
        t = torch.tensor([n], dtype=torch.int64, device=self.ctl)
        out = [torch.zeros_like(t) for _ in range(self.world)]
        dist.all_gather(out, t, group=self.group)
        return [int(x.item()) for x in out]

    def all_gather_pad(self, t: torch.Tensor, m: int) -> torch.Tensor:
        """[world * m] buffer; rank g's tensor at [g * m, g * m + len)."""
        dev = self.ctl if self.host_only else t.device
        out = torch.zeros(self.world * max(m, 1), dtype=t.dtype, device=dev)
        pad = torch.zeros(max(m, 1), dtype=t.dtype, device=dev)
        pad[: t.numel()] = t.to(dev)
        dist.all_gather(list(out.view(self.world, -1).unbind(0)), pad, group=self.group)
        return out.to(t.device)

    def all_to_all_v(self, out: torch.Tensor, inp: torch.Tensor, out_splits: list[int], in_splits: list[int]) -> None:
        if sum(out_splits) == 0 and sum(in_splits) == 0 and self.world == 1:
            return
        dist.all_to_all_single(out, inp, out_splits, in_splits, group=self.group)

    def all_gather_v_(self, buf: torch.Tensor, sizes: list[int]) -> None:
        """In place: rank g's segment [sum(sizes[:g]), +sizes[g]) of `buf` is sent to every rank
        (this rank's own segment must already be in place)."""
        off = 0
        for g, n in enumerate(sizes):
            if n:
                dist.broadcast(buf[off: off + n], src=self._src(g), group=self.group)
            off += n

    def all_gather_rows(self, row: list[int]) -> list[list[int]]:
        t = torch.tensor(row, dtype=torch.int64, device=self.ctl)
        out = [torch.zeros_like(t) for _ in range(self.world)]
        dist.all_gather(out, t, group=self.group)
        return [[int(v) for v in x.tolist()] for x in out]

    def space_key(self):
        return ("torch", id(self.group), str(self.device))

    def barrier(self) -> None:
        """Every rank's queued device work (e.g. peer stores) is complete before any returns."""
        if torch.cuda.is_available():
            torch.cuda.current_stream().synchronize()
        dist.barrier(group=self.group)

    def peer_views(self, bufs: dict) -> list[dict]:
        """The other ranks' buffers of the same names, mapped into this process through CUDA IPC
        (NVLink peer memory; the same GPU's memory when ranks share one): {name: PeerPtr}."""
        lib = load()
        mine = []
        for name in sorted(bufs):
            h = (ctypes.c_uint8 * 64)()
            off = ctypes.c_uint64(0)
            check(lib.gsh_ipc_handle(bufs[name].data_ptr(), h, ctypes.byref(off)), "gsh_ipc_handle")
            mine.append(list(bytes(h)) + [off.value & 0xFF_FFFF_FFFF_FFFF, bufs[name].numel()])
        flat = [v for rec in mine for v in rec]
        rows = self.all_gather_rows(flat)
        per = len(flat) // max(len(bufs), 1)
        views = []
        for g, row in enumerate(rows):
            if g == self.rank:
                views.append(dict(bufs))
                continue
            d = {}
            for i, name in enumerate(sorted(bufs)):
                rec = row[i * per: (i + 1) * per]
                d[name] = PeerPtr.open(bytes(v & 0xFF for v in rec[:64]), rec[64], rec[65])
            views.append(d)
        return views


class PeerPtr:
    """A peer process's device buffer mapped with gsh_ipc_open (base of its allocation + offset)."""

    _open: dict = {}   # handle bytes -> mapped base (one mapping per allocation and process)

    def __init__(self, ptr: int, n: int):
        self.ptr, self.n = ptr, n

    def data_ptr(self) -> int:
        return self.ptr

    def numel(self) -> int:
        return self.n

    @classmethod
    def open(cls, handle: bytes, offset: int, n: int) -> "PeerPtr":
        base = cls._open.get(handle)
        if base is None:
            p = ctypes.c_void_p(0)
            h = (ctypes.c_uint8 * 64).from_buffer_copy(handle)
            check(load().gsh_ipc_open(h, ctypes.byref(p)), "gsh_ipc_open")
            base = cls._open[handle] = p.value
        return cls(base + offset, n)


class LocalWorld:
    """G logical ranks in one process (one host thread each, any device), exchanging through
    device copies: the one-GPU multi-rank harness.  Every collective is a
    deposit / barrier / copy / barrier round; each rank synchronises its own stream before it
    deposits, so peers read finished data."""

    def __init__(self, world: int):
        self.world = world
        self.barrier = threading.Barrier(world)
        self.slots: list = [None] * world

    def comm(self, rank: int) -> "LocalComm":
        return LocalComm(self, rank)


class LocalComm:
    def __init__(self, w: LocalWorld, rank: int):
        self.w, self.rank, self.world = w, rank, w.world

    def _round(self, obj, fn):
        if torch.cuda.is_available():
            torch.cuda.current_stream().synchronize()
        self.w.slots[self.rank] = obj
        self.w.barrier.wait()
        try:
            r = fn(list(self.w.slots))
            if torch.cuda.is_available():
                torch.cuda.current_stream().synchronize()
        finally:
            self.w.barrier.wait()
        return r

    def all_reduce_(self, t: torch.Tensor) -> None:
        s = self._round(t, lambda xs: sum(x.clone() for x in xs))
        t.copy_(s)

    def all_gather_sizes(self, n: int) -> list[int]:
        return self._round(int(n), lambda xs: list(xs))

    def all_gather_pad(self, t: torch.Tensor, m: int) -> torch.Tensor:
        out = torch.zeros(self.world * max(m, 1), dtype=t.dtype, device=t.device)

        def fn(xs):
            for g, x in enumerate(xs):
                out[g * max(m, 1): g * max(m, 1) + x.numel()].copy_(x)
        self._round(t, fn)
        return out

    def all_to_all_v(self, out, inp, out_splits, in_splits) -> None:
        me = self.rank

        def fn(xs):
            o = 0
            for g, (x, isp) in enumerate(xs):
                n = isp[me]
                assert n == out_splits[g]
                if n:
                    src = sum(isp[:me])
                    out[o: o + n].copy_(x[src: src + n])
                o += out_splits[g]
        self._round((inp, list(in_splits)), fn)

    def all_gather_v_(self, buf, sizes) -> None:
        me = self.rank

        def fn(xs):
            off = 0
            for g, x in enumerate(xs):
                if g != me and sizes[g]:
                    buf[off: off + sizes[g]].copy_(x[off: off + sizes[g]])
                off += sizes[g]
        self._round(buf, fn)

    def all_gather_rows(self, row):
        return self._round(list(row), lambda xs: [list(x) for x in xs])

    def space_key(self):
        return ("local", id(self.w), self.rank)

    def barrier(self) -> None:
        self._round(None, lambda xs: None)

    def peer_views(self, bufs: dict) -> list[dict]:
        """In one process the peers' buffers are directly addressable: their tensors."""
        return self._round(dict(bufs), lambda xs: [dict(x) for x in xs])


# ------------------------------------------------------------------------------- CUDA ops
class CudaOps:
    """The production per-rank steps: every call is a libgsh.so entry point (include/gsh.h)."""

    def __init__(self, device: torch.device):
        self.dev = device
        self.events: list[tuple[str, torch.cuda.Event]] = []
        self.launches = 0   # libgsh kernels launched by the protocol steps (the joins report their own)

    # plumbing
    def tensor(self, vals, dtype=torch.int64):
        return torch.tensor(vals, dtype=dtype, device=self.dev)

    def empty(self, n: int):
        return torch.empty(max(int(n), 1), dtype=torch.int32, device=self.dev)[: int(n)]

    def stream(self):
        return _stream_handle(None, self.dev)

    def mark(self, name: str) -> None:
        e = torch.cuda.Event(enable_timing=True)
        e.record(torch.cuda.current_stream(self.dev))
        self.events.append((name, e))

    def phase_ms(self) -> dict:
        torch.cuda.current_stream(self.dev).synchronize()
        return {f"ms_{n}": float(a.elapsed_time(b)) for (_, a), (n, b) in zip(self.events, self.events[1:])}

    # steps
    def histogram(self, rk, sk, P):
        h = torch.empty(2 << P.part_bits, dtype=torch.int64, device=self.dev)
        R, S = _rel(rk, rk, "R"), _rel(sk, sk, "S")
        check(load().gsh_shard_histogram(ctypes.byref(R), ctypes.byref(S), ctypes.byref(P), h.data_ptr(),
                                         self.stream()), "gsh_shard_histogram")
        self.launches += (R.n > 0) + (S.n > 0)
        return h

    def candidates(self, state, rk, rp, sk, sp, P, hist):
        lib = load()
        R, S = _rel(rk, rp, "R"), _rel(sk, sp, "S")
        nb = int(lib.gsh_shard_workspace_bytes(R.n, S.n))
        state["cand_ws"] = ws = torch.empty(nb, dtype=torch.uint8, device=self.dev)
        cap = max(1024, (R.n + S.n) // 64)
        while True:
            out = torch.empty(cap, dtype=torch.int32, device=self.dev)
            n, ovf = ctypes.c_uint64(0), ctypes.c_uint32(0)
            st = lib.gsh_shard_candidates(ctypes.byref(R), ctypes.byref(S), ctypes.byref(P), hist.data_ptr(),
                                          ws.data_ptr(), ws.numel(), self.stream(), out.data_ptr(), cap,
                                          ctypes.byref(n), ctypes.byref(ovf))
            if st == _lib.GSH_ERR_INVALID and n.value > cap:
                cap = int(n.value)
                continue
            check(st, "gsh_shard_candidates")
            self.launches += 2 + (R.n > 0) + (S.n > 0)
            return out[: n.value], bool(ovf.value)

    def agree(self, state, gathered, sizes, stride):
        lib = load()
        G = len(sizes)
        ws = torch.empty(int(lib.gsh_shard_agree_workspace_bytes(G * max(stride, 1))), dtype=torch.uint8,
                         device=self.dev)
        state["agree_ws"] = ws
        cap = max(1, sum(sizes))
        uni = torch.empty(cap, dtype=torch.int32, device=self.dev)
        cnt = torch.zeros(2 * cap, dtype=torch.int64, device=self.dev)
        hs = (ctypes.c_uint64 * G)(*sizes)
        n = ctypes.c_uint64(0)
        cw = state["cand_ws"]
        check(lib.gsh_shard_agree(cw.data_ptr(), cw.numel(), gathered.data_ptr(), G, max(stride, 1), hs,
                                  ws.data_ptr(), ws.numel(), self.stream(), uni.data_ptr(), cnt.data_ptr(), cap,
                                  ctypes.byref(n)), "gsh_shard_agree")
        m = int(n.value)
        self.launches += 5 if sum(sizes) else 0
        return uni[:m], cnt[: 2 * m]

    def select(self, state, uni, cnt, P):
        lib = load()
        m = uni.numel()
        heavy = torch.empty(max(m, 1), dtype=torch.int32, device=self.dev)
        n = ctypes.c_uint64(0)
        ws = state.get("agree_ws")
        check(lib.gsh_shard_select(uni.data_ptr() if m else None, cnt.data_ptr() if m else None, m, ctypes.byref(P),
                                   ws.data_ptr() if ws is not None else None, ws.numel() if ws is not None else 0,
                                   self.stream(), heavy.data_ptr(), m, ctypes.byref(n)), "gsh_shard_select")
        nh = int(n.value)
        self.launches += (4 if m else 0) + (1 if nh else 0)
        heavy = heavy[:nh]
        sb = int(lib.gsh_heavy_set_bytes(nh))
        state["set"] = hset = torch.empty(max(sb, 256), dtype=torch.uint8, device=self.dev)
        state["set_bytes"] = sb
        check(lib.gsh_heavy_set_build(heavy.data_ptr() if nh else None, nh, hset.data_ptr(), sb, self.stream()),
              "gsh_heavy_set_build")
        return heavy

    def route_count(self, state, keys, rb):
        G1 = (1 << rb) + 1
        c = torch.empty(G1, dtype=torch.int64, device=self.dev)
        check(load().gsh_route_count(keys.data_ptr() if keys.numel() else None, keys.numel(), rb,
                                     state["set"].data_ptr() if state["set_bytes"] else None, state["set_bytes"],
                                     c.data_ptr(), self.stream()), "gsh_route_count")
        self.launches += keys.numel() > 0
        return [int(x) for x in c.cpu().tolist()]

    def route_scatter(self, state, keys, pays, rb, dst, heavy_copies: int = 1):
        """dst[d] = (keys_buffer, pays_buffer, offset): destination d's run starts at offset (d = G:
        skewed tuples; heavy_copies > 1: further copies of them follow in dst).  A buffer is a
        tensor or a PeerPtr (another rank's memory)."""
        if keys.numel() == 0:
            return
        ptrs = []
        for k, p, off in dst:
            ptrs += [k.data_ptr() + 4 * off if k.numel() else 0, p.data_ptr() + 4 * off if p.numel() else 0]
        d_dst = self.tensor([x - (1 << 64) if x >= (1 << 63) else x for x in ptrs])
        cur = torch.empty(len(dst) - heavy_copies + 1, dtype=torch.int64, device=self.dev)
        check(load().gsh_route_scatter(keys.data_ptr(), pays.data_ptr(), keys.numel(), rb,
                                       state["set"].data_ptr() if state["set_bytes"] else None, state["set_bytes"],
                                       d_dst.data_ptr(), heavy_copies, cur.data_ptr(), self.stream()),
              "gsh_route_scatter")
        state.setdefault("keep", []).append(d_dst)
        self.launches += 1

    def join(self, rk, rp, sk, sp, config, out=None):
        mode = "materialize" if out is not None else "count"
        r = join(rk, rp, sk, sp, mode=mode, out=out, config=config)
        self.launches += r.stats.get("launches", 0)
        return r.count, r.checksum, r.written, r.stats


# --------------------------------------------------------------------- peer-store exchange
_SPACES: dict = {}   # communicator identity -> PeerSpace (the IPC mappings outlive a call)


class PeerSpace:
    """A rank's receive buffers for the peer-store exchange, kept across calls (their IPC
    mappings are set up once): normal R / S keys and payloads, and the all-gathered skewed R.
    Capacities are decided from the all-gathered count matrix (identical on every rank), so
    all ranks grow together and re-share their buffers."""

    NAMES = ("rn_k", "rn_p", "sn_k", "sn_p", "rh_k", "rh_p")

    def __init__(self, ops):
        self.ops = ops
        self.caps = (-1, -1, -1)
        self.bufs: dict = {}
        self.views: list = []

    def ensure(self, comm, cap_rn: int, cap_sn: int, cap_rh: int) -> None:
        if cap_rn <= self.caps[0] and cap_sn <= self.caps[1] and cap_rh <= self.caps[2]:
            return
        grow = lambda c, old: max(c + (c >> 3) + 1024, old)   # noqa: E731  (headroom against regrowth)
        caps = (grow(cap_rn, self.caps[0]), grow(cap_sn, self.caps[1]), grow(cap_rh, self.caps[2]))
        comm.barrier()   # every peer is done with the old buffers
        self.bufs = {}
        for name, c in zip(self.NAMES, (caps[0], caps[0], caps[1], caps[1], caps[2], caps[2])):
            self.bufs[name] = self.ops.empty(c)
        self.caps = caps
        self.views = comm.peer_views(self.bufs)


def _route_p2p(rk, rp, sk, sp, rb, rc, sc, comm, ops, state):
    """Steps 2-3 with the exchange inside the route kernel: every tuple is stored straight into its
    destination rank's receive buffer (skewed R into every rank's), at an offset fixed by the
    all-gathered count matrix; a barrier then makes all peers' stores visible.  Returns this
    rank's (normal R, normal S, all skewed R, local skewed S) and the bytes it stored remotely."""
    G, me = comm.world, comm.rank
    M = comm.all_gather_rows(list(rc) + list(sc))          # row g: rank g's R counts, then S counts
    rcm = [row[: G + 1] for row in M]
    scm = [row[G + 1:] for row in M]
    need_rn = [sum(rcm[g][d] for g in range(G)) for d in range(G)]
    need_sn = [sum(scm[g][d] for g in range(G)) for d in range(G)]
    need_rh = sum(rcm[g][G] for g in range(G))
    key = comm.space_key()
    space = _SPACES.get(key)
    if space is None:
        space = _SPACES[key] = PeerSpace(ops)
    space.ensure(comm, max(need_rn), max(need_sn), need_rh)
    V = space.views
    off_rn = [sum(rcm[g][d] for g in range(me)) for d in range(G)]   # my run in each destination
    off_sn = [sum(scm[g][d] for g in range(me)) for d in range(G)]
    off_rh = sum(rcm[g][G] for g in range(me))
    Sh = (ops.empty(sc[G]), ops.empty(sc[G]))
    dst_r = [(V[d]["rn_k"], V[d]["rn_p"], off_rn[d]) for d in range(G)]
    dst_r += [(V[d]["rh_k"], V[d]["rh_p"], off_rh) for d in range(G)]     # skewed R: every rank
    dst_s = [(V[d]["sn_k"], V[d]["sn_p"], off_sn[d]) for d in range(G)] + [(Sh[0], Sh[1], 0)]
    ops.route_scatter(state, rk, rp, rb, dst_r, heavy_copies=G)
    ops.route_scatter(state, sk, sp, rb, dst_s)
    ops.mark("route")
    comm.barrier()
    ops.mark("exchange")
    B = space.bufs
    Rn = (B["rn_k"][: need_rn[me]], B["rn_p"][: need_rn[me]])
    Sn = (B["sn_k"][: need_sn[me]], B["sn_p"][: need_sn[me]])
    Rh = (B["rh_k"][:need_rh], B["rh_p"][:need_rh])
    remote = 8 * (sum(rc[d] for d in range(G) if d != me) + sum(sc[d] for d in range(G) if d != me)
                  + (G - 1) * rc[G])
    return Rn, Sn, Rh, Sh, remote, rcm


# ------------------------------------------------------------------------------- protocol
def shard_plan(n_r: int, n_s: int, world: int, config=None) -> GshShardParams:
    """gsh_shard_plan: the single-GPU rule's (B, L, T_h) for the global sizes + tau (host-only)."""
    P = GshShardParams()
    check(load().gsh_shard_plan(n_r, n_s, world, ctypes.byref(config) if config is not None else None,
                                ctypes.byref(P)), "gsh_shard_plan")
    return P


def _copy_cfg(c, **kw):
    n = _lib.GshConfig()
    if c is None:
        n = make_config()
    else:
        ctypes.memmove(ctypes.byref(n), ctypes.byref(c), ctypes.sizeof(c))
    for k, v in kw.items():
        setattr(n, k, v)
    return n


def _s64(x: int) -> int:
    x &= M64
    return x - (1 << 64) if x >= (1 << 63) else x


def agree_heavy(rk, rp, sk, sp, P, comm, ops, state):
    """Step 1: the globally agreed skewed keys (int32 h values, identical list on every rank)."""
    hist = ops.histogram(rk, sk, P)
    comm.all_reduce_(hist)
    cand, cand_ovf = ops.candidates(state, rk, rp, sk, sp, P, hist)
    sizes = comm.all_gather_sizes(cand.numel())
    stride = max(sizes) if sizes else 0
    state["cand_overflow"] = cand_ovf
    state["n_cand"] = sum(sizes)
    if stride == 0:
        return ops.select(state, cand[:0], ops.tensor([], dtype=torch.int64), P)
    gathered = comm.all_gather_pad(cand, stride)
    uni, cnt = ops.agree(state, gathered, sizes, stride)
    comm.all_reduce_(cnt)
    state["n_union"] = uni.numel()
    return ops.select(state, uni, cnt, P)


def _route_a2a(rk, rp, sk, sp, rb, rc, sc, comm, ops, state):
    """Steps 2-3 with collectives: the route kernel writes this rank's own normal tuples to the end
    of its receive buffer, its skewed R to its offset in the all-gathered R_H buffer, the rest to
    send buffers; then all_to_all of the normal tuples and the in-place all-gather of R_H."""
    G, me = comm.world, comm.rank
    send = ops.tensor([[rc[d], sc[d]] for d in range(G)]).reshape(-1)
    recv = ops.tensor([0] * (2 * G))
    comm.all_to_all_v(recv, send, [2] * G, [2] * G)
    recv = recv.reshape(G, 2).tolist()
    rh_sizes = comm.all_gather_sizes(rc[G])
    rr = [int(recv[g][0]) if g != me else 0 for g in range(G)]   # from other ranks
    rs = [int(recv[g][1]) if g != me else 0 for g in range(G)]
    rsend = [rc[d] if d != me else 0 for d in range(G)]
    ssend = [sc[d] if d != me else 0 for d in range(G)]
    nr_other, ns_other = sum(rr), sum(rs)
    Rn = (ops.empty(nr_other + rc[me]), ops.empty(nr_other + rc[me]))    # normal R: [others | own]
    Sn = (ops.empty(ns_other + sc[me]), ops.empty(ns_other + sc[me]))
    Rh = (ops.empty(sum(rh_sizes)), ops.empty(sum(rh_sizes)))            # skewed R of every rank
    Sh = (ops.empty(sc[G]), ops.empty(sc[G]))                            # local skewed S
    Rx = (ops.empty(sum(rsend)), ops.empty(sum(rsend)))                  # send buffers
    Sx = (ops.empty(sum(ssend)), ops.empty(sum(ssend)))

    def dst_list(own, own_off, x, xsend, heavy_buf, heavy_off):
        d, off = [], 0
        for g in range(G):
            if g == me:
                d.append((own[0], own[1], own_off))
            else:
                d.append((x[0], x[1], off))
                off += xsend[g]
        d.append((heavy_buf[0], heavy_buf[1], heavy_off))
        return d

    ops.route_scatter(state, rk, rp, rb, dst_list(Rn, nr_other, Rx, rsend, Rh, sum(rh_sizes[:me])))
    ops.route_scatter(state, sk, sp, rb, dst_list(Sn, ns_other, Sx, ssend, Sh, 0))
    ops.mark("route")
    for i in range(2):
        comm.all_to_all_v(Rn[i][:nr_other], Rx[i], rr, rsend)
        comm.all_to_all_v(Sn[i][:ns_other], Sx[i], rs, ssend)
    ops.mark("exchange")
    for i in range(2):
        comm.all_gather_v_(Rh[i], rh_sizes)
    ops.mark("broadcast")
    xbytes = 8 * (sum(rsend) + sum(ssend))
    bbytes = 8 * (sum(rh_sizes) - rh_sizes[me])
    return Rn, Sn, Rh, Sh, xbytes, bbytes, rh_sizes


def join_sharded(rk, rp, sk, sp, config=None, group=None, ops=None, comm=None, mode: str = "count", out=None,
                 exchange: str = "a2a"):
    """Hash-sharded GSH join of this rank's shards (any positional split of R and S over the ranks).

    exchange: "a2a" -- the route kernel fills send buffers, then all_to_all / all-gather
    collectives (NCCL); "p2p" -- the route kernel stores every tuple straight into its
    destination rank's receive buffer (peer memory: CUDA IPC over NVLink, or in-process), skewed R
    into every rank's, so the scatter IS the exchange and no send buffer exists.

    Returns a JoinResult whose count / checksum are GLOBAL (identical on all ranks); in
    "materialize" mode `out` ((capacity, 2) int32 CUDA tensor) receives this rank's pairs and
    `written` counts them.  stats: per-phase ms, exchanged bytes and their NVLink fraction."""
    if exchange not in ("a2a", "p2p"):
        raise ValueError("exchange must be 'a2a' or 'p2p'")
    if ops is None:
        rk, rp = _check_dev(rk, "r_keys"), _check_dev(rp, "r_payloads")
        sk, sp = _check_dev(sk, "s_keys"), _check_dev(sp, "s_payloads")
        ops = CudaOps(rk.device)
    if comm is None:
        comm = TorchComm(group, rk.device)
    G, me = comm.world, comm.rank
    if G & (G - 1):
        raise ValueError("world size must be a power of two (route bits)")
    if mode not in ("count", "materialize"):
        raise ValueError("mode must be 'count' or 'materialize'")
    state: dict = {}
    ops.mark("start")
    n = ops.tensor([rk.numel(), sk.numel()])
    comm.all_reduce_(n)
    n_r, n_s = (int(x) for x in n.tolist())
    P = shard_plan(n_r, n_s, G, config)
    rb = int(P.route_bits)
    heavy = agree_heavy(rk, rp, sk, sp, P, comm, ops, state)
    ops.mark("agree")

    # routing plan: destination counts, then every buffer laid out so the route kernel writes
    # each tuple to its final place
    rc = ops.route_count(state, rk, rb)
    sc = ops.route_count(state, sk, rb)
    if exchange == "p2p":
        Rn, Sn, Rh, Sh, xbytes, rcm = _route_p2p(rk, rp, sk, sp, rb, rc, sc, comm, ops, state)
        rh_sizes = [row[G] for row in rcm]
        bbytes = 0   # the skewed R copies are part of the peer stores (xbytes)
        ops.mark("broadcast")
    else:
        Rn, Sn, Rh, Sh, xbytes, bbytes, rh_sizes = _route_a2a(rk, rp, sk, sp, rb, rc, sc, comm, ops, state)
    # local joins: the routed normal shard under route_bits = rb, the skewed keys under 0
    cfg_n = _copy_cfg(config, route_bits=rb, timing=1)
    cfg_h = _copy_cfg(config, route_bits=0, timing=1)
    mat = mode == "materialize"
    o1 = out if mat else None
    c1, k1, w1, st1 = ops.join(Rn[0], Rn[1], Sn[0], Sn[1], cfg_n, o1)
    ops.mark("join_normal")
    o2 = out[w1:] if mat else None
    if Rh[0].numel() and Sh[0].numel():
        c2, k2, w2, st2 = ops.join(Rh[0], Rh[1], Sh[0], Sh[1], cfg_h, o2)
    else:
        c2, k2, w2, st2 = 0, 0, 0, {}
    ops.mark("join_heavy")
    t = ops.tensor([_s64(c1 + c2), _s64(k1 + k2)])
    comm.all_reduce_(t)
    gc, gk = (int(x) & M64 for x in t.tolist())
    ops.mark("reduce")
    phases = ops.phase_ms()
    stats = {
        "world": G, "rank": me, "route_bits": rb, "part_bits": int(P.part_bits),
        "large_threshold": int(P.large_threshold), "heavy_threshold": int(P.heavy_threshold),
        "cand_threshold": int(P.cand_threshold), "n_heavy_global": int(heavy.numel()),
        "n_candidates_gathered": state.get("n_cand", 0), "n_union": state.get("n_union", 0),
        "candidate_table_overflow": bool(state.get("cand_overflow", False)),
        "local_r": rk.numel(), "local_s": sk.numel(),
        "normal_r": Rn[0].numel(), "normal_s": Sn[0].numel(), "heavy_r": Rh[0].numel(), "heavy_s": Sh[0].numel(),
        "exchange": exchange, "exchange_send_bytes": xbytes, "broadcast_recv_bytes": bbytes,
        "count_normal": c1, "count_heavy": c2, "written": w1 + w2,
        "join_normal": st1, "join_heavy": st2, "launches": getattr(ops, "launches", 0),
    }
    stats.update(phases)
    for name, nbytes in (("exchange", xbytes), ("broadcast", bbytes)):
        ms = phases.get(f"ms_{name}", 0.0)
        gbs = nbytes / (ms * 1e6) if ms > 0 else None
        stats[f"{name}_GBps"] = gbs
        stats[f"{name}_nvlink_frac"] = gbs / NVLINK_GBS if gbs is not None else None
    return JoinResult(count=gc, checksum=gk, written=w1 + w2, overflow=bool(st1.get("overflow", 0) or
                                                                            st2.get("overflow", 0)),
                      pairs=(out[: w1 + w2] if mat else None), stats=stats)


def run_local(world: int, shards, config=None, mode: str = "count", out_capacity: int = 0, device=None,
              exchange: str = "a2a"):
    """Run join_sharded for `world` logical ranks on ONE device (threads + LocalWorld): the
    one-GPU multi-rank harness.  shards[g] = (rk, rp, sk, sp) CUDA tensors of rank g.  Returns the
    per-rank JoinResults (rank order)."""
    lw = LocalWorld(world)
    dev = torch.device(device) if device is not None else shards[0][0].device
    res: list = [None] * world
    err: list = []

    def worker(g):
        try:
            with torch.cuda.device(dev):
                s = torch.cuda.Stream(dev)
                with torch.cuda.stream(s):
                    out = (torch.empty((out_capacity, 2), dtype=torch.int32, device=dev)
                           if mode == "materialize" else None)
                    res[g] = join_sharded(*shards[g], config=config, comm=lw.comm(g), mode=mode, out=out,
                                          exchange=exchange)
                s.synchronize()
        except BaseException as e:  # surface the first failure, release the other ranks
            err.append(e)
            lw.barrier.abort()

    th = [threading.Thread(target=worker, args=(g,)) for g in range(world)]
    t0 = time.perf_counter()
    for t in th:
        t.start()
    for t in th:
        t.join()
    if err:
        raise err[0]
    for r in res:
        r.stats["wall_s"] = time.perf_counter() - t0
    return res


# ------------------------------------------------------- native driver (gsh_join_sharded)
EXCHANGES = {"a2a": _lib.GSH_EXCHANGE_A2A, "p2p": _lib.GSH_EXCHANGE_P2P}


class NativeComm:
    """A gsh_comm table (include/gsh.h) for the native driver: an NCCL communicator or one rank of
    a NativeLocalWorld.  close() releases what the library allocated for it."""

    def __init__(self, comm: _lib.GshComm, owner=None, destroy: bool = True):
        self.c, self._owner, self._destroy = comm, owner, destroy

    @property
    def rank(self) -> int:
        return int(self.c.rank)

    @property
    def world(self) -> int:
        return int(self.c.world)

    def close(self) -> None:
        if self._destroy and self.c.ctx:
            check(load().gsh_comm_destroy(ctypes.byref(self.c)), "gsh_comm_destroy")

    def abort(self) -> None:
        """Release the peers blocked in a collective (the comm's abort, when it has one)."""
        if self.c.abort:
            ctypes.CFUNCTYPE(None, ctypes.c_void_p)(self.c.abort)(self.c.ctx)


class NativeLocalWorld:
    """gsh_local_world_create: `world` ranks in this process, one host thread each (the one-GPU
    multi-rank harness of the native driver)."""

    def __init__(self, world: int):
        lw = ctypes.c_void_p(0)
        check(load().gsh_local_world_create(world, ctypes.byref(lw)), "gsh_local_world_create")
        self.ptr, self.world = lw.value, world

    def comm(self, rank: int) -> NativeComm:
        c = _lib.GshComm()
        check(load().gsh_comm_local(self.ptr, rank, ctypes.byref(c)), "gsh_comm_local")
        return NativeComm(c, owner=self, destroy=False)

    def close(self) -> None:
        if self.ptr:
            load().gsh_local_world_destroy(self.ptr)
            self.ptr = None


def nccl_comm(group=None, device=None, use_group_comm: bool = False) -> NativeComm:
    """An NCCL gsh_comm for this rank of `group` (default: the world).  use_group_comm=True wraps the
    process group's own ncclComm_t (gsh_comm_nccl; the group must be an initialised NCCL group);
    otherwise a new communicator is created (gsh_nccl_unique_id on the group's rank 0, broadcast over
    the group, gsh_comm_nccl_init on every rank)."""
    lib = load()
    pg = group if group is not None else dist.distributed_c10d._get_default_group()
    dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
    if use_group_comm:
        ptr = pg._get_backend(torch.device("cuda", dev.index))._comm_ptr()
        if not ptr:
            raise RuntimeError("the process group has no initialised NCCL communicator")
        c = _lib.GshComm()
        check(lib.gsh_comm_nccl(ptr, ctypes.byref(c)), "gsh_comm_nccl")
        return NativeComm(c)
    rank, world = dist.get_rank(pg), dist.get_world_size(pg)
    uid = (ctypes.c_uint8 * 128)()
    if rank == 0:
        check(lib.gsh_nccl_unique_id(uid), "gsh_nccl_unique_id")
    box = [bytes(uid)]
    dist.broadcast_object_list(box, src=dist.get_global_rank(pg, 0) if group is not None else 0, group=pg)
    uid = (ctypes.c_uint8 * 128).from_buffer_copy(box[0])
    c = _lib.GshComm()
    check(lib.gsh_comm_nccl_init(uid, world, rank, dev.index, ctypes.byref(c)), "gsh_comm_nccl_init")
    return NativeComm(c)


class ShardedJoin:
    """The native per-rank driver (gsh_sharded_create / gsh_join_sharded): the whole protocol of
    join_sharded -- agreement, routing, exchange, the two local joins, the reduction -- runs inside
    libgsh.so over the collectives of `comm`.  Buffers persist across calls (close() frees them)."""

    def __init__(self, comm: NativeComm, device=None):
        self.comm = comm
        self.device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        ctx = ctypes.c_void_p(0)
        check(load().gsh_sharded_create(ctypes.byref(comm.c), self.device.index, ctypes.byref(ctx)),
              "gsh_sharded_create")
        self.ctx = ctx.value

    def join(self, rk, rp, sk, sp, config=None, mode: str = "count", out=None, exchange: str = "p2p",
             stream=None) -> JoinResult:
        """This rank's shards in; the GLOBAL count / checksum out (identical on every rank); in
        "materialize" mode `out` ((capacity, 2) int32 CUDA tensor) receives this rank's pairs."""
        if exchange not in EXCHANGES:
            raise ValueError("exchange must be 'a2a' or 'p2p'")
        if mode not in ("count", "materialize"):
            raise ValueError("mode must be 'count' or 'materialize'")
        rk, rp = _check_dev(rk, "r_keys"), _check_dev(rp, "r_payloads")
        sk, sp = _check_dev(sk, "s_keys"), _check_dev(sp, "s_payloads")
        R, S = _rel(rk, rp, "R"), _rel(sk, sp, "S")
        o = None
        if mode == "materialize":
            if out is None or out.dim() != 2 or out.shape[1] != 2 or not out.is_cuda:
                raise ValueError("materialize needs out: a (capacity, 2) int32 CUDA tensor")
            o = _lib.GshOutput(out.data_ptr() if out.numel() else None, out.shape[0])
        res = _lib.GshShardedResult()
        st = load().gsh_join_sharded(self.ctx, ctypes.byref(R), ctypes.byref(S), int(mode == "materialize"),
                                     ctypes.byref(o) if o is not None else None,
                                     ctypes.byref(config) if config is not None else None, EXCHANGES[exchange],
                                     _stream_handle(stream, self.device), ctypes.byref(res))
        check(st, "gsh_join_sharded")
        w = int(res.written)
        stats = res.as_dict()
        stats.update(world=self.comm.world, rank=self.comm.rank, exchange=exchange, driver="native")
        for name, nbytes in (("exchange", int(res.exchange_bytes)), ("broadcast", int(res.broadcast_bytes))):
            ms = stats.get(f"ms_{name}", 0.0)
            gbs = nbytes / (ms * 1e6) if ms > 0 else None
            stats[f"{name}_GBps"] = gbs
            stats[f"{name}_nvlink_frac"] = gbs / NVLINK_GBS if gbs is not None else None
        return JoinResult(count=int(res.count), checksum=int(res.checksum), written=w, overflow=bool(res.overflow),
                          pairs=(out[:w] if mode == "materialize" else None), stats=stats)

    def close(self) -> None:
        if self.ctx:
            load().gsh_sharded_destroy(self.ctx)
            self.ctx = None


class LocalNativeRunner:
    """`world` logical ranks of the native driver on ONE device: a native local world, one
    ShardedJoin (persistent buffers) and one stream per rank; run() joins one set of shards with a
    host thread per rank (ctypes releases the GIL, so the ranks' protocol steps run concurrently)."""

    def __init__(self, world: int, device=None):
        self.world = world
        self.dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.lw = NativeLocalWorld(world)
        self.comms = [self.lw.comm(g) for g in range(world)]
        with torch.cuda.device(self.dev):
            self.drv = [ShardedJoin(c, self.dev) for c in self.comms]
            self.streams = [torch.cuda.Stream(self.dev) for _ in range(world)]

    def run(self, shards, config=None, mode: str = "count", outs=None, exchange: str = "p2p", configs=None):
        """shards[g] = (rk, rp, sk, sp) of rank g; outs[g]: rank g's (capacity, 2) output (materialize).
        Returns the per-rank JoinResults.  A failing rank aborts the world (the runner is then dead)."""
        res: list = [None] * self.world
        err: list = []
        ready = torch.cuda.Event()
        ready.record(torch.cuda.current_stream(self.dev))   # the shards are ready on the caller's stream

        def worker(g):
            try:
                with torch.cuda.device(self.dev), torch.cuda.stream(self.streams[g]):
                    self.streams[g].wait_event(ready)
                    cfg = configs[g] if configs is not None else config
                    res[g] = self.drv[g].join(*shards[g], config=cfg, mode=mode,
                                              out=outs[g] if outs is not None else None, exchange=exchange)
            except BaseException as e:  # noqa: BLE001  (the library aborted the world, or we do)
                err.append((g, e))
                self.comms[g].abort()

        th = [threading.Thread(target=worker, args=(g,)) for g in range(self.world)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        done = torch.cuda.current_stream(self.dev)
        for s in self.streams:
            done.wait_stream(s)
        if err:
            err.sort(key=lambda x: "peer rank failed" in str(x[1]))   # the root cause first
            raise err[0][1]
        return res

    def close(self) -> None:
        for d in self.drv:
            d.close()
        self.drv = []
        self.lw.close()


def run_local_native(world: int, shards, config=None, mode: str = "count", out_capacity: int = 0, device=None,
                     exchange: str = "p2p", repeat: int = 1, calls=None, configs=None):
    """The native driver for `world` logical ranks on ONE device (LocalNativeRunner).  shards[g] =
    (rk, rp, sk, sp) CUDA tensors of rank g; returns the per-rank JoinResults of the last of
    `repeat` calls (rank order).  calls: a list of such shard lists, joined one after another by the
    same per-rank drivers (buffer reuse and growth); the per-call results are then returned.
    configs: per-rank configs (default `config` everywhere)."""
    seq = list(calls) if calls is not None else [shards] * repeat
    dev = torch.device(device) if device is not None else seq[0][0][0].device
    runner = LocalNativeRunner(world, dev)
    try:
        outs = ([torch.empty((out_capacity, 2), dtype=torch.int32, device=dev) for _ in range(world)]
                if mode == "materialize" else None)
        got = [runner.run(sh, config=config, mode=mode, outs=outs, exchange=exchange, configs=configs) for sh in seq]
    finally:
        runner.close()
    return got if calls is not None else got[-1]


class _DevBytes:
    """A zero-copy uint8 view of raw device memory (CUDA array interface) for the callback comm."""

    def __init__(self, ptr: int, n: int):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (ptr, False), "version": 3,
                                         "strides": None}


def _dev_bytes(ptr, n: int) -> torch.Tensor:
    if n == 0:
        return torch.empty(0, dtype=torch.uint8, device="cuda")
    return torch.as_tensor(_DevBytes(int(ptr), int(n)), device="cuda")


_ALLRED = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p)
_ALLGATHER = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                              ctypes.c_void_p)
_P64 = ctypes.POINTER(ctypes.c_uint64)
_A2AV = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, _P64, _P64, ctypes.c_void_p, _P64, _P64,
                         ctypes.c_void_p)
_BARRIER = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p)


class TorchGroupComm(NativeComm):
    """A gsh_comm whose collectives are torch.distributed calls on `group` (any backend; payloads
    staged through host memory, so meant for gloo process groups, e.g. several processes sharing
    one GPU, where NCCL refuses to run).  The library calls back into Python for every collective;
    the peer-store exchange still shares its receive buffers through CUDA IPC."""

    def __init__(self, group=None):
        self.group = group
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        self._cbs = (_ALLRED(self._all_reduce), _ALLGATHER(self._all_gather), _A2AV(self._a2a),
                     _BARRIER(self._barrier))
        c = _lib.GshComm()
        c.rank, c.world, c.same_process = rank, world, 0
        c.ctx = None
        c.all_reduce_u64, c.all_gather, c.all_to_all_v, c.barrier = (ctypes.cast(f, ctypes.c_void_p) for f in self._cbs)
        super().__init__(c, destroy=False)

    @staticmethod
    def _sync(stream):
        torch.cuda.ExternalStream(int(stream or 0)).synchronize() if stream else torch.cuda.synchronize()

    def _guard(self, fn):
        try:
            fn()
            return _lib.GSH_OK
        except Exception:   # noqa: BLE001  (reported as a collective failure through the ABI)
            import traceback
            traceback.print_exc()
            return _lib.GSH_ERR_NCCL

    def _all_reduce(self, ctx, d, n, stream):
        def go():
            self._sync(stream)
            t = _dev_bytes(d, 8 * n)
            h = t.cpu().view(torch.int64)
            dist.all_reduce(h, group=self.group)
            t.copy_(h.view(torch.uint8))
            torch.cuda.synchronize()
        return self._guard(go)

    def _all_gather(self, ctx, send, recv, nbytes, stream):
        def go():
            self._sync(stream)
            src = _dev_bytes(send, nbytes).cpu()
            out = [torch.empty_like(src) for _ in range(self.c.world)]
            dist.all_gather(out, src, group=self.group)
            _dev_bytes(recv, nbytes * self.c.world).copy_(torch.cat(out))
            torch.cuda.synchronize()
        return self._guard(go)

    def _a2a(self, ctx, send, soff, sbytes, recv, roff, rbytes, stream):
        def go():
            self._sync(stream)
            G = self.c.world
            so, sb = [soff[g] for g in range(G)], [sbytes[g] for g in range(G)]
            ro, rbn = [roff[g] for g in range(G)], [rbytes[g] for g in range(G)]
            parts = [(_dev_bytes(send + so[g], sb[g]).cpu() if sb[g] else torch.empty(0, dtype=torch.uint8))
                     for g in range(G)]
            inp = torch.cat(parts)
            out = torch.empty(sum(rbn), dtype=torch.uint8)
            dist.all_to_all_single(out, inp, rbn, sb, group=self.group)
            o = 0
            for g in range(G):
                if rbn[g]:
                    _dev_bytes(recv + ro[g], rbn[g]).copy_(out[o: o + rbn[g]])
                o += rbn[g]
            torch.cuda.synchronize()
        return self._guard(go)

    def _barrier(self, ctx, stream):
        def go():
            self._sync(stream)
            dist.barrier(group=self.group)
        return self._guard(go)
