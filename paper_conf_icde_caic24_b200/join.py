"""Python API of the B200 GSH join: thin marshalling over the C-ABI (include/gsh.h).

Every step of the join runs in libgsh.so's CUDA kernels; PyTorch only provides device
memory (the workspace and outputs come from torch's caching allocator) and the stream.
Inputs are CUDA tensors of dtype int32 (or uint32) holding u32 bit patterns.  There is
no CPU path: calling with CPU tensors raises.
"""
from __future__ import annotations

import ctypes
import threading

import torch

from . import _lib
from ._lib import GshConfig, GshOutput, GshRelation, GshResult, check, load


def make_config(capacity: int = 0, pass_bits=None, heavy_threshold: int = 0, route_bits: int = 0,
                force_all_normal: bool = False, force_all_heavy: bool = False, timing: bool = False,
                large_threshold: int = 0, nm_table: int = 0, detect_mode: int = 0, sample_stride: int = 0,
                top_k: int = 0, prepass_bits: int = 0, input_side_only: bool = False,
                heavy_detail: bool = False, hybrid: bool = False, hybrid_stride: int = 0,
                hybrid_min: int = 0, hybrid_share: int = 0) -> GshConfig:
    """Build a gsh_config (see include/gsh.h for each field's meaning)."""
    cfg = _lib.default_config()
    cfg.capacity = int(capacity)
    if pass_bits is not None:
        cfg.pass_bits[0] = int(pass_bits[0])
        cfg.pass_bits[1] = int(pass_bits[1])
    cfg.heavy_threshold = int(heavy_threshold)
    cfg.route_bits = int(route_bits)
    cfg.force_all_normal = int(bool(force_all_normal))
    cfg.force_all_heavy = int(bool(force_all_heavy))
    cfg.timing = int(bool(timing))
    cfg.large_threshold = int(large_threshold)
    cfg.nm_table = int(nm_table)
    cfg.detect_mode = int(detect_mode)
    cfg.sample_stride = int(sample_stride)
    cfg.top_k = int(top_k)
    cfg.prepass_bits = int(prepass_bits)
    cfg.input_side_only = int(bool(input_side_only))
    cfg.heavy_detail = int(bool(heavy_detail))
    cfg.hybrid = int(bool(hybrid))
    cfg.hybrid_stride = int(hybrid_stride)
    cfg.hybrid_min = int(hybrid_min)
    cfg.hybrid_share = int(hybrid_share)
    return cfg


class JoinResult:
    """count, checksum (mod 2^64), written, overflow, pairs ((written, 2) int32 view of
    (payload_R, payload_S) or None) and stats (every gsh_result field, built on first access)."""

    __slots__ = ("count", "checksum", "written", "overflow", "pairs", "_stats", "_raw")

    def __init__(self, count: int, checksum: int, written: int = 0, overflow: bool = False,
                 pairs: torch.Tensor | None = None, stats: dict | None = None, raw=None):
        self.count, self.checksum, self.written, self.overflow, self.pairs = count, checksum, written, overflow, pairs
        self._stats, self._raw = stats, raw

    @property
    def stats(self) -> dict:
        if self._stats is None:
            self._stats = self._raw.as_dict() if self._raw is not None else {}
        return self._stats

    def __repr__(self) -> str:
        return (f"JoinResult(count={self.count}, checksum={self.checksum:#x}, written={self.written}, "
                f"overflow={self.overflow})")


def _check_dev(t: torch.Tensor, name: str) -> torch.Tensor:
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor (the GSH join has no CPU path)")
    if t.dtype not in (torch.int32, torch.uint32):
        raise TypeError(f"{name} must be int32/uint32, got {t.dtype}")
    if t.dim() != 1:
        raise ValueError(f"{name} must be 1-D")
    return t.contiguous()


def _rel(keys: torch.Tensor, pays: torch.Tensor, side: str) -> GshRelation:
    if keys.numel() != pays.numel():
        raise ValueError(f"{side}: keys and payloads differ in length")
    return GshRelation(keys.data_ptr() if keys.numel() else None, pays.data_ptr() if pays.numel() else None,
                       keys.numel())


def _stream_handle(stream, device=None) -> int | None:
    """cudaStream_t of `stream`; None = torch's current stream of `device` (per thread)."""
    if stream is None:
        return torch.cuda.current_stream(device).cuda_stream
    if isinstance(stream, torch.cuda.Stream):
        return stream.cuda_stream
    return int(stream)


class Workspace:
    """Grow-only device scratch buffer (torch caching allocator), one per (device, thread): calls
    from several host threads (e.g. logical ranks sharing a GPU) never share scratch."""

    def __init__(self):
        self._tls = threading.local()

    def get(self, nbytes: int, device: torch.device) -> torch.Tensor:
        idx = device.index if device.index is not None else torch.cuda.current_device()
        bufs = getattr(self._tls, "bufs", None)
        if bufs is None:
            bufs = self._tls.bufs = {}
        b = bufs.get(idx)
        if b is None or b.numel() < nbytes:
            bufs.pop(idx, None)
            b = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=torch.device("cuda", idx))
            bufs[idx] = b
        return b


_default_ws = Workspace()


def workspace_bytes(n_r: int, n_s: int, config: GshConfig | None = None) -> int:
    lib = load()
    nb = lib.gsh_workspace_bytes(n_r, n_s, ctypes.byref(config) if config is not None else None)
    if nb == 0:
        raise ValueError("invalid gsh_config")
    return int(nb)


def gbase_workspace_bytes(n_r: int, n_s: int, config: GshConfig | None = None) -> int:
    """Device workspace of the Gbase-style join (gsh_gbase_workspace_bytes: its bucket pools)."""
    nb = load().gsh_gbase_workspace_bytes(n_r, n_s, ctypes.byref(config) if config is not None else None)
    if nb == 0:
        raise ValueError("invalid gsh_config or more than 2^28 tuples per side")
    return int(nb)


def join(r_keys: torch.Tensor, r_payloads: torch.Tensor, s_keys: torch.Tensor, s_payloads: torch.Tensor,
         mode: str = "count", out: torch.Tensor | None = None, out_capacity: int | None = None,
         config: GshConfig | None = None, stream=None, workspace: torch.Tensor | None = None,
         impl: str = "gsh") -> JoinResult:
    """GSH equi-join of device-resident R and S (gsh_join, include/gsh.h).

    mode: "count" (count + checksum) or "materialize" (also (payload_R, payload_S) pairs into
    `out`, an int32 CUDA tensor of shape (capacity, 2), or a fresh one of out_capacity rows).
    impl: "gsh" (gsh_join) or "gbase" (gsh_join_gbase: the paper's skew-unaware comparison system,
    same result, for the GSH-vs-Gbase measurement).
    """
    if impl not in ("gsh", "gbase"):
        raise ValueError("impl must be 'gsh' or 'gbase'")
    lib = load()
    rk, rp = _check_dev(r_keys, "r_keys"), _check_dev(r_payloads, "r_payloads")
    sk, sp = _check_dev(s_keys, "s_keys"), _check_dev(s_payloads, "s_payloads")
    dev = rk.device
    R, S = _rel(rk, rp, "R"), _rel(sk, sp, "S")
    mat = mode == "materialize"
    if mode not in ("count", "materialize"):
        raise ValueError("mode must be 'count' or 'materialize'")
    outp = None
    if mat:
        if out is None:
            if out_capacity is None:
                raise ValueError("materialize needs out or out_capacity")
            out = torch.empty((int(out_capacity), 2), dtype=torch.int32, device=dev)
        if not out.is_cuda or out.dtype not in (torch.int32, torch.uint32) or out.dim() != 2 or out.shape[1] != 2:
            raise ValueError("out must be a CUDA int32 tensor of shape (capacity, 2)")
        if not out.is_contiguous():
            raise ValueError("out must be contiguous")
        outp = GshOutput(out.data_ptr() if out.numel() else None, out.shape[0])
    if workspace is not None:   # gsh_join itself rejects a too-small workspace (GSH_ERR_INVALID)
        ws = workspace
    else:
        nb = workspace_bytes(R.n, S.n, config) if impl == "gsh" else gbase_workspace_bytes(R.n, S.n, config)
        ws = _default_ws.get(nb, dev)
    res = GshResult()
    args = (ctypes.byref(R), ctypes.byref(S), _lib.GSH_OUT_MATERIALIZE if mat else _lib.GSH_OUT_COUNT,
            ctypes.byref(outp) if outp is not None else None, ws.data_ptr(), ws.numel(),
            ctypes.byref(config) if config is not None else None, _stream_handle(stream, dev), ctypes.byref(res))
    fn = lib.gsh_join if impl == "gsh" else lib.gsh_join_gbase
    if dev.index == torch.cuda.current_device():
        st = fn(*args)
    else:
        with torch.cuda.device(dev):
            st = fn(*args)
    check(st, "gsh_join" if impl == "gsh" else "gsh_join_gbase")
    return JoinResult(count=int(res.count), checksum=int(res.checksum), written=int(res.written),
                      overflow=bool(res.overflow), pairs=(out[: res.written] if mat else None), raw=res)


def join_host(r_keys, r_payloads, s_keys, s_payloads, mode: str = "count", out=None, out_capacity=None,
              config: GshConfig | None = None, device=None, stream=None,
              workspace: torch.Tensor | None = None) -> JoinResult:
    """End-to-end join of HOST tensors (gsh_join_host): H2D copy, join, D2H of the pairs.

    Inputs are CPU int32 tensors (pin_memory() for full bandwidth).  The device workspace is
    allocated on `device` (default: current CUDA device)."""
    lib = load()
    t = [r_keys, r_payloads, s_keys, s_payloads]
    for x in t:
        if not isinstance(x, torch.Tensor) or x.is_cuda or x.dtype not in (torch.int32, torch.uint32):
            raise TypeError("join_host takes CPU int32 tensors")
    rk, rp, sk, sp = (x.contiguous() for x in t)
    R, S = _rel(rk, rp, "R"), _rel(sk, sp, "S")
    mat = mode == "materialize"
    dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    outp = None
    cap = 0
    if mat:
        if out is None:
            out = torch.empty((int(out_capacity), 2), dtype=torch.int32, pin_memory=True)
        cap = out.shape[0]
        outp = GshOutput(out.data_ptr() if out.numel() else None, cap)
    nb = lib.gsh_host_workspace_bytes(R.n, S.n, 1 if mat else 0, cap,
                                      ctypes.byref(config) if config is not None else None)
    if nb == 0:
        raise ValueError("invalid gsh_config")
    ws = workspace if workspace is not None else _default_ws.get(int(nb), dev)
    res = GshResult()
    with torch.cuda.device(dev):
        st = lib.gsh_join_host(ctypes.byref(R), ctypes.byref(S), 1 if mat else 0,
                               ctypes.byref(outp) if outp is not None else None, ws.data_ptr(), ws.numel(),
                               ctypes.byref(config) if config is not None else None, _stream_handle(stream, dev),
                               ctypes.byref(res))
    check(st, "gsh_join_host")
    return JoinResult(count=int(res.count), checksum=int(res.checksum), written=int(res.written),
                      overflow=bool(res.overflow), pairs=(out[: res.written] if mat else None), raw=res)


# ------------------------------------------------------------------ step entry points
def hash_keys(keys: torch.Tensor, stream=None) -> torch.Tensor:
    """fmix32 of every key (gsh_hash_keys) -> int32 CUDA tensor."""
    lib = load()
    k = _check_dev(keys, "keys")
    out = torch.empty_like(k, dtype=torch.int32)
    with torch.cuda.device(k.device):
        check(lib.gsh_hash_keys(k.data_ptr() if k.numel() else None, out.data_ptr() if k.numel() else None,
                                k.numel(), _stream_handle(stream, k.device)), "gsh_hash_keys")
    return out


def radix_histogram(keys: torch.Tensor, hi_bits: int, nbits: int, stream=None) -> torch.Tensor:
    """Histogram of radix digits of fmix32(key) (gsh_radix_histogram) -> int64 tensor."""
    lib = load()
    k = _check_dev(keys, "keys")
    hist = torch.zeros(1 << nbits, dtype=torch.int64, device=k.device)
    with torch.cuda.device(k.device):
        check(lib.gsh_radix_histogram(k.data_ptr() if k.numel() else None, k.numel(), hi_bits, nbits,
                                      hist.data_ptr(), None, 0, _stream_handle(stream, k.device)), "gsh_radix_histogram")
    return hist


def partition(r_keys, r_payloads, s_keys, s_payloads, config: GshConfig | None = None, stream=None):
    """Partition phase only (gsh_partition).  Returns (part_r, part_s, off_r, off_s, (b1, b2)) where
    part_* are (n, 2) int32 tensors of (h, payload) grouped by partition and off_* int64 starts."""
    lib = load()
    rk, rp = _check_dev(r_keys, "r_keys"), _check_dev(r_payloads, "r_payloads")
    sk, sp = _check_dev(s_keys, "s_keys"), _check_dev(s_payloads, "s_payloads")
    dev = rk.device
    R, S = _rel(rk, rp, "R"), _rel(sk, sp, "S")
    nb = workspace_bytes(R.n, S.n, config)
    ws = _default_ws.get(nb, dev)
    # F is only known inside the library: size the offsets for the maximum fanout
    off_r = torch.zeros((1 << 16) + 1, dtype=torch.int64, device=dev)
    off_s = torch.zeros((1 << 16) + 1, dtype=torch.int64, device=dev)
    part_r = torch.empty((max(R.n, 1), 2), dtype=torch.int32, device=dev)
    part_s = torch.empty((max(S.n, 1), 2), dtype=torch.int32, device=dev)
    bits = (ctypes.c_uint32 * 2)()
    with torch.cuda.device(dev):
        check(lib.gsh_partition(ctypes.byref(R), ctypes.byref(S), ctypes.byref(config) if config is not None else None,
                                ws.data_ptr(), ws.numel(), _stream_handle(stream, dev), part_r.data_ptr(),
                                part_s.data_ptr(), off_r.data_ptr(), off_s.data_ptr(), bits), "gsh_partition")
    F = 1 << (bits[0] + bits[1])
    return part_r[: R.n], part_s[: S.n], off_r[: F + 1], off_s[: F + 1], (int(bits[0]), int(bits[1]))


def detect(r_keys, r_payloads, s_keys, s_payloads, config: GshConfig | None = None, stream=None, cap: int = 1 << 22):
    """Partition + skew detection (gsh_detect).  Returns (h, cnt_r, cnt_s, stats) as int64 CPU
    tensors sorted by h (h = fmix32 of each skewed key, as u32 values)."""
    lib = load()
    rk, rp = _check_dev(r_keys, "r_keys"), _check_dev(r_payloads, "r_payloads")
    sk, sp = _check_dev(s_keys, "s_keys"), _check_dev(s_payloads, "s_payloads")
    dev = rk.device
    R, S = _rel(rk, rp, "R"), _rel(sk, sp, "S")
    nb = workspace_bytes(R.n, S.n, config)
    ws = _default_ws.get(nb, dev)
    hk = (ctypes.c_uint32 * cap)()
    cr = (ctypes.c_uint32 * cap)()
    cs = (ctypes.c_uint32 * cap)()
    n = ctypes.c_uint64(0)
    res = GshResult()
    with torch.cuda.device(dev):
        check(lib.gsh_detect(ctypes.byref(R), ctypes.byref(S), ctypes.byref(config) if config is not None else None,
                             ws.data_ptr(), ws.numel(), _stream_handle(stream, dev), hk, cr, cs, cap, ctypes.byref(n),
                             ctypes.byref(res)), "gsh_detect")
    m = int(n.value)
    h = torch.tensor(list(hk[:m]), dtype=torch.int64)
    a = torch.tensor(list(cr[:m]), dtype=torch.int64)
    b = torch.tensor(list(cs[:m]), dtype=torch.int64)
    order = torch.argsort(h)
    return h[order], a[order], b[order], res.as_dict()


def join_detail(r_keys, r_payloads, s_keys, s_payloads, config: GshConfig | None = None, stream=None):
    """COUNT join with the skewed-key decomposition (gsh_config.heavy_detail +
    gsh_heavy_detail): returns (JoinResult, detail) where detail = dict of int64 CPU tensors
    h, cnt_r, cnt_s and uint64-valued checksum (C_k as Python ints in a list), one entry per
    skewed key.  result.count == normal_count + sum(cnt_r * cnt_s) and result.checksum ==
    normal_checksum + sum(C_k) mod 2^64."""
    lib = load()
    cfg = make_config(heavy_detail=True) if config is None else config
    cfg.heavy_detail = 1
    rk, rp = _check_dev(r_keys, "r_keys"), _check_dev(r_payloads, "r_payloads")
    sk, sp = _check_dev(s_keys, "s_keys"), _check_dev(s_payloads, "s_payloads")
    dev = rk.device
    ws = torch.empty(workspace_bytes(rk.numel(), sk.numel(), cfg), dtype=torch.uint8, device=dev)
    r = join(rk, rp, sk, sp, config=cfg, stream=stream, workspace=ws)
    cap = max(1, int(r.stats["n_heavy"]))
    hk, cr, cs = (ctypes.c_uint32 * cap)(), (ctypes.c_uint32 * cap)(), (ctypes.c_uint32 * cap)()
    ck = (ctypes.c_uint64 * cap)()
    n = ctypes.c_uint64(0)
    with torch.cuda.device(dev):
        check(lib.gsh_heavy_detail(rk.numel(), sk.numel(), ctypes.byref(cfg), ws.data_ptr(), ws.numel(),
                                   _stream_handle(stream, dev), hk, cr, cs, ck, cap, ctypes.byref(n)), "gsh_heavy_detail")
    m = int(n.value)
    detail = {"h": torch.tensor(list(hk[:m]), dtype=torch.int64), "cnt_r": torch.tensor(list(cr[:m]), dtype=torch.int64),
              "cnt_s": torch.tensor(list(cs[:m]), dtype=torch.int64), "checksum": [int(x) for x in ck[:m]]}
    return r, detail
