"""ctypes binding of libgsh.so (include/gsh.h).  Argument marshalling only.

The library is built in-tree by ``make`` (``__graft_entry__.build()``) into
``paper_conf_icde_caic24_b200/lib/libgsh.so``.  There is no fallback: if the library is
missing or cannot be loaded, importing the product API raises.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# GSH_LIB: experiments only (A/B builds of the same sources)
LIB_PATH = os.environ.get("GSH_LIB") or os.path.join(_HERE, "lib", "libgsh.so")
HEADER_PATH = os.path.join(os.path.dirname(_HERE), "include", "gsh.h")

u32 = ctypes.c_uint32
u64 = ctypes.c_uint64
i32 = ctypes.c_int32
vp = ctypes.c_void_p
p32 = ctypes.POINTER(ctypes.c_uint32)
p64 = ctypes.POINTER(ctypes.c_uint64)

GSH_OK, GSH_ERR_INVALID, GSH_ERR_NOMEM, GSH_ERR_CUDA, GSH_ERR_NCCL, GSH_ERR_INTERNAL = range(6)
GSH_OUT_COUNT, GSH_OUT_MATERIALIZE = 0, 1
GSH_EXCHANGE_A2A, GSH_EXCHANGE_P2P = 0, 1


class GshRelation(ctypes.Structure):
    _fields_ = [("keys", vp), ("payloads", vp), ("n", u64)]


class GshOutput(ctypes.Structure):
    _fields_ = [("pairs", vp), ("capacity", u64)]


class GshConfig(ctypes.Structure):
    _fields_ = [
        ("capacity", u32),
        ("pass_bits", i32 * 2),
        ("heavy_threshold", u32),
        ("route_bits", u32),
        ("force_all_normal", i32),
        ("force_all_heavy", i32),
        ("timing", i32),
        ("large_threshold", u32),
        ("nm_table", i32),
        ("detect_mode", i32),
        ("sample_stride", u32),
        ("top_k", u32),
        ("prepass_bits", i32),
        ("heavy_detail", i32),
        ("input_side_only", i32),
        ("hybrid", i32),
        ("hybrid_stride", u32),
        ("hybrid_min", u32),
        ("hybrid_share", u32),
    ]


class GshResult(ctypes.Structure):
    _fields_ = [
        ("count", u64),
        ("checksum", u64),
        ("written", u64),
        ("normal_count", u64),
        ("normal_checksum", u64),
        ("heavy_tuples_r", u64),
        ("heavy_tuples_s", u64),
        ("skew_pairs", u64),
        ("overflow", u32),
        ("n_heavy", u32),
        ("n_large", u32),
        ("detect_overflow", u32),
        ("pass_bits", u32 * 2),
        ("capacity", u32),
        ("heavy_threshold", u32),
        ("launches", u32),
        ("large_threshold", u32),
        ("nm_table", i32),
        ("ms_hist", ctypes.c_float),
        ("ms_pass1", ctypes.c_float),
        ("ms_pass2", ctypes.c_float),
        ("ms_detect", ctypes.c_float),
        ("ms_split", ctypes.c_float),
        ("ms_nmjoin", ctypes.c_float),
        ("ms_skewjoin", ctypes.c_float),
        ("ms_total", ctypes.c_float),
        ("prepass_bits", u32),
        ("ms_prepass", ctypes.c_float),
        ("large_tuples", u64),
        ("n_hybrid", u32),
        ("ms_sample", ctypes.c_float),
    ]

    def as_dict(self) -> dict:
        d = {}
        for name, _ in self._fields_:
            v = getattr(self, name)
            if name == "pass_bits":
                v = [int(v[0]), int(v[1])]
            d[name] = v
        return d


class GshShardParams(ctypes.Structure):
    _fields_ = [
        ("world", u32),
        ("route_bits", u32),
        ("part_bits", u32),
        ("large_threshold", u32),
        ("heavy_threshold", u32),
        ("cand_threshold", u32),
        ("force_all_normal", i32),
    ]


class GshComm(ctypes.Structure):
    """gsh_comm: a table of collectives (function pointers kept opaque: filled by the library's
    constructors gsh_comm_nccl / gsh_comm_nccl_init / gsh_comm_local)."""
    _fields_ = [("rank", u32), ("world", u32), ("same_process", u32), ("reserved", u32), ("ctx", vp),
                ("all_reduce_u64", vp), ("all_gather", vp), ("all_to_all_v", vp), ("barrier", vp), ("abort", vp)]


class GshShardedResult(ctypes.Structure):
    _fields_ = [
        ("count", u64), ("checksum", u64), ("written", u64), ("overflow", u32), ("n_heavy", u32),
        ("route_bits", u32), ("part_bits", u32), ("large_threshold", u32), ("heavy_threshold", u32),
        ("cand_threshold", u32), ("cand_overflow", u32), ("n_candidates", u64), ("n_union", u64),
        ("local_r", u64), ("local_s", u64), ("normal_r", u64), ("normal_s", u64), ("heavy_r", u64), ("heavy_s", u64),
        ("count_normal", u64), ("count_heavy", u64), ("exchange_bytes", u64), ("broadcast_bytes", u64),
        ("launches", u32), ("exchange", u32),
        ("ms_agree", ctypes.c_float), ("ms_route", ctypes.c_float), ("ms_exchange", ctypes.c_float),
        ("ms_join_heavy", ctypes.c_float), ("ms_join_normal", ctypes.c_float), ("ms_reduce", ctypes.c_float),
        ("ms_total", ctypes.c_float),
        ("normal", GshResult), ("heavy", GshResult),
    ]

    def as_dict(self) -> dict:
        d = {}
        for name, _ in self._fields_:
            v = getattr(self, name)
            d[name] = v.as_dict() if isinstance(v, GshResult) else v
        return d


# (name, restype, argtypes) for every entry point declared in include/gsh.h
_PROTOS = [
    ("gsh_config_default", None, [ctypes.POINTER(GshConfig)]),
    ("gsh_workspace_bytes", ctypes.c_size_t, [u64, u64, ctypes.POINTER(GshConfig)]),
    ("gsh_join", ctypes.c_int, [ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation), ctypes.c_int,
                                ctypes.POINTER(GshOutput), vp, ctypes.c_size_t, ctypes.POINTER(GshConfig), vp,
                                ctypes.POINTER(GshResult)]),
    ("gsh_gbase_workspace_bytes", ctypes.c_size_t, [u64, u64, ctypes.POINTER(GshConfig)]),
    ("gsh_join_gbase", ctypes.c_int, [ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation), ctypes.c_int,
                                      ctypes.POINTER(GshOutput), vp, ctypes.c_size_t, ctypes.POINTER(GshConfig), vp,
                                      ctypes.POINTER(GshResult)]),
    ("gsh_host_workspace_bytes", ctypes.c_size_t, [u64, u64, ctypes.c_int, u64, ctypes.POINTER(GshConfig)]),
    ("gsh_join_host", ctypes.c_int, [ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation), ctypes.c_int,
                                     ctypes.POINTER(GshOutput), vp, ctypes.c_size_t, ctypes.POINTER(GshConfig), vp,
                                     ctypes.POINTER(GshResult)]),
    ("gsh_heavy_detail", ctypes.c_int, [u64, u64, ctypes.POINTER(GshConfig), vp, ctypes.c_size_t, vp, p32, p32, p32,
                                        p64, u64, p64]),
    ("gsh_hash_keys", ctypes.c_int, [vp, vp, u64, vp]),
    ("gsh_radix_histogram", ctypes.c_int, [vp, u64, u32, u32, vp, vp, ctypes.c_size_t, vp]),
    ("gsh_partition", ctypes.c_int, [ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation),
                                     ctypes.POINTER(GshConfig), vp, ctypes.c_size_t, vp, vp, vp, vp, vp, p32]),
    ("gsh_detect", ctypes.c_int, [ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation),
                                  ctypes.POINTER(GshConfig), vp, ctypes.c_size_t, vp, p32, p32, p32, u64, p64,
                                  ctypes.POINTER(GshResult)]),
    ("gsh_shard_plan", ctypes.c_int, [u64, u64, u32, ctypes.POINTER(GshConfig), ctypes.POINTER(GshShardParams)]),
    ("gsh_shard_histogram", ctypes.c_int, [ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation),
                                           ctypes.POINTER(GshShardParams), vp, vp]),
    ("gsh_shard_workspace_bytes", ctypes.c_size_t, [u64, u64]),
    ("gsh_shard_candidates", ctypes.c_int, [ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation),
                                            ctypes.POINTER(GshShardParams), vp, vp, ctypes.c_size_t, vp, vp, u64,
                                            p64, p32]),
    ("gsh_shard_agree_workspace_bytes", ctypes.c_size_t, [u64]),
    ("gsh_shard_agree", ctypes.c_int, [vp, ctypes.c_size_t, vp, u32, u64, p64, vp, ctypes.c_size_t, vp, vp, vp, u64,
                                       p64]),
    ("gsh_shard_select", ctypes.c_int, [vp, vp, u64, ctypes.POINTER(GshShardParams), vp, ctypes.c_size_t, vp, vp, u64,
                                        p64]),
    ("gsh_heavy_set_bytes", ctypes.c_size_t, [u64]),
    ("gsh_heavy_set_build", ctypes.c_int, [vp, u64, vp, ctypes.c_size_t, vp]),
    ("gsh_route_count", ctypes.c_int, [vp, u64, u32, vp, ctypes.c_size_t, vp, vp]),
    ("gsh_route_scatter", ctypes.c_int, [vp, vp, u64, u32, vp, ctypes.c_size_t, vp, u32, vp, vp]),
    ("gsh_ipc_handle", ctypes.c_int, [vp, vp, p64]),
    ("gsh_ipc_open", ctypes.c_int, [vp, ctypes.POINTER(vp)]),
    ("gsh_ipc_close", ctypes.c_int, [vp]),
    ("gsh_comm_nccl", ctypes.c_int, [vp, ctypes.POINTER(GshComm)]),
    ("gsh_nccl_unique_id", ctypes.c_int, [vp]),
    ("gsh_comm_nccl_init", ctypes.c_int, [vp, u32, u32, ctypes.c_int, ctypes.POINTER(GshComm)]),
    ("gsh_comm_destroy", ctypes.c_int, [ctypes.POINTER(GshComm)]),
    ("gsh_local_world_create", ctypes.c_int, [u32, ctypes.POINTER(vp)]),
    ("gsh_comm_local", ctypes.c_int, [vp, u32, ctypes.POINTER(GshComm)]),
    ("gsh_local_world_destroy", ctypes.c_int, [vp]),
    ("gsh_sharded_create", ctypes.c_int, [ctypes.POINTER(GshComm), ctypes.c_int, ctypes.POINTER(vp)]),
    ("gsh_sharded_destroy", ctypes.c_int, [vp]),
    ("gsh_join_sharded", ctypes.c_int, [vp, ctypes.POINTER(GshRelation), ctypes.POINTER(GshRelation), ctypes.c_int,
                                        ctypes.POINTER(GshOutput), ctypes.POINTER(GshConfig), ctypes.c_int, vp,
                                        ctypes.POINTER(GshShardedResult)]),
    ("gsh_status_string", ctypes.c_char_p, [ctypes.c_int]),
    ("gsh_last_error", ctypes.c_char_p, []),
    ("gsh_version", ctypes.c_int, []),
    ("gsh_compiled_arch", ctypes.c_int, []),
]

EXPORTED = [name for name, _, _ in _PROTOS]

_lib = None


class GshError(RuntimeError):
    def __init__(self, status: int, where: str):
        lib = load()
        msg = f"{where}: {lib.gsh_status_string(status).decode()} ({lib.gsh_last_error().decode()})"
        super().__init__(msg)
        self.status = status


def load():
    """Load libgsh.so (raises OSError / FileNotFoundError if it is not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise FileNotFoundError(
                f"{LIB_PATH} not found: build the CUDA library first (python -c "
                "'import __graft_entry__ as g; g.build()' or `make`)")
        lib = ctypes.CDLL(LIB_PATH)
        for name, res, args in _PROTOS:
            fn = getattr(lib, name)
            fn.restype = res
            fn.argtypes = args
        _lib = lib
    return _lib


def check(status: int, where: str) -> None:
    if status != GSH_OK:
        raise GshError(status, where)


def default_config() -> GshConfig:
    cfg = GshConfig()
    load().gsh_config_default(ctypes.byref(cfg))
    return cfg
