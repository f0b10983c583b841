"""B200-native GSH: GPU Skew-conscious Hash join (Cai & Chen, ICDE 2024), sm_100a.

Public API (all GPU work runs in libgsh.so, include/gsh.h):
  join(...)            device-resident equi-join -> count, checksum, optional pairs
                       (impl="gbase": the paper's skew-unaware comparison system, same result)
  join_host(...)       end-to-end variant over host tensors
  make_config(...)     tuning / test hooks
  hash_keys, radix_histogram, partition, detect   -- single phases (parity tests)
  sharded.join_sharded -- multi-GPU hash sharding over torch.distributed (NCCL)
"""
from ._lib import GshError, LIB_PATH, load  # noqa: F401
from .join import (  # noqa: F401
    JoinResult,
    Workspace,
    detect,
    gbase_workspace_bytes,
    hash_keys,
    join,
    join_detail,
    join_host,
    make_config,
    partition,
    radix_histogram,
    workspace_bytes,
)

__version__ = "0.1.0"
