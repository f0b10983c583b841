"""Seeded synthetic workload generators shared by tests, smoke() and bench.py.

This module holds NO join arithmetic (no partition hash, no pair hash, no rule of the
method).  It only draws keys.  Both the CPU oracle and the CUDA path consume the arrays it
returns; it runs on any torch device and is bit-identical across devices (integer-only
sampling; the Zipf CDF is built once in float64 on the host and frozen into 63-bit
fixed-point thresholds).

Workload recipe (§V-A, SURVEY.md §8(c) readings #4-#6, #18):
  * Tuples are (u32 key, u32 payload), payload = row index (so payload == rid).
  * Zipf(theta) over ranks 1..N, p_k ∝ k^-theta, domain N = n by default (pinned by the
    1.79M top-key count of L59, see tests/test_datagen.py).  "an array of intervals" whose
    lengths are the probabilities (L132) -> inverse-CDF thresholds; "randomly assign a
    unique key to each interval" (L132) -> a seeded bijection rank -> u32 key; "generate
    a random number, and search it in the interval array" (L139) -> searchsorted.
  * R and S share the interval array and the rank -> key map (L139) but draw from
    independent counter-based RNG streams (R = 0, S = 1).
  * theta = 0 "1:1 PK-FK" (cfg2): R = n distinct keys, S key = R.key[uniform row].
  * Graph edges (cfg4): Zipf over vertex ranks, theta = 1/(gamma-1); src, dst iid.
"""
from .gen import (  # noqa: F401
    splitmix64,
    rand_u63,
    rank_to_key,
    zipf_thresholds,
    zipf_keys,
    zipf_relation,
    zipf_pair,
    pkfk_pair,
    uniform_pair,
    graph_pair,
    make_workload,
)
