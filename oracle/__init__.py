"""CPU oracle for the GSH equi-join -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything from this package.  The product path
(``paper_conf_icde_caic24_b200``) never imports it and shares no code with it: the C
oracle (``join_oracle.c``) and the numpy step references below carry their own copies
of every hash and rule.

Every function cites the passage it follows.  PAPER.md = /root/reference/PAPER.md
(Cai & Chen, "CPU and GPU Hash Joins on Skewed Data", ICDE 2024); SURVEY.md §8(c) holds
the readings where the paper is silent (listed again in DESIGN.md §3).

Pins (tests/test_oracle_*.py, all ``-m "not gpu"``):
  fmix32      SMHasher MurmurHash3_x86_32 published vectors (full hash rebuilt in the test)
  fmix64      inverse built from modular inverses of its constants (pow(c,-1,2**64));
              SURVEY §8(c) independent vectors
  pair_hash   inverse recovers (a<<32|b) -- pins operand order and salt
  join        brute-force nested loop; closed form sum_k cnt_R(k)*cnt_S(k) from
              np.unique histograms; metamorphic invariances; SURVEY §8(c) golden cases
  radix_histogram  pure-Python loop on small inputs; sum == n; PAPER.md L166 property
  heavy_rule  pure-Python dict counting on small inputs
No function here is "parity unpinned".
"""
from .oracle import (  # noqa: F401
    SALT,
    fmix32,
    fmix64,
    pair_hash,
    join,
    join_sorted_pairs,
    radix_digits,
    radix_histogram,
    heavy_rule,
    lib_path,
)
