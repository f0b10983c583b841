#!/usr/bin/env python
"""Regenerate tests/golden/survey_tiny_cases.json by brute force in plain Python integers.

Independent of oracle/ and of the CUDA path: the MurmurHash3 finalizers and the salted pair hash
are restated from their definitions (R2), and the join is a nested
loop over the literal inputs of SURVEY §8(c) P0.  The values must equal the survey author's
independent ones already committed (tests/test_oracle.py checks the oracle against them;
tests/test_golden_script.py checks this script against the file).

  python scripts/make_golden.py          # print the JSON
  python scripts/make_golden.py --write  # rewrite tests/golden/survey_tiny_cases.json
"""
import json
import os
import sys

M32, M64 = (1 << 32) - 1, (1 << 64) - 1
SALT = 0x9E3779B97F4A7C15
GOLDEN = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests", "golden",
                      "survey_tiny_cases.json")


def fmix32(h):
    """MurmurHash3 32-bit finalizer (the partition / identity hash h of SURVEY §8 notation)."""
    h ^= h >> 16
    h = (h * 0x85EBCA6B) & M32
    h ^= h >> 13
    h = (h * 0xC2B2AE35) & M32
    h ^= h >> 16
    return h


def fmix64(k):
    """MurmurHash3 64-bit finalizer."""
    k ^= k >> 33
    k = (k * 0xFF51AFD7ED558CCD) & M64
    k ^= k >> 33
    k = (k * 0xC4CEB9FE1A85EC53) & M64
    k ^= k >> 33
    return k


def pair_hash(a, b):
    """Checksum term of the result tuple (payload_R = a, payload_S = b): DESIGN.md R2."""
    return fmix64(((a << 32) | b) ^ SALT)


def nested_loop_join(R, S):
    """M = {(pR, pS) : kR == kS} by definition (§III)."""
    pairs = [(pr, ps) for kr, pr in R for ks, ps in S if kr == ks]
    return pairs, len(pairs), sum(pair_hash(a, b) for a, b in pairs) & M64


def build():
    R = [[5, 0], [7, 1], [5, 2], [4294967295, 3]]
    S = [[5, 10], [9, 11], [5, 12], [7, 13], [4294967295, 14], [0, 15]]
    pairs, cnt, chk = nested_loop_join(R, S)
    Ra = [[0, i] for i in range(100)]
    Sa = [[0, j] for j in range(200)]
    _, cnt_a, chk_a = nested_loop_join(Ra, Sa)
    return {
        "_source": "SURVEY.md §8(c) P0 golden tiny cases and test vectors, computed by the survey author's "
                   "independent throwaway script (/tmp/survey, not part of this repo). The paper (PAPER.md) prints "
                   "no worked example; these are an independent implementation's values of the definitions in "
                   "SURVEY §8(c).",
        "tiny": {"R": R, "S": S, "pairs": sorted([list(p) for p in pairs]), "count": cnt, "checksum": hex(chk)},
        "all_equal": {"nR": 100, "nS": 200, "key": 0, "count": cnt_a, "checksum": hex(chk_a)},
        "fmix32": {str(x): hex(fmix32(x)) for x in (0, 1, 4294967295)},
        "pair_hash": [[a, b, hex(pair_hash(a, b))] for a, b in ((0, 0), (0, 1), (1, 0), (M32, M32))],
    }


def main():
    g = build()
    if "--write" in sys.argv:
        with open(GOLDEN, "w") as f:
            json.dump(g, f, indent=2)
            f.write("\n")
    else:
        print(json.dumps(g, indent=2))


if __name__ == "__main__":
    main()
