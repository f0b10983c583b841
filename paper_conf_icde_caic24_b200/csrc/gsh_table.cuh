// gsh_table.cuh -- global-memory open-addressing tables keyed by h = fmix32(key).
//
// Slots hold (1 << 32 | h) so every u32 h is a legal key (0 marks an empty slot); linear
// probing from a multiplicative slot, bounded by kDetectMaxProbe (a table that fills degrades to
// "not found / overflow", never to an unbounded probe).  Used by skew detection (PAPER.md L107,
// "linear probing based hash table") and by the multi-GPU skew agreement.
#pragma once
#include <cstdint>

#include "gsh_internal.h"

namespace gsh {

__device__ __forceinline__ uint32_t gt_slot0(uint32_t h, uint32_t logcap) {
    return (h * 0x9E3779B1u) >> (32 - logcap);
}

// Insert-or-find h; returns slot or kNoHeavy when the probe budget is exhausted.
__device__ __forceinline__ uint32_t gt_insert(unsigned long long* keys, uint32_t h, uint32_t logcap) {
    const unsigned long long tag = (1ull << 32) | h;
    const uint32_t mask = (1u << logcap) - 1;
    uint32_t slot = gt_slot0(h, logcap);
    for (int probe = 0; probe < kDetectMaxProbe; ++probe) {
        unsigned long long cur = keys[slot];
        if (cur == tag) return slot;
        if (cur == 0) {
            unsigned long long prev = atomicCAS(&keys[slot], 0ull, tag);
            if (prev == 0 || prev == tag) return slot;
        }
        slot = (slot + 1) & mask;
    }
    return kNoHeavy;
}

__device__ __forceinline__ uint32_t gt_find(const unsigned long long* keys, uint32_t h, uint32_t logcap) {
    const unsigned long long tag = (1ull << 32) | h;
    const uint32_t mask = (1u << logcap) - 1;
    uint32_t slot = gt_slot0(h, logcap);
    for (int probe = 0; probe < kDetectMaxProbe; ++probe) {
        unsigned long long cur = keys[slot];
        if (cur == tag) return slot;
        if (cur == 0) return kNoHeavy;
        slot = (slot + 1) & mask;
    }
    return kNoHeavy;
}

inline uint32_t log2_pow2(uint64_t x) {
    uint32_t l = 0;
    while ((1ull << l) < x) ++l;
    return l;
}

}  // namespace gsh
