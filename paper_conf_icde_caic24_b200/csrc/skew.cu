// skew.cu -- GSH phases (2) and (3) (§IV-B), SURVEY.md §8(a) rows a5-a7.
//
//   a5 k_classify : "identify normal vs. large partitions by comparing the partition size with
//                   a pre-defined threshold" (L107).  large(p) <=> |R_p| > L or |S_p| > L
//                   (and both sides non-empty: a partition with an empty side yields nothing).
//   a6 k_detect   : exact per-key counts of every key of every large partition, both sides.
//                   Warp aggregation with __match_any_sync collapses a skewed key's tuples to
//                   one update per warp; counts live in an open-addressing table keyed by
//                   h = fmix32(key) (the paper's "linear probing based hash table", L107/L112,
//                   fed with all tuples instead of a 1 % sample -- DESIGN.md §3 reading R3).
//      k_select   : threshold pass compacting skewed keys into the side list H (L112 top-k,
//                   reading R4: max(cnt_R, cnt_S) >= T_h inside a large partition).
//   a7 k_split    : "checks each R tuple against the skewed keys.  If the tuple is skewed, it
//                   is appended to an array allocated for the associated skewed key ...
//                   Otherwise ... appends the tuple to a normal partition" (L114); same for S.
//                   Skewed arrays hold payloads only (every tuple of R_k has key k).
#include "gsh_device.cuh"
#include "gsh_internal.h"
#include "gsh_scan.cuh"
#include "gsh_table.cuh"

namespace gsh {

__device__ __forceinline__ uint32_t part_of(uint32_t h, uint32_t shift, uint32_t mask) {
    return (h >> shift) & mask;
}

// ------------------------------------------------------------------ a5: classify --
__global__ void k_classify(const uint32_t* __restrict__ cnt, uint32_t F, uint32_t L, int force_normal,
                           int force_heavy, uint32_t* __restrict__ large_list, uint32_t* __restrict__ large_idx,
                           uint32_t* __restrict__ part_heavy, DevState* st) {
    for (uint32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < F; p += gridDim.x * blockDim.x) {
        const uint32_t cr = cnt[p], cs = cnt[F + p];
        part_heavy[p] = 0;
        part_heavy[F + p] = 0;
        if (cs > 0 && cr > 0) atomicMax(&st->max_rlen, cr);
        const bool large = (cr > 0 && cs > 0) && !force_normal && (force_heavy || cr > L || cs > L);
        uint32_t idx = kNoHeavy;
        if (large) {
            idx = atomicAdd(&st->n_large, 1u);
            large_list[idx] = p;
            atomicAdd(&st->large_tuples[0], (unsigned long long)cr);
            atomicAdd(&st->large_tuples[1], (unsigned long long)cs);
        }
        large_idx[p] = idx;
    }
}

int launch_classify(const Plan& p, cudaStream_t s) {
    unsigned grid = (p.F + 255) / 256;
    k_classify<<<grid, 256, 0, s>>>(p.cnt, p.F, p.L, p.force_normal, p.force_heavy, p.large_list, p.large_idx,
                                    p.part_heavy, p.st);
    return 1;
}

// Work items of detect / split: ceil((|R_p| + |S_p|) / chunk) per large partition, never spanning
// two partitions.  Detect uses kDetectItem-tuple items (one shared-memory count table flush per
// item), split kDetectChunk-tuple items (every tuple held in registers across its two phases).

struct DetectItems {
    const uint32_t* cnt;
    const uint32_t* large_list;
    uint32_t F, chunk;
    __device__ uint64_t operator()(uint64_t i) const {
        uint32_t p = large_list[i];
        uint64_t t = uint64_t(cnt[p]) + cnt[F + p];
        return (t + chunk - 1) / chunk;
    }
};

// item -> large partition index, one thread per item (a binary search over the item prefix, done
// once here instead of by every thread of every claiming CTA: ~16 dependent loads per item)
__global__ void k_item_map(const uint64_t* __restrict__ prefix, uint32_t n_large, uint64_t bound,
                           uint32_t* __restrict__ item_li) {
    const uint64_t total = prefix[n_large];
    for (uint64_t it = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; it < umin64(total, bound);
         it += uint64_t(gridDim.x) * blockDim.x) {
        uint32_t lo = 0, hi = n_large;
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (prefix[mid] <= it) lo = mid; else hi = mid;
        }
        item_li[it] = lo;
    }
}

uint64_t detect_items_bound(uint64_t large_tuples, uint32_t n_large, uint32_t chunk) {
    return large_tuples / chunk + n_large + 1;
}

int launch_detect_prefix(const Plan& p, uint32_t n_large, uint64_t large_tuples, cudaStream_t s) {
    int l = launch_scan(DetectItems{p.cnt, p.large_list, p.F, kDetectChunk}, n_large, p.det_prefix, p.scan_scratch, s) +
            launch_scan(DetectItems{p.cnt, p.large_list, p.F, kDetectItem}, n_large, p.det_prefix2, p.scan_scratch, s);
    const uint64_t b1 = umin64(detect_items_bound(large_tuples, n_large, kDetectChunk), p.item_cap);
    const uint64_t b2 = umin64(detect_items_bound(large_tuples, n_large, kDetectItem), p.item_cap2);
    k_item_map<<<(unsigned)umin64((b1 + 255) / 256, uint64_t(p.num_sms) * 16), 256, 0, s>>>(p.det_prefix, n_large, b1,
                                                                                             p.item_li);
    k_item_map<<<(unsigned)umin64((b2 + 255) / 256, uint64_t(p.num_sms) * 16), 256, 0, s>>>(p.det_prefix2, n_large, b2,
                                                                                             p.item_li2);
    return l + 2;
}

struct LargeView {
    const uint2* part[2];     // final partitions (bufB)
    const uint64_t* start;    // [2][F + 1]
    const uint32_t* cnt;      // [2][F]
    const uint32_t* large_list;
    const uint64_t* det_prefix;
    uint32_t F, n_large, chunk;
    const uint32_t* item_li;   // item -> large partition index (k_item_map)
};

// The element range of one item: tuples [e0, e1) of the concatenation R_p ++ S_p.
struct ItemRange {
    uint32_t li, p, cr, cs;
    uint64_t e0, e1;
};

__device__ __forceinline__ ItemRange item_range(const LargeView& v, uint64_t it) {
    ItemRange r;
    r.li = v.item_li[it];
    r.p = v.large_list[r.li];
    r.cr = v.cnt[r.p];
    r.cs = v.cnt[v.F + r.p];
    uint64_t c = it - v.det_prefix[r.li];
    r.e0 = c * v.chunk;
    r.e1 = umin64(r.e0 + v.chunk, uint64_t(r.cr) + r.cs);
    return r;
}

__device__ __forceinline__ uint2 item_tuple(const LargeView& v, const ItemRange& r, uint64_t e, int& side) {
    side = e >= r.cr;
    uint64_t off = side ? (e - r.cr) : e;
    return v.part[side][v.start[size_t(side) * (v.F + 1) + r.p] + off];
}

// ------------------------------------------------------------------- a6: detect --
constexpr int kDetBlock = 256;

// FIND: count only keys already in the table (detect_mode 1: the sampled top-k keys).
template <bool FIND>
__global__ void __launch_bounds__(kDetBlock) k_detect(LargeView v, unsigned long long* gt_key, uint32_t* gt_cnt,
                                                     uint32_t cap_alloc, uint32_t logcap, DevState* st,
                                                     unsigned int* claim) {
    __shared__ unsigned int s_it;
    const uint64_t total = v.det_prefix[v.n_large];
    for (;;) {
        if (threadIdx.x == 0) s_it = atomicAdd(claim, 1u);
        __syncthreads();
        const uint64_t it = s_it;
        __syncthreads();
        if (it >= total) break;
        const ItemRange r = item_range(v, it);
        for (uint64_t base = r.e0; base < r.e1; base += kDetBlock) {
            const uint64_t e = base + threadIdx.x;
            const bool valid = e < r.e1;
            int side = 0;
            uint32_t h = 0;
            if (valid) h = item_tuple(v, r, e, side).x;
            const unsigned long long key = valid ? ((uint64_t(side) << 32) | h) : ((2ull << 32) | lane_id());
            const uint32_t peers = __match_any_sync(kFull, key);
            if (valid && (peers & lanemask_lt()) == 0) {
                const uint32_t slot = FIND ? gt_find(gt_key, h, logcap) : gt_insert(gt_key, h, logcap);
                if (slot == kNoHeavy) {
                    if (!FIND) st->detect_overflow = 1;
                } else {
                    atomicAdd(&gt_cnt[size_t(side) * cap_alloc + slot], (uint32_t)__popc(peers));
                }
            }
        }
    }
}

// Exact detection (detect_mode 0): per-item shared-memory count tables.  A CTA claims
// an item (<= kDetectItem tuples of ONE large partition), counts every key of it in a shared-memory
// linear-probing table keyed by h (0 marks an empty slot; the key with h = 0 has its own counters),
// then merges each distinct key ONCE into the global table -- a skewed key costs one global atomic
// per item instead of one per warp.  Every key lives in exactly one partition, so when the whole
// partition is this one item its counts are exact and only keys reaching T_h are merged (the rest
// are normal, and "not in the table" means normal to split and select); keys of partitions spanning
// several items are all merged.  A key that finds no shared slot within kDetSmemProbe goes to the
// global table directly (exact either way).
constexpr uint32_t kDetSmemSlots = 6144;   // 72 KB: three CTAs per SM
constexpr int kDetSmemProbe = 32;
constexpr size_t kDetSmemBytes = size_t(kDetSmemSlots) * 12;

__global__ void __launch_bounds__(kDetBlock, 3) k_detect_smem(LargeView v, unsigned long long* gt_key, uint32_t* gt_cnt,
                                                          uint32_t cap_alloc, uint32_t logcap, uint32_t Th,
                                                          int force_heavy, DevState* st, unsigned int* claim) {
    extern __shared__ uint32_t det_dyn[];
    uint32_t* s_key = det_dyn;                  // h, 0 = empty
    uint32_t* s_cr = det_dyn + kDetSmemSlots;
    uint32_t* s_cs = s_cr + kDetSmemSlots;
    __shared__ uint32_t s_zero[2];              // counts of the key with h = 0
    __shared__ unsigned int s_it;
    for (uint32_t i = threadIdx.x; i < kDetSmemSlots; i += kDetBlock) {
        s_key[i] = 0;
        s_cr[i] = 0;
        s_cs[i] = 0;
    }
    if (threadIdx.x < 2) s_zero[threadIdx.x] = 0;
    const uint64_t total = v.det_prefix[v.n_large];
    auto merge = [&](uint32_t h, uint32_t cr, uint32_t cs) {
        const uint32_t g = gt_insert(gt_key, h, logcap);
        if (g == kNoHeavy) {
            st->detect_overflow = 1;
        } else {
            if (cr) atomicAdd(&gt_cnt[g], cr);
            if (cs) atomicAdd(&gt_cnt[size_t(cap_alloc) + g], cs);
        }
    };
    // count k_r R and k_s S occurrences of h (K1: one occurrence of one side, which compiles to
    // ATOMS.POPC.INC: the lanes of a warp on one counter cost one instruction)
    auto count = [&](uint32_t h, uint32_t kr, uint32_t ks, bool K1) {
        if (h == 0) {
            if (kr) atomicAdd(&s_zero[0], kr);
            if (ks) atomicAdd(&s_zero[1], ks);
            return;
        }
        uint32_t slot = __umulhi(h * 0x9E3779B1u, kDetSmemSlots);
        for (int probe = 0; probe < kDetSmemProbe; ++probe) {
            const uint32_t cur = s_key[slot];
            bool hit = cur == h;
            if (!hit && cur == 0) {
                const uint32_t prev = atomicCAS(&s_key[slot], 0u, h);
                hit = prev == 0 || prev == h;
            }
            if (hit) {
                if (K1) {
                    atomicAdd(ks ? &s_cs[slot] : &s_cr[slot], 1u);
                } else {
                    if (kr) atomicAdd(&s_cr[slot], kr);
                    if (ks) atomicAdd(&s_cs[slot], ks);
                }
                return;
            }
            slot = slot + 1 == kDetSmemSlots ? 0 : slot + 1;
        }
        merge(h, kr, ks);   // shared table crowded: count globally
    };
    const uint32_t lane = lane_id();
    for (;;) {
        if (threadIdx.x == 0) s_it = atomicAdd(claim, 1u);
        __syncthreads();
        const uint64_t it = s_it;
        if (it >= total) break;
        const ItemRange r = item_range(v, it);
        const uint2* pr = v.part[0] + v.start[r.p];
        const uint2* ps = v.part[1] + v.start[size_t(v.F) + 1 + r.p];
        // the whole partition in this item: local counts are exact, merge only possible skewed keys
        const bool whole = r.e0 == 0 && r.e1 == uint64_t(r.cr) + r.cs;
        const uint32_t keep = (whole && !force_heavy) ? Th : 1u;
        // Warp reference key: lanes holding the warp's current reference key are counted in
        // registers (one ballot per side), so a skewed key's tuples cost no shared atomics; the
        // reference moves to another lane's key when it matched fewer than 8 lanes.
        uint32_t ref = 0, pend_r = 0, pend_s = 0;
        bool has_ref = false;
        constexpr int U = 8;   // independent loads in flight per thread; the next batch loads while
                               // this one is counted
        uint32_t hn[U];
        auto load = [&](uint64_t base) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint64_t e = base + uint64_t(u) * kDetBlock + threadIdx.x;
                hn[u] = e < r.e1 ? (e < r.cr ? pr[e].x : ps[e - r.cr].x) : 0u;
            }
        };
        load(r.e0);
        for (uint64_t base = r.e0; base < r.e1; base += uint64_t(U) * kDetBlock) {
            uint32_t h[U];
#pragma unroll
            for (int u = 0; u < U; ++u) h[u] = hn[u];
            if (base + uint64_t(U) * kDetBlock < r.e1) load(base + uint64_t(U) * kDetBlock);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint64_t e = base + uint64_t(u) * kDetBlock + threadIdx.x;
                const bool valid = e < r.e1, side = e >= r.cr;
                const bool isref = has_ref && valid && h[u] == ref;
                const uint32_t m1 = __ballot_sync(kFull, isref && side), ma = __ballot_sync(kFull, isref);
                pend_s += __popc(m1);
                pend_r += __popc(ma & ~m1);
                const bool other = valid && !isref;
                if (other) count(h[u], side ? 0u : 1u, side ? 1u : 0u, true);
                const uint32_t mo = __ballot_sync(kFull, other);
                if (__popc(ma) < 8 && mo) {
                    if (lane == 0 && (pend_r | pend_s)) count(ref, pend_r, pend_s, false);
                    pend_r = pend_s = 0;
                    ref = __shfl_sync(kFull, h[u], __ffs(mo) - 1);
                    has_ref = true;
                }
            }
        }
        if (lane == 0 && (pend_r | pend_s)) count(ref, pend_r, pend_s, false);
        __syncthreads();
        for (uint32_t i = threadIdx.x; i < kDetSmemSlots; i += kDetBlock) {   // merge + clear
            const uint32_t k = s_key[i];
            if (k) {
                const uint32_t cr = s_cr[i], cs = s_cs[i];
                if (max(cr, cs) >= keep) merge(k, cr, cs);
                s_key[i] = 0;
                s_cr[i] = 0;
                s_cs[i] = 0;
            }
        }
        if (threadIdx.x == 0 && (s_zero[0] | s_zero[1])) {
            if (max(s_zero[0], s_zero[1]) >= keep) merge(0u, s_zero[0], s_zero[1]);
            s_zero[0] = s_zero[1] = 0;
        }
        __syncthreads();
    }
}

int launch_detect(const Plan& p, uint32_t n_large, uint32_t gt_cap, cudaStream_t s) {
    if (n_large == 0) return 0;
    uint32_t logcap = 0;
    while ((1u << logcap) < gt_cap) ++logcap;
    if (p.detect_mode == 0) cudaMemsetAsync(p.gt_key, 0, size_t(gt_cap) * sizeof(unsigned long long), s);
    cudaMemsetAsync(p.gt_cnt, 0, size_t(gt_cap) * sizeof(uint32_t), s);
    cudaMemsetAsync(p.gt_cnt + p.gt_cap_alloc, 0, size_t(gt_cap) * sizeof(uint32_t), s);
    LargeView v{{p.bufB[0], p.bufB[1]}, p.start, p.cnt, p.large_list, p.det_prefix, p.F, n_large, kDetectChunk,
                p.item_li};
    if (p.detect_mode == 1)
        k_detect<true><<<p.num_sms * 8, kDetBlock, 0, s>>>(v, p.gt_key, p.gt_cnt, p.gt_cap_alloc, logcap, p.st,
                                                           &p.st->claim[2]);
    else {
        static std::once_flag attr_once[kMaxDevices];
        once_per_device(attr_once, [] {
            cudaFuncSetAttribute(k_detect_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kDetSmemBytes);
        });
        LargeView v2 = v;
        v2.det_prefix = p.det_prefix2;
        v2.chunk = kDetectItem;
        v2.item_li = p.item_li2;
        k_detect_smem<<<p.num_sms * 3, kDetBlock, kDetSmemBytes, s>>>(v2, p.gt_key, p.gt_cnt, p.gt_cap_alloc, logcap,
                                                                      p.Th, p.force_heavy, p.st, &p.st->claim[2]);
    }
    return 1;
}

// ------------------------------------------------- a6 (paper-literal): sample + top-k --
// "For each large partition, GSH samples (e.g., 1%) tuples to detect skewed keys.  GSH uses a
// linear probing based hash table to compute the frequencies of sampled keys.  After sampling,
// GSH marks the top-k most frequent keys in each large partition as the skewed key." (L107,
// L112).  One CTA per large partition: every sample_stride-th tuple of R_p ++ S_p (positions
// 0, stride, 2 stride, ...) is counted in a shared-memory linear-probing table; k rounds of a
// block arg-max over (count, h) pick the top-k, which are inserted into the global table whose
// exact counts k_detect<true> then takes.  A key whose probe sequence finds no free slot within
// kDetectMaxProbe is dropped (a nearly full table; a large partition's sample is dominated by
// its few skewed keys, so its distinct sampled keys are few); the choice affects
// performance only -- split and the NM-join stay exact for any set of skewed keys.
constexpr uint32_t kSampleSlots = 2048;
constexpr int kSampleBlock = 256;

__global__ void __launch_bounds__(kSampleBlock) k_sample_topk(LargeView v, uint32_t stride, uint32_t top_k,
                                                             unsigned long long* gt_key, uint32_t logcap,
                                                             DevState* st) {
    __shared__ unsigned long long s_key[kSampleSlots];   // (1 << 32 | h), 0 = empty
    __shared__ uint32_t s_cnt[kSampleSlots];
    __shared__ unsigned long long s_red[kSampleBlock / 32];
    for (uint32_t li = blockIdx.x; li < v.n_large; li += gridDim.x) {
        for (uint32_t i = threadIdx.x; i < kSampleSlots; i += kSampleBlock) {
            s_key[i] = 0;
            s_cnt[i] = 0;
        }
        __syncthreads();
        const uint32_t p = v.large_list[li];
        const uint32_t cr = v.cnt[p], cs = v.cnt[v.F + p];
        const uint64_t ns = (uint64_t(cr) + cs + stride - 1) / stride;
        for (uint64_t k = threadIdx.x; k < ns; k += kSampleBlock) {
            const uint64_t e = k * stride;
            const int side = e >= cr;
            const uint64_t off = side ? e - cr : e;
            const uint32_t h = v.part[side][v.start[size_t(side) * (v.F + 1) + p] + off].x;
            const unsigned long long tag = (1ull << 32) | h;
            uint32_t slot = (h * 0x9E3779B1u) >> (32 - 11);   // linear probing (kSampleSlots = 2^11)
            for (int probe = 0; probe < kDetectMaxProbe; ++probe) {
                const unsigned long long cur = s_key[slot];
                if (cur == tag) break;
                if (cur == 0) {
                    const unsigned long long prev = atomicCAS(&s_key[slot], 0ull, tag);
                    if (prev == 0 || prev == tag) break;
                }
                slot = (slot + 1) & (kSampleSlots - 1);
            }
            if (s_key[slot] == tag) atomicAdd(&s_cnt[slot], 1u);
        }
        __syncthreads();
        // top-k: k rounds of a block arg-max of (count << 32 | h) over the unchosen slots
        for (uint32_t r = 0; r < top_k; ++r) {
            unsigned long long best = 0;
            uint32_t bslot = 0;
            for (uint32_t i = threadIdx.x; i < kSampleSlots; i += kSampleBlock) {
                const unsigned long long w = s_cnt[i] ? ((unsigned long long)s_cnt[i] << 32) | uint32_t(s_key[i]) : 0ull;
                if (w > best) { best = w; bslot = i; }
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                const unsigned long long ob = __shfl_xor_sync(kFull, best, o);
                const uint32_t os = __shfl_xor_sync(kFull, bslot, o);
                if (ob > best) { best = ob; bslot = os; }
            }
            if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = best;
            __syncthreads();
            unsigned long long top = 0;
#pragma unroll
            for (int w = 0; w < kSampleBlock / 32; ++w) top = s_red[w] > top ? s_red[w] : top;
            if (top == 0) break;   // fewer than k distinct sampled keys (uniform across the block)
            // the owner of the winning slot retires it and publishes the key
            if ((threadIdx.x & 31) == 0 && best == top) {
                s_cnt[bslot] = 0;
                if (gt_insert(gt_key, uint32_t(top), logcap) == kNoHeavy) st->detect_overflow = 1;
            }
            __syncthreads();
        }
        __syncthreads();
    }
}

int launch_sample_topk(const Plan& p, uint32_t n_large, uint32_t gt_cap, cudaStream_t s) {
    if (n_large == 0) return 0;
    uint32_t logcap = 0;
    while ((1u << logcap) < gt_cap) ++logcap;
    cudaMemsetAsync(p.gt_key, 0, size_t(gt_cap) * sizeof(unsigned long long), s);
    LargeView v{{p.bufB[0], p.bufB[1]}, p.start, p.cnt, p.large_list, p.det_prefix, p.F, n_large, kDetectChunk,
                p.item_li};
    const unsigned grid = (unsigned)umin64(n_large, uint64_t(p.num_sms) * 8);
    k_sample_topk<<<grid, kSampleBlock, 0, s>>>(v, p.sample_stride, p.top_k, p.gt_key, logcap, p.st);
    return 1;
}

// ------------------------------------------------------------------- a6: select --
__global__ void k_select(const unsigned long long* __restrict__ gt_key, const uint32_t* __restrict__ gt_cnt,
                         uint32_t cap, uint32_t cap_alloc, uint32_t Th,
                         int force_heavy, uint32_t pshift, uint32_t pmask, uint32_t F, HeavyKey* __restrict__ H,
                         uint64_t h_max, uint32_t* __restrict__ part_heavy, DevState* st) {
    for (uint32_t slot = blockIdx.x * blockDim.x + threadIdx.x; slot < cap; slot += gridDim.x * blockDim.x) {
        const unsigned long long kw = gt_key[slot];
        if (kw == 0) continue;
        const uint32_t h = (uint32_t)kw;
        const uint32_t cr = gt_cnt[slot], cs = gt_cnt[cap_alloc + slot];
        const bool heavy = force_heavy || max(cr, cs) >= Th;
        if (heavy) {
            const uint32_t p = part_of(h, pshift, pmask);
            const uint32_t hid = atomicAdd(&st->n_heavy, 1u);
            if (hid >= h_max) {   // the side list is full: the call fails (GSH_ERR_INTERNAL)
                st->heavy_overflow = 1;
                continue;
            }
            H[hid] = HeavyKey{h, cr, cs, p};
            if (cr) atomicAdd(&part_heavy[p], cr);
            if (cs) atomicAdd(&part_heavy[F + p], cs);
            atomicAdd(&st->heavy_tuples[0], (unsigned long long)cr);
            atomicAdd(&st->heavy_tuples[1], (unsigned long long)cs);
            atomicAdd(&st->skew_pairs, (unsigned long long)cr * cs);
        }
    }
}

int launch_select(const Plan& p, uint32_t gt_cap, cudaStream_t s) {
    const uint32_t B = p.b1 + p.b2;
    const uint32_t pshift = B ? (32 - p.route_bits - B) : 0;
    unsigned grid = (unsigned)umin64((gt_cap + 255) / 256, uint64_t(p.num_sms) * 16);
    // detect_mode 1: the table holds exactly the sampled top-k keys, all skewed
    const uint32_t th = p.detect_mode == 1 ? 1u : p.Th;
    k_select<<<grid, 256, 0, s>>>(p.gt_key, p.gt_cnt, gt_cap, p.gt_cap_alloc, th, p.force_heavy, pshift,
                                  p.F - 1, p.F, p.H, p.h_max, p.part_heavy, p.st);
    return 1;
}

// ------------------------------------------------------------- offsets of H / normal --
struct HeavyCount {
    const HeavyKey* H;
    int side;
    __device__ uint64_t operator()(uint64_t k) const { return side ? H[k].cnt_s : H[k].cnt_r; }
};
struct HeavyTiles {
    const HeavyKey* H;
    __device__ uint64_t operator()(uint64_t k) const {
        uint64_t tr = (H[k].cnt_r + kSkewTileR - 1) / kSkewTileR;
        uint64_t ts = (H[k].cnt_s + kSkewTileS - 1) / kSkewTileS;
        return tr * ts;
    }
};
struct NormalRemainder {
    const uint32_t* cnt;
    const uint32_t* part_heavy;
    const uint32_t* large_list;
    uint32_t F;
    int side;
    __device__ uint64_t operator()(uint64_t li) const {
        uint32_t p = large_list[li];
        return uint64_t(cnt[side * F + p]) - part_heavy[side * F + p];
    }
};

// Per-key array offsets (R_k, S_k) and dense-tile prefix over H[0, n_heavy).  Entries keep their
// offsets when more are appended (hybrid keys first, then the residual detection's).
int launch_heavy_offsets(const Plan& p, uint32_t n_heavy, cudaStream_t s) {
    int l = 0;
    l += launch_scan(HeavyCount{p.H, 0}, n_heavy, p.h_off, p.scan_scratch, s);
    l += launch_scan(HeavyCount{p.H, 1}, n_heavy, p.h_off + (p.h_max + 1), p.scan_scratch, s);
    l += launch_scan(HeavyTiles{p.H}, n_heavy, p.h_tiles, p.scan_scratch, s);
    return l;
}

int launch_heavy_prefix(const Plan& p, uint32_t n_heavy, uint32_t n_large, cudaStream_t s) {
    int l = launch_heavy_offsets(p, n_heavy, s);
    l += launch_scan(NormalRemainder{p.cnt, p.part_heavy, p.large_list, p.F, 0}, n_large, p.nrm_off,
                     p.scan_scratch, s);
    l += launch_scan(NormalRemainder{p.cnt, p.part_heavy, p.large_list, p.F, 1}, n_large, p.nrm_off + (p.F + 1),
                     p.scan_scratch, s);
    cudaMemsetAsync(p.h_cur, 0, size_t(2) * p.h_max * sizeof(uint32_t), s);
    cudaMemsetAsync(p.nrm_cur, 0, size_t(2) * p.F * sizeof(uint32_t), s);
    return l;
}

// -------------------------------------------------------------------- a7: split --
// "checks each R tuple against the skewed keys.  If the tuple is skewed, it is appended to an
// array allocated for the associated skewed key ... Otherwise ... appends the tuple to a normal
// partition" (L114); same for S.  A CTA claims an item (<= kDetectChunk tuples of ONE large
// partition, 16 per thread, held in registers) and splits it in two phases: (1) every tuple gets
// its skewed-key id (global table lookup) and a rank inside the item -- per (side, key) for skewed
// tuples through a shared-memory table, per side for normal ones -- from shared-memory atomics
// (ATOMS.POPC.INC: lanes of a warp on one counter get consecutive ranks in one instruction);
// (2) one global atomic per distinct (side, key) and per side reserves the item's runs, and the
// tuples are written at base + rank (consecutive for runs of one key: coalesced).
constexpr uint32_t kSplitHidSlots = 2 * kDetectChunk;   // an item's distinct (side, key) always fit
constexpr int kSplitIpt = kDetectChunk / kSkewSplitBlock;
constexpr uint32_t kSplitSlotBits = kSplitHidSlots == 4096 ? 12 : kSplitHidSlots == 8192 ? 13 : 14;
constexpr size_t kSplitSmemBytes = size_t(kSplitHidSlots) * 8;
static_assert(kSplitIpt * kSkewSplitBlock == kDetectChunk, "split item = 8 tuples per thread");
static_assert((1u << kSplitSlotBits) == kSplitHidSlots, "slot hash bits");

// The split's skewed-key lookups go to a compact table of H only ((hid + 1) << 32 | h, 0 = empty,
// 2 slots per key: a few hundred KB, L2-resident) instead of the detection table (one slot per
// counted key, up to 256 MB: one DRAM sector per first probe of every tuple of a large partition).
__global__ void k_htab_build(const HeavyKey* __restrict__ H, uint32_t n_heavy, unsigned long long* htab,
                             uint32_t logcap) {
    const uint32_t mask = (1u << logcap) - 1;
    for (uint32_t hid = blockIdx.x * blockDim.x + threadIdx.x; hid < n_heavy; hid += gridDim.x * blockDim.x) {
        const uint32_t h = H[hid].h;
        const unsigned long long e = (uint64_t(hid + 1) << 32) | h;
        uint32_t s = gt_slot0(h, logcap);
        while (atomicCAS(&htab[s], 0ull, e) != 0ull) s = (s + 1) & mask;   // load <= 1/2: terminates
    }
}

__device__ __forceinline__ uint32_t htab_find(const unsigned long long* __restrict__ htab, uint32_t h,
                                              uint32_t logcap, uint32_t s) {
    const uint32_t mask = (1u << logcap) - 1;
    for (;;) {
        const unsigned long long e = htab[s];
        if (e == 0) return kNoHeavy;
        if ((uint32_t)e == h) return (uint32_t)(e >> 32) - 1;
        s = (s + 1) & mask;
    }
}

__global__ void __launch_bounds__(kSkewSplitBlock, 1024 / kSkewSplitBlock) k_split(LargeView v, const unsigned long long* __restrict__ htab,
                                                    uint32_t logcap,
                                                    const uint64_t* __restrict__ h_off, uint64_t h_stride,
                                                    uint32_t* h_cur, uint32_t h_max, uint32_t* heavy_pay_r,
                                                    uint32_t* heavy_pay_s, const uint64_t* __restrict__ nrm_off,
                                                    uint32_t* nrm_cur, uint2* out_r, uint2* out_s,
                                                    unsigned int* claim) {
    extern __shared__ uint32_t split_dyn[];
    uint32_t* s_key = split_dyn;                    // (hid << 1 | side) + 1, 0 = empty
    uint32_t* s_cnt = split_dyn + kSplitHidSlots;   // count, then the item's run base
    __shared__ uint32_t s_nrm[2], s_nbase[2];
    __shared__ uint32_t s_used[kSplitHidSlots];   // the item's claimed slots (the reservation walks only these)
    __shared__ uint32_t s_nused;
    __shared__ unsigned int s_it;
    for (uint32_t i = threadIdx.x; i < kSplitHidSlots; i += kSkewSplitBlock) {
        s_key[i] = 0;
        s_cnt[i] = 0;
    }
    if (threadIdx.x < 2) s_nrm[threadIdx.x] = 0;
    if (threadIdx.x == 0) s_nused = 0;
    const uint64_t total = v.det_prefix[v.n_large];
    for (;;) {
        if (threadIdx.x == 0) s_it = atomicAdd(claim, 1u);
        __syncthreads();
        const uint64_t it = s_it;
        if (it >= total) break;
        const ItemRange r = item_range(v, it);
        const uint2* pr = v.part[0] + v.start[r.p];
        const uint2* ps = v.part[1] + v.start[size_t(v.F) + 1 + r.p];
        uint2 t[kSplitIpt];
        // rk: skewed = shared slot << 16 | rank; normal = 1 << 31 | side << 16 | rank; none = ~0
        uint32_t rk[kSplitIpt];
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            const uint64_t e = r.e0 + uint64_t(j) * kSkewSplitBlock + threadIdx.x;
            t[j] = e < r.e1 ? (e < r.cr ? pr[e] : ps[e - r.cr]) : make_uint2(0, 0);
        }
        // skewed-key ids: the first probe of every tuple is issued before any is resolved (the
        // table holds only the skewed keys, so most first probes of normal tuples find an empty slot)
        uint32_t ids[kSplitIpt];
        {
            unsigned long long w0[kSplitIpt];
#pragma unroll
            for (int j = 0; j < kSplitIpt; ++j) w0[j] = htab[gt_slot0(t[j].x, logcap)];
#pragma unroll
            for (int j = 0; j < kSplitIpt; ++j)
                ids[j] = w0[j] == 0 ? kNoHeavy
                       : (uint32_t)w0[j] == t[j].x ? (uint32_t)(w0[j] >> 32) - 1
                       : htab_find(htab, t[j].x, logcap, (gt_slot0(t[j].x, logcap) + 1) & ((1u << logcap) - 1));
        }
        // Ranks: normal tuples by one shared atomic per (warp, side); skewed tuples of the warp's
        // reference key by one shared atomic per warp (lanes ranked by ballot prefix); other skewed
        // tuples one shared atomic each, the reference moving to one of their keys whenever it
        // matched fewer than 8 lanes (skewed items are dominated by one key).
        uint32_t ref = 0, ref_slot = 0;   // warp-uniform; key 0 = none
        const uint32_t lane = lane_id(), ltm = lanemask_lt();
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            const uint64_t e = r.e0 + uint64_t(j) * kSkewSplitBlock + threadIdx.x;
            const bool valid = e < r.e1;
            const uint32_t side = e >= r.cr;
            const uint32_t id = ids[j];
            const bool heavy = valid && id != kNoHeavy;
            const uint32_t key = heavy ? ((id << 1 | side) + 1) : 0u;
            uint32_t rr = 0xffffffffu;
#pragma unroll
            for (uint32_t sd = 0; sd < 2; ++sd) {
                const uint32_t m = __ballot_sync(kFull, valid && !heavy && side == sd);
                if (m) {
                    const uint32_t lead = __ffs(m) - 1;
                    uint32_t b = 0;
                    if (lane == lead) b = atomicAdd(&s_nrm[sd], (uint32_t)__popc(m));
                    b = __shfl_sync(kFull, b, lead);
                    if ((m >> lane) & 1u) rr = 1u << 31 | sd << 16 | (b + __popc(m & ltm));
                }
            }
            const uint32_t mr = __ballot_sync(kFull, heavy && key == ref);
            if (mr) {
                const uint32_t lead = __ffs(mr) - 1;
                uint32_t b = 0;
                if (lane == lead) b = atomicAdd(&s_cnt[ref_slot], (uint32_t)__popc(mr));
                b = __shfl_sync(kFull, b, lead);
                if ((mr >> lane) & 1u) rr = ref_slot << 16 | (b + __popc(mr & ltm));
            }
            const bool other = heavy && key != ref;
            if (other) {
                uint32_t slot = (key * 0x9E3779B1u) >> (32 - kSplitSlotBits);
                for (;;) {   // an item has <= kDetectChunk distinct keys: a free slot always exists
                    const uint32_t cur = s_key[slot];
                    if (cur == key) break;
                    if (cur == 0) {
                        const uint32_t prev = atomicCAS(&s_key[slot], 0u, key);
                        if (prev == 0) {
                            s_used[atomicAdd(&s_nused, 1u)] = slot;
                            break;
                        }
                        if (prev == key) break;
                    }
                    slot = (slot + 1) & (kSplitHidSlots - 1);
                }
                rr = slot << 16 | atomicAdd(&s_cnt[slot], 1u);
            }
            const uint32_t mo = __ballot_sync(kFull, other);
            if (__popc(mr) < 8 && mo) {
                const uint32_t lead = __ffs(mo) - 1;
                ref = __shfl_sync(kFull, key, lead);
                ref_slot = __shfl_sync(kFull, rr >> 16, lead);
            }
            rk[j] = rr;
        }
        __syncthreads();
        // reserve this item's runs: one global atomic per distinct (side, key) and per side
        for (uint32_t u = threadIdx.x; u < s_nused; u += kSkewSplitBlock) {
            const uint32_t i = s_used[u];
            const uint32_t key = s_key[i];
            const uint32_t id = (key - 1) >> 1, side = (key - 1) & 1u;
            s_cnt[i] = atomicAdd(&h_cur[size_t(side) * h_max + id], s_cnt[i]);
        }
        if (threadIdx.x < 2 && s_nrm[threadIdx.x])
            s_nbase[threadIdx.x] = atomicAdd(&nrm_cur[size_t(threadIdx.x) * v.F + r.li], s_nrm[threadIdx.x]);
        __syncthreads();
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            if (rk[j] == 0xffffffffu) continue;
            const uint32_t rank = rk[j] & 0xffffu;
            if (rk[j] >> 31) {
                const uint32_t side = (rk[j] >> 16) & 1u;
                uint2* dst = side ? out_s : out_r;
                dst[nrm_off[size_t(side) * (v.F + 1) + r.li] + s_nbase[side] + rank] = t[j];
            } else {
                const uint32_t slot = rk[j] >> 16;
                const uint32_t key = s_key[slot] - 1;
                uint32_t* dst = (key & 1u) ? heavy_pay_s : heavy_pay_r;
                dst[h_off[size_t(key & 1u) * h_stride + (key >> 1)] + s_cnt[slot] + rank] = t[j].y;
            }
        }
        __syncthreads();
        // clear the slots this item used (each thread its own tuples' slots; repeats are harmless)
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            if ((rk[j] >> 31) == 0) {
                s_key[rk[j] >> 16] = 0;
                s_cnt[rk[j] >> 16] = 0;
            }
        }
        if (threadIdx.x < 2) s_nrm[threadIdx.x] = 0;
        if (threadIdx.x == 0) s_nused = 0;
    }
}

int launch_split(const Plan& p, uint32_t n_large, uint32_t n_heavy, cudaStream_t s) {
    if (n_large == 0) return 0;
    uint64_t hc = 1024;
    while (hc < 2 * uint64_t(n_heavy) && hc < p.htab_cap) hc <<= 1;
    const uint32_t logcap = log2_pow2(hc);
    cudaMemsetAsync(p.htab, 0, hc * sizeof(unsigned long long), s);
    if (n_heavy)
        k_htab_build<<<(unsigned)umin64((n_heavy + 255) / 256, uint64_t(p.num_sms) * 8), 256, 0, s>>>(p.H, n_heavy,
                                                                                                p.htab, logcap);
    static std::once_flag attr_once[kMaxDevices];
    once_per_device(attr_once, [] {
        cudaFuncSetAttribute(k_split, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSplitSmemBytes);
    });
    LargeView v{{p.bufB[0], p.bufB[1]}, p.start, p.cnt, p.large_list, p.det_prefix, p.F, n_large, kDetectChunk,
                p.item_li};
    k_split<<<p.num_sms * (1024 / kSkewSplitBlock), kSkewSplitBlock, kSplitSmemBytes, s>>>(v, p.htab, logcap, p.h_off, p.h_max + 1,
                                                             p.h_cur, (uint32_t)p.h_max, p.heavy_pay[0],
                                                             p.heavy_pay[1], p.nrm_off, p.nrm_cur, p.bufA[0],
                                                             p.bufA[1], &p.st->claim[3]);
    return n_heavy ? 2 : 1;
}

// --------------------------------------------------------------- NM descriptors --
__global__ void k_nm_setup(const uint2* bufB0, const uint2* bufB1, const uint2* bufA0, const uint2* bufA1,
                           const uint64_t* start, const uint32_t* cnt, const uint32_t* large_idx,
                           const uint32_t* part_heavy, const uint64_t* nrm_off, uint32_t F, NmPart* nm) {
    for (uint32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < F; p += gridDim.x * blockDim.x) {
        NmPart d;
        const uint32_t li = large_idx[p];
        if (li == kNoHeavy) {
            d.r = bufB0 + start[p];
            d.s = bufB1 + start[F + 1 + p];
            d.rlen = cnt[p];
            d.slen = cnt[F + p];
        } else {
            d.r = bufA0 + nrm_off[li];
            d.s = bufA1 + nrm_off[F + 1 + li];
            d.rlen = cnt[p] - part_heavy[p];
            d.slen = cnt[F + p] - part_heavy[F + p];
        }
        nm[p] = d;
    }
}

struct NmItems {
    const NmPart* nm;
    uint32_t C;
    int chain;   // the streamed kernel's table (its R-side limit differs)
    __device__ uint64_t operator()(uint64_t p) const {
        const NmPart d = nm[p];
        if (d.rlen == 0 || d.slen == 0) return 0;
        if (ring_eligible(d.rlen, d.slen, chain != 0)) return 0;  // streamed kernel (nm_ring.cu)
        return uint64_t((d.rlen + C - 1) / C) * ((d.slen + kNmSlice - 1) / kNmSlice);
    }
};

int launch_nm_setup(const Plan& p, uint32_t n_large, cudaStream_t s) {
    (void)n_large;
    unsigned grid = (p.F + 255) / 256;
    k_nm_setup<<<grid, 256, 0, s>>>(p.bufB[0], p.bufB[1], p.bufA[0], p.bufA[1], p.start, p.cnt, p.large_idx,
                                    p.part_heavy, p.nrm_off, p.F, p.nm);
    return 1 + launch_scan(NmItems{p.nm, p.C, p.nm_chain}, p.F, p.nm_prefix, p.scan_scratch, s);
}

}  // namespace gsh

