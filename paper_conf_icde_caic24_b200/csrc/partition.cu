// partition.cu -- GSH phase (1): "partitions input tables into shared memory sized partitions
// ... a simple count then partition procedure ... two passes" (§IV-B(1)).
//
// SURVEY.md §8(a) rows a1-a4:
//   a1 k_hist2d        : h = fmix32(key); joint (d1,d2) histogram of BOTH passes from one read
//                        of the keys (4 B/tuple).  Per-CTA shared-memory counters (packed u16 with
//                        exact wrap accounting above 2^15 bins) updated by shared-memory atomics.
//   a2 k_hist_reduce + scans : per-partition counts and start offsets, pass-1 chunk offsets.
//   a3/a4 k_scatter    : static-offset scatter -- every unit's (pass-1 chunk / pass-2 (digit,
//                        group)) bucket offsets come from scans of the histogram, so there is no
//                        look-back.  Tiles arrive by TMA, ranks come from ATOMS.POPC.INC, tuples
//                        are staged in shared memory in bucket order and written as whole 32 B
//                        sectors (a carry holds each bucket's partial sector).  16 B/tuple per
//                        pass; pass-2 units never cross a pass-1 partition.
#include <cstdio>
#include <cstdlib>

#include <type_traits>

#include "gsh_device.cuh"
#include "gsh_internal.h"
#include "gsh_scan.cuh"

namespace gsh {

// ---------------------------------------------------------------------- hash (debug) --
__global__ void k_hash(const uint32_t* __restrict__ keys, uint32_t* __restrict__ out, uint64_t n) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
        out[i] = hash32(keys[i]);
}

int launch_hash(const uint32_t* keys, uint32_t* out, uint64_t n, cudaStream_t s) {
    if (n == 0) return 0;
    unsigned grid = (unsigned)((n + 255) / 256);
    if (grid > 148u * 16u) grid = 148u * 16u;
    k_hash<<<grid, 256, 0, s>>>(keys, out, n);
    return 1;
}

// ------------------------------------------------------------------- a1: histogram --
// One read of the keys yields the (d1, d2) histogram of BOTH partition passes, per pass-1 work
// unit (a "slice" of unit_chunks chunks: the pass-1 scatter's unit IS the histogram slice, so
// the pass-1 digit counts of a unit are the joint counts summed over d2 -- one shared atomic
// per key).
// F <= 2^15: u32 counters in shared memory, atomicAdd(.., 1) = hardware-aggregated
// ATOMS.POPC.INC (skewed digits cost no more than spread ones; __match_any_sync costs ~64
// cycles -- scripts/microbench_warp_ops.cu).
// F > 2^15 (up to 2^16 bins): packed u16 counters, two bins per 32-bit word, so ONE CTA holds
// all bins in 128 KB and every key is hashed once.  A u16 can wrap (a bin reaching 2^16 keys in
// one slice, heavy skew only), so wraps are accounted for from the atomics' return values (all
// updates of a word are serialised, each returns the old word):
//   * the lane whose increment takes a half from 0xffff to 0 sees old half == 0xffff;
//   * a low-half wrap carries +1 into the high half -- recorded as a -1 correction of the high
//     bin, and if that carry itself wrapped the high half (old high == 0xffff) as a high wrap.
// true(low) = low + 65536 * wraps(low); true(high) = high + 65536 * wraps(high) - carries.
// The (bin, delta) events of a slice are applied at its flush: a slice holds <= kHistMaxUnitChunks
// * 2^14 = 2^20 keys, so at most 16 wraps of 3 events each.
constexpr uint32_t kHistMaxEvents = 128;
static_assert(kScatterChunk == 16 * kHistBlock, "a full chunk is 4 uint4 per histogram thread");
static_assert(3 * ((uint64_t(kHistMaxUnitChunks) * kScatterChunk) >> 16) <= kHistMaxEvents, "wrap events of a slice");

// Hybrid partition (hybrid.cu): the sampled skewed keys' table (u32 h per slot, kHybEmpty = empty,
// then u16 ids); load <= 1/4, so most misses end at their first slot.
__device__ __forceinline__ uint32_t hyb_slot(uint32_t h) { return (h * 0x9E3779B1u) >> (32 - kHybLogSlots); }
// The lookup of h whose first slot's key k0 = key[hyb_slot(h)] is already loaded (callers issue all
// their first probes before resolving any: independent shared loads instead of a dependent chain).
__device__ __forceinline__ uint32_t hyb_resolve(const uint32_t* key, const uint16_t* id, uint32_t h, uint32_t k0) {
    if (h == kHybEmpty || k0 == kHybEmpty) return kNoHeavy;   // kHybEmpty is never chosen
    uint32_t s = hyb_slot(h);
    if (k0 == h) return id[s];
    for (;;) {
        s = (s + 1) & (kHybSlots - 1);
        const uint32_t k = key[s];
        if (k == h) return id[s];
        if (k == kHybEmpty) return kNoHeavy;
    }
}
__device__ __forceinline__ uint32_t hyb_find(const uint32_t* key, const uint16_t* id, uint32_t h) {
    return hyb_resolve(key, id, h, key[hyb_slot(h)]);
}
// Both first slots loaded unconditionally, resolved with selects; the probe loop runs only when
// both hold other keys (rare at load <= 1/4), so the common case has no divergent path.
__device__ __forceinline__ uint32_t hyb_find2(const uint32_t* key, const uint16_t* id, uint32_t h) {
    const uint32_t s0 = hyb_slot(h), s1 = (s0 + 1) & (kHybSlots - 1);
    const uint32_t ka = key[s0], kb = key[s1];
    if (h == kHybEmpty || ka == kHybEmpty) return kNoHeavy;
    if (ka == h) return id[s0];
    if (kb == h) return id[s1];
    if (kb == kHybEmpty) return kNoHeavy;
    return hyb_find(key, id, h);
}

// CHECK (route_bits > 0): also verify the caller's gsh_config.route_bits assertion -- every tuple
// shares the top route_bits of h -- by OR-ing t and ~t over all keys (t = those bits): they are all
// equal iff (OR t) & (OR ~t) has no bit set.  The NM-join's chained table relies on it.
// HYB (gsh_config.hybrid): a key of the sampled skewed set is counted per (side, key) -- hyb_cnt,
// the sizes of R_k / S_k -- instead of in its digit bins, so every later offset covers the
// partitioned (normal) tuples only.
template <bool FAST16, bool CHECK, bool HYB>
__global__ void __launch_bounds__(kHistBlock, 1)
k_hist2d(const uint32_t* __restrict__ k0, uint64_t n0, const uint32_t* __restrict__ k1, uint64_t n1,
         uint32_t shift, uint32_t nbits, uint32_t b2, uint32_t* __restrict__ partial, uint32_t* __restrict__ c1cnt,
         uint32_t nu0, uint32_t nu1, uint32_t unit_chunks, uint32_t rshift, DevState* st,
         uint32_t* __restrict__ slice_dom, const uint32_t* __restrict__ hyb_tab, uint32_t n_h0,
         uint32_t* __restrict__ hyb_cnt, uint32_t* __restrict__ hyb_slice, uint32_t* __restrict__ hyb_ref) {
    __shared__ uint32_t s_href;   // HYB: max over the slice's keys of (count << 9 | id)
    __shared__ uint32_t s_hkey[HYB ? kHybSlots : 1];
    __shared__ uint16_t s_hid[HYB ? kHybSlots : 1];
    __shared__ uint32_t s_hc[HYB ? kHybMaxKeys : 1];
    if (HYB) {
        for (uint32_t i = threadIdx.x; i < kHybSlots; i += blockDim.x) {
            s_hkey[i] = hyb_tab[i];
            s_hid[i] = reinterpret_cast<const uint16_t*>(hyb_tab + kHybSlots)[i];
        }
        for (uint32_t i = threadIdx.x; i < kHybMaxKeys; i += blockDim.x) s_hc[i] = 0;
        if (threadIdx.x == 0) s_href = 0;
    }
    static_assert(kHybMaxKeys <= 512 && kHistMaxUnitChunks * kScatterChunk <= (1u << 22), "(count << 9 | id) fits");
    uint32_t r_or = 0, r_nor = 0;
    __shared__ uint32_t s_dom;
    extern __shared__ uint32_t cnt[];
    __shared__ uint32_t c1s[256];
    __shared__ uint32_t ev_bin[kHistMaxEvents];
    __shared__ int32_t ev_delta[kHistMaxEvents];
    __shared__ uint32_t n_ev;
    const uint32_t F = 1u << nbits;
    const uint32_t mask = F - 1;
    const bool packed = F > (1u << 15);
    // digits above bit 16 do not see fmix32's last xor-shift (it only changes the low half)
    const bool top16 = shift >= 16;
    const uint32_t nwords = packed ? F / 2 : F;
    const uint32_t d1n = (F >> b2) ? (F >> b2) : 1;
    const uint32_t per_d = packed ? ((1u << b2) >> 1) : (1u << b2);   // counter words per pass-1 digit
    auto event = [&](uint32_t bin, int32_t d) {
        const uint32_t e = atomicAdd(&n_ev, 1u);
        if (e < kHistMaxEvents) {
            ev_bin[e] = bin;
            ev_delta[e] = d;
        }
    };
    // inc = 1 << (16 * (bin & 1)) and m = its half's mask, without variable shifts (the
    // histogram is ALU-bound): a wrap is old's half == 0xffff, i.e. (~old & m) == 0
    auto wrap_events = [&](uint32_t bin, uint32_t old) {   // rare: a u16 wrapped
        const uint32_t s16 = (bin & 1u) << 4;
        event(bin, 65536);
        if (s16 == 0) {
            event(bin | 1u, -1);
            if ((old >> 16) == 0xffffu) event(bin | 1u, 65536);
        }
    };
    auto count_exact = [&](uint32_t bin) {
        const uint32_t inc = umax32((bin & 1u) << 16, 1u);
        const uint32_t m = inc * 0xffffu;
        const uint32_t old = atomicAdd(&cnt[bin >> 1], inc);
        if (__builtin_expect((~old & m) == 0, 0)) wrap_events(bin, old);
    };
    // Packed counters, a batch of keys: every atomic is issued before any returned value is
    // tested, so their shared-memory round trips overlap (one per key otherwise: the wrap test
    // of key i would hold back the atomic of key i + 1).
    auto count_exact_batch = [&](const uint32_t (&bins)[8]) {
        uint32_t old[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) old[q] = atomicAdd(&cnt[bins[q] >> 1], umax32((bins[q] & 1u) << 16, 1u));
        auto rest = [&](int q) { return ~old[q] & (umax32((bins[q] & 1u) << 16, 1u) * 0xffffu); };   // 0: wrapped
        uint32_t mn = rest(0);
#pragma unroll
        for (int q = 1; q < 8; ++q) mn = umin32(mn, rest(q));
        if (__builtin_expect(mn == 0, 0))
#pragma unroll
            for (int q = 0; q < 8; ++q)
                if (rest(q) == 0) wrap_events(bins[q], old[q]);
    };
    auto bin_of = [&](uint32_t key) -> uint32_t {
        if (FAST16) return hash32_top(key) >> 16;
        const uint32_t hk = top16 ? hash32_top(key) : hash32(key);
        if (CHECK) {
            const uint32_t t = hk >> rshift;
            r_or |= t;
            r_nor |= ~t;
        }
        return (hk >> shift) & mask;
    };
    auto count_key = [&](uint32_t key) {
        if (HYB) {
            const uint32_t hk = hash32(key);
            if (CHECK) {
                const uint32_t t = hk >> rshift;
                r_or |= t;
                r_nor |= ~t;
            }
            const uint32_t hid = hyb_find(s_hkey, s_hid, hk);
            if (hid != kNoHeavy) {
                atomicAdd(&s_hc[hid], 1u);   // no return value: warp-aggregated in hardware
                return;
            }
            const uint32_t bin = (hk >> shift) & mask;
            if (packed) count_exact(bin); else atomicAdd(&cnt[bin], 1u);
        } else if (FAST16) {
            count_exact(hash32_top(key) >> 16);
        } else {
            const uint32_t hk = top16 ? hash32_top(key) : hash32(key);
            if (CHECK) {
                const uint32_t t = hk >> rshift;
                r_or |= t;
                r_nor |= ~t;
            }
            const uint32_t bin = (hk >> shift) & mask;
            if (packed) count_exact(bin); else atomicAdd(&cnt[bin], 1u);
        }
    };
    for (uint32_t w = threadIdx.x; w < nwords; w += blockDim.x) cnt[w] = 0;
    if (threadIdx.x < 256) c1s[threadIdx.x] = 0;
    if (threadIdx.x == 0) n_ev = 0;
    __syncthreads();
    for (uint32_t it = blockIdx.x; it < nu0 + nu1; it += gridDim.x) {
        const int side = it >= nu0;
        const uint32_t sl = it - (side ? nu0 : 0);
        const uint32_t nu = side ? nu1 : nu0;
        const uint32_t* keys = side ? k1 : k0;
        const uint64_t n = side ? n1 : n0;
        const uint32_t nch = (uint32_t)((n + kScatterChunk - 1) / kScatterChunk);
        uint32_t* c1out = c1cnt + (side ? size_t(nu0) * 256 : 0);
        const bool vec = ((reinterpret_cast<uintptr_t>(keys) & 15u) == 0);
        const uint32_t c0 = sl * unit_chunks, cend = umin32(c0 + unit_chunks, nch);
        // Full chunks are loaded one chunk ahead (16 keys per thread in registers), so the
        // loads of chunk c+1 are in flight while chunk c is counted.
        uint4 v[4];
        auto load_chunk = [&](uint32_t c) {
            const uint4* kv = reinterpret_cast<const uint4*>(keys + uint64_t(c) * kScatterChunk);
#pragma unroll
            for (int u = 0; u < 4; ++u) v[u] = ld_stream_u4(kv + threadIdx.x + u * kHistBlock);
        };
        auto chunk_full = [&](uint32_t c) { return vec && uint64_t(c + 1) * kScatterChunk <= n; };
        if (c0 < cend && chunk_full(c0)) load_chunk(c0);
        for (uint32_t c = c0; c < cend; ++c) {
            const uint64_t cb = uint64_t(c) * kScatterChunk;
            const uint64_t ce = umin64(cb + kScatterChunk, n);
            if (chunk_full(c)) {
                uint4 cur[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) cur[u] = v[u];
                if (c + 1 < cend && chunk_full(c + 1)) load_chunk(c + 1);
                if (HYB && packed) {
                    // four keys at a time, no divergent path in the common case: both first probe
                    // slots of every key loaded up front (load <= 1/4: a third is rarely needed),
                    // then predicated atomics -- the bin counter of a normal key, the per-key
                    // counter of a sampled skewed one -- and one batched wrap test
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const uint32_t kk[4] = {cur[u].x, cur[u].y, cur[u].z, cur[u].w};
                        uint32_t hk[4], ka[4], kb[4], hid[4];
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            hk[q] = hash32(kk[q]);
                            if (CHECK) {
                                const uint32_t t = hk[q] >> rshift;
                                r_or |= t;
                                r_nor |= ~t;
                            }
                            const uint32_t s0 = hyb_slot(hk[q]);
                            ka[q] = s_hkey[s0];
                            kb[q] = s_hkey[(s0 + 1) & (kHybSlots - 1)];
                        }
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            const uint32_t s0 = hyb_slot(hk[q]);
                            uint32_t id = kNoHeavy;
                            if (hk[q] != kHybEmpty && ka[q] != kHybEmpty) {
                                if (ka[q] == hk[q]) id = s_hid[s0];
                                else if (kb[q] == hk[q]) id = s_hid[(s0 + 1) & (kHybSlots - 1)];
                                else if (kb[q] != kHybEmpty) id = hyb_find(s_hkey, s_hid, hk[q]);   // rare
                            }
                            hid[q] = id;
                        }
                        uint32_t old[4], rest = 0xffffffffu;
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            const uint32_t bin = (hk[q] >> shift) & mask;
                            const uint32_t inc = umax32((bin & 1u) << 16, 1u);
                            old[q] = 0;
                            if (hid[q] == kNoHeavy) old[q] = atomicAdd(&cnt[bin >> 1], inc);
                            else atomicAdd(&s_hc[hid[q]], 1u);
                        }
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            const uint32_t bin = (hk[q] >> shift) & mask;
                            const uint32_t m = umax32((bin & 1u) << 16, 1u) * 0xffffu;
                            rest = umin32(rest, hid[q] == kNoHeavy ? (~old[q] & m) : 1u);
                        }
                        if (__builtin_expect(rest == 0, 0))
#pragma unroll
                            for (int q = 0; q < 4; ++q) {
                                const uint32_t bin = (hk[q] >> shift) & mask;
                                const uint32_t m = umax32((bin & 1u) << 16, 1u) * 0xffffu;
                                if (hid[q] == kNoHeavy && (~old[q] & m) == 0) wrap_events(bin, old[q]);
                            }
                    }
                } else if (!HYB && packed) {
#pragma unroll
                    for (int h2 = 0; h2 < 2; ++h2) {
                        const uint32_t bins[8] = {bin_of(cur[2 * h2].x), bin_of(cur[2 * h2].y),
                                                  bin_of(cur[2 * h2].z), bin_of(cur[2 * h2].w),
                                                  bin_of(cur[2 * h2 + 1].x), bin_of(cur[2 * h2 + 1].y),
                                                  bin_of(cur[2 * h2 + 1].z), bin_of(cur[2 * h2 + 1].w)};
                        count_exact_batch(bins);
                    }
                } else {
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const uint32_t kk[4] = {cur[u].x, cur[u].y, cur[u].z, cur[u].w};
#pragma unroll
                        for (int q = 0; q < 4; ++q) count_key(kk[q]);
                    }
                }
            } else {  // the ragged last chunk, or keys not 16-byte aligned
                uint64_t done = cb;
                if (vec) {
                    const uint4* kv = reinterpret_cast<const uint4*>(keys + cb);
                    const uint64_t nv = (ce - cb) / 4;
                    for (uint64_t i = threadIdx.x; i < nv; i += blockDim.x) {
                        const uint4 w = ld_stream_u4(kv + i);
                        const uint32_t kk[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
                        for (int q = 0; q < 4; ++q) count_key(kk[q]);
                    }
                    done = cb + nv * 4;
                }
                for (uint64_t j = done + threadIdx.x; j < ce; j += blockDim.x) count_key(keys[j]);
            }
        }
        __syncthreads();
        if (HYB)   // the slice's skewed-key counts (every slice belongs to one side) and their totals
            for (uint32_t i = threadIdx.x; i < n_h0; i += blockDim.x) {
                const uint32_t c = s_hc[i];
                hyb_slice[(size_t(side ? nu0 : 0) + sl) * kHybMaxKeys + i] = c;
                if (c) {
                    atomicAdd(&hyb_cnt[side * kHybMaxKeys + i], c);
                    atomicMax(&s_href, c << 9 | i);
                    s_hc[i] = 0;
                }
            }
        // flush this slice's joint counts (and their per-d1 sums) and reset
        uint32_t* row = partial + (size_t(side ? nu0 : 0) + sl) * F;
        for (uint32_t w = threadIdx.x; w < nwords; w += blockDim.x) {
            const uint32_t x = cnt[w];
            uint32_t val;
            if (packed) {
                reinterpret_cast<uint2*>(row)[w] = make_uint2(x & 0xffffu, x >> 16);
                val = (x & 0xffffu) + (x >> 16);
            } else {
                row[w] = x;
                val = x;
            }
            cnt[w] = 0;
            const uint32_t d = (packed ? 2 * w : w) >> b2;
            if (per_d >= 32) {   // the warp's 32 words share one digit (whole warps: nwords % 32 == 0)
                const uint32_t sum = __reduce_add_sync(kFull, val);
                if ((threadIdx.x & 31) == 0 && sum) atomicAdd(&c1s[d], sum);
            } else if (val) {
                atomicAdd(&c1s[d], val);
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) {  // wrap corrections (sequential so repeated bins add up)
            for (uint32_t e = 0; e < umin32(n_ev, kHistMaxEvents); ++e) {
                row[ev_bin[e]] += ev_delta[e];
                c1s[ev_bin[e] >> b2] += ev_delta[e];
            }
            n_ev = 0;
        }
        __syncthreads();
        // the slice's dominant pass-1 digit (>= 1/8 of it: skewed data), for the pass-1 scatter
        const uint64_t slen = umin64(n, uint64_t(cend) * kScatterChunk) - uint64_t(c0) * kScatterChunk;
        if (threadIdx.x == 0) s_dom = 0;
        __syncthreads();
        if (threadIdx.x < d1n) {
            const uint32_t c = c1s[threadIdx.x];
            c1out[size_t(threadIdx.x) * nu + sl] = c;
            c1s[threadIdx.x] = 0;
            const uint32_t w = __reduce_max_sync(__activemask(),
                                                 (uint32_t)umin64(slen ? uint64_t(c) * 256 / slen : 0, 256) << 8 | threadIdx.x);
            if ((threadIdx.x & 31) == 0) atomicMax(&s_dom, w);
        }
        __syncthreads();
        if (threadIdx.x == 0) slice_dom[(side ? nu0 : 0) + sl] = (s_dom >> 8) >= 32 ? (s_dom & 255u) : 0xffffffffu;
        if (HYB && threadIdx.x == 0) {   // the slice's reference skewed key (pass 1 ranks it by ballot)
            hyb_ref[(side ? nu0 : 0) + sl] = (s_href >> 9) >= 64 ? (s_href & 511u) : kNoHeavy;
            s_href = 0;
        }
    }
    if (CHECK) {
        r_or = __reduce_or_sync(kFull, r_or);
        r_nor = __reduce_or_sync(kFull, r_nor);
        if ((threadIdx.x & 31) == 0 && (r_or & r_nor & ((1u << (32 - rshift)) - 1))) atomicOr(&st->route_mismatch, 1u);
    }
}

int launch_hist(const Plan& p, const uint32_t* k0, const uint32_t* k1, cudaStream_t s) {
    const uint32_t nbits = p.b1 + p.b2;
    const uint32_t shift = nbits ? (32 - p.route_bits - nbits) : 0;
    const uint32_t F = 1u << nbits;
    const size_t smem = size_t(F > (1u << 15) ? F / 2 : F) * 4;
    static std::once_flag attr_once[kMaxDevices];
    once_per_device(attr_once, [] {
        cudaFuncSetAttribute(k_hist2d<false, false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024);
        cudaFuncSetAttribute(k_hist2d<false, true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024);
        cudaFuncSetAttribute(k_hist2d<true, false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024);
        cudaFuncSetAttribute(k_hist2d<false, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024);
        cudaFuncSetAttribute(k_hist2d<false, true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024);
    });
    const bool fast16 = nbits == 16 && p.route_bits == 0 && p.b2 == 8;
    const uint32_t rshift = 32 - p.route_bits;
    // (Rejected, kept in history: CTA pairs each counting one half of 2^16 u32 bins -- every key
    // hashed twice, ALU-bound at 0.76 ms for 2^28 keys; a cluster pair exchanging bins through
    // DSMEM atomics, 3.6 ms, or DSMEM loads, 1.0 ms.)
    auto go = [&](auto kern) {
        kern<<<p.hist_grid, kHistBlock, smem, s>>>(k0, p.n[0], k1, p.n[1], shift, nbits, p.b2, p.hist_partial,
                                                   p.c1cnt, p.nu1[0], p.nu1[1], p.unit_chunks, rshift, p.st,
                                                   p.slice_dom, p.hyb_tab, p.n_h0, p.hyb_cnt, p.hyb_slice,
                                                   p.hyb_ref);
    };
    if (p.n_h0) {
        if (p.route_bits) go(k_hist2d<false, true, true>);
        else go(k_hist2d<false, false, true>);
    } else if (fast16) {
        go(k_hist2d<true, false, false>);
    } else if (p.route_bits) {
        go(k_hist2d<false, true, false>);
    } else {
        go(k_hist2d<false, false, false>);
    }
    return 1;
}

// --------------------------------------------- a2: reduce partials + pass-2 unit plan --
// One CTA per pass-1 partition row (side, d1); thread b handles final partition p = (d1, b).
//
// Pass-2 units: a unit is a range of consecutive histogram slices [c0, c1) of ONE pass-1
// partition: the runs those slices wrote into partition d1 in pass 1, contiguous there.  Slice s
// belongs to unit floor(P_incl(s) / T) (P_incl = tuples of d1 in slices <= s), so units hold about
// T tuples and a slice whose run alone exceeds T is a unit of its own: a skewed pass-1 partition
// (38 % of a side at theta = 1.5) spreads over many CTAs instead of one.  Units of large rows
// (>= 4x the mean row) are allocated from the front of the unit list, the rest from the back, so
// the dynamic claim order runs the biggest units first (longest-processing-time-first).
//
// Then per thread: cnt[side][p] = |R_p| / |S_p|, and off2[u][b] = tuples of p in the slices before
// unit u's first one (u's write offset in partition p, relative to the partition start).
constexpr int kSlicesPerThread = 16;
constexpr uint32_t kMaxSlices = 256 * kSlicesPerThread;   // >= 2^32 tuples / (64 chunks of 16K)

__global__ void __launch_bounds__(256) k_hist_reduce(const uint32_t* __restrict__ partial,
                                                     const uint32_t* __restrict__ c1cnt, uint32_t* __restrict__ cnt,
                                                     uint32_t* __restrict__ off2, uint4* __restrict__ uinfo,
                                                     uint32_t F, uint32_t b1, uint32_t b2, uint32_t ns0, uint32_t ns1,
                                                     uint32_t T, uint32_t big, uint32_t ucap, DevState* st) {
    __shared__ uint32_t starts[kMaxSlices + 1];
    __shared__ uint32_t scan_tmp[256 / 32 + 1];
    __shared__ uint32_t s_base, s_units;
    const uint32_t side = blockIdx.x >> b1, d1 = blockIdx.x & ((1u << b1) - 1);
    const uint32_t ns = side ? ns1 : ns0;
    const uint32_t* row = c1cnt + (side ? size_t(ns0) * 256 : 0) + size_t(d1) * ns;
    // (1) unit starts of this row: thread t owns slices [16t, 16t + 16) (ns <= kMaxSlices)
    constexpr int K = kSlicesPerThread;
    uint32_t v[K], loc = 0;
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const uint32_t sl = K * threadIdx.x + k;
        v[k] = sl < ns ? row[sl] : 0u;
        loc += v[k];
    }
    uint32_t rtot = 0;
    uint32_t pex = block_excl_scan_u32<256>(loc, &rtot, scan_tmp);   // tuples before my first slice
    uint32_t flag = 0, nflag = 0;   // flag bit k: slice K t + k starts a unit
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const uint32_t sl = K * threadIdx.x + k;
        const uint32_t pin = pex + v[k];
        // start: slice 0 of a non-empty row, or the unit id floor(P_incl / T) advances past a
        // non-empty prefix (leading empty slices stay in unit 0)
        const bool f = (sl < ns) && ((sl == 0 && rtot > 0) || (pex > 0 && pin / T > pex / T));
        flag |= uint32_t(f) << k;
        nflag += f;
        pex = pin;
    }
    __syncthreads();   // scan_tmp reuse
    uint32_t units = 0;
    uint32_t j = block_excl_scan_u32<256>(nflag, &units, scan_tmp);
#pragma unroll
    for (int k = 0; k < K; ++k)
        if ((flag >> k) & 1u) starts[j++] = K * threadIdx.x + k;
    if (threadIdx.x == 0) {
        starts[units] = ns;
        uint32_t base = 0;
        if (units) {
            if (rtot >= big) base = atomicAdd(&st->u2_front, units);
            else base = ucap - atomicAdd(&st->u2_back, units) - units;
        }
        s_base = base;
        s_units = units;
    }
    __syncthreads();
    const uint32_t ub = s_base, uc = s_units;
    for (uint32_t q = threadIdx.x; q < uc; q += blockDim.x)
        uinfo[ub + q] = make_uint4(side << 8 | d1, starts[q], starts[q + 1], 0xffffffffu);
    // (2) per final partition p = (d1, b): running sum over slices, recorded at unit starts
    const uint32_t b = threadIdx.x;
    uint32_t run = 0;
    if (b < (1u << b2)) {
        const uint32_t bin = (d1 << b2) | b;
        const uint32_t* base = partial + size_t(side ? ns0 : 0) * F + bin;
        uint32_t jj = 0, next = uc ? starts[0] : 0xffffffffu;
        for (uint32_t s = 0; s < ns; s += 8) {   // 8 loads in flight per thread
            uint32_t x[8];
#pragma unroll
            for (int k = 0; k < 8; ++k) x[k] = (s + k < ns) ? base[size_t(s + k) * F] : 0u;
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                if (s + k == next) {
                    off2[(size_t(ub + jj) << b2) + b] = run;
                    ++jj;
                    next = jj < uc ? starts[jj] : 0xffffffffu;
                }
                run += x[k];
            }
        }
        cnt[size_t(side) * F + bin] = run;
    }
    // (3) the row's dominant final partition (>= 1/8 of the row: skewed data) for every unit of
    // the row: the pass-2 scatter ranks its tuples with ballots instead of shared atomics
    const uint32_t w = __reduce_max_sync(kFull, (uint32_t)umin64(rtot ? uint64_t(run) * 256 / rtot : 0, 256) << 8 | b);
    __syncthreads();   // scan_tmp is free
    if ((threadIdx.x & 31) == 0) scan_tmp[threadIdx.x >> 5] = w;
    __syncthreads();
    uint32_t best = 0;
    for (int i = 0; i < 8; ++i) best = umax32(best, scan_tmp[i]);
    const uint32_t dom = (best >> 8) >= 32 ? (best & 255u) : 0xffffffffu;
    for (uint32_t q = threadIdx.x; q < uc; q += blockDim.x) uinfo[ub + q].w = dom;
}

struct CountAt {
    const uint32_t* c;
    __device__ uint64_t operator()(uint64_t i) const { return c[i]; }
};

// Pass-1 unit counts in (digit, unit) order: the exclusive scan in that order IS the output
// offset of unit u's bucket-d run (start of bucket d + runs of d in earlier units).
struct ChunkDigit {
    const uint32_t* c1;   // [256][nu1] digit-major
    __device__ uint64_t operator()(uint64_t i) const { return c1[i]; }
};

int launch_hist_reduce_scan(const Plan& p, cudaStream_t s) {
    const uint32_t F = p.F;
    const uint64_t mean_row = (p.n[0] + p.n[1]) / (2ull << p.b1);
    const uint32_t big = (uint32_t)umin64(4 * mean_row + 1, 0xffffffffull);
    k_hist_reduce<<<2u << p.b1, 256, 0, s>>>(p.hist_partial, p.c1cnt, p.cnt, p.off2, p.u2_info, F, p.b1, p.b2,
                                             p.nu1[0], p.nu1[1], p.u2_target, big, p.u2_max[0] + p.u2_max[1], p.st);
    // four independent scans in one launch triple: partition starts per side, pass-1
    // (digit, unit) offsets per side
    ScanSegs g{};
    g.k = 4;
    uint64_t off = 0;
    for (int side = 0; side < 2; ++side) {
        g.in[side] = p.cnt + size_t(side) * F;
        g.out[side] = p.start + size_t(side) * (F + 1);
        g.n[side] = F;
        const uint64_t m = uint64_t(p.nu1[side]) * 256;
        g.in[2 + side] = p.c1cnt + (side ? size_t(p.nu1[0]) * 256 : 0);
        g.out[2 + side] = p.off1 + off;
        g.n[2 + side] = m;
        off += m + 1;
    }
    return 1 + launch_scan_u32_multi(g, p.scan_scratch, s);
}

// ------------------------------------------------------------- a3/a4: tile scatter --
// Work unit: pass 1 = one pass-1 chunk (kScatterChunk input tuples); pass 2 = (pass-1 digit d1,
// chunk group g) = the runs that the chunks of group g wrote into pass-1 partition d1 -- a
// contiguous slice of that partition.  Every unit's per-bucket output offsets are known before
// the pass (histogram pass + scans: "count then partition"), so a CTA streams its
// unit with no cross-CTA dependency and writes each bucket as ONE contiguous run, which lets it
// combine writes into whole 32-byte sectors (partial-sector stores cost ~1.7x on this part:
// scripts/microbench_scatter_ceiling.cu).
struct ScatterArgs {
    const uint32_t* keys[2];   // pass 1 input (SoA)
    const uint32_t* pays[2];
    const uint2* in[2];        // pass 2 input (AoS pass-1 output)
    uint2* out[2];
    const uint64_t* start[2];  // final partition starts [F + 1] per side
    const uint64_t* off1[2];   // [256 * nu1 + 1] per side: start of unit u's run of digit d at d*nu1 + u
    const uint32_t* off2;      // [pass-2 unit][2^b2]: unit's write offset in each of its partitions
    const uint4* u2_info;      // pass-2 units (side << 8 | d1, first slice, end slice, dominant bucket)
    const uint32_t* p1_dom;    // pass-1 units: dominant pass-1 digit of the slice, or 0xffffffff
    const unsigned int* u2_fb;      // (front, back) unit counts (device, from k_hist_reduce)
    uint32_t u2_cap;           // unit list capacity: front units at [0, f), back units at [cap - b, cap)
    uint64_t n[2];
    uint32_t nu1[2];           // pass-1 units (= histogram slices) per side
    uint32_t unit_len;         // tuples per pass-1 unit
    uint32_t pass, b1, b2, route_bits;
    unsigned int* unit_ctr;
    // hybrid pass 1 (HYB): sampled skewed keys' table, their count, R_k / S_k offsets, cursors, arrays
    const uint32_t* hyb_tab;
    uint32_t n_h0;
    const uint64_t* hyb_off[2];   // per side [kHybMaxKeys][nu1]: (key, unit) write offsets
    const uint32_t* hyb_ref;      // per pass-1 unit: its most frequent skewed key (ballot-ranked) or ~0
    uint32_t* heavy_pay[2];
};

struct ScatterSmem {
    uint32_t tcnt[256];                 // tile bucket counters -> ranks
    uint32_t local_start[256];          // bucket start inside the staged tile
    uint32_t run[256];                  // next output index of bucket b for this unit
    uint32_t wpos[256];                 // first index of bucket b not yet written to memory
    uint2 gw[256];                      // bucket b: (output index of stage position 0 (mod 2^32),
                                        //            write-out limit for the current tile)
    uint32_t tailpos[256];              // stage position of bucket b's carried tail
    uint2 cbuf[256][4];                 // carry: < 4 tuples (one 32 B sector) per bucket
    uint32_t carry[256];                // tuples in cbuf[b]
    uint32_t scan_tmp[33];
    uint32_t claim;
    uint32_t wdom[32];                  // per warp: tuples of the dominant bucket in this tile
    uint32_t wdoff[32];                 // their exclusive prefix over warps
    uint64_t mbar;                      // TMA completion of the tile buffer
};

struct UnitInfo {
    int side;
    uint32_t d1, grp, len;
    uint32_t dom;   // dominant bucket of the unit (skewed data) or 0xffffffff
    uint64_t begin;
};

// Pass 1: unit u = histogram slice (side 1 from units0 on).  Pass 2: claim index u maps to the
// unit list's front part [0, units0) or, shifted by back_off, its back part.
__device__ __forceinline__ UnitInfo unit_info(const ScatterArgs& a, uint32_t u, uint32_t units0, uint32_t back_off,
                                              bool p1) {
    UnitInfo ui;
    ui.side = (u >= units0) ? 1 : 0;
    const uint32_t lu = u - (ui.side ? units0 : 0);
    const uint32_t nch = a.nu1[ui.side];
    if (p1) {
        ui.d1 = 0;
        ui.grp = lu;
        ui.begin = uint64_t(lu) * a.unit_len;
        ui.len = (uint32_t)umin64(a.unit_len, a.n[ui.side] - ui.begin);
        ui.dom = a.p1_dom[u];
    } else {
        const uint32_t li = u < units0 ? u : u + back_off;
        const uint4 inf = a.u2_info[li];
        ui.side = (int)(inf.x >> 8);
        ui.d1 = inf.x & 255u;
        ui.grp = li;
        const uint32_t nc = a.nu1[ui.side];
        ui.begin = a.off1[ui.side][size_t(ui.d1) * nc + inf.y];
        ui.len = (uint32_t)(a.off1[ui.side][size_t(ui.d1) * nc + inf.z] - ui.begin);
        ui.dom = inf.w;
    }
    return ui;
}

// Which tile elements arrive by TMA bulk copy (pass 1, SoA): [head, head + nbulk); element i lives
// at shared index i + shift.  The rest (a tail that is not a multiple of 16 bytes, or everything
// when the SoA inputs are not 16-byte aligned) is loaded by its owning thread with ordinary loads.
struct LoadPlan {
    uint32_t head, nbulk, shift;
};

__device__ __forceinline__ LoadPlan load_plan(const ScatterArgs& a, int side, uint64_t begin, uint32_t len, bool p1) {
    LoadPlan lp;
    if (p1) {
        const uintptr_t k = reinterpret_cast<uintptr_t>(a.keys[side] + begin);
        const uintptr_t q = reinterpret_cast<uintptr_t>(a.pays[side] + begin);
        const bool al = ((k | q) & 15u) == 0;
        lp.head = al ? 0 : len;
        lp.nbulk = al ? (len & ~3u) : 0;
        lp.shift = 0;
    } else {  // pass 2 always copies the 16-byte-aligned superset (see tile_geo)
        lp.head = 0;
        lp.nbulk = len;
        lp.shift = 0;
    }
    return lp;
}

// Tile q of a unit [begin, begin + len).  Pass 1: TILE-aligned tiles of the (chunk-aligned) unit.
// Pass 2 (AoS, 8-byte tuples): the first tile is one tuple shorter when `begin` is odd, so every
// tile's 16-byte-aligned superset [tb - off, tb + ql rounded up to even) holds at most TILE tuples
// and arrives by ONE bulk copy; the superset's extra (neighbouring units') tuples are masked.  The
// workspace keeps >= 1 tuple of slack after each side, so the round-up never leaves it.
struct TileGeo {
    uint64_t tb;
    uint32_t ql, off;
};

template <int TILE>
__device__ __forceinline__ uint32_t tile_count(bool p1, uint64_t begin, uint32_t len) {
    return p1 ? (len + TILE - 1) / TILE : (len + uint32_t(begin & 1) + TILE - 1) / TILE;
}

template <int TILE>
__device__ __forceinline__ TileGeo tile_geo(bool p1, uint64_t begin, uint32_t len, uint32_t q) {
    TileGeo g;
    if (p1) {
        g.tb = begin + uint64_t(q) * TILE;
        g.ql = umin32(TILE, len - q * TILE);
        g.off = 0;
    } else {
        const uint32_t lead = uint32_t(begin & 1);
        if (q == 0) {
            g.tb = begin;
            g.ql = umin32(TILE - lead, len);
            g.off = lead;
        } else {
            g.tb = begin - lead + uint64_t(q) * TILE;
            g.ql = (uint32_t)umin64(TILE, begin + len - g.tb);
            g.off = 0;
        }
    }
    return g;
}

// Thread 0: arm `bar` and issue the bulk copies of tile g (read once: evict-first).
__device__ __forceinline__ void tile_issue(const ScatterArgs& a, int side, const TileGeo& g, bool p1, uint32_t* kdst,
                                           uint32_t* pdst, uint2* adst, uint64_t* bar, uint64_t pol) {
    if (p1) {
        const LoadPlan lp = load_plan(a, side, g.tb, g.ql, p1);
        const uint32_t bytes = lp.nbulk * 4;
        mbar_arrive_expect_tx(bar, 2 * bytes);
        if (bytes) {
            bulk_g2s_hint(kdst, a.keys[side] + g.tb, bytes, bar, pol);
            bulk_g2s_hint(pdst, a.pays[side] + g.tb, bytes, bar, pol);
        }
    } else {
        const uint32_t bytes = ((g.ql + g.off + 1) & ~1u) * 8;
        mbar_arrive_expect_tx(bar, bytes);
        if (bytes) bulk_g2s_hint(adst, a.in[side] + (g.tb - g.off), bytes, bar, pol);
    }
}

// TMAST: whole-sector bucket runs leave the staging buffer as TMA bulk stores (one per bucket
// and tile, issued by the bucket's thread) instead of per-tuple stores.
// HYB (pass 1, gsh_config.hybrid -- CSH's hybrid partition, L90-L91, L100): a tuple of a sampled
// skewed key is ranked per key in the tile (rank | 0x4000), the unit's running offset of the key
// (from the histogram pass: no atomics) places the tile's run in R_k / S_k, and its payload is
// stored there instead of being staged: it never reaches a partition.
template <int BLOCK, int IPT, int PASS, bool TMAST, bool HYB = false>
__global__ void __launch_bounds__(BLOCK, kScatterMinBlocks) k_scatter(ScatterArgs a) {
    constexpr int TILE = BLOCK * IPT;
    static_assert(TILE < 0x7fff, "ranks are packed as u16: bit 15 = dominant bucket, 0xffff = masked");
    extern __shared__ __align__(128) unsigned char smem_raw[];
    ScatterSmem& S = *reinterpret_cast<ScatterSmem*>(smem_raw);
    unsigned char* buf0 = smem_raw + ((sizeof(ScatterSmem) + 127) & ~size_t(127));
    uint32_t* ok = reinterpret_cast<uint32_t*>(buf0);   // pass 1: keys -> h
    uint32_t* op = ok + TILE + 4;                       // pass 1: payloads
    uint2* o2 = reinterpret_cast<uint2*>(buf0);         // pass 2: (h, payload)
    uint2* stage = reinterpret_cast<uint2*>(buf0 + (size_t(TILE) + 4) * 8);
    unsigned char* hyb0 = buf0 + (size_t(TILE) + 4) * 8 + (size_t(TILE) + 4 * 256 + 4) * 8;
    uint32_t* hkey = reinterpret_cast<uint32_t*>(hyb0);                        // [kHybSlots]
    uint32_t* hcnt = hkey + kHybSlots;                                          // [kHybMaxKeys] tile ranks
    uint32_t* hbase = hcnt + kHybMaxKeys;                                       // [kHybMaxKeys] run starts
    uint32_t* hrun = hbase + kHybMaxKeys;                                       // [kHybMaxKeys] unit cursors
    uint32_t* hwref = hrun + kHybMaxKeys;                                       // [32] per warp: ref-key tuples
    uint32_t* hwoff = hwref + 32;                                               // [32] their prefix over warps
    uint16_t* hid16 = reinterpret_cast<uint16_t*>(hwoff + 32);                  // [kHybSlots]
    static_assert(!HYB || PASS == 1, "hybrid routing happens in pass 1");
    static_assert(!HYB || BLOCK * IPT < 0x2000, "hybrid ranks are tagged 0x4000 | [0x2000 ref |] rank");

    const uint32_t tid = threadIdx.x;
    constexpr bool p1 = (PASS == 1);
    const uint32_t bits = p1 ? a.b1 : a.b2;
    const uint32_t nb = 1u << bits;
    const uint32_t dmask = nb - 1;
    const uint32_t dshift = (32 - a.route_bits - a.b1 - (p1 ? 0 : a.b2)) & 31;
    const uint32_t lowbits = p1 ? a.b2 : 0;
    const uint32_t units0 = p1 ? a.nu1[0] : a.u2_fb[0];
    const uint32_t total = p1 ? a.nu1[0] + a.nu1[1] : a.u2_fb[0] + a.u2_fb[1];
    const uint32_t back_off = p1 ? 0u : a.u2_cap - total;
    const uint64_t rpol = policy_evict_first(), wpol = policy_evict_first();

    if (tid < 256) S.tcnt[tid] = 0;
    if (HYB) {
        for (uint32_t i = tid; i < kHybSlots; i += BLOCK) {
            hkey[i] = a.hyb_tab[i];
            hid16[i] = reinterpret_cast<const uint16_t*>(a.hyb_tab + kHybSlots)[i];
        }
        for (uint32_t i = tid; i < kHybMaxKeys; i += BLOCK) hcnt[i] = 0;
    }
    if (tid == 0) {
        mbar_init(&S.mbar, 1);
        S.claim = atomicAdd(a.unit_ctr, 1u);
    }
    __syncthreads();
    uint32_t u = S.claim;
    __syncthreads();   // every thread has read the first claim before thread 0 claims again
    uint32_t par = 0;
    bool issued = false;   // first tile of unit u already in flight
    while (u < total) {
        const UnitInfo ui = unit_info(a, u, units0, back_off, p1);
        const uint32_t ntile = tile_count<TILE>(p1, ui.begin, ui.len);
        if (ntile == 0) {  // empty unit (pass 2: digit absent from the group)
            __syncthreads();
            if (tid == 0) S.claim = atomicAdd(a.unit_ctr, 1u);
            __syncthreads();
            u = S.claim;
            continue;
        }
        if (tid == 0 && !issued)
            tile_issue(a, ui.side, tile_geo<TILE>(p1, ui.begin, ui.len, 0), p1, ok, op, o2, &S.mbar, rpol);
        if (tid < nb) {
            uint32_t r0;
            const uint32_t pidx = ((ui.d1 << bits) | tid) << lowbits;
            if (p1) r0 = (uint32_t)a.off1[ui.side][size_t(tid) * a.nu1[ui.side] + ui.grp];
            else r0 = (uint32_t)a.start[ui.side][pidx] + a.off2[(size_t(ui.grp) << a.b2) + tid];
            S.run[tid] = r0;
            S.wpos[tid] = r0;
            S.carry[tid] = 0;
        }
        if constexpr (HYB)   // the unit's offset of every skewed key (read after the first barrier)
            for (uint32_t i = tid; i < a.n_h0; i += BLOCK) {
                GSH_BOUNDS(ui.grp < a.nu1[ui.side], "hybrid pass 1: unit index");
                hrun[i] = (uint32_t)a.hyb_off[ui.side][size_t(i) * a.nu1[ui.side] + ui.grp];
            }
        const uint32_t href = HYB ? a.hyb_ref[u] : kNoHeavy;   // pass 1: u indexes the slices
        // Dominant bucket (skewed data: one key's bucket holds >= 1/8 of the slice / pass-1
        // partition, from the histogram pass): its tuples are ranked with warp ballots and per-warp
        // register counters instead of shared-memory atomics, which serialise when most lanes of
        // every warp hit the same counter.
        const uint32_t dom = ui.dom;
        const bool dom_on = dom != 0xffffffffu;
        // (the first sync of the tile loop orders run[] before its use)
        uint32_t un = total;
        for (uint32_t q = 0; q < ntile; ++q) {
            const TileGeo geo = tile_geo<TILE>(p1, ui.begin, ui.len, q);
            const uint32_t ql = geo.ql;
            const uint64_t tb = geo.tb;
            const LoadPlan lp = load_plan(a, ui.side, tb, ql, p1);
            // pass 2 always takes the vector path (masked superset); pass 1 when the tile is whole
            const bool full = !p1 || ((ql == TILE) && lp.head == 0 && lp.nbulk == TILE);
            const bool last = (q + 1 == ntile);
            if (tid == 0 && last) S.claim = atomicAdd(a.unit_ctr, 1u);
            // TMA-prefetch the next tile (of this unit, or the first of the next unit) into the
            // input buffer once this tile's input has been consumed
            auto issue_next = [&]() {
                if (tid == 0) {
                    if (!last) {
                        tile_issue(a, ui.side, tile_geo<TILE>(p1, ui.begin, ui.len, q + 1), p1, ok, op, o2, &S.mbar,
                                   rpol);
                    } else if (un < total) {
                        const UnitInfo nx = unit_info(a, un, units0, back_off, p1);
                        if (nx.len)
                            tile_issue(a, nx.side, tile_geo<TILE>(p1, nx.begin, nx.len, 0), p1, ok, op, o2, &S.mbar,
                                       rpol);
                    }
                }
            };
            mbar_wait(&S.mbar, par);
            par ^= 1;
            uint32_t rk[IPT / 2];  // ranks, packed 2 x u16 (bit 15: dominant-bucket rank; 0xffff: masked)
            uint32_t wrun = 0;     // this warp's dominant-bucket tuples so far in this tile
            uint32_t wref = 0;     // HYB: this warp's tuples of the unit's reference skewed key
            // rank of one tuple of bucket b: dominant bucket by ballot, others by shared atomics
            // full tile: the input stays in registers from the ranking to the staging step, so
            // the input buffer is free (and the next tile's TMA issued) after the first barrier
            constexpr int NV = p1 ? IPT / 4 : IPT / 2;
            uint4 xa[NV], xb[p1 ? NV : 1];
            // (two instantiations of the full-tile ranking: DOM = the unit has a dominant bucket)
            auto rank_tile = [&](auto dom_tag) {
                constexpr bool DOM = decltype(dom_tag)::value;
                auto rank_of = [&](bool valid, uint32_t b) -> uint32_t {
                    if constexpr (DOM) {
                        const bool isd = valid && b == dom;
                        const uint32_t m = __ballot_sync(kFull, isd);
                        uint32_t r = 0xffffu;
                        if (isd) r = 0x8000u | (wrun + __popc(m & lanemask_lt()));
                        else if (valid) r = atomicAdd(&S.tcnt[b], 1u);
                        wrun += __popc(m);
                        return r;
                    } else {
                        return valid ? atomicAdd(&S.tcnt[b], 1u) : 0xffffu;
                    }
                };
                if (p1) {    // uint4 = 4 keys; slot 4 * v + c of element 4 * (v * BLOCK + tid) + c
                    // a sampled skewed key's tuple: ranked among its key's tuples in the tile
                    auto rank1 = [&](uint32_t h) -> uint32_t {
                        if constexpr (HYB) {
                            // the reference key by ballot (0x2000 | rank in the warp's run), other
                            // skewed keys by shared atomics
                            const uint32_t hid = hyb_find2(hkey, hid16, h);
                            const uint32_t r = rank_of(hid == kNoHeavy, (h >> dshift) & dmask);
                            const bool isref = hid != kNoHeavy && hid == href;
                            const uint32_t m = __ballot_sync(kFull, isref);
                            uint32_t hr = 0;
                            if (isref) hr = 0x2000u | (wref + __popc(m & lanemask_lt()));
                            else if (hid != kNoHeavy) hr = atomicAdd(&hcnt[hid], 1u);
                            wref += __popc(m);
                            return hid == kNoHeavy ? r : (0x4000u | hr);
                        } else {
                            return rank_of(true, (h >> dshift) & dmask);
                        }
                    };
#pragma unroll
                    for (int v = 0; v < NV; ++v) {
                        uint4 x = reinterpret_cast<const uint4*>(ok)[v * BLOCK + tid];
                        xb[v] = reinterpret_cast<const uint4*>(op)[v * BLOCK + tid];
                        x.x = hash32(x.x); x.y = hash32(x.y); x.z = hash32(x.z); x.w = hash32(x.w);
                        xa[v] = x;
                        const uint32_t r0 = rank1(x.x);
                        const uint32_t r1 = rank1(x.y);
                        const uint32_t r2 = rank1(x.z);
                        const uint32_t r3 = rank1(x.w);
                        rk[2 * v] = r0 | (r1 << 16);
                        rk[2 * v + 1] = r2 | (r3 << 16);
                    }
                } else {     // uint4 = 2 AoS tuples: shared slots 2u, 2u + 1 = tile elements 2u - off, ...
#pragma unroll
                    for (int v = 0; v < NV; ++v) {
                        const uint32_t i0 = 2 * (v * BLOCK + tid) - geo.off;   // wraps for slot 0 when off = 1
                        const uint4 x = reinterpret_cast<const uint4*>(o2)[v * BLOCK + tid];
                        xa[v] = x;
                        // 0xffff = not in this tile
                        const uint32_t r0 = rank_of(i0 < ql, (x.x >> dshift) & dmask);
                        const uint32_t r1 = rank_of(i0 + 1 < ql, (x.z >> dshift) & dmask);
                        rk[v] = r0 | (r1 << 16);
                    }
                }
            };
            if (full) {  // whole tile arrived by TMA: vector shared loads, no bounds checks
                if (dom_on) rank_tile(std::true_type{});
                else rank_tile(std::false_type{});
                fence_proxy_async_smem();  // reads of the input tile precede the next TMA writes
            } else {
#pragma unroll
                for (int jj = 0; jj < IPT; ++jj) {
                    const uint32_t i = jj * BLOCK + tid;
                    uint32_t r = 0;
                    if (i < ql) {
                        const bool bulk = (i - lp.head) < lp.nbulk;
                        uint32_t h;
                        if (p1) {
                            uint32_t k;
                            if (bulk) {
                                k = ok[i];
                            } else {
                                k = a.keys[ui.side][tb + i];
                                op[i] = a.pays[ui.side][tb + i];
                            }
                            h = hash32(k);
                            ok[i] = h;
                        } else {
                            if (bulk) {
                                h = o2[i + lp.shift].x;
                            } else {
                                const uint2 e = a.in[ui.side][tb + i];
                                o2[i + lp.shift] = e;
                                h = e.x;
                            }
                        }
                        uint32_t hid = kNoHeavy;
                        if constexpr (HYB) hid = hyb_find2(hkey, hid16, h);
                        r = hid == kNoHeavy ? atomicAdd(&S.tcnt[(h >> dshift) & dmask], 1u)
                                            : (0x4000u | atomicAdd(&hcnt[hid], 1u));
                    }
                    if (jj & 1) rk[jj >> 1] |= r << 16; else rk[jj >> 1] = r;
                }
            }
            if ((tid & 31) == 0) S.wdom[tid >> 5] = wrun;
            if (HYB && (tid & 31) == 0) hwref[tid >> 5] = wref;
            // the previous tile's bulk stores must have read the staging buffer before any thread
            // writes it again (after the barrier below)
            if (TMAST && tid < nb) bulk_wait_read0();
            __syncthreads();
            if (last) un = S.claim;
            if (full) issue_next();
            // Write combining: bucket b's staged run = [carry from the previous tile | this tile's
            // tuples]; only whole 32-byte sectors are written, the < 4-tuple remainder carries
            // over (the unit's last tile flushes everything).  u32 offsets (n < 2^32).
            if constexpr (HYB) {   // place this tile's run of every skewed key it holds
                for (uint32_t i = tid; i < a.n_h0; i += BLOCK) {
                    const uint32_t c = hcnt[i];
                    if (c && i != href) {
                        hbase[i] = hrun[i];
                        hrun[i] += c;
                        hcnt[i] = 0;
                    }
                }
                if (href != kNoHeavy && tid < 32) {   // the reference key: ballot ranks (full tiles)
                    constexpr uint32_t NW = BLOCK / 32;   // + atomic ranks (ragged tiles), never both
                    const uint32_t c = tid < NW ? hwref[tid] : 0u;
                    uint32_t x = c;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint32_t y = __shfl_up_sync(kFull, x, o);
                        if (tid >= (uint32_t)o) x += y;
                    }
                    if (tid < NW) hwoff[tid] = x - c;
                    const uint32_t tot = __shfl_sync(kFull, x, 31) + hcnt[href];
                    if (tid == 0) {
                        hbase[href] = hrun[href];
                        hrun[href] += tot;
                        hcnt[href] = 0;
                    }
                }
            }
            uint32_t tc = (tid < nb) ? S.tcnt[tid] : 0u;
            if (dom_on) {
                constexpr uint32_t NW = BLOCK / 32;
                if (tid == dom)
                    for (uint32_t w = 0; w < NW; ++w) tc += S.wdom[w];
                if (tid < 32) {   // exclusive prefix of the warps' dominant counts
                    const uint32_t c = tid < NW ? S.wdom[tid] : 0u;
                    uint32_t x = c;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint32_t y = __shfl_up_sync(kFull, x, o);
                        if (tid >= (uint32_t)o) x += y;
                    }
                    if (tid < NW) S.wdoff[tid] = x - c;
                }
            }
            const uint32_t cin = (tid < nb) ? S.carry[tid] : 0u;
            uint32_t all;
            // TMAST: one spare slot per bucket so the run starts at the parity of its output index
            // (16-byte alignment of both ends of the bulk store)
            uint32_t lstart = block_excl_scan_1bar<256 / 32>(tc + cin + ((TMAST && tid < nb) ? 1u : 0u), &all, S.scan_tmp);
            uint32_t my_w0 = 0, my_ew = 0;
            if (tid < nb) {
                const uint32_t nxt = S.run[tid] + tc;
                const uint32_t w0 = S.wpos[tid];
                uint32_t ew = last ? nxt : (nxt & ~3u);
                if (ew < w0) ew = w0;
                if (TMAST) lstart += (lstart ^ w0) & 1u;
                my_w0 = w0;
                my_ew = ew;
                S.local_start[tid] = lstart + cin;
                S.gw[tid] = make_uint2(w0 - lstart, ew);
                S.tailpos[tid] = lstart + (ew - w0);
                for (uint32_t k = 0; k < cin; ++k) stage[lstart + k] = S.cbuf[tid][k];
                S.wpos[tid] = ew;
                S.run[tid] = nxt;
                S.carry[tid] = nxt - ew;
                S.tcnt[tid] = 0;
            }
            __syncthreads();
            if (full) {
                // staging position of a tuple of bucket b with rank r (bit 15: dominant bucket)
                const uint32_t dbase = dom_on ? S.local_start[dom & 255u] + S.wdoff[tid >> 5] : 0u;
                auto spos = [&](uint32_t b, uint32_t r) {
                    return (r & 0x8000u) ? dbase + (r & 0x7fffu) : S.local_start[b] + r;
                };
                if (p1) {
                    // staged, or (hybrid: rank tagged 0x4000, dominant bit clear) stored into R_k / S_k
                    auto put = [&](uint32_t h, uint32_t pay, uint32_t r) {
                        if (HYB && (r & 0xc000u) == 0x4000u) {
                            const uint32_t pos = (r & 0x2000u) ? hbase[href] + hwoff[tid >> 5] + (r & 0x1fffu)
                                                               : hbase[hyb_find2(hkey, hid16, h)] + (r & 0x1fffu);
                            GSH_BOUNDS(pos < a.n[ui.side], "hybrid pass 1: skewed payload position");
                            a.heavy_pay[ui.side][pos] = pay;
                        } else
                            stage[spos((h >> dshift) & dmask, r)] = make_uint2(h, pay);
                    };
#pragma unroll
                    for (int v = 0; v < NV; ++v) {
                        const uint4 h4 = xa[v], p4 = xb[v];
                        put(h4.x, p4.x, rk[2 * v] & 0xffffu);
                        put(h4.y, p4.y, rk[2 * v] >> 16);
                        put(h4.z, p4.z, rk[2 * v + 1] & 0xffffu);
                        put(h4.w, p4.w, rk[2 * v + 1] >> 16);
                    }
                } else {   // ranks < TILE <= 0x7fff, so 0xffff marks a masked slot
#pragma unroll
                    for (int v = 0; v < NV; ++v) {
                        const uint4 x = xa[v];
                        const uint32_t r0 = rk[v] & 0xffffu, r1 = rk[v] >> 16;
                        if (r0 != 0xffffu) stage[spos((x.x >> dshift) & dmask, r0)] = make_uint2(x.x, x.y);
                        if (r1 != 0xffffu) stage[spos((x.z >> dshift) & dmask, r1)] = make_uint2(x.z, x.w);
                    }
                }
            } else {
#pragma unroll
                for (int jj = 0; jj < IPT; ++jj) {
                    const uint32_t i = jj * BLOCK + tid;
                    if (i < ql) {
                        const uint2 e = p1 ? make_uint2(ok[i], op[i]) : o2[i + lp.shift];
                        const uint32_t r = (jj & 1) ? (rk[jj >> 1] >> 16) : (rk[jj >> 1] & 0xffffu);
                        if (HYB && (r & 0xc000u) == 0x4000u) {
                            const uint32_t pos = hbase[hyb_find2(hkey, hid16, e.x)] + (r & 0x1fffu);
                            GSH_BOUNDS(pos < a.n[ui.side], "hybrid pass 1 (ragged tile): skewed payload position");
                            a.heavy_pay[ui.side][pos] = e.y;
                        }
                        else
                            stage[S.local_start[(e.x >> dshift) & dmask] + r] = e;
                    }
                }
                fence_proxy_async_smem();  // reads of the input tile precede the next TMA writes
            }
            if (TMAST) fence_proxy_async_smem();  // staging writes precede the bulk stores' reads
            __syncthreads();
            if (!full) issue_next();
            // the < 4-tuple tail of each bucket moves to its carry slot; whole sectors go out
            if (tid < nb)
                for (uint32_t k = 0; k < S.carry[tid]; ++k) S.cbuf[tid][k] = stage[S.tailpos[tid] + k];
            uint2* out = a.out[ui.side];
            if (TMAST) {
                // bucket tid's run [w0, ew) sits at stage[lstart ...]: an odd first index and an
                // odd last one go out as single stores, the even-aligned middle as one bulk store
                if (tid < nb && my_ew > my_w0) {
                    const uint32_t hs = my_w0 & 1u;
                    if (hs) st_stream_u2(out + my_w0, stage[lstart], wpol);
                    const uint32_t a0 = my_w0 + hs;
                    const uint32_t n2 = (my_ew - a0) & ~1u;
                    if (n2) bulk_s2g_hint(out + a0, stage + lstart + hs, n2 * 8, wpol);
                    if (a0 + n2 < my_ew) st_stream_u2(out + (my_ew - 1), stage[lstart + (my_ew - 1 - my_w0)], wpol);
                    bulk_commit();
                }
            } else {
#pragma unroll 4
                for (uint32_t i = tid; i < all; i += BLOCK) {
                    const uint2 e = stage[i];
                    const uint2 ge = S.gw[(e.x >> dshift) & dmask];
                    const uint32_t g = ge.x + i;
                    GSH_BOUNDS(g >= ge.y || g < a.n[ui.side], "scatter: output position");
                    if (g < ge.y) st_stream_u2(out + g, e, wpol);
                }
            }
            // No barrier here: the next tile's ranking touches only the input buffer and tcnt
            // (reset in phase B), and everything this write-out reads (stage, gw, carry,
            // tailpos) is rewritten only after the next tile's first barrier.
        }
        u = un;
        issued = true;  // the next unit's first tile (if any, and non-empty) is in flight
        if (u < total && unit_info(a, u, units0, back_off, p1).len == 0) issued = false;
    }
    if (TMAST && tid < nb) bulk_wait0();  // shared memory must outlive the bulk stores' reads
}

size_t scatter_smem_bytes(int tile, bool hyb = false) {
    // input tile (+4 slack) and staging = tile + up to 3 carried tuples per bucket (+ the hybrid
    // table, tile ranks and run starts)
    return ((sizeof(ScatterSmem) + 127) & ~size_t(127)) + (size_t(tile) + 4) * 8 + (size_t(tile) + 4 * 256 + 4) * 8 +
           (hyb ? size_t(kHybSlots) * 6 + size_t(kHybMaxKeys) * 12 + 64 * 4 : 0);
}

template <int BLOCK, int IPT, int PASS, bool TMAST, bool HYB = false>
int launch_scatter_pass(const Plan& p, const ScatterArgs& a, cudaStream_t s) {
    const size_t smem = scatter_smem_bytes(BLOCK * IPT, HYB);
    static std::once_flag attr_once[kMaxDevices];   // > 48 KB of dynamic shared memory: opt in once per device
    once_per_device(attr_once, [&] {
        cudaFuncSetAttribute(k_scatter<BLOCK, IPT, PASS, TMAST, HYB>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smem);
    });
    static int occ_dev[kMaxDevices] = {0};   // per kernel instance and device: query once
    int dev = 0;
    cudaGetDevice(&dev);
    int& occ = occ_dev[dev >= 0 && dev < kMaxDevices ? dev : 0];
    if (occ < 1) {
        int o = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, k_scatter<BLOCK, IPT, PASS, TMAST, HYB>, BLOCK, smem);
        occ = o < 1 ? 1 : o;
    }
    k_scatter<BLOCK, IPT, PASS, TMAST, HYB><<<(unsigned)(p.num_sms * occ), BLOCK, smem, s>>>(a);
    return 1;
}
template <int BLOCK, int IPT, bool TMAST>
int launch_scatter_cfg(const Plan& p, const ScatterArgs& a, cudaStream_t s) {
    return a.pass == 1 ? launch_scatter_pass<BLOCK, IPT, 1, TMAST>(p, a, s)
                       : launch_scatter_pass<BLOCK, IPT, 2, TMAST>(p, a, s);
}

int launch_scatter(const Plan& p, int pass, const uint32_t* const keys[2], const uint32_t* const pays[2],
                   cudaStream_t s) {
    ScatterArgs a;
    uint64_t o1 = 0;
    for (int side = 0; side < 2; ++side) {
        a.keys[side] = keys ? keys[side] : nullptr;
        a.pays[side] = pays ? pays[side] : nullptr;
        a.in[side] = (pass == 2) ? p.bufA[side] : nullptr;
        a.out[side] = (pass == 1) ? p.bufA[side] : p.bufB[side];
        a.start[side] = p.start + size_t(side) * (p.F + 1);
        a.off1[side] = p.off1 + o1;
        o1 += uint64_t(p.nu1[side]) * 256 + 1;
        a.n[side] = p.n[side];
        a.nu1[side] = p.nu1[side];
    }
    a.off2 = p.off2;
    a.u2_info = p.u2_info;
    a.u2_fb = &p.st->u2_front;
    a.p1_dom = p.slice_dom;
    a.u2_cap = p.u2_max[0] + p.u2_max[1];
    a.unit_len = p.unit_chunks * kScatterChunk;
    a.pass = pass;
    a.b1 = p.b1;
    a.b2 = p.b2;
    a.route_bits = p.route_bits;
    a.unit_ctr = &p.st->claim[pass - 1];
    a.hyb_tab = p.hyb_tab;
    a.hyb_ref = p.hyb_ref;
    a.n_h0 = p.n_h0;
    for (int side = 0; side < 2; ++side) {
        a.hyb_off[side] = p.hyb_off + (side ? size_t(p.nu1[0]) * kHybMaxKeys + 1 : 0);
        a.heavy_pay[side] = p.heavy_pay[side];
    }
    static int cfg = -1;
    if (cfg < 0) {
        const char* e = getenv("GSH_SCATTER_CFG");  // experiments only
        cfg = e ? atoi(e) : 0;
    }
    // (TMA bulk stores per bucket run, cfg 1, measured slower on cfg2: 1.12 / 1.24 ms vs
    // 1.06 / 1.17 ms for the per-tuple whole-sector stores -- barrier-bound, ALU 49 % vs 28 %)
    // Tile shapes per pass (measured on cfg2, scripts/gpu_variants.sh): the largest tiles that
    // still let two CTAs share an SM's 227 KB win -- pass 1 (SoA, hashes in-kernel) 256 x 20 =
    // 5120 tuples (0.927 ms; 512 x 8: 1.013, 512 x 16 at one CTA/SM: 0.944), pass 2 (AoS)
    // 448 x 12 = 5376 tuples (0.976 ms; 512 x 8: 1.032, 384 x 12: 1.011, 512 x 12: 1.187).
    // Tiles need not divide a unit: a unit's ragged last tile takes the scalar path.
    if (cfg == 1) return launch_scatter_cfg<kScatterBlock, kScatterIpt, true>(p, a, s);
    if (pass == 1 && p.n_h0) return launch_scatter_pass<kScatterBlock1, kScatterIptHyb, 1, false, true>(p, a, s);
    return pass == 1 ? launch_scatter_pass<kScatterBlock1, kScatterIpt1, 1, false>(p, a, s)
                     : launch_scatter_pass<kScatterBlock2, kScatterIpt, 2, false>(p, a, s);
}

// ----------------------------------------------- standalone radix histogram (ABI) --
// Shared-memory bins, one window of up to 2^15 digits per CTA (128 KB of u32 counters): a
// 16-bit histogram runs as two windows (blockIdx.y), each CTA reading its key range once per
// window and counting the keys whose digit falls in it.  atomicAdd(.., 1) without a return value
// is the hardware-aggregated ATOMS.POPC.INC (no __match_any_sync: ~64 cycles per call).
constexpr uint32_t kHistWindowBits = 15;

__global__ void __launch_bounds__(1024, 1) k_radix_hist(const uint32_t* __restrict__ keys, uint64_t n,
                                                        uint32_t shift, uint32_t mask,
                                                        unsigned long long* __restrict__ hist) {
    extern __shared__ uint32_t hs[];
    const uint32_t wlen = umin64(uint64_t(mask) + 1, 1u << kHistWindowBits);
    const uint32_t wlo = blockIdx.y * wlen;
    for (uint32_t i = threadIdx.x; i < wlen; i += blockDim.x) hs[i] = 0;
    __syncthreads();
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += 4 * stride) {
        uint32_t k[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) k[j] = i + j * stride < n ? __ldcs(keys + i + j * stride) : 0u;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const uint32_t bin = ((hash32(k[j]) >> shift) & mask) - wlo;
            if (i + j * stride < n && bin < wlen) atomicAdd(&hs[bin], 1u);
        }
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < wlen; i += blockDim.x)
        if (hs[i]) atomicAdd(&hist[wlo + i], (unsigned long long)hs[i]);
}

int launch_radix_hist(const uint32_t* keys, uint64_t n, uint32_t hi_bits, uint32_t nbits, uint64_t* hist,
                      cudaStream_t s) {
    if (n == 0) return 0;
    const uint32_t F = 1u << nbits;
    const uint32_t shift = nbits ? (32 - hi_bits - nbits) : 0;
    const uint32_t wlen = F < (1u << kHistWindowBits) ? F : (1u << kHistWindowBits);
    static std::once_flag attr_once[kMaxDevices];   // > 48 KB of dynamic shared memory: opt in once per device
    once_per_device(attr_once, [&] {
        cudaFuncSetAttribute(k_radix_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, (4u << kHistWindowBits));
    });
    const dim3 grid((unsigned)umin64((n + 4095) / 4096, 148), F / wlen);
    k_radix_hist<<<grid, 1024, size_t(wlen) * 4, s>>>(keys, n, shift, F - 1,
                                                      reinterpret_cast<unsigned long long*>(hist));
    return 1;
}

}  // namespace gsh
