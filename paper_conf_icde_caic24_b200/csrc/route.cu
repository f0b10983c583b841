// route.cu -- multi-GPU hash sharding kernels.  Not in the
// paper (single A100); the north star adds it: normal keys are routed by the top
// route bits of h = fmix32(key), tuples of agreed skewed keys go to a separate "heavy" bucket
// (S_k stays local, R_k is all-gathered by the driver), so no GPU receives a skewed key's S.
//
// Skewed keys are identified by their hash h (fmix32 is a bijection), sorted ascending.
#include <type_traits>

#include "gsh_device.cuh"
#include "gsh_internal.h"
#include "gsh_scan.cuh"

namespace gsh {

// ---------------------------------------------------------------------------------------------
// Split pass (DESIGN.md §5 "split pass"): beyond 2^28 tuples per side the two radix passes
// (<= 2^16 partitions) leave partitions larger than the NM ring stages, so gsh_join first splits
// both relations by `rb` hash bits below the `skip` bits already consumed (multi-GPU routing) and
// joins each of the 2^rb sub-problems separately.  Equal keys have equal h, so every match lies
// inside one sub-problem (partitioning by the hash of the key).  SoA in, SoA out.
// Bucket peers are found with rb + 1 ballots (no __match_any_sync); one shared-memory atomic per
// (warp, bucket) and one global cursor atomic per (tile, bucket).

__device__ __forceinline__ uint32_t split_dest(uint32_t k, uint32_t skip, uint32_t rb) {
    return (hash32_top(k) << skip) >> (32 - rb);   // skip + rb <= 16: the top half of h
}

// lanes of this warp holding the same bucket d (valid lanes only)
__device__ __forceinline__ uint32_t split_peers(bool v, uint32_t d, uint32_t rb) {
    uint32_t peers = __ballot_sync(kFull, v);
    for (uint32_t b = 0; b < rb; ++b) {
        const bool bit = (d >> b) & 1u;
        const uint32_t m = __ballot_sync(kFull, bit);
        peers &= bit ? m : ~m;
    }
    return peers;
}

constexpr int kSplitBlock = 512;
constexpr int kSplitIpt = 16;
constexpr uint64_t kSplitTile = uint64_t(kSplitBlock) * kSplitIpt;

// 8 independent key loads per thread in flight (one per 512-key stride of a 4096-key tile), so the
// pass streams at HBM rate rather than at one load per thread's latency.
__global__ void __launch_bounds__(kSplitBlock) k_split_count(const uint32_t* __restrict__ keys, uint64_t n,
                                                            uint32_t skip, uint32_t rb, unsigned long long* counts) {
    constexpr int kIpt = 8;
    constexpr uint64_t kTile = uint64_t(kSplitBlock) * kIpt;
    __shared__ uint32_t c[256];
    const uint32_t G = 1u << rb;
    for (uint32_t i = threadIdx.x; i < G; i += blockDim.x) c[i] = 0;
    __syncthreads();
    const uint64_t ntiles = (n + kTile - 1) / kTile;
    for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        uint32_t k[kIpt];
#pragma unroll
        for (int j = 0; j < kIpt; ++j) {
            const uint64_t i = t * kTile + uint64_t(j) * kSplitBlock + threadIdx.x;
            k[j] = i < n ? __ldcs(keys + i) : 0u;
        }
#pragma unroll
        for (int j = 0; j < kIpt; ++j) {
            const bool v = t * kTile + uint64_t(j) * kSplitBlock + threadIdx.x < n;
            const uint32_t d = v ? split_dest(k[j], skip, rb) : 0u;
            const uint32_t peers = split_peers(v, d, rb);
            if (v && (peers & lanemask_lt()) == 0) atomicAdd(&c[d], (uint32_t)__popc(peers));
        }
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < G; i += blockDim.x)
        if (c[i]) atomicAdd(&counts[i], (unsigned long long)c[i]);
}

// One 8192-tuple tile per iteration: rank every tuple within its bucket (ballot peers + one shared
// atomic per (warp, bucket)), reserve each bucket's run with one global atomic, permute the tile
// into shared memory grouped by bucket, then write it out with consecutive threads on consecutive
// addresses of a run (coalesced; only run ends touch partial sectors).
constexpr size_t kSplitSmem = kSplitTile * (4 + 4 + 1);   // k_split_scatter: keys, payloads, buckets

__global__ void __launch_bounds__(kSplitBlock, 2) k_split_scatter(const uint32_t* __restrict__ keys,
                                                              const uint32_t* __restrict__ pays, uint64_t n,
                                                              uint32_t skip, uint32_t rb,
                                                              const uint64_t* __restrict__ off,
                                                              unsigned long long* cur, uint32_t* __restrict__ ok,
                                                              uint32_t* __restrict__ op) {
    extern __shared__ uint4 split_dyn[];
    uint32_t* s_k = reinterpret_cast<uint32_t*>(split_dyn);
    uint32_t* s_p = s_k + kSplitTile;
    uint8_t* s_d = reinterpret_cast<uint8_t*>(s_p + kSplitTile);
    __shared__ uint32_t cnt[256], pre[256];
    __shared__ unsigned long long base[256];
    const uint32_t G = 1u << rb;
    const uint64_t ntiles = (n + kSplitTile - 1) / kSplitTile;
    for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        for (uint32_t i = threadIdx.x; i < G; i += blockDim.x) cnt[i] = 0;
        __syncthreads();
        const uint64_t t0 = t * kSplitTile;
        uint32_t k[kSplitIpt], p[kSplitIpt], dr[kSplitIpt];  // dr = bucket << 16 | rank in tile
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            const uint64_t idx = t0 + uint64_t(j) * kSplitBlock + threadIdx.x;
            const bool v = idx < n;
            k[j] = v ? keys[idx] : 0u;
            p[j] = v ? pays[idx] : 0u;
        }
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            const bool v = t0 + uint64_t(j) * kSplitBlock + threadIdx.x < n;
            const uint32_t d = v ? split_dest(k[j], skip, rb) : 0u;
            const uint32_t peers = split_peers(v, d, rb);
            const uint32_t leader = peers ? __ffs(peers) - 1 : 0;
            uint32_t b = 0;
            if (v && lane_id() == leader) b = atomicAdd(&cnt[d], (uint32_t)__popc(peers));
            b = __shfl_sync(kFull, b, leader);  // every lane calls; invalid lanes discard it
            dr[j] = v ? (d << 16 | (b + __popc(peers & lanemask_lt()))) : 0xffffffffu;
        }
        __syncthreads();
        for (uint32_t i = threadIdx.x; i < G; i += blockDim.x)
            base[i] = cnt[i] ? off[i] + atomicAdd(&cur[i], (unsigned long long)cnt[i]) : 0ull;
        if (threadIdx.x < 32) {   // exclusive scan of the tile's bucket counts (8 buckets per lane)
            uint32_t c[8], s = 0;
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const uint32_t i = threadIdx.x * 8 + q;
                c[q] = i < G ? cnt[i] : 0u;
                s += c[q];
            }
            uint32_t incl = s;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, incl, o);
                if (threadIdx.x >= (uint32_t)o) incl += y;
            }
            uint32_t e = incl - s;
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const uint32_t i = threadIdx.x * 8 + q;
                if (i < G) pre[i] = e;
                e += c[q];
            }
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            if (dr[j] != 0xffffffffu) {
                const uint32_t d = dr[j] >> 16, q = pre[d] + (dr[j] & 0xffffu);
                s_k[q] = k[j];
                s_p[q] = p[j];
                s_d[q] = (uint8_t)d;
            }
        }
        __syncthreads();
        const uint32_t tn = (uint32_t)umin64(kSplitTile, n - t0);
        for (uint32_t i = threadIdx.x; i < tn; i += kSplitBlock) {
            const uint32_t d = s_d[i];
            const uint64_t pos = base[d] + (i - pre[d]);
            ok[pos] = s_k[i];
            op[pos] = s_p[i];
        }
        __syncthreads();  // cnt / base / pre / staging reused by the next tile
    }
}

// ---- rb <= 3 (G <= 8; auto mode up to 2^31 tuples per side): no atomics.  Every lane of a warp
// computes the warp's G bucket masks from rb + 1 ballots, so per-(warp, bucket) counts and ranks
// stay in warp-uniform registers.  The count kernel writes per-(bucket, tile) counts, one scan
// (bucket-major) gives every tile its write offset in each bucket, and the scatter needs neither
// a shared nor a global atomic.
template <int RB>
__device__ __forceinline__ void split_masks(bool v, uint32_t d, uint32_t (&eq)[1 << RB]) {
    const uint32_t m = __ballot_sync(kFull, v);
    uint32_t mb[RB];
#pragma unroll
    for (int b = 0; b < RB; ++b) mb[b] = __ballot_sync(kFull, (d >> b) & 1u);
#pragma unroll
    for (int g = 0; g < (1 << RB); ++g) {
        uint32_t e = m;
#pragma unroll
        for (int b = 0; b < RB; ++b) e &= ((g >> b) & 1) ? mb[b] : ~mb[b];
        eq[g] = e;
    }
}

// Element of slot j (0..kSplitIpt) of this thread within tile t0: scalar layout = one element per
// 512-stride; VEC layout = 4 consecutive elements per uint4 (slots 4v..4v+3 of vector v).  Any
// bijection onto the tile is correct: counts are per tile, ranks are computed where they are used.
template <bool VEC>
__device__ __forceinline__ uint64_t split_elem(uint64_t t0, int j) {
    return VEC ? t0 + (uint64_t((j >> 2) * kSplitBlock + threadIdx.x) << 2) + (j & 3)
               : t0 + uint64_t(j) * kSplitBlock + threadIdx.x;
}

template <bool VEC>
__device__ __forceinline__ void split_load(const uint32_t* __restrict__ src, uint64_t t0, uint64_t n,
                                           uint32_t (&x)[kSplitIpt]) {
    if (VEC && t0 + kSplitTile <= n) {
#pragma unroll
        for (int v = 0; v < kSplitIpt / 4; ++v) {
            const uint4 w = __ldcs(reinterpret_cast<const uint4*>(src + split_elem<true>(t0, 4 * v)));
            x[4 * v] = w.x; x[4 * v + 1] = w.y; x[4 * v + 2] = w.z; x[4 * v + 3] = w.w;
        }
    } else {
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            const uint64_t i = split_elem<VEC>(t0, j);
            x[j] = i < n ? __ldcs(src + i) : 0u;
        }
    }
}

constexpr int kSplitWarps = kSplitBlock / 32;

// Per-thread bucket counts of a tile live in one u64 of eight 8-bit fields (<= 16 elements per
// thread): an element costs its hash, one shift and one add -- no ballots or popcounts.  Sums over
// a warp or the tile widen the fields to 16 bits: word q of wide16() holds buckets 2q' and 2q'+2
// (even bytes) or 2q'+1 and 2q'+3 (odd bytes) of each half.
__device__ __forceinline__ void wide16(uint64_t c, uint32_t (&w)[4]) {
    const uint32_t lo = uint32_t(c), hi = uint32_t(c >> 32);
    w[0] = lo & 0x00ff00ffu;          // buckets 0, 2
    w[1] = (lo >> 8) & 0x00ff00ffu;   // buckets 1, 3
    w[2] = hi & 0x00ff00ffu;          // buckets 4, 6
    w[3] = (hi >> 8) & 0x00ff00ffu;   // buckets 5, 7
}
// word and bit offset of bucket g in wide16()'s layout
__device__ __forceinline__ uint32_t w16_word(uint32_t g) { return (g & 1u) | ((g >> 2) << 1); }
__device__ __forceinline__ uint32_t w16_shift(uint32_t g) { return ((g >> 1) & 1u) << 4; }

template <int RB, bool VEC>
__global__ void __launch_bounds__(kSplitBlock, 2) k_split_count_tiles(const uint32_t* __restrict__ keys, uint64_t n,
                                                                     uint32_t skip, uint32_t* __restrict__ tile_cnt,
                                                                     unsigned long long* counts) {
    constexpr int G = 1 << RB;
    constexpr int NWD = G <= 4 ? 2 : 4;   // 16-bit-field words in use
    __shared__ uint32_t s_c[2][G];        // tile totals, double-buffered by tile parity
    const uint64_t ntiles = (n + kSplitTile - 1) / kSplitTile;
    if (threadIdx.x < 2 * G) (&s_c[0][0])[threadIdx.x] = 0;
    __syncthreads();
    // the next tile's keys are loaded while this tile's counts are reduced (k[] is free by then)
    uint32_t k[kSplitIpt];
    auto load = [&](uint64_t tt) {
        if (tt < ntiles) split_load<VEC>(keys, tt * kSplitTile, n, k);
    };
    load(blockIdx.x);
    for (uint64_t t = blockIdx.x, par = 0; t < ntiles; t += gridDim.x, par ^= 1) {
        const uint64_t t0 = t * kSplitTile;
        using C = typename std::conditional<(G <= 4), uint32_t, uint64_t>::type;   // 8-bit fields
        C c = 0;
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            const bool v = split_elem<VEC>(t0, j) < n;
            c += v ? (C(1) << (8 * split_dest(k[j], skip, RB))) : C(0);
        }
        load(t + gridDim.x);
        uint32_t w[4];
        wide16(c, w);
#pragma unroll
        for (int q = 0; q < NWD; ++q) w[q] = __reduce_add_sync(kFull, w[q]);
        if (lane_id() == 0) {
#pragma unroll
            for (int g = 0; g < G; ++g) {
                const uint32_t x = (w[w16_word(g)] >> w16_shift(g)) & 0xffffu;
                if (x) atomicAdd(&s_c[par][g], x);
            }
        }
        __syncthreads();
        if (threadIdx.x < G) {   // read and reset this parity's totals (reused two tiles later)
            const uint32_t cg = s_c[par][threadIdx.x];
            s_c[par][threadIdx.x] = 0;
            tile_cnt[uint64_t(threadIdx.x) * ntiles + t] = cg;
            if (cg) atomicAdd(&counts[threadIdx.x], (unsigned long long)cg);
        }
    }
}

// Scatter of one 8192-tuple tile: every element's bucket and its rank among the thread's own
// elements of that bucket come from the packed counter; a block scan of the widened counters
// gives each thread's offset per bucket; the tile is permuted into shared memory (bucket-grouped)
// and written out with consecutive threads on consecutive addresses of each bucket's run (the
// bucket of a staged position is found from the tile's bucket starts, so none is stored).
template <int RB, bool VEC>
__global__ void __launch_bounds__(kSplitBlock, 2) k_split_scatter_tiles(
    const uint32_t* __restrict__ keys, const uint32_t* __restrict__ pays, uint64_t n, uint32_t skip,
    const uint64_t* __restrict__ off, const uint64_t* __restrict__ tpfx, uint32_t* __restrict__ ok,
    uint32_t* __restrict__ op) {
    constexpr int G = 1 << RB;
    constexpr int NWD = G <= 4 ? 2 : 4;
    extern __shared__ uint4 split_dyn[];
    uint32_t* s_k = reinterpret_cast<uint32_t*>(split_dyn);
    uint32_t* s_p = s_k + kSplitTile;
    __shared__ uint32_t s_wt[kSplitWarps][4];   // per-warp widened totals
    __shared__ uint32_t pre[G + 1];
    __shared__ unsigned long long base[G];
    const uint64_t ntiles = (n + kSplitTile - 1) / kSplitTile;
    const uint32_t warp = threadIdx.x >> 5, lane = lane_id();
    // the next tile is loaded into k[] / p[] before this tile's write-out (they are free once the
    // tile sits permuted in shared memory), so its load latency overlaps the stores
    uint32_t k[kSplitIpt], p[kSplitIpt];
    uint32_t dr[kSplitIpt / 4];   // byte j: bucket << 5 | rank among the thread's elements of that bucket
    static_assert(kSplitIpt % 4 == 0 && kSplitIpt <= 31, "ranks fit 5 bits, four per word");
    auto load = [&](uint64_t tt) {
        if (tt < ntiles) {
            split_load<VEC>(keys, tt * kSplitTile, n, k);
            split_load<VEC>(pays, tt * kSplitTile, n, p);
        }
    };
    load(blockIdx.x);
    for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const uint64_t t0 = t * kSplitTile;
        using C = typename std::conditional<(G <= 4), uint32_t, uint64_t>::type;   // 8-bit fields
        C c = 0;
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            const bool v = split_elem<VEC>(t0, j) < n;
            const uint32_t d = split_dest(k[j], skip, RB);
            const uint32_t b = d << 5 | uint32_t((c >> (8 * d)) & 0xffu);
            if ((j & 3) == 0) dr[j >> 2] = 0;
            dr[j >> 2] |= b << (8 * (j & 3));
            c += v ? (C(1) << (8 * d)) : C(0);
        }
        // block exclusive scan of the widened counters (thread order)
        uint32_t ex[4] = {0, 0, 0, 0};   // this thread's exclusive prefix per bucket (16-bit fields)
        {
            uint32_t w[4];
            wide16(c, w);
#pragma unroll
            for (int q = 0; q < NWD; ++q) {
                uint32_t x = w[q];
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(kFull, x, o);
                    if (lane >= (uint32_t)o) x += y;
                }
                ex[q] = x - w[q];
                if (lane == 31) s_wt[warp][q] = x;
            }
        }
        __syncthreads();
        for (uint32_t v2 = 0; v2 < warp; ++v2) {
#pragma unroll
            for (int q = 0; q < NWD; ++q) ex[q] += s_wt[v2][q];
        }
        if (threadIdx.x == 0) {   // bucket starts inside the tile
            uint32_t tot[4] = {0, 0, 0, 0};
            for (int v2 = 0; v2 < kSplitWarps; ++v2) {
#pragma unroll
                for (int q = 0; q < NWD; ++q) tot[q] += s_wt[v2][q];
            }
            uint32_t run = 0;
#pragma unroll
            for (int g = 0; g < G; ++g) {
                pre[g] = run;
                run += (tot[w16_word(g)] >> w16_shift(g)) & 0xffffu;
            }
            pre[G] = run;
        }
        if (threadIdx.x < G) {
            const uint32_t g = threadIdx.x;
            base[g] = off[g] + (tpfx[uint64_t(g) * ntiles + t] - tpfx[uint64_t(g) * ntiles]);
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < kSplitIpt; ++j) {
            if (split_elem<VEC>(t0, j) < n) {
                const uint32_t b = (dr[j >> 2] >> (8 * (j & 3))) & 0xffu, d = b >> 5;
                const uint32_t wd = w16_word(d);   // register select, not a dynamically indexed array
                const uint32_t e4 = wd == 0 ? ex[0] : wd == 1 ? ex[1] : wd == 2 ? ex[2] : ex[3];
                const uint32_t q = pre[d] + ((e4 >> w16_shift(d)) & 0xffffu) + (b & 31u);
                s_k[q] = k[j];
                s_p[q] = p[j];
            }
        }
        __syncthreads();
        load(t + gridDim.x);
        const uint32_t tn = (uint32_t)umin64(kSplitTile, n - t0);
        uint32_t pr[G + 1];
#pragma unroll
        for (int g = 0; g <= G; ++g) pr[g] = pre[g];
        for (uint32_t i = threadIdx.x; i < tn; i += kSplitBlock) {
            uint32_t d = 0;
#pragma unroll
            for (int g = 1; g < G; ++g) d += i >= pr[g] ? 1u : 0u;
            const uint64_t pos = base[d] + (i - pr[d]);
            ok[pos] = s_k[i];
            op[pos] = s_p[i];
        }
        __syncthreads();
    }
}

struct TileCount {
    const uint32_t* c;
    __device__ uint64_t operator()(uint64_t i) const { return c[i]; }
};

uint64_t split_tiles(uint64_t n) { return (n + kSplitTile - 1) / kSplitTile; }

// rb in 1..3: per-(bucket, tile) counts into tile_cnt[G * ntiles], bucket totals added to counts[G]
template <bool VEC>
void split_count_tiles_rb(const uint32_t* keys, uint64_t n, uint32_t skip, uint32_t rb, uint32_t* tile_cnt,
                          unsigned long long* c, unsigned grid, cudaStream_t s) {
    if (rb == 1) k_split_count_tiles<1, VEC><<<grid, kSplitBlock, 0, s>>>(keys, n, skip, tile_cnt, c);
    else if (rb == 2) k_split_count_tiles<2, VEC><<<grid, kSplitBlock, 0, s>>>(keys, n, skip, tile_cnt, c);
    else k_split_count_tiles<3, VEC><<<grid, kSplitBlock, 0, s>>>(keys, n, skip, tile_cnt, c);
}

// rb in 1..3: per-(bucket, tile) counts into tile_cnt[G * ntiles], bucket totals added to counts[G]
int launch_split_count_tiles(const uint32_t* keys, uint64_t n, uint32_t skip, uint32_t rb, uint32_t* tile_cnt,
                             uint64_t* counts, cudaStream_t s) {
    if (n == 0) return 0;
    const unsigned grid = (unsigned)umin64(split_tiles(n), 148 * 4);
    auto* c = reinterpret_cast<unsigned long long*>(counts);
    if ((reinterpret_cast<uintptr_t>(keys) & 15u) == 0) split_count_tiles_rb<true>(keys, n, skip, rb, tile_cnt, c, grid, s);
    else split_count_tiles_rb<false>(keys, n, skip, rb, tile_cnt, c, grid, s);
    return 1;
}

// exclusive bucket-major prefix of tile_cnt (G * ntiles + 1 values) into tpfx
int launch_split_tile_scan(const uint32_t* tile_cnt, uint64_t n, uint32_t rb, uint64_t* tpfx, uint64_t* scratch,
                           cudaStream_t s) {
    if (n == 0) return 0;
    return launch_scan(TileCount{tile_cnt}, (uint64_t(1) << rb) * split_tiles(n), tpfx, scratch, s);
}

template <int RB, bool VEC>
void split_scatter_tiles_one(const uint32_t* keys, const uint32_t* pays, uint64_t n, uint32_t skip,
                             const uint64_t* off, const uint64_t* tpfx, uint32_t* ok, uint32_t* op, cudaStream_t s) {
    static std::once_flag attr_once[kMaxDevices];   // > 48 KB of dynamic shared memory: opt in once per device
    once_per_device(attr_once, [&] {
        cudaFuncSetAttribute(k_split_scatter_tiles<RB, VEC>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)kSplitSmem);
    });
    const unsigned grid = (unsigned)umin64(split_tiles(n), 148 * 2);
    k_split_scatter_tiles<RB, VEC><<<grid, kSplitBlock, kSplitSmem, s>>>(keys, pays, n, skip, off, tpfx, ok, op);
}

int launch_split_scatter_tiles(const uint32_t* keys, const uint32_t* pays, uint64_t n, uint32_t skip, uint32_t rb,
                               const uint64_t* off, const uint64_t* tpfx, uint32_t* ok, uint32_t* op,
                               cudaStream_t s) {
    if (n == 0) return 0;
    const bool vec = ((reinterpret_cast<uintptr_t>(keys) | reinterpret_cast<uintptr_t>(pays)) & 15u) == 0;
    if (vec) {
        if (rb == 1) split_scatter_tiles_one<1, true>(keys, pays, n, skip, off, tpfx, ok, op, s);
        else if (rb == 2) split_scatter_tiles_one<2, true>(keys, pays, n, skip, off, tpfx, ok, op, s);
        else split_scatter_tiles_one<3, true>(keys, pays, n, skip, off, tpfx, ok, op, s);
    } else {
        if (rb == 1) split_scatter_tiles_one<1, false>(keys, pays, n, skip, off, tpfx, ok, op, s);
        else if (rb == 2) split_scatter_tiles_one<2, false>(keys, pays, n, skip, off, tpfx, ok, op, s);
        else split_scatter_tiles_one<3, false>(keys, pays, n, skip, off, tpfx, ok, op, s);
    }
    return 1;
}

int launch_split_count(const uint32_t* keys, uint64_t n, uint32_t skip, uint32_t rb, uint64_t* counts,
                       cudaStream_t s) {
    if (n == 0) return 0;
    unsigned grid = (unsigned)umin64((n + kSplitBlock * 8 - 1) / (kSplitBlock * 8), 148 * 4);
    k_split_count<<<grid, kSplitBlock, 0, s>>>(keys, n, skip, rb, reinterpret_cast<unsigned long long*>(counts));
    return 1;
}

int launch_split_scatter(const uint32_t* keys, const uint32_t* pays, uint64_t n, uint32_t skip, uint32_t rb,
                         const uint64_t* off, uint64_t* cur, uint32_t* ok, uint32_t* op, cudaStream_t s) {
    if (n == 0) return 0;
    unsigned grid = (unsigned)umin64((n + kSplitTile - 1) / kSplitTile, 148 * 4);
    static std::once_flag attr_once[kMaxDevices];   // > 48 KB of dynamic shared memory: opt in once per device
    once_per_device(attr_once, [&] {
        cudaFuncSetAttribute(k_split_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSplitSmem);
    });
    k_split_scatter<<<grid, kSplitBlock, kSplitSmem, s>>>(keys, pays, n, skip, rb, off,
                                                 reinterpret_cast<unsigned long long*>(cur), ok, op);
    return 1;
}

}  // namespace gsh
