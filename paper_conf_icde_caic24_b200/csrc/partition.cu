// partition.cu -- GSH phase (1): "partitions input tables into shared memory sized partitions
// ... a simple count then partition procedure ... two passes" (§IV-B(1)).
//
// SURVEY.md §8(a) rows a1-a4:
//   a1 k_hist2d        : h = fmix32(key); joint (d1,d2) histogram of BOTH passes from one read
//                        of the keys (4 B/tuple).  Per-CTA packed-u16 shared-memory counters with
//                        warp aggregation (__match_any_sync) so skewed digits do not serialise.
//   a2 k_hist_reduce + scans : per-partition counts and start offsets, pass-1 chunk offsets.
//   a3/a4 k_scatter    : Onesweep-style scatter -- dynamic tile ids, per-tile bucket ranks via
//                        __match_any_sync, decoupled look-back across tiles per bucket, tiles
//                        staged in shared memory in bucket order, then written as contiguous
//                        runs (coalesced 8 B AoS stores).  16 B/tuple per pass.  Pass-2 tiles
//                        never cross a pass-1 partition; the look-back chain restarts there.
#include <cstdio>
#include <cstdlib>

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
// One read of the keys yields the (d1, d2) histogram of BOTH partition passes.  Counters are
// u32 in shared memory incremented with atomicAdd(.., 1), which sm_100a executes as a
// warp-aggregated ATOMS.POPC.INC: lanes hitting the same bin are combined in hardware, so
// skewed digits cost no more than spread ones (measured: ~1 SM-cycle per warp-op either way,
// while __match_any_sync costs ~64 -- scripts/microbench_warp_ops.cu, profiles/).
// 2^16 u32 bins do not fit one CTA (256 KB), so for F > 2^15 two CTAs read the same chunk
// (the second read is served by L2) and each counts one half of the bins in 128 KB.
__device__ __forceinline__ void hist_one(uint32_t* cnt, uint32_t key, uint32_t shift, uint32_t mask, uint32_t lo,
                                         uint32_t nb) {
    const uint32_t bin = ((hash32(key) >> shift) & mask) - lo;
    if (bin < nb) atomicAdd(&cnt[bin], 1u);
}

// The same read also yields, per pass-1 chunk (kScatterChunk consecutive tuples), the chunk's
// pass-1 digit counts: "count then partition" at chunk granularity, so pass 1
// needs neither a second read nor a cross-CTA look-back (its offsets come from one scan).
__global__ void __launch_bounds__(kHistBlock, 1)
k_hist2d(const uint32_t* __restrict__ k0, uint64_t n0, const uint32_t* __restrict__ k1, uint64_t n1,
         uint32_t shift, uint32_t nbits, uint32_t b2, uint32_t* __restrict__ partial, uint32_t* __restrict__ c1cnt,
         uint32_t nch0, uint32_t nch1) {
    extern __shared__ uint32_t cnt[];
    __shared__ uint32_t c1[256];
    const uint32_t F = 1u << nbits;
    const uint32_t mask = F - 1;
    const bool split = F > (1u << 15);
    // digits above bit 16 do not see fmix32's last xor-shift (it only changes the low half)
    const bool top16 = shift >= 16;
    const uint32_t groups = split ? gridDim.x / 2 : gridDim.x;
    const uint32_t g = split ? blockIdx.x >> 1 : blockIdx.x;
    const uint32_t nb = split ? F / 2 : F;
    const uint32_t lo = split ? (blockIdx.x & 1) * nb : 0;
    const uint32_t d1lo = lo >> b2, d1n = (nb >> b2) ? (nb >> b2) : 1;
    for (int side = 0; side < 2; ++side) {
        const uint32_t* keys = side ? k1 : k0;
        const uint64_t n = side ? n1 : n0;
        const uint32_t nch = side ? nch1 : nch0;
        uint32_t* c1out = c1cnt + (side ? size_t(nch0) * 256 : 0);
        for (uint32_t w = threadIdx.x; w < nb; w += blockDim.x) cnt[w] = 0;
        if (threadIdx.x < 256) c1[threadIdx.x] = 0;
        __syncthreads();
        const bool vec = ((reinterpret_cast<uintptr_t>(keys) & 15u) == 0);
        for (uint32_t c = g; c < nch; c += groups) {
            const uint64_t cb = uint64_t(c) * kScatterChunk;
            const uint64_t ce = umin64(cb + kScatterChunk, n);
            uint64_t done = cb;
            if (vec) {
                const uint4* kv = reinterpret_cast<const uint4*>(keys + cb);
                const uint64_t nv = (ce - cb) / 4;
                uint64_t i = threadIdx.x;
                for (; i + 3ull * blockDim.x < nv; i += 4ull * blockDim.x) {
                    uint4 v[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) v[u] = ld_stream_u4(kv + i + u * blockDim.x);
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const uint32_t kk[4] = {v[u].x, v[u].y, v[u].z, v[u].w};
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            const uint32_t bin = ((top16 ? hash32_top(kk[q]) : hash32(kk[q])) >> shift) & mask;
                            if (bin - lo < nb) {
                                atomicAdd(&cnt[bin - lo], 1u);
                                atomicAdd(&c1[bin >> b2], 1u);
                            }
                        }
                    }
                }
                for (; i < nv; i += blockDim.x) {
                    const uint4 v = ld_stream_u4(kv + i);
                    const uint32_t kk[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const uint32_t bin = ((top16 ? hash32_top(kk[q]) : hash32(kk[q])) >> shift) & mask;
                        if (bin - lo < nb) {
                            atomicAdd(&cnt[bin - lo], 1u);
                            atomicAdd(&c1[bin >> b2], 1u);
                        }
                    }
                }
                done = cb + nv * 4;
            }
            for (uint64_t j = done + threadIdx.x; j < ce; j += blockDim.x) {
                const uint32_t bin = ((top16 ? hash32_top(keys[j]) : hash32(keys[j])) >> shift) & mask;
                if (bin - lo < nb) {
                    atomicAdd(&cnt[bin - lo], 1u);
                    atomicAdd(&c1[bin >> b2], 1u);
                }
            }
            __syncthreads();
            if (threadIdx.x < d1n) {
                c1out[size_t(d1lo + threadIdx.x) * nch + c] = c1[d1lo + threadIdx.x];
                c1[d1lo + threadIdx.x] = 0;
            }
            __syncthreads();
        }
        uint32_t* row = partial + (size_t(side) * groups + g) * F + lo;
        for (uint32_t w = threadIdx.x; w < nb; w += blockDim.x) row[w] = cnt[w];
        __syncthreads();
    }
}

int launch_hist(const Plan& p, const uint32_t* k0, const uint32_t* k1, cudaStream_t s) {
    const uint32_t nbits = p.b1 + p.b2;
    const uint32_t shift = nbits ? (32 - p.route_bits - nbits) : 0;
    const uint32_t F = 1u << nbits;
    const size_t smem = size_t(F > (1u << 15) ? F / 2 : F) * 4;
    static bool attr_set = false;
    if (!attr_set) {
        cudaFuncSetAttribute(k_hist2d, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024);
        attr_set = true;
    }
    // (A cluster-pair variant that hashes each key once and increments the partner's half
    // through DSMEM atomics measured 3.6 ms vs 0.5 ms here: remote shared-memory atomics are
    // far slower than re-hashing an L2-resident chunk.)
    k_hist2d<<<p.hist_grid, kHistBlock, smem, s>>>(k0, p.n[0], k1, p.n[1], shift, nbits, p.b2, p.hist_partial,
                                                   p.c1cnt, p.nch1[0], p.nch1[1]);
    return 1;
}

// --------------------------------------------------- a2: reduce partials + prefix scans --
// cnt[side][bin] = sum over chunk groups of partial[side][group][bin]
__global__ void k_hist_reduce(const uint32_t* __restrict__ partial, uint32_t* __restrict__ cnt, uint32_t F,
                              uint32_t groups) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < 2 * F; i += gridDim.x * blockDim.x) {
        const uint32_t side = i / F, bin = i % F;
        const uint32_t* base = partial + size_t(side) * groups * F + bin;
        uint32_t s = 0;
        for (uint32_t g = 0; g < groups; ++g) s += base[size_t(g) * F];
        cnt[i] = s;
    }
}

struct CountAt {
    const uint32_t* c;
    __device__ uint64_t operator()(uint64_t i) const { return c[i]; }
};

// Pass-1 chunk counts, read in (digit, chunk) order: the exclusive scan in that order IS the
// output offset of chunk c's bucket-d run (start of bucket d + runs of d in earlier chunks).
struct ChunkDigit {
    const uint32_t* c1;   // [256][nch] digit-major
    __device__ uint64_t operator()(uint64_t i) const { return c1[i]; }
};

int launch_hist_reduce_scan(const Plan& p, cudaStream_t s) {
    const uint32_t F = p.F;
    const uint32_t groups = F > (1u << 15) ? p.hist_grid / 2 : p.hist_grid;
    unsigned grid = (2 * F + 255) / 256;
    k_hist_reduce<<<grid, 256, 0, s>>>(p.hist_partial, p.cnt, F, groups);
    int l = 1;
    for (int side = 0; side < 2; ++side)
        l += launch_scan(CountAt{p.cnt + size_t(side) * F}, F, p.start + size_t(side) * (F + 1), p.scan_scratch, s);
    uint64_t off = 0;
    for (int side = 0; side < 2; ++side) {
        const uint64_t m = uint64_t(p.nch1[side]) * 256;
        if (m)
            l += launch_scan(ChunkDigit{p.c1cnt + (side ? size_t(p.nch1[0]) * 256 : 0)}, m,
                             p.off1 + off, p.scan_scratch, s);
        off += m + 1;
    }
    return l;
}

// ------------------------------------------------------------- a3/a4: tile scatter --
struct ScatterArgs {
    const uint32_t* keys[2];   // pass 1 input (SoA); pass 2: nullptr
    const uint32_t* pays[2];
    const uint2* in[2];        // pass 2 input (AoS)
    uint2* out[2];
    const uint64_t* start[2];  // partition start offsets [F + 1] per side
    void* status[2];           // look-back words [tiles][256] per side (u32 or u64)
    uint64_t n[2];
    uint32_t pass, b1, b2, route_bits;
    unsigned int* tile_ctr;
    const uint64_t* off1[2];   // pass 1: [256][nch] chunk/bucket output offsets (no count phase)
    uint32_t nch1[2];
    uint32_t dbg;              // experiment switches (GSH_SCATTER_DEBUG), 0 in production
};

// Look-back status word: 2 flag bits (0 = not ready, 1 = tile aggregate, 2 = inclusive prefix)
// above the value.  u32 words (30-bit values) unless a side holds >= 2^30 tuples.
template <typename W>
struct LB {
    static constexpr int kShift = sizeof(W) * 8 - 2;
    static constexpr W kAgg = W(1) << kShift;
    static constexpr W kInc = W(2) << kShift;
    static constexpr W kMask = (W(1) << kShift) - 1;
    __device__ static W load(const W* p) {
        if constexpr (sizeof(W) == 8) {
            return ld_volatile_u64(reinterpret_cast<const uint64_t*>(p));
        } else {
            W v;
            asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
            return v;
        }
    }
    __device__ static void store(W* p, W v) {
        if constexpr (sizeof(W) == 8) {
            st_volatile_u64(reinterpret_cast<uint64_t*>(p), v);
        } else {
            asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
        }
    }
};

// Work unit = a CHUNK of kScatterChunk tuples inside one segment (the whole side in pass 1, one
// pass-1 partition in pass 2).  A CTA first COUNTS its chunk (TMA tiles, bucket counts only),
// publishes the chunk's bucket aggregates and looks back over preceding chunks (decoupled
// look-back at chunk granularity: 8x fewer, 8x longer-lived units than tiles, so the look-back
// depth stays short), then re-streams the chunk (from L2) and SCATTERS it tile by tile with
// per-CTA running bucket offsets -- no cross-CTA dependency per tile.
struct ScatterSmem {
    uint32_t cnt[256];                  // chunk bucket counts (count phase)
    uint32_t tcnt[256];                 // tile bucket counters -> ranks (scatter phase)
    uint32_t local_start[256];          // bucket start inside the tile
    uint32_t run[256];                  // next output index of bucket b for this chunk
    uint32_t wpos[256];                 // first index of bucket b not yet written to memory
    uint32_t gbase[256];                // output index of stage position 0 of bucket b (mod 2^32)
    uint32_t endw[256];                 // write-out limit of bucket b for the current tile
    uint32_t tailpos[256];              // stage position of bucket b's carried tail
    uint2 cbuf[256][4];                 // carry: < 4 tuples (one 32 B sector) per bucket
    uint32_t carry[256];                // tuples in cbuf[b]
    uint32_t segch[2][257];             // chunk prefix over segments per side
    uint32_t scan_tmp[33];
    uint32_t claim;
    uint64_t mbar[2];                   // TMA completion, one per tile buffer
};

struct ChunkInfo {
    int side;
    uint32_t lc, seg, first_chunk, chunk_in_seg, len;
    uint64_t begin;
};

__device__ __forceinline__ ChunkInfo chunk_info(const ScatterArgs& a, const ScatterSmem& S, uint32_t t,
                                                uint32_t chunks0, uint32_t nseg, bool p1) {
    ChunkInfo ci;
    ci.side = (t >= chunks0) ? 1 : 0;
    ci.lc = t - (ci.side ? chunks0 : 0);
    uint32_t lo = 0, hi = nseg;  // largest s with segch[s] <= lc
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (S.segch[ci.side][mid] <= ci.lc) lo = mid; else hi = mid;
    }
    ci.seg = lo;
    ci.first_chunk = S.segch[ci.side][lo];
    ci.chunk_in_seg = ci.lc - ci.first_chunk;
    const uint64_t seg_b = p1 ? 0 : a.start[ci.side][uint64_t(lo) << a.b2];
    const uint64_t seg_e = p1 ? a.n[ci.side] : a.start[ci.side][uint64_t(lo + 1) << a.b2];
    ci.begin = seg_b + uint64_t(ci.chunk_in_seg) * kScatterChunk;
    ci.len = (uint32_t)umin64(kScatterChunk, seg_e - ci.begin);
    return ci;
}

// Which tile elements arrive by TMA bulk copy: [head, head + nbulk); element i lives at shared
// index i + shift (keeps the bulk destination 16-byte aligned).  The rest (an unaligned first
// AoS tuple, a tail that is not a multiple of 16 bytes, or everything when the SoA inputs are
// not 16-byte aligned) is loaded by its owning thread with ordinary loads.
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
    } else {
        const uintptr_t ip = reinterpret_cast<uintptr_t>(a.in[side] + begin);
        lp.head = umin32((ip & 15u) ? 1u : 0u, len);
        lp.nbulk = (len - lp.head) & ~1u;
        lp.shift = lp.head ? 1u : 0u;
    }
    return lp;
}

// Thread 0: arm `bar` and issue the bulk copies of tile [begin, begin + len).  keys_only: pass-1
// count phase (payloads not needed).  kdst/pdst: pass-1 key / payload buffers; adst: pass-2 AoS.
__device__ __forceinline__ void tile_issue(const ScatterArgs& a, int side, uint64_t begin, uint32_t len, bool p1,
                                           bool keys_only, uint32_t* kdst, uint32_t* pdst, uint2* adst,
                                           uint64_t* bar) {
    // count phase (keys_only): the chunk is re-read by the scatter phase -> keep it in L2;
    // scatter phase: last use -> evict first.  (Pass-1 payloads are only read once.)
    const uint64_t pol = keys_only ? policy_evict_last() : policy_evict_first();
    const LoadPlan lp = load_plan(a, side, begin, len, p1);
    if (p1) {
        const uint32_t bytes = lp.nbulk * 4;
        mbar_arrive_expect_tx(bar, keys_only ? bytes : 2 * bytes);
        if (bytes) {
            bulk_g2s_hint(kdst, a.keys[side] + begin, bytes, bar, pol);
            if (!keys_only) bulk_g2s_hint(pdst, a.pays[side] + begin, bytes, bar, pol);
        }
    } else {
        const uint32_t bytes = lp.nbulk * 8;
        mbar_arrive_expect_tx(bar, bytes);
        if (bytes) bulk_g2s_hint(adst + lp.head + lp.shift, a.in[side] + begin + lp.head, bytes, bar, pol);
    }
}

template <typename W, int BLOCK, int IPT>
__global__ void __launch_bounds__(BLOCK) k_scatter(ScatterArgs a) {
    constexpr int TILE = BLOCK * IPT;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    ScatterSmem& S = *reinterpret_cast<ScatterSmem*>(smem_raw);
    unsigned char* buf0 = smem_raw + ((sizeof(ScatterSmem) + 127) & ~size_t(127));
    unsigned char* buf1 = buf0 + (size_t(TILE) + 4) * 8;
    // scatter phase: buf0 = input tile ("orig"), buf1 = bucket-ordered staging
    uint32_t* ok = reinterpret_cast<uint32_t*>(buf0);   // pass 1: keys -> h
    uint32_t* op = ok + TILE + 4;               // pass 1: payloads
    uint2* o2 = reinterpret_cast<uint2*>(buf0);         // pass 2: (h, payload)
    uint2* stage = reinterpret_cast<uint2*>(buf1);

    const uint32_t tid = threadIdx.x;
    const bool p1 = (a.pass == 1);
    const uint32_t bits = p1 ? a.b1 : a.b2;
    const uint32_t nb = 1u << bits;
    const uint32_t dmask = nb - 1;
    const uint32_t dshift = (32 - a.route_bits - a.b1 - (p1 ? 0 : a.b2)) & 31;
    const uint32_t nseg = p1 ? 1 : (1u << a.b1);
    const uint32_t lowbits = p1 ? a.b2 : 0;

    // chunk prefix over segments (pass 1: one segment per side)
    for (int side = 0; side < 2; ++side) {
        if (p1) {
            if (tid == 0) {
                S.segch[side][0] = 0;
                S.segch[side][1] = (uint32_t)((a.n[side] + kScatterChunk - 1) / kScatterChunk);
            }
        } else {
            uint32_t v = 0;
            if (tid < nseg) {
                const uint64_t b = a.start[side][uint64_t(tid) << a.b2];
                const uint64_t e = a.start[side][uint64_t(tid + 1) << a.b2];
                v = (uint32_t)((e - b + kScatterChunk - 1) / kScatterChunk);
            }
            uint32_t tot;
            const uint32_t ex = block_excl_scan_u32<BLOCK>(v, &tot, S.scan_tmp);
            if (tid < nseg) S.segch[side][tid] = ex;
            if (tid == 0) S.segch[side][nseg] = tot;
        }
    }
    if (tid == 0) {
        mbar_init(&S.mbar[0], 1);
        mbar_init(&S.mbar[1], 1);
        S.claim = atomicAdd(a.tile_ctr, 1u);
    }
    if (tid < 256) S.tcnt[tid] = 0;
    __syncthreads();
    const uint32_t chunks0 = S.segch[0][nseg];
    const uint32_t total = chunks0 + S.segch[1][nseg];
    uint32_t par0 = 0, par1 = 0;
    const uint64_t wpol = policy_evict_first();

    for (uint32_t t = S.claim; t < total;) {
        const ChunkInfo ci = chunk_info(a, S, t, chunks0, nseg, p1);
        const uint32_t ntile = (ci.len + TILE - 1) / TILE;

        // ------------------------------------------------ count phase (double-buffered TMA)
        if (tid < 256) S.cnt[tid] = 0;
        // pass 1 gets its chunk offsets from the histogram pass: no count phase, no look-back
        const bool stat = p1 && a.off1[ci.side] != nullptr;
        const uint32_t ncount = (stat || (a.dbg & 1)) ? 0 : ntile;
        if (tid == 0 && ncount) {
            fence_proxy_async_smem();
            tile_issue(a, ci.side, ci.begin, umin32(TILE, ci.len), p1, true, ok, nullptr, o2, &S.mbar[0]);
        }
        __syncthreads();
        for (uint32_t q = 0; q < ncount; ++q) {
            const uint32_t qb = q * TILE;
            const uint32_t ql = umin32(TILE, ci.len - qb);
            unsigned char* cur = (q & 1) ? buf1 : buf0;
            if (tid == 0 && q + 1 < ncount) {
                unsigned char* nxt = (q & 1) ? buf0 : buf1;
                tile_issue(a, ci.side, ci.begin + qb + TILE, umin32(TILE, ci.len - qb - TILE), p1,
                           true, reinterpret_cast<uint32_t*>(nxt), nullptr, reinterpret_cast<uint2*>(nxt),
                           &S.mbar[(q + 1) & 1]);
            }
            if (q & 1) { mbar_wait(&S.mbar[1], par1); par1 ^= 1; } else { mbar_wait(&S.mbar[0], par0); par0 ^= 1; }
            const LoadPlan lp = load_plan(a, ci.side, ci.begin + qb, ql, p1);
#pragma unroll 4
            for (uint32_t i = tid; i < ql; i += BLOCK) {
                const bool bulk = (i - lp.head) < lp.nbulk;
                uint32_t h;
                if (p1) h = hash32(bulk ? reinterpret_cast<const uint32_t*>(cur)[i] : a.keys[ci.side][ci.begin + qb + i]);
                else h = bulk ? reinterpret_cast<const uint2*>(cur)[i + lp.shift].x : a.in[ci.side][ci.begin + qb + i].x;
                atomicAdd(&S.cnt[(h >> dshift) & dmask], 1u);
            }
            fence_proxy_async_smem();
            __syncthreads();
        }
        // first scatter tile: its TMA overlaps the look-back below
        if (tid == 0)
            tile_issue(a, ci.side, ci.begin, umin32(TILE, ci.len), p1, false, ok, op, o2, &S.mbar[0]);

        // --------------------------------------- chunk-level decoupled look-back, one bucket/thread
        if (stat) {
            if (tid < nb) {
                S.run[tid] = (uint32_t)a.off1[ci.side][size_t(tid) * a.nch1[ci.side] + ci.lc];
                S.wpos[tid] = S.run[tid];
                S.carry[tid] = 0;
            }
        } else if (tid < nb) {
            const uint32_t tot = S.cnt[tid];
            W* st = reinterpret_cast<W*>(a.status[ci.side]);
            const size_t me = size_t(ci.lc) * 256 + tid;
            uint64_t excl = 0;
            if (ci.chunk_in_seg == 0) {
                LB<W>::store(st + me, LB<W>::kInc | W(tot));
            } else {
                LB<W>::store(st + me, LB<W>::kAgg | W(tot));
                // walk back in windows of 4 predecessors (independent loads in flight)
                int64_t j = int64_t(ci.lc) - 1;
                const int64_t stop = int64_t(ci.first_chunk);
                bool done = false;
                while (!done) {
                    W v[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) v[u] = (j - u >= stop) ? LB<W>::load(st + size_t(j - u) * 256 + tid) : W(0);
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        if (done || j - u < stop) continue;
                        W x = v[u];
                        while ((x >> LB<W>::kShift) == 0) x = LB<W>::load(st + size_t(j - u) * 256 + tid);
                        excl += x & LB<W>::kMask;
                        if ((x >> LB<W>::kShift) == 2) done = true;
                    }
                    j -= 4;
                    if (j < stop) done = true;
                }
                LB<W>::store(st + me, LB<W>::kInc | W(excl + tot));
            }
            const uint64_t pidx = ((uint64_t(ci.seg) << bits) | tid) << lowbits;
            S.run[tid] = (uint32_t)(a.start[ci.side][pidx] + excl);
            S.wpos[tid] = S.run[tid];
            S.carry[tid] = 0;
        }
        // (the first sync of the tile loop below orders run[] before its use)

        // ------------------------------------------------------------------ scatter phase
        if (a.dbg & 4) {
            if (tid == 0) { mbar_wait(&S.mbar[0], par0); S.claim = atomicAdd(a.tile_ctr, 1u); }
            par0 ^= 1;
            __syncthreads();
            t = S.claim;
            __syncthreads();
            continue;
        }
        for (uint32_t q = 0; q < ntile; ++q) {
            const uint32_t qb = q * TILE;
            const uint32_t ql = umin32(TILE, ci.len - qb);
            const uint64_t tb = ci.begin + qb;
            const LoadPlan lp = load_plan(a, ci.side, tb, ql, p1);
            const bool full = (ql == TILE) && lp.head == 0 && lp.nbulk == TILE;
            mbar_wait(&S.mbar[0], par0);
            par0 ^= 1;
            uint32_t rk[IPT / 2];  // ranks, packed 2 x u16
            if (full) {  // whole tile arrived by TMA: vector shared loads, no bounds checks
                if (p1) {    // uint4 = 4 keys; slot jj = 4 * v + c of element 4 * (v * BLOCK + tid) + c
#pragma unroll
                    for (int v = 0; v < IPT / 4; ++v) {
                        uint4* k4 = reinterpret_cast<uint4*>(ok) + v * BLOCK + tid;
                        uint4 x = *k4;
                        x.x = hash32(x.x); x.y = hash32(x.y); x.z = hash32(x.z); x.w = hash32(x.w);
                        *k4 = x;
                        const uint32_t r0 = atomicAdd(&S.tcnt[(x.x >> dshift) & dmask], 1u);
                        const uint32_t r1 = atomicAdd(&S.tcnt[(x.y >> dshift) & dmask], 1u);
                        const uint32_t r2 = atomicAdd(&S.tcnt[(x.z >> dshift) & dmask], 1u);
                        const uint32_t r3 = atomicAdd(&S.tcnt[(x.w >> dshift) & dmask], 1u);
                        rk[2 * v] = r0 | (r1 << 16);
                        rk[2 * v + 1] = r2 | (r3 << 16);
                    }
                } else {     // uint4 = 2 AoS tuples; slot jj = 2 * v + c
#pragma unroll
                    for (int v = 0; v < IPT / 2; ++v) {
                        const uint4 x = reinterpret_cast<const uint4*>(o2)[v * BLOCK + tid];
                        const uint32_t r0 = atomicAdd(&S.tcnt[(x.x >> dshift) & dmask], 1u);
                        const uint32_t r1 = atomicAdd(&S.tcnt[(x.z >> dshift) & dmask], 1u);
                        rk[v] = r0 | (r1 << 16);
                    }
                }
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
                                k = a.keys[ci.side][tb + i];
                                op[i] = a.pays[ci.side][tb + i];
                            }
                            h = hash32(k);
                            ok[i] = h;
                        } else {
                            if (bulk) {
                                h = o2[i + lp.shift].x;
                            } else {
                                const uint2 e = a.in[ci.side][tb + i];
                                o2[i + lp.shift] = e;
                                h = e.x;
                            }
                        }
                        r = atomicAdd(&S.tcnt[(h >> dshift) & dmask], 1u);
                    }
                    if (jj & 1) rk[jj >> 1] |= r << 16; else rk[jj >> 1] = r;
                }
            }
            __syncthreads();
            // Write combining: bucket b's staged run = [carry from the previous tile | this tile's
            // tuples]; only whole 32-byte sectors are written (partial-sector writes cost ~1.7x,
            // scripts/microbench_scatter_ceiling.cu), the < 4-tuple remainder carries over.
            // Positions are u32 offsets into the side's output (n < 2^32).
            const uint32_t tc = (tid < nb) ? S.tcnt[tid] : 0u;
            const uint32_t cin = (tid < nb) ? S.carry[tid] : 0u;
            uint32_t all;
            const uint32_t lstart = block_excl_scan_u32<BLOCK>(tc + cin, &all, S.scan_tmp);
            if (tid < nb) {
                const uint32_t nxt = S.run[tid] + tc;
                const uint32_t w0 = S.wpos[tid];
                uint32_t ew = (q + 1 == ntile) ? nxt : (nxt & ~3u);
                if (ew < w0) ew = w0;
                S.local_start[tid] = lstart + cin;
                S.gbase[tid] = w0 - lstart;
                S.endw[tid] = ew;
                S.tailpos[tid] = lstart + (ew - w0);
                for (uint32_t k = 0; k < cin; ++k) stage[lstart + k] = S.cbuf[tid][k];
                S.wpos[tid] = ew;
                S.run[tid] = nxt;
                S.carry[tid] = nxt - ew;
                S.tcnt[tid] = 0;
            }
            __syncthreads();
            if (full) {
                if (p1) {
#pragma unroll
                    for (int v = 0; v < IPT / 4; ++v) {
                        const uint4 h4 = reinterpret_cast<const uint4*>(ok)[v * BLOCK + tid];
                        const uint4 p4 = reinterpret_cast<const uint4*>(op)[v * BLOCK + tid];
                        stage[S.local_start[(h4.x >> dshift) & dmask] + (rk[2 * v] & 0xffffu)] = make_uint2(h4.x, p4.x);
                        stage[S.local_start[(h4.y >> dshift) & dmask] + (rk[2 * v] >> 16)] = make_uint2(h4.y, p4.y);
                        stage[S.local_start[(h4.z >> dshift) & dmask] + (rk[2 * v + 1] & 0xffffu)] =
                            make_uint2(h4.z, p4.z);
                        stage[S.local_start[(h4.w >> dshift) & dmask] + (rk[2 * v + 1] >> 16)] =
                            make_uint2(h4.w, p4.w);
                    }
                } else {
#pragma unroll
                    for (int v = 0; v < IPT / 2; ++v) {
                        const uint4 x = reinterpret_cast<const uint4*>(o2)[v * BLOCK + tid];
                        stage[S.local_start[(x.x >> dshift) & dmask] + (rk[v] & 0xffffu)] = make_uint2(x.x, x.y);
                        stage[S.local_start[(x.z >> dshift) & dmask] + (rk[v] >> 16)] = make_uint2(x.z, x.w);
                    }
                }
            } else {
#pragma unroll
                for (int jj = 0; jj < IPT; ++jj) {
                    const uint32_t i = jj * BLOCK + tid;
                    if (i < ql) {
                        const uint2 e = p1 ? make_uint2(ok[i], op[i]) : o2[i + lp.shift];
                        const uint32_t r = (jj & 1) ? (rk[jj >> 1] >> 16) : (rk[jj >> 1] & 0xffffu);
                        stage[S.local_start[(e.x >> dshift) & dmask] + r] = e;
                    }
                }
            }
            if (tid == 0 && q + 1 == ntile) S.claim = atomicAdd(a.tile_ctr, 1u);
            fence_proxy_async_smem();  // reads of the input tile precede the next TMA writes
            __syncthreads();
            if (tid == 0 && q + 1 < ntile)
                tile_issue(a, ci.side, tb + TILE, umin32(TILE, ci.len - qb - TILE), p1, false,
                           ok, op, o2, &S.mbar[0]);
            // the < 4-tuple tail of each bucket moves to its carry slot; whole sectors go out
            if (tid < nb)
                for (uint32_t k = 0; k < S.carry[tid]; ++k) S.cbuf[tid][k] = stage[S.tailpos[tid] + k];
            uint2* out = a.out[ci.side];
#pragma unroll 4
            for (uint32_t i = tid; i < all; i += BLOCK) {
                const uint2 e = stage[i];
                const uint32_t d = (e.x >> dshift) & dmask;
                const uint32_t g = S.gbase[d] + i;
                if (g < S.endw[d]) st_stream_u2(out + g, e, wpol);
            }
            __syncthreads();
        }
        t = S.claim;
    }
}

size_t scatter_smem_bytes(int tile) {
    // buf0: input tile (+4 slack); buf1: staging = tile + up to 3 carried tuples per bucket
    return ((sizeof(ScatterSmem) + 127) & ~size_t(127)) + (size_t(tile) + 4) * 8 + (size_t(tile) + 3 * 256 + 4) * 8;
}

bool scatter_wide_status(const Plan& p) { return p.n[0] >= (1ull << 30) || p.n[1] >= (1ull << 30); }

template <typename W, int BLOCK, int IPT>
int launch_scatter_cfg(const Plan& p, const ScatterArgs& a, cudaStream_t s) {
    const size_t smem = scatter_smem_bytes(BLOCK * IPT);
    static bool attr_set = false;
    if (!attr_set) {
        cudaFuncSetAttribute(k_scatter<W, BLOCK, IPT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        attr_set = true;
    }
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_scatter<W, BLOCK, IPT>, BLOCK, smem);
    if (occ < 1) occ = 1;
    k_scatter<W, BLOCK, IPT><<<(unsigned)(p.num_sms * occ), BLOCK, smem, s>>>(a);
    return 1;
}

template <typename W>
int launch_scatter_w(const Plan& p, const ScatterArgs& a, cudaStream_t s) {
    static int cfg = -1;
    if (cfg < 0) {
        const char* e = getenv("GSH_SCATTER_CFG");
        cfg = e ? atoi(e) : 1;
    }
    switch (cfg) {
        case 0: return launch_scatter_cfg<W, 256, 8>(p, a, s);
        case 2: return launch_scatter_cfg<W, 256, 16>(p, a, s);
        case 3: return launch_scatter_cfg<W, 1024, 8>(p, a, s);
        default: return launch_scatter_cfg<W, 512, 8>(p, a, s);
    }
}

int launch_scatter(const Plan& p, int pass, const uint32_t* const keys[2], const uint32_t* const pays[2],
                   cudaStream_t s) {
    const bool wide = scatter_wide_status(p);
    const size_t wbytes = wide ? 8 : 4;
    ScatterArgs a;
    for (int side = 0; side < 2; ++side) {
        a.keys[side] = keys ? keys[side] : nullptr;
        a.pays[side] = pays ? pays[side] : nullptr;
        a.in[side] = (pass == 2) ? p.bufA[side] : nullptr;
        a.out[side] = (pass == 1) ? p.bufA[side] : p.bufB[side];
        a.start[side] = p.start + size_t(side) * (p.F + 1);
        a.n[side] = p.n[side];
    }
    a.status[0] = p.status;
    a.status[1] = reinterpret_cast<unsigned char*>(p.status) + size_t(p.max_chunks[0]) * 256 * wbytes;
    a.pass = pass;
    a.b1 = p.b1;
    a.b2 = p.b2;
    a.route_bits = p.route_bits;
    a.tile_ctr = &p.st->claim[pass - 1];
    for (int side = 0; side < 2; ++side) {
        a.off1[side] = (pass == 1) ? p.off1 + (side ? uint64_t(p.nch1[0]) * 256 + 1 : 0) : nullptr;
        a.nch1[side] = p.nch1[side];
    }
    {
        const char* e = getenv("GSH_SCATTER_DEBUG");
        a.dbg = e ? (uint32_t)atoi(e) : 0u;
    }
    // status words must be zero before the pass
    cudaMemsetAsync(p.status, 0, size_t(p.max_chunks[0] + p.max_chunks[1]) * 256 * wbytes, s);
    return wide ? launch_scatter_w<unsigned long long>(p, a, s) : launch_scatter_w<uint32_t>(p, a, s);
}

// ----------------------------------------------- standalone radix histogram (ABI) --
// Shared-memory bins for up to 2^14 digits; wider histograms aggregate per warp and go
// straight to global atomics.
__global__ void k_radix_hist(const uint32_t* __restrict__ keys, uint64_t n, uint32_t shift, uint32_t mask,
                             unsigned long long* __restrict__ hist, int use_smem) {
    extern __shared__ uint32_t hs[];
    if (use_smem) {
        for (uint32_t i = threadIdx.x; i <= mask; i += blockDim.x) hs[i] = 0;
        __syncthreads();
    }
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i - threadIdx.x < n;
         i += uint64_t(gridDim.x) * blockDim.x) {
        bool v = i < n;
        uint32_t bin = v ? ((hash32(keys[i]) >> shift) & mask) : (0x80000000u | lane_id());
        uint32_t peers = __match_any_sync(kFull, bin);
        if (v && (peers & lanemask_lt()) == 0) {
            if (use_smem) atomicAdd(&hs[bin], (uint32_t)__popc(peers));
            else atomicAdd(&hist[bin], (unsigned long long)__popc(peers));
        }
    }
    if (use_smem) {
        __syncthreads();
        for (uint32_t i = threadIdx.x; i <= mask; i += blockDim.x)
            if (hs[i]) atomicAdd(&hist[i], (unsigned long long)hs[i]);
    }
}

int launch_radix_hist(const uint32_t* keys, uint64_t n, uint32_t hi_bits, uint32_t nbits, uint64_t* hist,
                      cudaStream_t s) {
    if (n == 0) return 0;
    const uint32_t F = 1u << nbits;
    const uint32_t shift = nbits ? (32 - hi_bits - nbits) : 0;
    const int use_smem = nbits <= 14;
    size_t smem = use_smem ? size_t(F) * 4 : 0;
    static bool attr_set = false;
    if (!attr_set) {
        cudaFuncSetAttribute(k_radix_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
        attr_set = true;
    }
    unsigned grid = (unsigned)umin64((n + 1023) / 1024, 148);
    k_radix_hist<<<grid, 1024, smem, s>>>(keys, n, shift, F - 1, reinterpret_cast<unsigned long long*>(hist),
                                          use_smem);
    return 1;
}

}  // namespace gsh
