// partition.cu -- GSH phase (1): "partitions input tables into shared memory sized partitions
// ... a simple count then partition procedure ... two passes" (§IV-B(1)).
//
// SURVEY.md §8(a) rows a1-a4:
//   a1 k_hist2d        : h = fmix32(key); joint (d1,d2) histogram of BOTH passes from one read
//                        of the keys (4 B/tuple).  Per-CTA packed-u16 shared-memory counters with
//                        warp aggregation (__match_any_sync) so skewed digits do not serialise.
//   a2 k_hist_reduce / k_part_scan : per-partition counts and start offsets.
//   a3/a4 k_scatter    : Onesweep-style scatter -- dynamic tile ids, per-tile bucket ranks via
//                        __match_any_sync, decoupled look-back across tiles per bucket, tiles
//                        staged in shared memory in bucket order, then written as contiguous
//                        runs (coalesced 8 B AoS stores).  16 B/tuple per pass.  Pass-2 tiles
//                        never cross a pass-1 partition; the look-back chain restarts there.
#include <cstdio>

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

__global__ void __launch_bounds__(kHistBlock, 1)
k_hist2d(const uint32_t* __restrict__ k0, uint64_t n0, const uint32_t* __restrict__ k1, uint64_t n1,
         uint32_t shift, uint32_t nbits, uint32_t* __restrict__ partial) {
    extern __shared__ uint32_t cnt[];
    const uint32_t F = 1u << nbits;
    const uint32_t mask = F - 1;
    const bool split = F > (1u << 15);
    const uint32_t nchunks = split ? gridDim.x / 2 : gridDim.x;
    const uint32_t chunk = split ? blockIdx.x >> 1 : blockIdx.x;
    const uint32_t nb = split ? F / 2 : F;
    const uint32_t lo = split ? (blockIdx.x & 1) * nb : 0;
    for (int side = 0; side < 2; ++side) {
        const uint32_t* keys = side ? k1 : k0;
        const uint64_t n = side ? n1 : n0;
        for (uint32_t w = threadIdx.x; w < nb; w += blockDim.x) cnt[w] = 0;
        __syncthreads();
        const bool vec = ((reinterpret_cast<uintptr_t>(keys) & 15u) == 0);
        const uint64_t nv = vec ? n / 4 : 0;
        const uint64_t b = nv * chunk / nchunks, e = nv * (chunk + 1) / nchunks;
        const uint4* kv = reinterpret_cast<const uint4*>(keys);
        uint64_t i = b + threadIdx.x;
        for (; i + 3ull * blockDim.x < e; i += 4ull * blockDim.x) {
            uint4 v[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) v[u] = ld_stream_u4(kv + i + u * blockDim.x);
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                hist_one(cnt, v[u].x, shift, mask, lo, nb);
                hist_one(cnt, v[u].y, shift, mask, lo, nb);
                hist_one(cnt, v[u].z, shift, mask, lo, nb);
                hist_one(cnt, v[u].w, shift, mask, lo, nb);
            }
        }
        for (; i < e; i += blockDim.x) {
            uint4 v = ld_stream_u4(kv + i);
            hist_one(cnt, v.x, shift, mask, lo, nb);
            hist_one(cnt, v.y, shift, mask, lo, nb);
            hist_one(cnt, v.z, shift, mask, lo, nb);
            hist_one(cnt, v.w, shift, mask, lo, nb);
        }
        // scalar remainder (all keys when unaligned, else the n % 4 tail) -> chunk 0
        if (chunk == 0)
            for (uint64_t j = nv * 4 + threadIdx.x; j < n; j += blockDim.x) hist_one(cnt, keys[j], shift, mask, lo, nb);
        __syncthreads();
        uint32_t* row = partial + (size_t(side) * nchunks + chunk) * F + lo;
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
    k_hist2d<<<p.hist_grid, kHistBlock, smem, s>>>(k0, p.n[0], k1, p.n[1], shift, nbits, p.hist_partial);
    return 1;
}

// --------------------------------------------------- a2: reduce partials + prefix scan --
// cnt[side][bin] = sum over chunks of partial[side][chunk][bin]
__global__ void k_hist_reduce(const uint32_t* __restrict__ partial, uint32_t* __restrict__ cnt, uint32_t F,
                              uint32_t nchunks) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < 2 * F; i += gridDim.x * blockDim.x) {
        const uint32_t side = i / F, bin = i % F;
        const uint32_t* base = partial + size_t(side) * nchunks * F + bin;
        uint32_t s = 0;
        for (uint32_t g = 0; g < nchunks; ++g) s += base[size_t(g) * F];
        cnt[i] = s;
    }
}

// One CTA per side: start[side][0..F] = exclusive scan of cnt[side][*].
__global__ void __launch_bounds__(1024) k_part_scan(const uint32_t* __restrict__ cnt, uint64_t* __restrict__ start,
                                                    uint32_t F) {
    __shared__ uint64_t wsum[33];
    const uint32_t side = blockIdx.x;
    const uint32_t* c = cnt + size_t(side) * F;
    uint64_t* o = start + size_t(side) * (F + 1);
    const uint32_t per = (F + 1023) / 1024;
    const uint32_t b = threadIdx.x * per;
    uint64_t local = 0;
    for (uint32_t j = 0; j < per; ++j)
        if (b + j < F) local += c[b + j];
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint64_t incl = warp_incl_scan_u64(local);
    if (lane == 31) wsum[w] = incl;
    __syncthreads();
    if (w == 0) {
        uint64_t v = wsum[lane];
        uint64_t t = warp_incl_scan_u64(v);
        wsum[lane] = t - v;
        if (lane == 31) wsum[32] = t;
    }
    __syncthreads();
    uint64_t run = wsum[w] + incl - local;
    for (uint32_t j = 0; j < per; ++j)
        if (b + j < F) {
            o[b + j] = run;
            run += c[b + j];
        }
    if (threadIdx.x == 0) o[F] = wsum[32];
}

int launch_hist_reduce_scan(const Plan& p, cudaStream_t s) {
    const uint32_t F = p.F;
    const uint32_t nchunks = F > (1u << 15) ? p.hist_grid / 2 : p.hist_grid;
    unsigned grid = (2 * F + 255) / 256;
    k_hist_reduce<<<grid, 256, 0, s>>>(p.hist_partial, p.cnt, F, nchunks);
    k_part_scan<<<2, 1024, 0, s>>>(p.cnt, p.start, F);
    return 2;
}

// ------------------------------------------------------------- a3/a4: tile scatter --
struct ScatterArgs {
    const uint32_t* keys[2];   // pass 1 input (SoA); pass 2: nullptr
    const uint32_t* pays[2];
    const uint2* in[2];        // pass 2 input (AoS)
    uint2* out[2];
    const uint64_t* start[2];  // partition start offsets [F + 1] per side
    uint64_t* status[2];       // look-back words [tiles][256] per side
    uint64_t n[2];
    uint32_t pass, b1, b2, route_bits;
    unsigned int* tile_ctr;
};

constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagInc = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;
constexpr int kWarps = kScatterBlock / 32;

struct ScatterSmem {
    uint32_t bcnt[256];                 // per-tile bucket counters (ATOMS.POPC.INC ranks)
    uint32_t local_start[256];          // bucket start inside the tile
    unsigned long long gbase[256];      // global index of tile element 0 of bucket b
    uint32_t segtiles[2][257];          // tile prefix over segments per side
    uint32_t scan_tmp[kWarps + 1];
    uint32_t claim;
};

__global__ void __launch_bounds__(kScatterBlock, 2) k_scatter(ScatterArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    ScatterSmem& S = *reinterpret_cast<ScatterSmem*>(smem_raw);
    uint2* stage = reinterpret_cast<uint2*>(smem_raw + ((sizeof(ScatterSmem) + 15) & ~size_t(15)));

    const uint32_t tid = threadIdx.x;
    const bool p1 = (a.pass == 1);
    const uint32_t bits = p1 ? a.b1 : a.b2;
    const uint32_t nb = 1u << bits;
    const uint32_t dmask = nb - 1;
    const uint32_t dshift = (32 - a.route_bits - a.b1 - (p1 ? 0 : a.b2)) & 31;
    const uint32_t nseg = p1 ? 1 : (1u << a.b1);
    const uint32_t lowbits = p1 ? a.b2 : 0;

    // tile prefix over segments (pass 1: one segment per side)
    for (int side = 0; side < 2; ++side) {
        if (p1) {
            if (tid == 0) {
                S.segtiles[side][0] = 0;
                S.segtiles[side][1] = (uint32_t)((a.n[side] + kScatterTile - 1) / kScatterTile);
            }
        } else {
            // thread t < nseg computes tiles of segment t; serial scan by warp 0 below
            uint32_t v = 0;
            if (tid < nseg) {
                uint64_t b = a.start[side][uint64_t(tid) << a.b2];
                uint64_t e = a.start[side][uint64_t(tid + 1) << a.b2];
                v = (uint32_t)((e - b + kScatterTile - 1) / kScatterTile);
            }
            uint32_t tot;
            uint32_t ex = block_excl_scan_u32<kScatterBlock>(v, &tot, S.scan_tmp);
            if (tid < nseg) S.segtiles[side][tid] = ex;
            if (tid == 0) S.segtiles[side][nseg] = tot;
        }
    }
    __syncthreads();
    const uint32_t tiles0 = S.segtiles[0][nseg];
    const uint32_t total = tiles0 + S.segtiles[1][nseg];

    for (;;) {
        if (tid == 0) S.claim = atomicAdd(a.tile_ctr, 1u);
        __syncthreads();
        const uint32_t t = S.claim;
        if (t >= total) break;
        const int side = (t >= tiles0) ? 1 : 0;
        const uint32_t lt = t - (side ? tiles0 : 0);
        // segment: largest s with segtiles[s] <= lt
        uint32_t lo = 0, hi = nseg;
        while (hi - lo > 1) {
            uint32_t mid = (lo + hi) >> 1;
            if (S.segtiles[side][mid] <= lt) lo = mid; else hi = mid;
        }
        const uint32_t seg = lo;
        const uint32_t first_tile = S.segtiles[side][seg];
        const uint32_t tile_in_seg = lt - first_tile;
        const uint64_t seg_b = p1 ? 0 : a.start[side][uint64_t(seg) << a.b2];
        const uint64_t seg_e = p1 ? a.n[side] : a.start[side][uint64_t(seg + 1) << a.b2];
        const uint64_t begin = seg_b + uint64_t(tile_in_seg) * kScatterTile;
        const uint32_t len = (uint32_t)umin64(kScatterTile, seg_e - begin);

        if (tid < 256) S.bcnt[tid] = 0;
        __syncthreads();

        // load + rank: atomicAdd(.., 1) on a per-tile bucket counter returns a unique rank
        // (hardware-aggregated for lanes of the same bucket, so skew does not serialise)
        uint32_t hv[kScatterIpt], pv[kScatterIpt], rk[kScatterIpt / 2];  // ranks packed 2 x u16
        if (p1) {
            const uint32_t* kp = a.keys[side] + begin;
            const uint32_t* pp = a.pays[side] + begin;
#pragma unroll
            for (int j = 0; j < kScatterIpt; ++j) {
                uint32_t i = j * kScatterBlock + tid;
                bool v = i < len;
                hv[j] = v ? ld_stream_u32(kp + i) : 0u;
                pv[j] = v ? ld_stream_u32(pp + i) : 0u;
            }
#pragma unroll
            for (int j = 0; j < kScatterIpt; ++j) hv[j] = hash32(hv[j]);
        } else {
            const uint2* ip = a.in[side] + begin;
#pragma unroll
            for (int j = 0; j < kScatterIpt; ++j) {
                uint32_t i = j * kScatterBlock + tid;
                uint2 e = (i < len) ? ld_stream_u2(ip + i) : make_uint2(0, 0);
                hv[j] = e.x;
                pv[j] = e.y;
            }
        }
#pragma unroll
        for (int j = 0; j < kScatterIpt; ++j) {
            uint32_t i = j * kScatterBlock + tid;
            uint32_t r = 0;
            if (i < len) r = atomicAdd(&S.bcnt[(hv[j] >> dshift) & dmask], 1u);
            if (j & 1) rk[j >> 1] |= r << 16; else rk[j >> 1] = r;
        }
        __syncthreads();

        // bucket totals -> block scan -> local starts
        const uint32_t tot = (tid < nb) ? S.bcnt[tid] : 0u;
        uint32_t all;
        uint32_t lstart = block_excl_scan_u32<kScatterBlock>(tid < nb ? tot : 0u, &all, S.scan_tmp);
        if (tid < nb) S.local_start[tid] = lstart;

        // decoupled look-back, one bucket per thread
        if (tid < nb) {
            uint64_t* st = a.status[side];
            const size_t me = size_t(lt) * 256 + tid;
            uint64_t excl = 0;
            if (tile_in_seg == 0) {
                st_volatile_u64(st + me, kFlagInc | tot);
            } else {
                st_volatile_u64(st + me, kFlagAgg | tot);
                for (int64_t j = int64_t(lt) - 1; j >= int64_t(first_tile); --j) {
                    uint64_t v;
                    do { v = ld_volatile_u64(st + size_t(j) * 256 + tid); } while ((v >> 62) == 0);
                    excl += v & kValMask;
                    if ((v >> 62) == 2) break;
                }
                st_volatile_u64(st + me, kFlagInc | (excl + tot));
            }
            const uint64_t pidx = ((uint64_t(seg) << bits) | tid) << lowbits;
            S.gbase[tid] = a.start[side][pidx] + excl - lstart;
        }
        __syncthreads();

        // scatter into shared staging in bucket order
#pragma unroll
        for (int j = 0; j < kScatterIpt; ++j) {
            uint32_t i = j * kScatterBlock + tid;
            if (i < len) {
                uint32_t d = (hv[j] >> dshift) & dmask;
                uint32_t r = (j & 1) ? (rk[j >> 1] >> 16) : (rk[j >> 1] & 0xffffu);
                uint32_t pos = S.local_start[d] + r;
                stage[pos] = make_uint2(hv[j], pv[j]);
            }
        }
        __syncthreads();

        // write out contiguous bucket runs
        uint2* out = a.out[side];
#pragma unroll 4
        for (uint32_t i = tid; i < len; i += kScatterBlock) {
            uint2 e = stage[i];
            uint32_t d = (e.x >> dshift) & dmask;
            out[S.gbase[d] + i] = e;
        }
        __syncthreads();
    }
}

size_t scatter_smem_bytes() {
    return ((sizeof(ScatterSmem) + 15) & ~size_t(15)) + size_t(kScatterTile) * sizeof(uint2);
}

int launch_scatter(const Plan& p, int pass, const uint32_t* const keys[2], const uint32_t* const pays[2],
                   cudaStream_t s) {
    ScatterArgs a;
    for (int side = 0; side < 2; ++side) {
        a.keys[side] = keys ? keys[side] : nullptr;
        a.pays[side] = pays ? pays[side] : nullptr;
        a.in[side] = (pass == 2) ? p.bufA[side] : nullptr;
        a.out[side] = (pass == 1) ? p.bufA[side] : p.bufB[side];
        a.start[side] = p.start + size_t(side) * (p.F + 1);
        a.status[side] = p.status + size_t(side) * p.max_tiles[0] * 256;
        a.n[side] = p.n[side];
    }
    a.status[1] = p.status + size_t(p.max_tiles[0]) * 256;
    a.pass = pass;
    a.b1 = p.b1;
    a.b2 = p.b2;
    a.route_bits = p.route_bits;
    a.tile_ctr = &p.st->claim[pass - 1];
    const size_t smem = scatter_smem_bytes();
    static bool attr_set = false;
    if (!attr_set) {
        cudaFuncSetAttribute(k_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        attr_set = true;
    }
    // status words must be zero before the pass
    cudaMemsetAsync(p.status, 0, size_t(p.max_tiles[0] + p.max_tiles[1]) * 256 * sizeof(uint64_t), s);
    unsigned grid = (unsigned)p.num_sms * 2;
    k_scatter<<<grid, kScatterBlock, smem, s>>>(a);
    return 1;
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
