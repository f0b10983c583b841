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
// Packed u16 counters: word w holds bins 2w (low half) and 2w+1 (high half).  When a half
// crosses 0x8000 the crossing warp moves 0x8000 to the global spill counter, so a half never
// exceeds 0x8000 + (adds in flight) < 0x10000 and never carries into its neighbour.
__device__ __forceinline__ void hist_add(uint32_t* cnt, uint32_t bin, uint32_t c, uint32_t* spill) {
    const uint32_t sh = (bin & 1u) * 16u;
    uint32_t old = atomicAdd(&cnt[bin >> 1], c << sh);
    uint32_t ov = (old >> sh) & 0xffffu;
    if (ov < 0x8000u && ov + c >= 0x8000u) {
        atomicSub(&cnt[bin >> 1], 0x8000u << sh);
        atomicAdd(&spill[bin], 0x8000u);
    }
}

__device__ __forceinline__ void hist_key(uint32_t* cnt, uint32_t* spill, uint32_t key, bool valid,
                                         uint32_t shift, uint32_t mask) {
    uint32_t bin = valid ? ((hash32(key) >> shift) & mask) : (0x80000000u | lane_id());
    uint32_t peers = __match_any_sync(kFull, bin);
    if (valid && (peers & lanemask_lt()) == 0) hist_add(cnt, bin, __popc(peers), spill);
}

// grid = (hist_grid, 2): blockIdx.y = side.  Writes this CTA's counters to partial[side][bx][*].
__global__ void __launch_bounds__(kHistBlock, 1)
k_hist2d(const uint32_t* __restrict__ k0, uint64_t n0, const uint32_t* __restrict__ k1, uint64_t n1,
         uint32_t shift, uint32_t nbits, uint16_t* __restrict__ partial, uint32_t* __restrict__ spill) {
    extern __shared__ uint32_t cnt[];
    const int side = blockIdx.y;
    const uint32_t* keys = side ? k1 : k0;
    const uint64_t n = side ? n1 : n0;
    const uint32_t F = 1u << nbits;
    const uint32_t words = (F + 1) / 2;
    const uint32_t mask = F - 1;
    uint32_t* sp = spill + size_t(side) * F;
    for (uint32_t w = threadIdx.x; w < words; w += blockDim.x) cnt[w] = 0;
    __syncthreads();

    // contiguous chunk per CTA, in units of 4 keys (uint4) when the pointer is 16 B aligned
    const uint64_t G = gridDim.x;
    const bool vec = ((reinterpret_cast<uintptr_t>(keys) & 15u) == 0);
    if (vec) {
        const uint64_t nv = n / 4;
        const uint64_t b = nv * blockIdx.x / G, e = nv * (blockIdx.x + 1) / G;
        const uint4* kv = reinterpret_cast<const uint4*>(keys);
        // block-uniform loop bounds (full-warp __match_any_sync below)
        uint64_t base = b;
        for (; base + 2ull * blockDim.x <= e; base += 2ull * blockDim.x) {
            const uint64_t i = base + threadIdx.x;
            uint4 a = ld_stream_u4(kv + i);
            uint4 c = ld_stream_u4(kv + i + blockDim.x);
            hist_key(cnt, sp, a.x, true, shift, mask);
            hist_key(cnt, sp, a.y, true, shift, mask);
            hist_key(cnt, sp, a.z, true, shift, mask);
            hist_key(cnt, sp, a.w, true, shift, mask);
            hist_key(cnt, sp, c.x, true, shift, mask);
            hist_key(cnt, sp, c.y, true, shift, mask);
            hist_key(cnt, sp, c.z, true, shift, mask);
            hist_key(cnt, sp, c.w, true, shift, mask);
        }
        for (; base < e; base += blockDim.x) {
            const uint64_t i = base + threadIdx.x;
            bool v = i < e;
            uint4 a = v ? ld_stream_u4(kv + i) : make_uint4(0, 0, 0, 0);
            hist_key(cnt, sp, a.x, v, shift, mask);
            hist_key(cnt, sp, a.y, v, shift, mask);
            hist_key(cnt, sp, a.z, v, shift, mask);
            hist_key(cnt, sp, a.w, v, shift, mask);
        }
        // scalar tail (n % 4 keys) handled by the last CTA
        if (blockIdx.x == G - 1) {
            uint64_t t0 = nv * 4;
            uint64_t j = t0 + threadIdx.x;
            if (j - threadIdx.x < n) {
                bool v = j < n;
                hist_key(cnt, sp, v ? keys[j] : 0u, v, shift, mask);
            }
        }
    } else {
        const uint64_t b = n * blockIdx.x / G, e = n * (blockIdx.x + 1) / G;
        for (uint64_t i = b + threadIdx.x; i - threadIdx.x < e; i += blockDim.x) {
            bool v = i < e;
            hist_key(cnt, sp, v ? keys[i] : 0u, v, shift, mask);
        }
    }
    __syncthreads();
    uint32_t* row = reinterpret_cast<uint32_t*>(partial + (size_t(side) * G + blockIdx.x) * (F < 2 ? 2 : F));
    for (uint32_t w = threadIdx.x; w < words; w += blockDim.x) row[w] = cnt[w];
}

int launch_hist(const Plan& p, const uint32_t* k0, const uint32_t* k1, cudaStream_t s) {
    const uint32_t nbits = p.b1 + p.b2;
    const uint32_t shift = (32 - p.route_bits - nbits) & 31;
    const uint32_t F = 1u << nbits;
    size_t smem = size_t((F + 1) / 2) * 4;
    static bool attr_set = false;
    if (!attr_set) {
        cudaFuncSetAttribute(k_hist2d, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024);
        attr_set = true;
    }
    cudaMemsetAsync(p.hist_spill, 0, size_t(2) * F * sizeof(uint32_t), s);
    dim3 grid(p.hist_grid, 2);
    k_hist2d<<<grid, kHistBlock, smem, s>>>(k0, p.n[0], k1, p.n[1], nbits ? shift : 0, nbits, p.hist_partial,
                                            p.hist_spill);
    return 1;
}

// --------------------------------------------------- a2: reduce partials + prefix scan --
// cnt[side][bin] = sum_g partial[side][g][bin] + spill[side][bin]
__global__ void k_hist_reduce(const uint16_t* __restrict__ partial, const uint32_t* __restrict__ spill,
                              uint32_t* __restrict__ cnt, uint32_t F, uint32_t G) {
    const uint32_t rowlen = F < 2 ? 2 : F;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < 2 * F; i += gridDim.x * blockDim.x) {
        const uint32_t side = i / F, bin = i % F;
        const uint16_t* base = partial + size_t(side) * G * rowlen + bin;
        uint32_t s = spill[i];
        for (uint32_t g = 0; g < G; ++g) s += base[size_t(g) * rowlen];
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
    unsigned grid = (2 * F + 255) / 256;
    k_hist_reduce<<<grid, 256, 0, s>>>(p.hist_partial, p.hist_spill, p.cnt, F, p.hist_grid);
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
    uint16_t wc[kWarps][256];           // per-warp bucket counters -> per-warp exclusive prefix
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

    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
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

        for (uint32_t i = tid; i < kWarps * 256 / 2; i += kScatterBlock) reinterpret_cast<uint32_t*>(S.wc)[i] = 0;
        __syncthreads();

        // load + rank within warp
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
        const uint32_t lt_mask = lanemask_lt();
#pragma unroll
        for (int j = 0; j < kScatterIpt; ++j) {
            uint32_t i = j * kScatterBlock + tid;
            bool v = i < len;
            uint32_t d = (hv[j] >> dshift) & dmask;
            uint32_t key = v ? d : (0x100u | lane);
            uint32_t peers = __match_any_sync(kFull, key);
            uint32_t before = v ? S.wc[warp][d] : 0u;
            __syncwarp();
            uint32_t r = before + __popc(peers & lt_mask);
            if (v && (peers & lt_mask) == 0) S.wc[warp][d] = (uint16_t)(before + __popc(peers));
            __syncwarp();
            if (j & 1) rk[j >> 1] |= r << 16; else rk[j >> 1] = r;
        }
        __syncthreads();

        // per-bucket: exclusive prefix over warps, bucket totals, block scan -> local starts
        uint32_t tot = 0;
        if (tid < nb) {
#pragma unroll
            for (int w = 0; w < kWarps; ++w) {
                uint32_t c = S.wc[w][tid];
                S.wc[w][tid] = (uint16_t)tot;
                tot += c;
            }
        }
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
                uint32_t pos = S.local_start[d] + S.wc[warp][d] + r;
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
