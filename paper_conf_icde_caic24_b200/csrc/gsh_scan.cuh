// gsh_scan.cuh -- generic device-wide exclusive scan of u64 values v(i) (reduce-then-scan).
//
// Used for the small bookkeeping prefixes of the method (partition work items, skewed-key
// array offsets, dense-tile counts).  Input values come from a functor so no temporary
// array is materialised.  out[0..n] receives the exclusive prefix, out[n] the total.
#pragma once
#include <cstdint>

#include "gsh_device.cuh"

namespace gsh {

constexpr int kScanBlock = 512;
constexpr int kScanIpt = 8;
constexpr int kScanTile = kScanBlock * kScanIpt;  // 4096 elements per CTA

template <class Fn>
__device__ __forceinline__ void k_scan_reduce_body(const Fn& fn, uint64_t n, uint32_t block, uint64_t* bsum) {
    __shared__ uint64_t red[kScanBlock / 32];
    const uint64_t base = uint64_t(block) * kScanTile;
    uint64_t acc = 0;
#pragma unroll
    for (int j = 0; j < kScanIpt; ++j) {
        uint64_t i = base + uint64_t(j) * kScanBlock + threadIdx.x;
        if (i < n) acc += fn(i);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(kFull, acc, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t t = 0;
        for (int w = 0; w < kScanBlock / 32; ++w) t += red[w];
        bsum[block] = t;
    }
}
// u32 array as a scan input
struct U32At {
    const uint32_t* in;
    __device__ uint64_t operator()(uint64_t i) const { return in[i]; }
};

template <class Fn>
__global__ void __launch_bounds__(kScanBlock) k_scan_reduce(Fn fn, uint64_t n, uint64_t* bsum) {
    k_scan_reduce_body(fn, n, blockIdx.x, bsum);
}

__device__ __forceinline__ uint64_t warp_incl_scan_u64(uint64_t x) {
    const uint32_t lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= (uint32_t)o) x += y;
    }
    return x;
}

// Single-CTA exclusive scan of nb block sums (in place); bsum[nb] = total.
__device__ __forceinline__ void scan_blocks_body(uint64_t* bsum, uint64_t nb) {
    __shared__ uint64_t wsum[33];
    uint64_t carry = 0;
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint64_t base = 0; base < nb; base += 1024) {
        uint64_t i = base + threadIdx.x;
        uint64_t v = (i < nb) ? bsum[i] : 0;
        uint64_t incl = warp_incl_scan_u64(v);
        if (lane == 31) wsum[w] = incl;
        __syncthreads();
        if (w == 0) {
            uint64_t s = wsum[lane];
            uint64_t t = warp_incl_scan_u64(s);
            wsum[lane] = t - s;
            if (lane == 31) wsum[32] = t;
        }
        __syncthreads();
        if (i < nb) bsum[i] = carry + wsum[w] + incl - v;
        carry += wsum[32];
        __syncthreads();
    }
    if (threadIdx.x == 0) bsum[nb] = carry;
}

template <int Dummy = 0>
__global__ void __launch_bounds__(1024) k_scan_blocks(uint64_t* bsum, uint64_t nb) {
    scan_blocks_body(bsum, nb);
}

template <class Fn>
__device__ __forceinline__ void scan_final_body(const Fn& fn, uint64_t n, uint32_t block, uint32_t nblocks,
                                                const uint64_t* bsum, uint64_t* out) {
    __shared__ uint64_t wsum[kScanBlock / 32 + 1];
    const uint64_t base = uint64_t(block) * kScanTile;
    // blocked arrangement: thread t owns elements [base + t*IPT, base + t*IPT + IPT)
    uint64_t v[kScanIpt];
    uint64_t local = 0;
#pragma unroll
    for (int j = 0; j < kScanIpt; ++j) {
        uint64_t i = base + uint64_t(threadIdx.x) * kScanIpt + j;
        v[j] = (i < n) ? fn(i) : 0;
        local += v[j];
    }
    uint64_t incl = warp_incl_scan_u64(local);
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (lane == 31) wsum[w] = incl;
    __syncthreads();
    if (w == 0) {
        uint64_t s = (lane < kScanBlock / 32) ? wsum[lane] : 0;
        uint64_t t = warp_incl_scan_u64(s);
        if (lane < kScanBlock / 32) wsum[lane] = t - s;
    }
    __syncthreads();
    uint64_t run = bsum[block] + wsum[w] + incl - local;
#pragma unroll
    for (int j = 0; j < kScanIpt; ++j) {
        uint64_t i = base + uint64_t(threadIdx.x) * kScanIpt + j;
        if (i < n) out[i] = run;
        run += v[j];
    }
    if (block == nblocks - 1 && threadIdx.x == kScanBlock - 1) out[n] = run;
}

template <class Fn>
__global__ void __launch_bounds__(kScanBlock) k_scan_final(Fn fn, uint64_t n, const uint64_t* bsum,
                                                          uint64_t* out) {
    scan_final_body(fn, n, blockIdx.x, gridDim.x, bsum, out);
}

template <class Fn>
int launch_scan(const Fn& fn, uint64_t n, uint64_t* out, uint64_t* scratch, cudaStream_t s) {
    if (n == 0) {
        cudaMemsetAsync(out, 0, sizeof(uint64_t), s);
        return 0;
    }
    uint64_t nb = (n + kScanTile - 1) / kScanTile;
    k_scan_reduce<Fn><<<(unsigned)nb, kScanBlock, 0, s>>>(fn, n, scratch);
    k_scan_blocks<0><<<1, 1024, 0, s>>>(scratch, nb);
    k_scan_final<Fn><<<(unsigned)nb, kScanBlock, 0, s>>>(fn, n, scratch, out);
    return 3;
}

// ---- several independent u32 -> u64 exclusive scans in ONE reduce/blocks/final launch triple
// (the histogram's per-partition and per-(digit, unit) counts: 4 segments, 3 launches, not 12).
// Segment g: out_g[0..n_g) = exclusive prefix of in_g, out_g[n_g] = total; its block sums live
// at scratch[sb_g .. sb_g + nb_g] (sb_g = sum over earlier segments of nb + 1).
constexpr int kMaxScanSegs = 4;
struct ScanSegs {
    const uint32_t* in[kMaxScanSegs];
    uint64_t* out[kMaxScanSegs];
    uint64_t n[kMaxScanSegs];
    uint32_t b0[kMaxScanSegs + 1];   // first block of each segment (exclusive prefix of nb)
    int k;
};

__device__ __forceinline__ int scan_seg_of(const ScanSegs& g, uint32_t block) {
    int q = 0;
    while (q + 1 < g.k && block >= g.b0[q + 1]) ++q;
    return q;
}

template <int Dummy = 0>
__global__ void __launch_bounds__(kScanBlock) k_mscan_reduce(ScanSegs g, uint64_t* scratch) {
    const int q = scan_seg_of(g, blockIdx.x);
    const uint32_t bl = blockIdx.x - g.b0[q];
    k_scan_reduce_body(U32At{g.in[q]}, g.n[q], bl, scratch + g.b0[q] + q);
}

template <int Dummy = 0>
__global__ void __launch_bounds__(1024) k_mscan_blocks(ScanSegs g, uint64_t* scratch) {
    const int q = blockIdx.x;
    scan_blocks_body(scratch + g.b0[q] + q, g.b0[q + 1] - g.b0[q]);
}

template <int Dummy = 0>
__global__ void __launch_bounds__(kScanBlock) k_mscan_final(ScanSegs g, const uint64_t* scratch) {
    const int q = scan_seg_of(g, blockIdx.x);
    const uint32_t bl = blockIdx.x - g.b0[q];
    scan_final_body(U32At{g.in[q]}, g.n[q], bl, g.b0[q + 1] - g.b0[q], scratch + g.b0[q] + q, g.out[q]);
}

// scratch needs sum over segments of (nb + 1) elements.  Empty segments get out[0] = 0.
inline int launch_scan_u32_multi(ScanSegs g, uint64_t* scratch, cudaStream_t s) {
    uint32_t nbt = 0;
    int l = 0;
    for (int q = 0; q < g.k; ++q) {
        g.b0[q] = nbt;
        nbt += (uint32_t)((g.n[q] + kScanTile - 1) / kScanTile);
        if (g.n[q] == 0) cudaMemsetAsync(g.out[q], 0, sizeof(uint64_t), s);
    }
    g.b0[g.k] = nbt;
    if (nbt == 0) return l;
    k_mscan_reduce<0><<<nbt, kScanBlock, 0, s>>>(g, scratch);
    k_mscan_blocks<0><<<g.k, 1024, 0, s>>>(g, scratch);
    k_mscan_final<0><<<nbt, kScanBlock, 0, s>>>(g, scratch);
    return l + 3;
}

}  // namespace gsh
