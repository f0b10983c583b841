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
__global__ void __launch_bounds__(kScanBlock) k_scan_reduce(Fn fn, uint64_t n, uint64_t* bsum) {
    __shared__ uint64_t red[kScanBlock / 32];
    const uint64_t base = uint64_t(blockIdx.x) * kScanTile;
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
        bsum[blockIdx.x] = t;
    }
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
template <int Dummy = 0>
__global__ void __launch_bounds__(1024) k_scan_blocks(uint64_t* bsum, uint64_t nb) {
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

template <class Fn>
__global__ void __launch_bounds__(kScanBlock) k_scan_final(Fn fn, uint64_t n, const uint64_t* bsum,
                                                          uint64_t* out) {
    __shared__ uint64_t wsum[kScanBlock / 32 + 1];
    const uint64_t base = uint64_t(blockIdx.x) * kScanTile;
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
    uint64_t run = bsum[blockIdx.x] + wsum[w] + incl - local;
#pragma unroll
    for (int j = 0; j < kScanIpt; ++j) {
        uint64_t i = base + uint64_t(threadIdx.x) * kScanIpt + j;
        if (i < n) out[i] = run;
        run += v[j];
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == kScanBlock - 1) out[n] = run;
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

}  // namespace gsh
