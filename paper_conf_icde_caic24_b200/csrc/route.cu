// route.cu -- multi-GPU hash sharding kernels.  Not in the
// paper (single A100); the north star adds it: normal keys are routed by the top
// route bits of h = fmix32(key), tuples of agreed skewed keys go to a separate "heavy" bucket
// (S_k stays local, R_k is all-gathered by the driver), so no GPU receives a skewed key's S.
//
// Skewed keys are identified by their hash h (fmix32 is a bijection), sorted ascending.
#include "gsh_device.cuh"
#include "gsh_internal.h"
#include "gsh_scan.cuh"

namespace gsh {

__device__ __forceinline__ bool sorted_find(const uint32_t* a, uint64_t n, uint32_t x, uint64_t* where) {
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        uint32_t v = a[mid];
        if (v < x) lo = mid + 1; else hi = mid;
    }
    *where = lo;
    return lo < n && a[lo] == x;
}

__device__ __forceinline__ uint32_t route_dest(uint32_t h, uint32_t rb, const uint32_t* hk, uint64_t nh) {
    uint64_t w;
    if (nh && sorted_find(hk, nh, h, &w)) return 1u << rb;  // heavy bucket G
    return rb ? (h >> (32 - rb)) : 0u;
}

__global__ void k_route_count(const uint32_t* __restrict__ keys, uint64_t n, uint32_t rb,
                              const uint32_t* __restrict__ hk, uint64_t nh, unsigned long long* counts) {
    __shared__ uint32_t c[257];
    const uint32_t G1 = (1u << rb) + 1;
    for (uint32_t i = threadIdx.x; i < G1; i += blockDim.x) c[i] = 0;
    __syncthreads();
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i - threadIdx.x < n;
         i += uint64_t(gridDim.x) * blockDim.x) {
        const bool v = i < n;
        const uint32_t d = v ? route_dest(hash32(keys[i]), rb, hk, nh) : (0x10000u | lane_id());
        const uint32_t peers = __match_any_sync(kFull, d);
        if (v && (peers & lanemask_lt()) == 0) atomicAdd(&c[d], (uint32_t)__popc(peers));
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < G1; i += blockDim.x)
        if (c[i]) atomicAdd(&counts[i], (unsigned long long)c[i]);
}

int launch_route_count(const uint32_t* keys, uint64_t n, uint32_t rb, const uint32_t* hk, uint64_t nh,
                       uint64_t* counts, cudaStream_t s) {
    if (n == 0) return 0;
    unsigned grid = (unsigned)umin64((n + 1023) / 1024, 148 * 4);
    k_route_count<<<grid, 1024, 0, s>>>(keys, n, rb, hk, nh, reinterpret_cast<unsigned long long*>(counts));
    return 1;
}

__global__ void k_route_scatter(const uint32_t* __restrict__ keys, const uint32_t* __restrict__ pays, uint64_t n,
                                uint32_t rb, const uint32_t* __restrict__ hk, uint64_t nh,
                                const uint64_t* __restrict__ off, unsigned long long* cur, uint32_t* ok,
                                uint32_t* op) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i - threadIdx.x < n;
         i += uint64_t(gridDim.x) * blockDim.x) {
        const bool v = i < n;
        uint32_t k = 0, p = 0;
        if (v) { k = keys[i]; p = pays[i]; }
        const uint32_t d = v ? route_dest(hash32(k), rb, hk, nh) : (0x10000u | lane_id());
        const uint32_t peers = __match_any_sync(kFull, d);
        const uint32_t leader = __ffs(peers) - 1;
        unsigned long long b = 0;
        if (v && lane_id() == leader) b = atomicAdd(&cur[d], (unsigned long long)__popc(peers));
        b = __shfl_sync(kFull, b, leader);
        if (v) {
            const uint64_t pos = off[d] + b + __popc(peers & lanemask_lt());
            ok[pos] = k;
            op[pos] = p;
        }
    }
}

int launch_route_scatter(const uint32_t* keys, const uint32_t* pays, uint64_t n, uint32_t rb, const uint32_t* hk,
                         uint64_t nh, const uint64_t* off, uint64_t* cur, uint32_t* ok, uint32_t* op,
                         cudaStream_t s) {
    if (n == 0) return 0;
    unsigned grid = (unsigned)umin64((n + 511) / 512, 148 * 8);
    k_route_scatter<<<grid, 512, 0, s>>>(keys, pays, n, rb, hk, nh, off, reinterpret_cast<unsigned long long*>(cur),
                                         ok, op);
    return 1;
}

__global__ void k_count_keys(const uint32_t* __restrict__ keys, uint64_t n, const uint32_t* __restrict__ q,
                             uint64_t m, unsigned long long* counts) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i - threadIdx.x < n;
         i += uint64_t(gridDim.x) * blockDim.x) {
        const bool v = i < n;
        uint64_t w = 0;
        const bool hit = v && sorted_find(q, m, hash32(keys[i]), &w);
        const unsigned long long key = hit ? w : ((1ull << 40) | lane_id());
        const uint32_t peers = __match_any_sync(kFull, key);
        if (hit && (peers & lanemask_lt()) == 0) atomicAdd(&counts[w], (unsigned long long)__popc(peers));
    }
}

int launch_count_keys(const uint32_t* keys, uint64_t n, const uint32_t* q, uint64_t m, uint64_t* counts,
                      cudaStream_t s) {
    if (n == 0 || m == 0) return 0;
    unsigned grid = (unsigned)umin64((n + 511) / 512, 148 * 8);
    k_count_keys<<<grid, 512, 0, s>>>(keys, n, q, m, reinterpret_cast<unsigned long long*>(counts));
    return 1;
}

}  // namespace gsh
