// gsh_device.cuh -- device-side primitives shared by the GSH kernels (sm_100a).
//
// Nothing here is shared with oracle/ (the oracle carries its own hashes).
#pragma once
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

namespace gsh {

__host__ __device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ uint32_t umin32(uint32_t a, uint32_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ uint32_t umax32(uint32_t a, uint32_t b) { return a > b ? a : b; }

constexpr uint32_t kFull = 0xffffffffu;

// Bounds checks of computed indices, compiled in only for the checking build
// (scripts/build_variant.sh bounds "-DGSH_CHECK_BOUNDS"; compute-sanitizer is not available on the
// GPU pool): a violation prints its site and traps, so the calling test fails with a CUDA error.
#ifdef GSH_CHECK_BOUNDS
#define GSH_BOUNDS(cond, what)                                                                       \
    do {                                                                                             \
        if (!(cond)) {                                                                               \
            printf("GSH_BOUNDS violated: %s (%s:%d) block %d thread %d\n", what, __FILE__, __LINE__,  \
                   (int)blockIdx.x, (int)threadIdx.x);                                              \
            __trap();                                                                                \
        }                                                                                            \
    } while (0)
#else
#define GSH_BOUNDS(cond, what) \
    do {                       \
    } while (0)
#endif

// h = fmix32(key): the MurmurHash3 32-bit finalizer, a bijection on u32, so equality of h
// is equality of keys.  Partition digits are taken from h, most significant bits first
// (SURVEY.md §8(c) reading #7; PAPER.md L106 gives no partition hash).
__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16;
    x *= 0x85ebca6bu;
    x ^= x >> 13;
    x *= 0xc2b2ae35u;
    x ^= x >> 16;
    return x;
}

// fmix32 without its final xor-shift: identical to hash32 in bits 16..31 (the last step
// h ^= h >> 16 only changes the low half); used where only high digits are needed.
__device__ __forceinline__ uint32_t hash32_top(uint32_t x) {
    x ^= x >> 16;
    x *= 0x85ebca6bu;
    x ^= x >> 13;
    x *= 0xc2b2ae35u;
    return x;
}

// Checksum term of one join result tuple (a = payload_R, b = payload_S), SURVEY.md §8(c)
// reading #2: mix64(((u64)a << 32 | b) ^ 0x9E3779B97F4A7C15), mix64 = MurmurHash3 fmix64.
__device__ __forceinline__ uint64_t mix64(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return k;
}
constexpr uint64_t kPairSalt = 0x9E3779B97F4A7C15ull;
__device__ __forceinline__ uint64_t pair_term(uint32_t a, uint32_t b) {
    return mix64(((uint64_t(a) << 32) | uint64_t(b)) ^ kPairSalt);
}

// Row-hoisted form of pair_term for the dense skewed-key tiles (a fixed per row):
//   x = (hi, lo) with hi = a ^ salt_hi, lo = b ^ salt_lo.  First xor-shift touches only lo
//   (x >> 33 = hi >> 1), first multiply's hi*c1_lo term is per-row.  ~12 int ops / pair.
struct RowHoist {
    uint32_t hi;        // a ^ salt_hi
    uint32_t hi_shr1;   // hi >> 1
    uint32_t hi_c1lo;   // hi * c1_lo (low 32 bits)
};
__device__ __forceinline__ RowHoist row_hoist(uint32_t a) {
    RowHoist r;
    r.hi = a ^ uint32_t(kPairSalt >> 32);
    r.hi_shr1 = r.hi >> 1;
    r.hi_c1lo = r.hi * 0xed558ccdu;
    return r;
}
__device__ __forceinline__ uint32_t col_lo(uint32_t b) { return b ^ uint32_t(kPairSalt); }

__device__ __forceinline__ uint64_t pair_term_hoisted(const RowHoist& r, uint32_t lo_b) {
    // x ^= x >> 33
    uint32_t lo = lo_b ^ r.hi_shr1;
    uint32_t hi = r.hi;
    // x *= c1  (c1 = 0xff51afd7_ed558ccd)
    uint64_t p = uint64_t(lo) * 0xed558ccdull;                // lo*c1_lo (wide)
    uint32_t nhi = uint32_t(p >> 32) + r.hi_c1lo + lo * 0xff51afd7u;
    lo = uint32_t(p);
    hi = nhi;
    // x ^= x >> 33
    lo ^= hi >> 1;
    // x *= c2  (c2 = 0xc4ceb9fe_1a85ec53)
    p = uint64_t(lo) * 0x1a85ec53ull;
    nhi = uint32_t(p >> 32) + hi * 0x1a85ec53u + lo * 0xc4ceb9feu;
    lo = uint32_t(p);
    hi = nhi;
    // x ^= x >> 33
    lo ^= hi >> 1;
    return (uint64_t(hi) << 32) | lo;
}

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31u; }
__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Relaxed 64-bit global loads/stores for decoupled look-back status words (single-copy
// atomic for aligned 8-byte accesses; the flag and value live in the same word).
__device__ __forceinline__ uint64_t ld_volatile_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_volatile_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Streaming loads that do not allocate in L1 (inputs are read exactly once).
__device__ __forceinline__ uint32_t ld_stream_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ uint2 ld_stream_u2(const uint2* p) {
    uint2 v;
    asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p));
    return v;
}
__device__ __forceinline__ uint4 ld_stream_u4(const uint4* p) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

// ---- TMA bulk copies (cp.async.bulk, SASS UBLKCP) with mbarrier completion ------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
// One arrival that also announces `bytes` of transaction (bulk copies) on this phase.
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t done = 0;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    } while (!done);
}
// Plain arrival (no transaction bytes).
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// Non-blocking: has the phase with this parity completed?
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
    uint32_t done;
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return done != 0;
}
// Named barrier over `count` threads (a subset of the CTA; id 0 is __syncthreads).
__device__ __forceinline__ void named_sync(uint32_t id, uint32_t count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
// Global -> shared bulk copy; dst, src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
// L2 cache policies (createpolicy): keep lines that will be re-read soon, drop streamed ones.
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void bulk_g2s_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                              uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
        "%4;" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}
__device__ __forceinline__ void st_stream_u2(uint2* p, uint2 v, uint64_t policy) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u32 [%0], {%1, %2}, %3;" ::"l"(p), "r"(v.x), "r"(v.y),
                 "l"(policy)
                 : "memory");
}
// Shared -> global bulk copy (TMA store, SASS UBLKCP); dst, src 16-byte aligned, bytes a
// multiple of 16.  Completion is tracked per thread by bulk groups.
__device__ __forceinline__ void bulk_s2g_hint(void* dst, const void* src, uint32_t bytes, uint64_t policy) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
                 "r"(smem_u32(src)), "r"(bytes), "l"(policy)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// Wait until this thread's bulk stores have READ their shared-memory source (it may be reused).
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
// Wait until this thread's bulk stores are complete.
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
// Order this thread's generic-proxy shared-memory accesses before later async-proxy (TMA) ones.
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// Block-wide reduction of (count, checksum) followed by one u64 atomic each.
template <int BLOCK>
__device__ __forceinline__ void block_flush_u64x2(uint64_t a, uint64_t b, unsigned long long* ga,
                                                  unsigned long long* gb) {
    __shared__ uint64_t sa[BLOCK / 32], sb[BLOCK / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        a += __shfl_xor_sync(kFull, a, o);
        b += __shfl_xor_sync(kFull, b, o);
    }
    const int w = threadIdx.x >> 5;
    if ((threadIdx.x & 31) == 0) { sa[w] = a; sb[w] = b; }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t ta = 0, tb = 0;
#pragma unroll
        for (int i = 0; i < BLOCK / 32; ++i) { ta += sa[i]; tb += sb[i]; }
        if (ta) atomicAdd(ga, (unsigned long long)ta);
        if (tb) atomicAdd(gb, (unsigned long long)tb);
    }
}

// Block-wide exclusive scan where only the first NW warps hold non-zero values, with ONE
// barrier: warp scans, the NW warp totals through shared memory, every thread sums the totals of
// the warps before it (broadcast loads).  The caller must separate reuses of `smem` by a barrier.
template <int NW>
__device__ __forceinline__ uint32_t block_excl_scan_1bar(uint32_t v, uint32_t* total, uint32_t* smem /*NW*/) {
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= (uint32_t)o) x += y;
    }
    if (lane == 31 && w < (uint32_t)NW) smem[w] = x;
    __syncthreads();
    uint32_t base = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < NW; ++i) {
        const uint32_t t = smem[i];
        base += ((uint32_t)i < w) ? t : 0u;
        tot += t;
    }
    *total = tot;
    return base + x - v;
}

// Block-wide exclusive scan of one u32 per thread; returns exclusive prefix, *total = sum.
template <int BLOCK>
__device__ __forceinline__ uint32_t block_excl_scan_u32(uint32_t v, uint32_t* total, uint32_t* smem /*BLOCK/32+1*/) {
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= (uint32_t)o) x += y;
    }
    if (lane == 31) smem[w] = x;
    __syncthreads();
    if (w == 0) {
        uint32_t s = (lane < BLOCK / 32) ? smem[lane] : 0;
        uint32_t t = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(kFull, t, o);
            if (lane >= (uint32_t)o) t += y;
        }
        if (lane < BLOCK / 32) smem[lane] = t - s;
        if (lane == BLOCK / 32 - 1) smem[BLOCK / 32] = t;
    }
    __syncthreads();
    uint32_t r = smem[w] + x - v;
    *total = smem[BLOCK / 32];
    __syncthreads();
    return r;
}

}  // namespace gsh
