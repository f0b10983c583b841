// shard.cu -- per-rank steps of the multi-GPU hash-sharded GSH join (SURVEY.md §8(a) row a11,
// §8(e)).  Not in the paper (one A100, §V-A); the north star adds sharding over one
// 8xB200 node.  The host driver (paper_conf_icde_caic24_b200/sharded.py) calls these entry points
// between collectives; every data-path step is a kernel here.
//
//   skew agreement (PAPER.md L107 large partitions + L112 skewed keys, on the WHOLE input):
//     k_shard_large    large(p) from the all-reduced global partition histogram
//     k_cand_count     exact local counts of every key of a globally large partition (table T)
//     k_cand_select    candidates: local max(cnt_R, cnt_S) >= tau = ceil(T_h / G)  (pigeonhole:
//                      a key with global count >= T_h reaches tau on some rank)
//     k_agree_*        union of the all-gathered candidates, deduplicated by FIRST OCCURRENCE in
//                      the gathered buffer (identical on every rank, so the union's order is too)
//                      + this rank's exact counts of each union key, looked up in T
//     k_select_*       after the all-reduce of those counts: heavy iff max >= T_h, compacted
//                      in union order (a scan, no atomics: every rank gets the same list)
//   routing (north star: "normal keys are routed by high radix bits ... heavy keys keep S local
//   while their R tuples are broadcast"):
//     k_route_count / k_route_scatter   destination d = top route_bits of h, or G for a tuple of a
//                      skewed key (found in an open-addressing set); tuples are written straight
//                      into per-destination buffers the driver lays out (its own received segment,
//                      the all-gathered R_H buffer, the send buffer), so no copy follows.
#include <cstring>
#include <dlfcn.h>

#include "gsh_device.cuh"
#include "gsh_internal.h"
#include "gsh_scan.cuh"
#include "gsh_table.cuh"

namespace gsh {

constexpr uint32_t kMaxShardWorld = 256;
constexpr uint64_t kCandMaxSlots = 1ull << 27;

// ------------------------------------------------------------------ large partitions --
__global__ void k_shard_large(const unsigned long long* __restrict__ hist, uint32_t F, uint32_t L, int force_normal,
                              uint8_t* __restrict__ large, unsigned long long* __restrict__ nlarge) {
    unsigned long long t = 0;   // global tuples in large partitions (sizes the local count table)
    for (uint32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < F; p += gridDim.x * blockDim.x) {
        const unsigned long long cr = hist[p], cs = hist[F + p];
        const bool lg = !force_normal && cr > 0 && cs > 0 && (cr > L || cs > L);
        large[p] = lg ? 1 : 0;
        if (lg) t += cr + cs;
    }
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(kFull, t, o);
    if (lane_id() == 0 && t) atomicAdd(nlarge, t);
}

// -------------------------------------------------- exact local counts of large keys --
__global__ void k_cand_count(const uint32_t* __restrict__ keys, uint64_t n, int side, uint32_t pshift,
                             const uint8_t* __restrict__ large, unsigned long long* gt_key, uint32_t* gt_cnt,
                             uint32_t cap, uint32_t logcap, unsigned int* overflow) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i - threadIdx.x < n;
         i += uint64_t(gridDim.x) * blockDim.x) {
        bool v = i < n;
        const uint32_t h = v ? hash32(keys[i]) : 0u;
        v = v && large[pshift < 32 ? (h >> pshift) : 0u];
        const unsigned long long key = v ? h : ((1ull << 32) | lane_id());
        const uint32_t peers = __match_any_sync(kFull, key);
        if (v && (peers & lanemask_lt()) == 0) {
            const uint32_t slot = gt_insert(gt_key, h, logcap);
            if (slot == kNoHeavy) *overflow = 1;
            else atomicAdd(&gt_cnt[size_t(side) * cap + slot], (uint32_t)__popc(peers));
        }
    }
}

__global__ void k_cand_select(const unsigned long long* __restrict__ gt_key, const uint32_t* __restrict__ gt_cnt,
                              uint32_t cap, uint32_t threshold, uint32_t* out, unsigned long long outcap,
                              unsigned long long* nout) {
    for (uint32_t slot = blockIdx.x * blockDim.x + threadIdx.x; slot < cap; slot += gridDim.x * blockDim.x) {
        const unsigned long long kw = gt_key[slot];
        if (kw == 0) continue;
        if (max(gt_cnt[slot], gt_cnt[cap + slot]) >= threshold) {
            const unsigned long long i = atomicAdd(nout, 1ull);
            if (i < outcap) out[i] = (uint32_t)kw;
        }
    }
}

// Layout of the per-rank agreement workspace: [state 256 B][large u8[2^16]][T keys][T cnt_R][T cnt_S].
struct CandWs {
    unsigned long long* nout;
    unsigned int* overflow;
    uint32_t* slots_used;   // T's slot count (log2 in the high byte is recomputed from it)
    unsigned long long* nlarge;   // global tuples in large partitions
    uint8_t* large;
    unsigned long long* key;
    uint32_t* cnt;
    uint32_t cap;
};

static uint32_t cand_slots(uint64_t nR, uint64_t nS) {
    uint64_t c = 1024;
    while (c < 2 * (nR + nS) && c < kCandMaxSlots) c <<= 1;
    return (uint32_t)c;
}

static CandWs cand_ws(void* ws, uint32_t cap) {
    unsigned char* b = reinterpret_cast<unsigned char*>(ws);
    CandWs w;
    w.nout = reinterpret_cast<unsigned long long*>(b);
    w.overflow = reinterpret_cast<unsigned int*>(b + 8);
    w.slots_used = reinterpret_cast<uint32_t*>(b + 12);
    w.nlarge = reinterpret_cast<unsigned long long*>(b + 16);
    w.large = b + 256;
    w.key = reinterpret_cast<unsigned long long*>(b + 256 + 65536);
    w.cnt = reinterpret_cast<uint32_t*>(w.key + cap);
    w.cap = cap;
    return w;
}

static size_t cand_ws_bytes(uint32_t cap) { return 256 + 65536 + size_t(cap) * 16; }

// ------------------------------------------------------------------------- agreement --
struct GatherView {
    const uint32_t* buf;
    uint64_t stride;
    uint32_t G;
    uint32_t size[kMaxShardWorld];
    __device__ __forceinline__ bool valid(uint64_t i) const {
        const uint32_t g = (uint32_t)(i / stride);
        return g < G && (i - uint64_t(g) * stride) < size[g];
    }
};

__global__ void k_agree_first(GatherView v, unsigned long long* dkey, uint32_t* didx, uint32_t logcap,
                              unsigned int* overflow) {
    const uint64_t n = uint64_t(v.G) * v.stride;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
        if (!v.valid(i)) continue;
        const uint32_t slot = gt_insert(dkey, v.buf[i], logcap);
        if (slot == kNoHeavy) *overflow = 1;
        else atomicMin(&didx[slot], (uint32_t)i);
    }
}

struct FirstOcc {
    GatherView v;
    const unsigned long long* dkey;
    const uint32_t* didx;
    uint32_t logcap;
    __device__ uint64_t operator()(uint64_t i) const {
        if (!v.valid(i)) return 0;
        const uint32_t slot = gt_find(dkey, v.buf[i], logcap);
        return (slot != kNoHeavy && didx[slot] == (uint32_t)i) ? 1 : 0;
    }
};

__global__ void k_agree_emit(FirstOcc f, const uint64_t* __restrict__ pos, const unsigned long long* __restrict__ tkey,
                             const uint32_t* __restrict__ tcnt, uint32_t tcap, uint32_t tlog, uint32_t* __restrict__ uni,
                             unsigned long long* __restrict__ cnt) {
    const uint64_t n = uint64_t(f.v.G) * f.v.stride;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
        if (!f(i)) continue;
        const uint32_t h = f.v.buf[i];
        const uint64_t q = pos[i];
        uni[q] = h;
        const uint32_t slot = gt_find(tkey, h, tlog);
        cnt[2 * q] = slot == kNoHeavy ? 0ull : tcnt[slot];
        cnt[2 * q + 1] = slot == kNoHeavy ? 0ull : tcnt[size_t(tcap) + slot];
    }
}

// ---------------------------------------------------------------------- heavy select --
struct IsHeavy {
    const unsigned long long* cnt;
    unsigned long long th;
    __device__ uint64_t operator()(uint64_t i) const { return max(cnt[2 * i], cnt[2 * i + 1]) >= th ? 1 : 0; }
};

__global__ void k_select_emit(IsHeavy f, uint64_t m, const uint64_t* __restrict__ pos, const uint32_t* __restrict__ uni,
                              uint32_t* __restrict__ heavy) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < m; i += uint64_t(gridDim.x) * blockDim.x)
        if (f(i)) heavy[pos[i]] = uni[i];
}

// ------------------------------------------------------------------------- heavy set --
__global__ void k_set_build(const uint32_t* __restrict__ hk, uint64_t n, unsigned long long* set, uint32_t logcap,
                            unsigned int* fail) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
        if (gt_insert(set, hk[i], logcap) == kNoHeavy) *fail = 1;
}

struct HeavySet {
    const unsigned long long* slot;
    uint32_t logcap;   // 0 = empty set
    __device__ __forceinline__ bool has(uint32_t h) const {
        return logcap && gt_find(slot, h, logcap) != kNoHeavy;
    }
};

__device__ __forceinline__ uint32_t route_dest(uint32_t h, uint32_t rb, const HeavySet& hs) {
    if (hs.has(h)) return 1u << rb;  // heavy bucket G
    return rb ? (h >> (32 - rb)) : 0u;
}

// ---------------------------------------------------------------------------- routing --
__global__ void k_route_count(const uint32_t* __restrict__ keys, uint64_t n, uint32_t rb, HeavySet hs,
                              unsigned long long* counts) {
    __shared__ uint32_t c[kMaxShardWorld + 1];
    const uint32_t G1 = (1u << rb) + 1;
    for (uint32_t i = threadIdx.x; i < G1; i += blockDim.x) c[i] = 0;
    __syncthreads();
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
        if (i < n) atomicAdd(&c[route_dest(hash32(__ldcs(keys + i)), rb, hs)], 1u);   // ATOMS.POPC.INC
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < G1; i += blockDim.x)
        if (c[i]) atomicAdd(&counts[i], (unsigned long long)c[i]);
}

// One 8192-tuple tile per iteration: rank each tuple within its destination (match_any peers +
// one shared atomic per (warp, destination)), reserve each destination's run with one global
// atomic on its cursor, permute the tile into shared memory grouped by destination, then write
// runs with consecutive threads on consecutive addresses of the destination buffer.
constexpr int kRouteBlock = 512;
constexpr int kRouteIpt = 8;
constexpr uint32_t kRouteTile = kRouteBlock * kRouteIpt;
constexpr size_t kRouteSmem = size_t(kRouteTile) * (4 + 4 + 2);

__global__ void __launch_bounds__(kRouteBlock, 2) k_route_scatter(const uint32_t* __restrict__ keys,
                                                              const uint32_t* __restrict__ pays, uint64_t n,
                                                              uint32_t rb, HeavySet hs,
                                                              const unsigned long long* __restrict__ dst,
                                                              uint32_t heavy_copies, unsigned long long* cur) {
    extern __shared__ uint4 route_dyn[];
    uint32_t* s_k = reinterpret_cast<uint32_t*>(route_dyn);
    uint32_t* s_p = s_k + kRouteTile;
    uint16_t* s_d = reinterpret_cast<uint16_t*>(s_p + kRouteTile);
    __shared__ uint32_t cnt[kMaxShardWorld + 1], pre[kMaxShardWorld + 1];
    __shared__ unsigned long long base[kMaxShardWorld + 1], wk[kMaxShardWorld + 1], wp[kMaxShardWorld + 1];
    const uint32_t G1 = (1u << rb) + 1;
    const uint32_t dbits = rb + 2;   // destinations 0..G (normal, heavy) and G1 (invalid) fit
    const uint64_t ntiles = (n + kRouteTile - 1) / kRouteTile;
    for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        for (uint32_t i = threadIdx.x; i < G1; i += blockDim.x) cnt[i] = 0;
        __syncthreads();
        const uint64_t t0 = t * kRouteTile;
        uint32_t k[kRouteIpt], p[kRouteIpt], dr[kRouteIpt];  // dr = destination << 16 | rank in tile
#pragma unroll
        for (int j = 0; j < kRouteIpt; ++j) {
            const uint64_t idx = t0 + uint64_t(j) * kRouteBlock + threadIdx.x;
            const bool v = idx < n;
            k[j] = v ? __ldcs(keys + idx) : 0u;
            p[j] = v ? __ldcs(pays + idx) : 0u;
        }
#pragma unroll
        for (int j = 0; j < kRouteIpt; ++j) {
            const bool v = t0 + uint64_t(j) * kRouteBlock + threadIdx.x < n;
            const uint32_t d = v ? route_dest(hash32(k[j]), rb, hs) : G1;   // G1: invalid lanes' own class
            // lanes with the same destination: AND of rb + 2 bit ballots (cheaper than match_any)
            uint32_t peers = kFull;
#pragma unroll
            for (uint32_t b = 0; b < 10; ++b) {
                if (b < dbits) {
                    const uint32_t m = __ballot_sync(kFull, (d >> b) & 1u);
                    peers &= ((d >> b) & 1u) ? m : ~m;
                }
            }
            const uint32_t leader = __ffs(peers) - 1;
            uint32_t b = 0;
            if (v && lane_id() == leader) b = atomicAdd(&cnt[d], (uint32_t)__popc(peers));
            b = __shfl_sync(kFull, b, leader);
            dr[j] = v ? (d << 16 | (b + __popc(peers & lanemask_lt()))) : 0xffffffffu;
        }
        __syncthreads();
        if (threadIdx.x < 32) {   // exclusive scan of the tile's destination counts
            constexpr int kPer = (kMaxShardWorld + 1 + 31) / 32;
            uint32_t c[kPer], s = 0;
#pragma unroll
            for (int q = 0; q < kPer; ++q) {
                const uint32_t i = threadIdx.x * kPer + q;
                c[q] = i < G1 ? cnt[i] : 0u;
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
            for (int q = 0; q < kPer; ++q) {
                const uint32_t i = threadIdx.x * kPer + q;
                if (i < G1) pre[i] = e;
                e += c[q];
            }
        }
        __syncthreads();
        // reserve each destination's run; wk / wp: write addresses biased so that tile position i of
        // destination d's run lands at wk[d] + 4 i (unsigned wrap-around is intended)
        for (uint32_t i = threadIdx.x; i < G1; i += blockDim.x) {
            const unsigned long long b = cnt[i] ? atomicAdd(&cur[i], (unsigned long long)cnt[i]) : 0ull;
            const unsigned long long bias = 4ull * (b - pre[i]);
            wk[i] = dst[2 * i] + bias;
            wp[i] = dst[2 * i + 1] + bias;
            base[i] = b;
        }
#pragma unroll
        for (int j = 0; j < kRouteIpt; ++j) {
            if (dr[j] != 0xffffffffu) {
                const uint32_t d = dr[j] >> 16, q = pre[d] + (dr[j] & 0xffffu);
                s_k[q] = k[j];
                s_p[q] = p[j];
                s_d[q] = (uint16_t)d;
            }
        }
        __syncthreads();
        const uint32_t tn = (uint32_t)umin64(kRouteTile, n - t0);
        for (uint32_t i = threadIdx.x; i < tn; i += kRouteBlock) {
            const uint32_t d = s_d[i];
            *reinterpret_cast<uint32_t*>(wk[d] + 4ull * i) = s_k[i];
            *reinterpret_cast<uint32_t*>(wp[d] + 4ull * i) = s_p[i];
        }
        if (heavy_copies > 1) {   // the skewed run again into every further R_H buffer (peer GPUs')
            const uint32_t h0 = pre[G1 - 1], hn = cnt[G1 - 1];
            const unsigned long long hb = base[G1 - 1];
            for (uint32_t c = 1; c < heavy_copies; ++c)
                for (uint32_t i = threadIdx.x; i < hn; i += kRouteBlock) {
                    reinterpret_cast<uint32_t*>(dst[2 * (G1 - 1 + c)])[hb + i] = s_k[h0 + i];
                    reinterpret_cast<uint32_t*>(dst[2 * (G1 - 1 + c) + 1])[hb + i] = s_p[h0 + i];
                }
        }
        __syncthreads();
    }
}

__global__ void __launch_bounds__(1024, 1)
k_route_from_hist(const unsigned long long* __restrict__ hist, uint32_t B, uint32_t rb,
                  const uint32_t* __restrict__ uni, IsHeavy global, const unsigned long long* __restrict__ cloc,
                  uint64_t m, unsigned long long* __restrict__ out) {
    __shared__ unsigned long long acc[2][kMaxShardWorld + 1];
    const uint32_t G = 1u << rb, F = 1u << B;
    for (uint32_t i = threadIdx.x; i <= G; i += blockDim.x) acc[0][i] = acc[1][i] = 0;
    __syncthreads();
    const uint32_t dshift = B - rb;   // partition p = top B bits of h; its destination = top rb bits
    {   // each thread sums a contiguous range of partitions, flushing when the destination changes
        const uint32_t per = (F + blockDim.x - 1) / blockDim.x, p0 = threadIdx.x * per, p1 = min(F, p0 + per);
        unsigned long long sr = 0, ss = 0;
        uint32_t dcur = p0 >> dshift;
        for (uint32_t p = p0; p < p1; ++p) {
            if ((p >> dshift) != dcur) {
                atomicAdd(&acc[0][dcur], sr);
                atomicAdd(&acc[1][dcur], ss);
                sr = ss = 0;
                dcur = p >> dshift;
            }
            sr += hist[p];
            ss += hist[F + p];
        }
        if (p0 < p1) {
            atomicAdd(&acc[0][dcur], sr);
            atomicAdd(&acc[1][dcur], ss);
        }
    }
    for (uint64_t u = threadIdx.x; u < m; u += blockDim.x) {
        if (!global(u)) continue;
        const uint32_t d = rb ? (uni[u] >> (32 - rb)) : 0u;
        const unsigned long long cr = cloc[2 * u], cs = cloc[2 * u + 1];
        if (cr) {
            atomicAdd(&acc[0][d], 0ull - cr);
            atomicAdd(&acc[0][G], cr);
        }
        if (cs) {
            atomicAdd(&acc[1][d], 0ull - cs);
            atomicAdd(&acc[1][G], cs);
        }
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i <= G; i += blockDim.x) {
        out[i] = acc[0][i];
        out[G + 1 + i] = acc[1][i];
    }
}

int launch_route_counts_from_hist(const uint64_t* hist_local, uint32_t part_bits, uint32_t route_bits,
                                  const uint32_t* uni, const uint64_t* cnt_global, const uint64_t* cnt_local,
                                  uint64_t m, uint32_t heavy_threshold, uint64_t* out, cudaStream_t s) {
    IsHeavy f{reinterpret_cast<const unsigned long long*>(cnt_global), heavy_threshold};
    k_route_from_hist<<<1, 1024, 0, s>>>(reinterpret_cast<const unsigned long long*>(hist_local), part_bits,
                                         route_bits, uni, f, reinterpret_cast<const unsigned long long*>(cnt_local),
                                         m, reinterpret_cast<unsigned long long*>(out));
    return 1;
}

// Per-device one-time opt-in for > 48 KB of dynamic shared memory.
static bool route_attr(cudaStream_t) {
    static std::once_flag attr_once[kMaxDevices];
    once_per_device(attr_once, [] {
        cudaFuncSetAttribute(k_route_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kRouteSmem);
    });
    return true;
}

// Heavy-set buffer: [256-byte header: u32 build-failure flag][slots u64[2^logcap]], 2^logcap the
// largest power of two (>= 1024) that fits; an empty set (n_heavy = 0) may be a NULL buffer.
static HeavySet heavy_set_view(const void* set, size_t set_bytes) {
    HeavySet hs{nullptr, 0};
    if (set && set_bytes >= 256 + 1024 * 8) {
        uint64_t slots = 1024;
        while (256 + slots * 2 * 8 <= set_bytes && slots < (1ull << 31)) slots <<= 1;
        hs.slot = reinterpret_cast<const unsigned long long*>(reinterpret_cast<const unsigned char*>(set) + 256);
        hs.logcap = log2_pow2(slots);
    }
    return hs;
}

}  // namespace gsh

using namespace gsh;

namespace gsh {
gsh_status api_fail(gsh_status s, const char* msg);   // api.cu: sets the thread-local message
gsh_status api_cuda(const char* where);               // api.cu: maps cudaGetLastError()
bool shard_plan_params(uint64_t nR, uint64_t nS, const gsh_config* cfg, uint32_t* B, uint32_t* L, uint32_t* Th);
}  // namespace gsh

extern "C" {

gsh_status gsh_shard_plan(uint64_t n_r_global, uint64_t n_s_global, uint32_t world, const gsh_config* cfg,
                          gsh_shard_params* out) {
    if (!out) return api_fail(GSH_ERR_INVALID, "out is NULL");
    if (world == 0 || world > kMaxShardWorld || (world & (world - 1)))
        return api_fail(GSH_ERR_INVALID, "world must be a power of two <= 256");
    uint32_t B = 0, L = 0, Th = 0;
    if (!shard_plan_params(n_r_global, n_s_global, cfg, &B, &L, &Th)) return api_fail(GSH_ERR_INVALID, "invalid gsh_config");
    std::memset(out, 0, sizeof(*out));
    out->world = world;
    out->route_bits = log2_pow2(world);
    out->part_bits = B;
    out->large_threshold = L;
    out->heavy_threshold = Th;
    out->cand_threshold = (Th + world - 1) / world;
    if (out->cand_threshold == 0) out->cand_threshold = 1;
    out->force_all_normal = cfg ? cfg->force_all_normal : 0;
    return GSH_OK;
}

gsh_status gsh_shard_histogram(const gsh_relation* R, const gsh_relation* S, const gsh_shard_params* p,
                               uint64_t* d_hist, void* stream) {
    if (!R || !S || !p || !d_hist) return api_fail(GSH_ERR_INVALID, "NULL argument");
    if ((R->n && !R->keys) || (S->n && !S->keys) || p->part_bits > 16) return api_fail(GSH_ERR_INVALID, "bad argument");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const size_t F = size_t(1) << p->part_bits;
    cudaMemsetAsync(d_hist, 0, 2 * F * 8, s);
    launch_radix_hist(R->keys, R->n, 0, p->part_bits, d_hist, s);
    launch_radix_hist(S->keys, S->n, 0, p->part_bits, d_hist + F, s);
    return api_cuda("shard_histogram");
}

size_t gsh_shard_workspace_bytes(uint64_t n_r, uint64_t n_s) { return cand_ws_bytes(cand_slots(n_r, n_s)); }

gsh_status gsh_shard_candidates(const gsh_relation* R, const gsh_relation* S, const gsh_shard_params* p,
                                const uint64_t* d_hist_global, void* workspace, size_t workspace_bytes, void* stream,
                                uint32_t* d_cand, uint64_t cap, uint64_t* h_n, uint32_t* h_overflow) {
    if (!R || !S || !p || !d_hist_global || !h_n || (cap && !d_cand)) return api_fail(GSH_ERR_INVALID, "NULL argument");
    if ((R->n && !R->keys) || (S->n && !S->keys) || p->part_bits > 16) return api_fail(GSH_ERR_INVALID, "bad argument");
    const uint32_t cap_t = cand_slots(R->n, S->n);
    if (!workspace || workspace_bytes < cand_ws_bytes(cap_t) || (reinterpret_cast<uintptr_t>(workspace) & 255u))
        return api_fail(GSH_ERR_INVALID, "workspace NULL, misaligned or smaller than gsh_shard_workspace_bytes");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const uint32_t F = 1u << p->part_bits;
    cudaMemsetAsync(workspace, 0, 256, s);
    k_shard_large<<<(F + 255) / 256, 256, 0, s>>>(reinterpret_cast<const unsigned long long*>(d_hist_global), F,
                                                  p->large_threshold, p->force_all_normal,
                                                  cand_ws(workspace, cap_t).large, cand_ws(workspace, cap_t).nlarge);
    // the count table only needs room for this rank's tuples of large partitions (<= the global
    // number): size it from the global count, so a skew-free input clears and scans ~nothing
    unsigned long long nlarge = 0;
    cudaError_t ce = cudaMemcpyAsync(&nlarge, cand_ws(workspace, cap_t).nlarge, 8, cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return api_cuda("shard_candidates large count");
    uint32_t cap_u = 1024;
    const uint64_t local_large = umin64(nlarge, R->n + S->n);
    while (cap_u < 2 * local_large && cap_u < cap_t) cap_u <<= 1;
    CandWs w = cand_ws(workspace, cap_u);
    const uint32_t logcap = log2_pow2(cap_u);
    cudaMemsetAsync(w.key, 0, size_t(cap_u) * 16, s);
    cudaMemcpyAsync(w.slots_used, &cap_u, 4, cudaMemcpyHostToDevice, s);
    const uint32_t pshift = p->part_bits ? 32 - p->part_bits : 32;
    if (nlarge) {
        if (R->n)
            k_cand_count<<<148 * 8, 512, 0, s>>>(R->keys, R->n, 0, pshift, w.large, w.key, w.cnt, cap_u, logcap,
                                                 w.overflow);
        if (S->n)
            k_cand_count<<<148 * 8, 512, 0, s>>>(S->keys, S->n, 1, pshift, w.large, w.key, w.cnt, cap_u, logcap,
                                                 w.overflow);
        k_cand_select<<<148 * 4, 256, 0, s>>>(w.key, w.cnt, cap_u, p->cand_threshold, d_cand, cap, w.nout);
    }
    gsh_status st = api_cuda("shard_candidates");
    if (st != GSH_OK) return st;
    unsigned long long hs[2] = {0, 0};
    ce = cudaMemcpyAsync(hs, workspace, 16, cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return api_cuda("shard_candidates sync");
    *h_n = hs[0];
    if (h_overflow) *h_overflow = (uint32_t)(hs[1] & 0xffffffffu);
    if (hs[0] > cap) return api_fail(GSH_ERR_INVALID, "candidate capacity too small (see *h_n)");
    return GSH_OK;
}

size_t gsh_shard_agree_workspace_bytes(uint64_t n_gathered) {
    uint64_t slots = 1024;
    while (slots < 2 * n_gathered) slots <<= 1;
    const uint64_t scan = (uint64_t(n_gathered) / kScanTile + 4) * 8;
    return 256 + slots * 12 + ((scan + 255) & ~uint64_t(255)) + ((n_gathered + 1) * 8 + 256);
}

gsh_status gsh_shard_agree(const void* cand_ws_ptr, size_t cand_ws_bytes_in, const uint32_t* d_gathered,
                           uint32_t world, uint64_t stride, const uint64_t* h_sizes, void* workspace,
                           size_t workspace_bytes, void* stream, uint32_t* d_union, uint64_t* d_counts, uint64_t cap,
                           uint64_t* h_n) {
    if (!cand_ws_ptr || !h_sizes || !h_n || (cap && (!d_union || !d_counts))) return api_fail(GSH_ERR_INVALID, "NULL argument");
    if (world == 0 || world > kMaxShardWorld) return api_fail(GSH_ERR_INVALID, "bad world");
    if (uint64_t(world) * stride >= (1ull << 32)) return api_fail(GSH_ERR_INVALID, "gathered buffer too large");
    uint64_t tot = 0;
    GatherView v;
    v.buf = d_gathered;
    v.stride = stride;
    v.G = world;
    for (uint32_t g = 0; g < world; ++g) {
        if (h_sizes[g] > stride) return api_fail(GSH_ERR_INVALID, "size exceeds stride");
        v.size[g] = (uint32_t)h_sizes[g];
        tot += h_sizes[g];
    }
    *h_n = 0;
    if (tot && !d_gathered) return api_fail(GSH_ERR_INVALID, "NULL gathered buffer");
    if (!workspace || workspace_bytes < gsh_shard_agree_workspace_bytes(uint64_t(world) * stride) ||
        (reinterpret_cast<uintptr_t>(workspace) & 255u))
        return api_fail(GSH_ERR_INVALID, "workspace NULL, misaligned or too small");
    // the candidate workspace's local count table T (exact local counts of large-partition keys)
    uint32_t cap_t = 0;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    {
        const unsigned char* b = reinterpret_cast<const unsigned char*>(cand_ws_ptr);
        cudaError_t ce = cudaMemcpyAsync(&cap_t, b + 12, 4, cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return api_cuda("shard_agree table size");
        if (cap_t < 1024 || (cap_t & (cap_t - 1)) || cand_ws_bytes(cap_t) > cand_ws_bytes_in)
            return api_fail(GSH_ERR_INVALID, "candidate workspace not initialised by gsh_shard_candidates");
    }
    CandWs t = cand_ws(const_cast<void*>(cand_ws_ptr), cap_t);
    const uint64_t n = uint64_t(world) * stride;
    uint64_t slots = 1024;
    while (slots < 2 * n) slots <<= 1;
    unsigned char* b = reinterpret_cast<unsigned char*>(workspace);
    unsigned int* ovf = reinterpret_cast<unsigned int*>(b);
    unsigned long long* dkey = reinterpret_cast<unsigned long long*>(b + 256);
    uint32_t* didx = reinterpret_cast<uint32_t*>(dkey + slots);
    uint64_t* scratch = reinterpret_cast<uint64_t*>(b + 256 + slots * 12);
    const uint64_t scan = (n / kScanTile + 4) * 8;
    uint64_t* pos = reinterpret_cast<uint64_t*>(reinterpret_cast<unsigned char*>(scratch) + ((scan + 255) & ~uint64_t(255)));
    if (tot == 0) return GSH_OK;
    const uint32_t logcap = log2_pow2(slots);
    cudaMemsetAsync(b, 0, 256, s);
    cudaMemsetAsync(dkey, 0, slots * 8, s);
    cudaMemsetAsync(didx, 0xff, slots * 4, s);
    const unsigned grid = (unsigned)umin64((n + 255) / 256, 148 * 8);
    k_agree_first<<<grid, 256, 0, s>>>(v, dkey, didx, logcap, ovf);
    FirstOcc f{v, dkey, didx, logcap};
    launch_scan(f, n, pos, scratch, s);
    uint64_t m = 0;
    unsigned int hovf = 0;
    cudaError_t ce = cudaMemcpyAsync(&m, pos + n, 8, cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaMemcpyAsync(&hovf, ovf, 4, cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return api_cuda("shard_agree sync");
    if (hovf) return api_fail(GSH_ERR_INTERNAL, "union table overflow");
    *h_n = m;
    if (m > cap) return api_fail(GSH_ERR_INVALID, "union capacity too small (see *h_n)");
    k_agree_emit<<<grid, 256, 0, s>>>(f, pos, t.key, t.cnt, cap_t, log2_pow2(cap_t), d_union,
                                      reinterpret_cast<unsigned long long*>(d_counts));
    return api_cuda("shard_agree");
}

gsh_status gsh_shard_select(const uint32_t* d_union, const uint64_t* d_counts, uint64_t m, const gsh_shard_params* p,
                            void* workspace, size_t workspace_bytes, void* stream, uint32_t* d_heavy, uint64_t cap,
                            uint64_t* h_n) {
    if (!p || !h_n || (m && (!d_union || !d_counts)) || (cap && !d_heavy)) return api_fail(GSH_ERR_INVALID, "NULL argument");
    *h_n = 0;
    if (m == 0) return GSH_OK;
    const uint64_t scan = (m / kScanTile + 4) * 8;
    const size_t need = ((scan + 255) & ~uint64_t(255)) + (m + 1) * 8;
    if (!workspace || workspace_bytes < need || (reinterpret_cast<uintptr_t>(workspace) & 255u))
        return api_fail(GSH_ERR_INVALID, "workspace NULL, misaligned or too small (gsh_shard_agree_workspace_bytes(m))");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    uint64_t* scratch = reinterpret_cast<uint64_t*>(workspace);
    uint64_t* pos = reinterpret_cast<uint64_t*>(reinterpret_cast<unsigned char*>(workspace) + ((scan + 255) & ~uint64_t(255)));
    IsHeavy f{reinterpret_cast<const unsigned long long*>(d_counts), p->heavy_threshold};
    launch_scan(f, m, pos, scratch, s);
    uint64_t nh = 0;
    cudaError_t ce = cudaMemcpyAsync(&nh, pos + m, 8, cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return api_cuda("shard_select sync");
    *h_n = nh;
    if (nh > cap) return api_fail(GSH_ERR_INVALID, "heavy capacity too small (see *h_n)");
    const unsigned grid = (unsigned)umin64((m + 255) / 256, 148 * 8);
    k_select_emit<<<grid, 256, 0, s>>>(f, m, pos, d_union, d_heavy);
    return api_cuda("shard_select");
}

size_t gsh_heavy_set_bytes(uint64_t n_heavy) {
    if (n_heavy == 0) return 0;
    uint64_t slots = 1024;
    while (slots < 2 * n_heavy) slots <<= 1;
    return 256 + slots * 8;
}

gsh_status gsh_heavy_set_build(const uint32_t* d_heavy, uint64_t n, void* d_set, size_t set_bytes, void* stream) {
    if (n == 0) return GSH_OK;
    if (!d_heavy || !d_set || set_bytes < gsh_heavy_set_bytes(n) || (reinterpret_cast<uintptr_t>(d_set) & 255u))
        return api_fail(GSH_ERR_INVALID, "set buffer NULL, misaligned or smaller than gsh_heavy_set_bytes");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const HeavySet hs = heavy_set_view(d_set, set_bytes);
    unsigned int* fail = reinterpret_cast<unsigned int*>(d_set);
    cudaMemsetAsync(d_set, 0, 256 + (size_t(1) << hs.logcap) * 8, s);
    const unsigned grid = (unsigned)umin64((n + 255) / 256, 148 * 8);
    k_set_build<<<grid, 256, 0, s>>>(d_heavy, n, const_cast<unsigned long long*>(hs.slot), hs.logcap, fail);
    unsigned int hf = 0;
    cudaError_t ce = cudaMemcpyAsync(&hf, fail, 4, cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return api_cuda("set build");
    if (hf) return api_fail(GSH_ERR_INTERNAL, "heavy set probe budget exhausted");
    return GSH_OK;
}

gsh_status gsh_route_count(const uint32_t* d_keys, uint64_t n, uint32_t route_bits, const void* d_set,
                           size_t set_bytes, uint64_t* d_counts, void* stream) {
    if (route_bits > 8) return api_fail(GSH_ERR_INVALID, "route_bits > 8");
    if ((n && !d_keys) || !d_counts) return api_fail(GSH_ERR_INVALID, "NULL pointer");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    cudaMemsetAsync(d_counts, 0, ((1u << route_bits) + 1) * 8, s);
    if (n) {
        const unsigned grid = (unsigned)umin64((n + 1023) / 1024, 148 * 4);
        k_route_count<<<grid, 1024, 0, s>>>(d_keys, n, route_bits, heavy_set_view(d_set, set_bytes),
                                            reinterpret_cast<unsigned long long*>(d_counts));
    }
    return api_cuda("route_count");
}

gsh_status gsh_route_scatter(const uint32_t* d_keys, const uint32_t* d_payloads, uint64_t n, uint32_t route_bits,
                             const void* d_set, size_t set_bytes, const uint64_t* d_dst, uint32_t heavy_copies,
                             uint64_t* d_cursor, void* stream) {
    if (route_bits > 8) return api_fail(GSH_ERR_INVALID, "route_bits > 8");
    if (heavy_copies < 1 || heavy_copies > kMaxShardWorld) return api_fail(GSH_ERR_INVALID, "bad heavy_copies");
    if (n && (!d_keys || !d_payloads || !d_dst || !d_cursor)) return api_fail(GSH_ERR_INVALID, "NULL pointer");
    if (n == 0) return GSH_OK;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    if (!route_attr(s)) return api_cuda("route_scatter attribute");
    cudaMemsetAsync(d_cursor, 0, ((1u << route_bits) + 1) * 8, s);
    const unsigned grid = (unsigned)umin64((n + kRouteTile - 1) / kRouteTile, 148 * 2);
    k_route_scatter<<<grid, kRouteBlock, kRouteSmem, s>>>(d_keys, d_payloads, n, route_bits,
                                                          heavy_set_view(d_set, set_bytes),
                                                          reinterpret_cast<const unsigned long long*>(d_dst),
                                                          heavy_copies,
                                                          reinterpret_cast<unsigned long long*>(d_cursor));
    return api_cuda("route_scatter");
}

// CUDA IPC: a device allocation shared with the other processes of the node (peer GPUs over
// NVLink, or another process on the same GPU), for the route kernel's direct peer stores.  A
// handle names a whole cudaMalloc allocation; the caller's buffer (a caching-allocator
// sub-range) is its base + *offset, found with the driver's cuMemGetAddressRange (looked up at
// run time, so libgsh loads without a driver, e.g. for the CPU tests).
typedef int (*CuMemGetAddressRange)(unsigned long long*, size_t*, unsigned long long);
static CuMemGetAddressRange cu_range() {
    static CuMemGetAddressRange fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_NOLOAD);
        if (!h) h = dlopen("libcuda.so.1", RTLD_NOW);
        if (h) fn = reinterpret_cast<CuMemGetAddressRange>(dlsym(h, "cuMemGetAddressRange_v2"));
    });
    return fn;
}

gsh_status gsh_ipc_handle(const void* d_ptr, void* handle, uint64_t* offset) {
    if (!d_ptr || !handle || !offset) return api_fail(GSH_ERR_INVALID, "NULL pointer");
    const CuMemGetAddressRange range = cu_range();
    if (!range) return api_fail(GSH_ERR_CUDA, "cuMemGetAddressRange unavailable (no CUDA driver)");
    unsigned long long base = 0;
    size_t size = 0;
    if (range(&base, &size, reinterpret_cast<unsigned long long>(d_ptr)) != 0)
        return api_fail(GSH_ERR_CUDA, "cuMemGetAddressRange failed");
    cudaIpcMemHandle_t h;
    const cudaError_t e = cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base));
    if (e != cudaSuccess) {
        cudaGetLastError();
        return api_fail(GSH_ERR_CUDA, cudaGetErrorString(e));
    }
    std::memcpy(handle, &h, sizeof(h));
    *offset = reinterpret_cast<unsigned long long>(d_ptr) - base;
    return GSH_OK;
}

gsh_status gsh_ipc_open(const void* handle, void** d_ptr) {
    if (!handle || !d_ptr) return api_fail(GSH_ERR_INVALID, "NULL pointer");
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, sizeof(h));
    const cudaError_t e = cudaIpcOpenMemHandle(d_ptr, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return api_fail(GSH_ERR_CUDA, cudaGetErrorString(e));
    }
    return GSH_OK;
}

gsh_status gsh_ipc_close(void* d_ptr) {
    if (!d_ptr) return GSH_OK;
    const cudaError_t e = cudaIpcCloseMemHandle(d_ptr);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return api_fail(GSH_ERR_CUDA, cudaGetErrorString(e));
    }
    return GSH_OK;
}

}  // extern "C"
