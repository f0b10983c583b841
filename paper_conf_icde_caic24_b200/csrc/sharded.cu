// sharded.cu -- the native multi-GPU driver: gsh_join_sharded and its communicators
// (SURVEY.md §8(b) "gsh_join_sharded(..., ncclComm_t)", §8(e)).  Not in the paper,
// which runs on one A100 (§V-A): the north star adds hash sharding over one
// 8xB200 node.
//
// gsh_join_sharded is the per-rank protocol of shard.cu's steps, run in the library between the
// collectives of a gsh_comm table:
//   sizes -> all_reduce                 gsh_shard_plan: the single-GPU (B, L, T_h) of the whole input
//   histogram -> all_reduce             globally large partitions (L107)
//   candidates -> all_gather            local max(cnt_R, cnt_S) >= ceil(T_h / G) (pigeonhole)
//   agree -> all_reduce -> select       skewed iff global max(cnt_R, cnt_S) >= T_h (L112)
//   route counts -> all_gather          the G x 2(G+1) count matrix: every rank derives every
//                                       buffer offset from it, identically
//   route scatter + exchange            a2a: send buffers, skewed R all-gathered on the compute
//                                       stream, the normal all_to_all_v on a second stream while
//                                       the skewed-key join runs; p2p: the route kernel stores
//                                       into the peers' receive buffers (CUDA IPC), one barrier
//   gsh_join x 2                        routed normal shard (route_bits = log2 G), all skewed R x
//                                       local skewed S (route_bits = 0)
//   (count, checksum) -> all_reduce     mod 2^64: the single-GPU result bit-exactly
//
// Communicators: NCCL (libnccl.so.2 resolved at run time, the process's loaded copy first, so an
// ncclComm_t of torch's process group is driven by the library that created it), and an
// in-process local world (G host threads = G ranks; device copies behind host barriers).
#include <algorithm>
#include <condition_variable>
#include <cstring>
#include <dlfcn.h>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include <nccl.h>   // types and enums only: the functions are looked up with dlsym

#include "gsh_internal.h"

namespace gsh {
gsh_status api_fail(gsh_status s, const char* msg);   // api.cu: sets the thread-local message
gsh_status api_cuda(const char* where);               // api.cu: maps cudaGetLastError()
}  // namespace gsh

using namespace gsh;

namespace {

constexpr uint32_t kMaxWorld = 256;

gsh_status cuda_status(cudaError_t e, const char* where) {
    if (e == cudaSuccess) return GSH_OK;
    cudaGetLastError();
    return api_fail(GSH_ERR_CUDA, (std::string(where) + ": " + cudaGetErrorString(e)).c_str());
}

// --------------------------------------------------------------------------- NCCL --
struct NcclApi {
    bool ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    ncclResult_t (*CommCount)(const ncclComm_t, int*) = nullptr;
    ncclResult_t (*CommUserRank)(const ncclComm_t, int*) = nullptr;
};

const NcclApi& nccl_api() {
    static NcclApi a;
    static std::once_flag once;
    std::call_once(once, [] {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW);
        if (!h) return;
#define GSH_NCCL_SYM(x) a.x = reinterpret_cast<decltype(a.x)>(dlsym(h, "nccl" #x))
        GSH_NCCL_SYM(GetUniqueId);
        GSH_NCCL_SYM(CommInitRank);
        GSH_NCCL_SYM(CommDestroy);
        GSH_NCCL_SYM(AllReduce);
        GSH_NCCL_SYM(AllGather);
        GSH_NCCL_SYM(Send);
        GSH_NCCL_SYM(Recv);
        GSH_NCCL_SYM(GroupStart);
        GSH_NCCL_SYM(GroupEnd);
        GSH_NCCL_SYM(GetErrorString);
        GSH_NCCL_SYM(CommCount);
        GSH_NCCL_SYM(CommUserRank);
#undef GSH_NCCL_SYM
        a.ok = a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.AllReduce && a.AllGather && a.Send &&
               a.Recv && a.GroupStart && a.GroupEnd && a.GetErrorString && a.CommCount && a.CommUserRank;
    });
    return a;
}

gsh_status nccl_status(ncclResult_t r, const char* where) {
    if (r == ncclSuccess) return GSH_OK;
    const NcclApi& a = nccl_api();
    std::string m = std::string(where) + ": " + (a.GetErrorString ? a.GetErrorString(r) : "NCCL error");
    return api_fail(GSH_ERR_NCCL, m.c_str());
}

struct NcclCtx {
    ncclComm_t comm = nullptr;
    bool owned = false;
    uint64_t* d_one = nullptr;   // barrier scratch
};

gsh_status nccl_all_reduce(void* ctx, uint64_t* d, uint64_t n, void* stream) {
    if (n == 0) return GSH_OK;
    NcclCtx* c = static_cast<NcclCtx*>(ctx);
    return nccl_status(nccl_api().AllReduce(d, d, n, ncclUint64, ncclSum, c->comm, (cudaStream_t)stream),
                       "ncclAllReduce");
}

gsh_status nccl_all_gather(void* ctx, const void* send, void* recv, uint64_t bytes, void* stream) {
    if (bytes == 0) return GSH_OK;
    NcclCtx* c = static_cast<NcclCtx*>(ctx);
    return nccl_status(nccl_api().AllGather(send, recv, bytes, ncclUint8, c->comm, (cudaStream_t)stream),
                       "ncclAllGather");
}

gsh_status nccl_all_to_all_v(void* ctx, const void* send, const uint64_t* soff, const uint64_t* sbytes, void* recv,
                             const uint64_t* roff, const uint64_t* rbytes, void* stream) {
    NcclCtx* c = static_cast<NcclCtx*>(ctx);
    const NcclApi& a = nccl_api();
    int G = 0;
    gsh_status st = nccl_status(a.CommCount(c->comm, &G), "ncclCommCount");
    if (st != GSH_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    st = nccl_status(a.GroupStart(), "ncclGroupStart");
    if (st != GSH_OK) return st;
    for (int g = 0; g < G && st == GSH_OK; ++g) {
        if (sbytes[g])
            st = nccl_status(a.Send(static_cast<const char*>(send) + soff[g], sbytes[g], ncclUint8, g, c->comm, s),
                             "ncclSend");
        if (st == GSH_OK && rbytes[g])
            st = nccl_status(a.Recv(static_cast<char*>(recv) + roff[g], rbytes[g], ncclUint8, g, c->comm, s),
                             "ncclRecv");
    }
    const gsh_status se = nccl_status(a.GroupEnd(), "ncclGroupEnd");
    return st != GSH_OK ? st : se;
}

gsh_status nccl_barrier(void* ctx, void* stream) {
    NcclCtx* c = static_cast<NcclCtx*>(ctx);
    cudaStream_t s = (cudaStream_t)stream;
    if (!c->d_one) {
        gsh_status st = cuda_status(cudaMalloc(&c->d_one, 8), "barrier scratch");
        if (st != GSH_OK) return st;
        cudaMemsetAsync(c->d_one, 0, 8, s);
    }
    gsh_status st = nccl_status(nccl_api().AllReduce(c->d_one, c->d_one, 1, ncclUint64, ncclSum, c->comm, s),
                                "ncclAllReduce(barrier)");
    if (st != GSH_OK) return st;
    return cuda_status(cudaStreamSynchronize(s), "barrier sync");
}

gsh_status fill_nccl(NcclCtx* c, gsh_comm* out) {
    const NcclApi& a = nccl_api();
    int G = 0, r = 0;
    gsh_status st = nccl_status(a.CommCount(c->comm, &G), "ncclCommCount");
    if (st == GSH_OK) st = nccl_status(a.CommUserRank(c->comm, &r), "ncclCommUserRank");
    if (st != GSH_OK) return st;
    std::memset(out, 0, sizeof(*out));
    out->rank = (uint32_t)r;
    out->world = (uint32_t)G;
    out->same_process = 0;
    out->ctx = c;
    out->all_reduce_u64 = nccl_all_reduce;
    out->all_gather = nccl_all_gather;
    out->all_to_all_v = nccl_all_to_all_v;
    out->barrier = nccl_barrier;
    out->abort = nullptr;
    return GSH_OK;
}

// -------------------------------------------------------------------- local world --
struct PtrSet {
    const unsigned long long* p[kMaxWorld];
};

__global__ void k_sum_u64(unsigned long long* __restrict__ dst, PtrSet src, uint32_t G, uint64_t n) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
        unsigned long long s = 0;
        for (uint32_t g = 0; g < G; ++g) s += src.p[g][i];
        dst[i] = s;
    }
}

struct LocalWorld;
struct LocalRank {
    LocalWorld* w = nullptr;
    uint32_t rank = 0;
    void* tmp = nullptr;   // all-reduce staging (this rank's device memory)
    size_t tmp_cap = 0;
};

struct LocalWorld {
    struct Slot {
        const void* p = nullptr;
        const uint64_t* off = nullptr;
        const uint64_t* bytes = nullptr;
    };
    uint32_t G = 0;
    std::mutex m;
    std::condition_variable cv;
    uint32_t arrived = 0;
    uint64_t gen = 0;
    bool aborted = false;
    std::vector<Slot> slot;
    std::vector<LocalRank> ranks;

    bool wait() {
        std::unique_lock<std::mutex> l(m);
        if (aborted) return false;
        const uint64_t g = gen;
        if (++arrived == G) {
            arrived = 0;
            ++gen;
            cv.notify_all();
            return true;
        }
        cv.wait(l, [&] { return gen != g || aborted; });
        return gen != g;
    }
    void abort() {
        std::lock_guard<std::mutex> l(m);
        aborted = true;
        cv.notify_all();
    }
};

gsh_status local_peer_failed() { return api_fail(GSH_ERR_INTERNAL, "local world: a peer rank failed (aborted)"); }

gsh_status local_sync(cudaStream_t s) { return cuda_status(cudaStreamSynchronize(s), "local world sync"); }

gsh_status local_all_reduce(void* ctx, uint64_t* d, uint64_t n, void* stream) {
    LocalRank* r = static_cast<LocalRank*>(ctx);
    LocalWorld* w = r->w;
    cudaStream_t s = (cudaStream_t)stream;
    gsh_status st = local_sync(s);
    w->slot[r->rank].p = d;
    if (!w->wait()) return local_peer_failed();
    if (st == GSH_OK && n && r->tmp_cap < n * 8) {
        if (r->tmp) cudaFree(r->tmp);
        r->tmp = nullptr;
        r->tmp_cap = 0;
        st = cuda_status(cudaMalloc(&r->tmp, n * 8), "local all-reduce staging");
        if (st == GSH_OK) r->tmp_cap = n * 8;
    }
    if (st == GSH_OK && n) {
        PtrSet ps;
        for (uint32_t g = 0; g < w->G; ++g) ps.p[g] = static_cast<const unsigned long long*>(w->slot[g].p);
        const unsigned grid = (unsigned)std::min<uint64_t>((n + 255) / 256, 148 * 4);
        k_sum_u64<<<grid, 256, 0, s>>>(static_cast<unsigned long long*>(r->tmp), ps, w->G, n);
        st = cuda_status(cudaGetLastError(), "local all-reduce kernel");
        if (st == GSH_OK) st = local_sync(s);
    }
    if (!w->wait()) return local_peer_failed();   // every rank has read every buffer
    if (st == GSH_OK && n) st = cuda_status(cudaMemcpyAsync(d, r->tmp, n * 8, cudaMemcpyDefault, s), "local all-reduce");
    return st;
}

gsh_status local_all_gather(void* ctx, const void* send, void* recv, uint64_t bytes, void* stream) {
    LocalRank* r = static_cast<LocalRank*>(ctx);
    LocalWorld* w = r->w;
    cudaStream_t s = (cudaStream_t)stream;
    gsh_status st = local_sync(s);
    w->slot[r->rank].p = send;
    if (!w->wait()) return local_peer_failed();
    for (uint32_t g = 0; g < w->G && st == GSH_OK && bytes; ++g)
        st = cuda_status(cudaMemcpyAsync(static_cast<char*>(recv) + g * bytes, w->slot[g].p, bytes, cudaMemcpyDefault, s),
                         "local all-gather");
    if (st == GSH_OK) st = local_sync(s);
    if (!w->wait()) return local_peer_failed();
    return st;
}

gsh_status local_all_to_all_v(void* ctx, const void* send, const uint64_t* soff, const uint64_t* sbytes, void* recv,
                              const uint64_t* roff, const uint64_t* rbytes, void* stream) {
    LocalRank* r = static_cast<LocalRank*>(ctx);
    LocalWorld* w = r->w;
    const uint32_t me = r->rank;
    cudaStream_t s = (cudaStream_t)stream;
    gsh_status st = local_sync(s);
    w->slot[me].p = send;
    w->slot[me].off = soff;
    w->slot[me].bytes = sbytes;
    if (!w->wait()) return local_peer_failed();
    for (uint32_t g = 0; g < w->G && st == GSH_OK; ++g) {
        const uint64_t n = w->slot[g].bytes[me];
        if (n != rbytes[g]) {
            st = api_fail(GSH_ERR_INVALID, "all_to_all_v: send and receive sizes differ");
            break;
        }
        if (n)
            st = cuda_status(cudaMemcpyAsync(static_cast<char*>(recv) + roff[g],
                                             static_cast<const char*>(w->slot[g].p) + w->slot[g].off[me], n,
                                             cudaMemcpyDefault, s),
                             "local all-to-all");
    }
    if (st == GSH_OK) st = local_sync(s);
    if (!w->wait()) return local_peer_failed();
    return st;
}

gsh_status local_barrier(void* ctx, void* stream) {
    LocalRank* r = static_cast<LocalRank*>(ctx);
    gsh_status st = local_sync((cudaStream_t)stream);
    if (!r->w->wait()) return local_peer_failed();
    return st;
}

void local_abort(void* ctx) { static_cast<LocalRank*>(ctx)->w->abort(); }

}  // namespace

// ------------------------------------------------------------------ driver state --
struct gsh_sharded {
    struct Buf {
        void* p = nullptr;
        size_t cap = 0;
    };
    gsh_comm c{};
    int dev = 0;
    cudaStream_t xs = nullptr;     // exchange stream (a2a: normal all_to_all_v beside the skewed join)
    cudaEvent_t ev[10] = {};
    Buf ctl, hist, hloc, cloc, candws, cand, gathered, agreews, uni, cnt, heavy, set, mat, sh, rx, sx, wsn, wsh;
    Buf rn, sn, rh;                // receive buffers: keys [0, cap), payloads [cap, 2 cap)
    uint64_t cap_rn = 0, cap_sn = 0, cap_rh = 0;   // p2p: the world-wide capacities (tuples)
    bool shared = false;           // p2p: rn / sn / rh are known to the peers
    std::vector<void*> peer_rn, peer_sn, peer_rh;
    std::vector<void*> ipc_mapped;
};

namespace {

// Grow-only device buffer; `keep` preserves the contents (stream-ordered copy).
gsh_status ensure(gsh_sharded::Buf& b, size_t bytes, cudaStream_t s, bool keep = false) {
    if (b.cap >= bytes) return GSH_OK;
    const size_t cap = std::max<size_t>(bytes + bytes / 8, 256);
    void* p = nullptr;
    gsh_status st = cuda_status(cudaMalloc(&p, cap), "driver buffer");
    if (st != GSH_OK) return st;
    if (keep && b.p) {
        st = cuda_status(cudaMemcpyAsync(p, b.p, b.cap, cudaMemcpyDeviceToDevice, s), "driver buffer copy");
        if (st == GSH_OK) st = cuda_status(cudaStreamSynchronize(s), "driver buffer copy");
    }
    if (b.p) cudaFree(b.p);
    b.p = p;
    b.cap = cap;
    return st;
}

void release(gsh_sharded::Buf& b) {
    if (b.p) cudaFree(b.p);
    b.p = nullptr;
    b.cap = 0;
}

void close_peers(gsh_sharded* x) {
    for (void* p : x->ipc_mapped) cudaIpcCloseMemHandle(p);
    x->ipc_mapped.clear();
    cudaGetLastError();
    x->peer_rn.clear();
    x->peer_sn.clear();
    x->peer_rh.clear();
    x->shared = false;
}

template <class T>
T* at(const gsh_sharded::Buf& b, size_t byte_off = 0) {
    return reinterpret_cast<T*>(static_cast<char*>(b.p) + byte_off);
}

// p2p: receive buffers of the world-wide capacities, shared with every peer (raw pointers in one
// process, CUDA IPC handles across processes).  All ranks take the same decisions (the
// capacities come from the all-gathered count matrix), so they grow and re-share together.
gsh_status ensure_shared(gsh_sharded* x, uint64_t need_rn, uint64_t need_sn, uint64_t need_rh, cudaStream_t s) {
    const gsh_comm& c = x->c;
    if (x->shared && need_rn <= x->cap_rn && need_sn <= x->cap_sn && need_rh <= x->cap_rh) return GSH_OK;
    auto grow = [](uint64_t need, uint64_t old) { return std::max<uint64_t>(need + (need >> 3) + 1024, old); };
    gsh_status st = c.barrier(c.ctx, s);   // every peer is done with the old buffers
    if (st != GSH_OK) return st;
    close_peers(x);
    release(x->rn);
    release(x->sn);
    release(x->rh);
    x->cap_rn = grow(need_rn, x->cap_rn);
    x->cap_sn = grow(need_sn, x->cap_sn);
    x->cap_rh = grow(need_rh, x->cap_rh);
    if ((st = ensure(x->rn, x->cap_rn * 8, s)) != GSH_OK) return st;
    if ((st = ensure(x->sn, x->cap_sn * 8, s)) != GSH_OK) return st;
    if ((st = ensure(x->rh, x->cap_rh * 8, s)) != GSH_OK) return st;
    const uint32_t G = c.world;
    const size_t rec = c.same_process ? 3 * 8 : 3 * sizeof(cudaIpcMemHandle_t);
    std::vector<unsigned char> mine(rec), all(size_t(G) * rec);
    void* bases[3] = {x->rn.p, x->sn.p, x->rh.p};
    if (c.same_process) {
        std::memcpy(mine.data(), bases, 24);
    } else {
        for (int i = 0; i < 3; ++i) {
            cudaIpcMemHandle_t h;
            if ((st = cuda_status(cudaIpcGetMemHandle(&h, bases[i]), "cudaIpcGetMemHandle")) != GSH_OK) return st;
            std::memcpy(mine.data() + i * sizeof(h), &h, sizeof(h));
        }
    }
    const size_t ctl_need = rec * (G + 1);
    if ((st = ensure(x->mat, ctl_need, s)) != GSH_OK) return st;
    unsigned char* d = at<unsigned char>(x->mat);
    if ((st = cuda_status(cudaMemcpyAsync(d, mine.data(), rec, cudaMemcpyHostToDevice, s), "share")) != GSH_OK) return st;
    if ((st = c.all_gather(c.ctx, d, d + rec, rec, s)) != GSH_OK) return st;
    if ((st = cuda_status(cudaMemcpyAsync(all.data(), d + rec, G * rec, cudaMemcpyDeviceToHost, s), "share")) != GSH_OK)
        return st;
    if ((st = cuda_status(cudaStreamSynchronize(s), "share")) != GSH_OK) return st;
    x->peer_rn.assign(G, nullptr);
    x->peer_sn.assign(G, nullptr);
    x->peer_rh.assign(G, nullptr);
    for (uint32_t g = 0; g < G; ++g) {
        void* p[3];
        if (g == c.rank) {
            std::memcpy(p, bases, 24);
        } else if (c.same_process) {
            std::memcpy(p, all.data() + g * rec, 24);
        } else {
            for (int i = 0; i < 3; ++i) {
                cudaIpcMemHandle_t h;
                std::memcpy(&h, all.data() + g * rec + i * sizeof(h), sizeof(h));
                if ((st = cuda_status(cudaIpcOpenMemHandle(&p[i], h, cudaIpcMemLazyEnablePeerAccess),
                                      "cudaIpcOpenMemHandle")) != GSH_OK)
                    return st;
                x->ipc_mapped.push_back(p[i]);
            }
        }
        x->peer_rn[g] = p[0];
        x->peer_sn[g] = p[1];
        x->peer_rh[g] = p[2];
    }
    x->shared = true;
    return GSH_OK;
}

float ms_between(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
        cudaGetLastError();
        return 0.f;
    }
    return ms;
}

gsh_status run_sharded(gsh_sharded* x, const gsh_relation* R, const gsh_relation* S, gsh_out_mode mode,
                       const gsh_output* out, const gsh_config* cfg_in, gsh_exchange exch, cudaStream_t s,
                       gsh_sharded_result* res) {
    const gsh_comm& c = x->c;
    const uint32_t G = c.world, me = c.rank;
    gsh_status st = GSH_OK;
#define CK(expr)                         \
    do {                                 \
        if ((st = (expr)) != GSH_OK) return st; \
    } while (0)
    CK(cuda_status(cudaSetDevice(x->dev), "cudaSetDevice"));
    uint32_t launches = 0;
    cudaEventRecord(x->ev[0], s);

    // ---- global sizes and the plan (the single-GPU rule on the whole input)
    CK(ensure(x->ctl, 16 + 16 * (G + 1) + 64, s));
    uint64_t* d_ctl = at<uint64_t>(x->ctl);
    uint64_t hn[2] = {R->n, S->n};
    CK(cuda_status(cudaMemcpyAsync(d_ctl, hn, 16, cudaMemcpyHostToDevice, s), "sizes"));
    CK(c.all_reduce_u64(c.ctx, d_ctl, 2, s));
    CK(cuda_status(cudaMemcpyAsync(hn, d_ctl, 16, cudaMemcpyDeviceToHost, s), "sizes"));
    CK(cuda_status(cudaStreamSynchronize(s), "sizes"));
    gsh_shard_params P;
    CK(gsh_shard_plan(hn[0], hn[1], G, cfg_in, &P));
    const uint32_t rb = P.route_bits;
    res->route_bits = rb;
    res->part_bits = P.part_bits;
    res->large_threshold = P.large_threshold;
    res->heavy_threshold = P.heavy_threshold;
    res->cand_threshold = P.cand_threshold;

    // ---- skew agreement
    const size_t F = size_t(1) << P.part_bits;
    CK(ensure(x->hist, 2 * F * 8, s));
    CK(gsh_shard_histogram(R, S, &P, at<uint64_t>(x->hist), s));
    launches += (R->n > 0) + (S->n > 0);
    const bool counts_from_hist = rb <= P.part_bits;   // route counts from the local histogram
    if (counts_from_hist) {
        CK(ensure(x->hloc, 2 * F * 8, s));
        CK(cuda_status(cudaMemcpyAsync(x->hloc.p, x->hist.p, 2 * F * 8, cudaMemcpyDeviceToDevice, s), "local hist"));
    }
    CK(c.all_reduce_u64(c.ctx, at<uint64_t>(x->hist), 2 * F, s));
    const size_t cws = gsh_shard_workspace_bytes(R->n, S->n);
    CK(ensure(x->candws, cws, s));
    uint64_t cap = std::max<uint64_t>(1024, (R->n + S->n) / 64), nc = 0;
    uint32_t covf = 0;
    for (;;) {
        CK(ensure(x->cand, cap * 4, s));
        st = gsh_shard_candidates(R, S, &P, at<uint64_t>(x->hist), x->candws.p, x->candws.cap, s, at<uint32_t>(x->cand),
                                  cap, &nc, &covf);
        if (st == GSH_ERR_INVALID && nc > cap) {
            cap = nc;
            continue;
        }
        CK(st);
        break;
    }
    launches += 2 + (R->n > 0) + (S->n > 0);
    uint64_t* d_sz = d_ctl + 2;   // [mine: n, overflow | gathered: G x (n, overflow)]
    uint64_t hs[2] = {nc, covf};
    CK(cuda_status(cudaMemcpyAsync(d_sz, hs, 16, cudaMemcpyHostToDevice, s), "candidate sizes"));
    CK(c.all_gather(c.ctx, d_sz, d_sz + 2, 16, s));
    std::vector<uint64_t> gs(2 * G);
    CK(cuda_status(cudaMemcpyAsync(gs.data(), d_sz + 2, 16 * G, cudaMemcpyDeviceToHost, s), "candidate sizes"));
    CK(cuda_status(cudaStreamSynchronize(s), "candidate sizes"));
    std::vector<uint64_t> sizes(G);
    uint64_t stride = 0, total = 0;
    for (uint32_t g = 0; g < G; ++g) {
        sizes[g] = gs[2 * g];
        stride = std::max(stride, sizes[g]);
        total += sizes[g];
        res->cand_overflow |= gs[2 * g + 1] ? 1u : 0u;
    }
    res->n_candidates = total;
    uint64_t nh = 0, m = 0;
    if (stride) {
        CK(ensure(x->cand, stride * 4, s, /*keep=*/true));
        CK(ensure(x->gathered, G * stride * 4, s));
        CK(c.all_gather(c.ctx, x->cand.p, x->gathered.p, stride * 4, s));
        CK(ensure(x->agreews, gsh_shard_agree_workspace_bytes(uint64_t(G) * stride), s));
        CK(ensure(x->uni, total * 4, s));
        CK(ensure(x->cnt, total * 16, s));
        CK(gsh_shard_agree(x->candws.p, x->candws.cap, at<uint32_t>(x->gathered), G, stride, sizes.data(),
                           x->agreews.p, x->agreews.cap, s, at<uint32_t>(x->uni), at<uint64_t>(x->cnt), total, &m));
        launches += 5;
        res->n_union = m;
        if (counts_from_hist) {
            CK(ensure(x->cloc, std::max<uint64_t>(m, 1) * 16, s));
            CK(cuda_status(cudaMemcpyAsync(x->cloc.p, x->cnt.p, m * 16, cudaMemcpyDeviceToDevice, s), "local counts"));
        }
        CK(c.all_reduce_u64(c.ctx, at<uint64_t>(x->cnt), 2 * m, s));
        CK(ensure(x->heavy, std::max<uint64_t>(m, 1) * 4, s));
        CK(gsh_shard_select(at<uint32_t>(x->uni), at<uint64_t>(x->cnt), m, &P, x->agreews.p, x->agreews.cap, s,
                            at<uint32_t>(x->heavy), m, &nh));
        launches += m ? 4 : 0;
    }
    res->n_heavy = (uint32_t)nh;
    const size_t sb = gsh_heavy_set_bytes(nh);
    if (nh) {
        CK(ensure(x->set, sb, s));
        CK(gsh_heavy_set_build(at<uint32_t>(x->heavy), nh, x->set.p, sb, s));
        launches += 1;
    }
    const void* set = nh ? x->set.p : nullptr;
    cudaEventRecord(x->ev[1], s);

    // ---- routing plan: the count matrix (row g: rank g's R counts per destination, then S's)
    const uint32_t W = 2 * (G + 1);
    CK(ensure(x->mat, size_t(W) * (G + 1) * 8, s));
    uint64_t* d_mat = at<uint64_t>(x->mat);
    if (counts_from_hist && !covf) {
        // no second read of the keys: the local histogram's destination sums minus the skewed keys'
        // exact local counts (this rank's count table did not overflow)
        launch_route_counts_from_hist(at<uint64_t>(x->hloc), P.part_bits, rb, m ? at<uint32_t>(x->uni) : nullptr,
                                      m ? at<uint64_t>(x->cnt) : nullptr, m ? at<uint64_t>(x->cloc) : nullptr, m,
                                      P.heavy_threshold, d_mat + size_t(W) * G, s);
        launches += 1;
        CK(api_cuda("route counts"));
    } else {
        CK(gsh_route_count(R->keys, R->n, rb, set, sb, d_mat + size_t(W) * G, s));
        CK(gsh_route_count(S->keys, S->n, rb, set, sb, d_mat + size_t(W) * G + G + 1, s));
        launches += (R->n > 0) + (S->n > 0);
    }
    CK(c.all_gather(c.ctx, d_mat + size_t(W) * G, d_mat, W * 8, s));
    std::vector<uint64_t> M(size_t(W) * G);
    CK(cuda_status(cudaMemcpyAsync(M.data(), d_mat, M.size() * 8, cudaMemcpyDeviceToHost, s), "count matrix"));
    CK(cuda_status(cudaStreamSynchronize(s), "count matrix"));
    auto rc = [&](uint32_t g, uint32_t d) { return M[size_t(g) * W + d]; };
    auto sc = [&](uint32_t g, uint32_t d) { return M[size_t(g) * W + G + 1 + d]; };
    std::vector<uint64_t> need_rn(G, 0), need_sn(G, 0), off_rn(G, 0), off_sn(G, 0);
    uint64_t need_rh = 0, off_rh_me = 0;
    std::vector<uint64_t> off_rh(G, 0);
    for (uint32_t g = 0; g < G; ++g) {
        off_rh[g] = need_rh;
        need_rh += rc(g, G);
        for (uint32_t d = 0; d < G; ++d) {
            if (g < me) {
                off_rn[d] += rc(g, d);   // my run in destination d's receive buffer
                off_sn[d] += sc(g, d);
            }
            need_rn[d] += rc(g, d);
            need_sn[d] += sc(g, d);
        }
    }
    off_rh_me = off_rh[me];
    const uint64_t nrn = need_rn[me], nsn = need_sn[me], nrh = need_rh, nsh = sc(me, G);
    CK(ensure(x->sh, std::max<uint64_t>(nsh, 1) * 8, s));
    uint32_t* shk = at<uint32_t>(x->sh);
    uint32_t* shp = shk + std::max<uint64_t>(nsh, 1);
    std::vector<uint64_t> dr(2 * (2 * G + 1), 0), ds(2 * (G + 1), 0);
    uint64_t Lrn, Lsn, Lrh;   // layout capacities (payloads start at keys + L)
    uint64_t xbytes = 0, bbytes = 0;
    auto addr = [](void* base, uint64_t idx) { return uint64_t(reinterpret_cast<uintptr_t>(base)) + 4 * idx; };
    if (exch == GSH_EXCHANGE_P2P) {
        uint64_t mx_rn = 0, mx_sn = 0;
        for (uint32_t d = 0; d < G; ++d) {
            mx_rn = std::max(mx_rn, need_rn[d]);
            mx_sn = std::max(mx_sn, need_sn[d]);
        }
        CK(ensure_shared(x, mx_rn, mx_sn, need_rh, s));
        Lrn = x->cap_rn;
        Lsn = x->cap_sn;
        Lrh = x->cap_rh;
        for (uint32_t d = 0; d < G; ++d) {
            dr[2 * d] = addr(x->peer_rn[d], off_rn[d]);
            dr[2 * d + 1] = addr(x->peer_rn[d], Lrn + off_rn[d]);
            ds[2 * d] = addr(x->peer_sn[d], off_sn[d]);
            ds[2 * d + 1] = addr(x->peer_sn[d], Lsn + off_sn[d]);
            dr[2 * (G + d)] = addr(x->peer_rh[d], off_rh_me);          // skewed R: every rank's copy
            dr[2 * (G + d) + 1] = addr(x->peer_rh[d], Lrh + off_rh_me);
            if (d != me) xbytes += 8 * (rc(me, d) + sc(me, d) + rc(me, G));
        }
    } else {
        close_peers(x);   // a2a buffers are private (a later p2p call re-shares)
        Lrn = std::max<uint64_t>(nrn, 1);
        Lsn = std::max<uint64_t>(nsn, 1);
        Lrh = std::max<uint64_t>(nrh, 1);
        CK(ensure(x->rn, Lrn * 8, s));
        CK(ensure(x->sn, Lsn * 8, s));
        CK(ensure(x->rh, Lrh * 8, s));
        uint64_t nrx = 0, nsx = 0;
        for (uint32_t d = 0; d < G; ++d)
            if (d != me) {
                nrx += rc(me, d);
                nsx += sc(me, d);
            }
        CK(ensure(x->rx, std::max<uint64_t>(nrx, 1) * 8, s));
        CK(ensure(x->sx, std::max<uint64_t>(nsx, 1) * 8, s));
        const uint64_t Lrx = std::max<uint64_t>(nrx, 1), Lsx = std::max<uint64_t>(nsx, 1);
        uint64_t orx = 0, osx = 0;
        for (uint32_t d = 0; d < G; ++d) {
            if (d == me) {
                dr[2 * d] = addr(x->rn.p, off_rn[me]);
                dr[2 * d + 1] = addr(x->rn.p, Lrn + off_rn[me]);
                ds[2 * d] = addr(x->sn.p, off_sn[me]);
                ds[2 * d + 1] = addr(x->sn.p, Lsn + off_sn[me]);
            } else {
                dr[2 * d] = addr(x->rx.p, orx);
                dr[2 * d + 1] = addr(x->rx.p, Lrx + orx);
                ds[2 * d] = addr(x->sx.p, osx);
                ds[2 * d + 1] = addr(x->sx.p, Lsx + osx);
                orx += rc(me, d);
                osx += sc(me, d);
            }
        }
        dr[2 * G] = addr(x->rh.p, off_rh_me);
        dr[2 * G + 1] = addr(x->rh.p, Lrh + off_rh_me);
        xbytes = 8 * (nrx + nsx);
        bbytes = 8 * (nrh - rc(me, G));
    }
    ds[2 * G] = addr(shk, 0);
    ds[2 * G + 1] = addr(shp, 0);
    // device copies of the destination tables (+ the scatter cursors) after the control words
    CK(ensure(x->ctl, (2 + 2 * (G + 1) + dr.size() + ds.size() + G + 1) * 8, s, true));
    d_ctl = at<uint64_t>(x->ctl);
    uint64_t* d_dr = d_ctl + 2 + 2 * (G + 1);
    uint64_t* d_ds = d_dr + dr.size();
    uint64_t* d_cur = d_ds + ds.size();
    CK(cuda_status(cudaMemcpyAsync(d_dr, dr.data(), dr.size() * 8, cudaMemcpyHostToDevice, s), "route table"));
    CK(cuda_status(cudaMemcpyAsync(d_ds, ds.data(), ds.size() * 8, cudaMemcpyHostToDevice, s), "route table"));
    const uint32_t copies = exch == GSH_EXCHANGE_P2P ? G : 1;
    CK(gsh_route_scatter(R->keys, R->payloads, R->n, rb, set, sb, d_dr, copies, d_cur, s));
    CK(gsh_route_scatter(S->keys, S->payloads, S->n, rb, set, sb, d_ds, 1, d_cur, s));
    launches += (R->n > 0) + (S->n > 0);
    cudaEventRecord(x->ev[2], s);

    uint32_t* rnk = at<uint32_t>(x->rn);
    uint32_t* snk = at<uint32_t>(x->sn);
    uint32_t* rhk = at<uint32_t>(x->rh);
    gsh_relation Rn{rnk, rnk + Lrn, nrn}, Sn{snk, snk + Lsn, nsn}, Rh{rhk, rhk + Lrh, nrh}, Sh{shk, shp, nsh};
    gsh_config cn, ch;
    if (cfg_in)
        cn = *cfg_in;
    else
        gsh_config_default(&cn);
    cn.route_bits = rb;
    ch = cn;
    ch.route_bits = 0;
    const bool mat = mode == GSH_OUT_MATERIALIZE;
    gsh_output oh{mat ? out->pairs : nullptr, mat ? out->capacity : 0};
    gsh_result& rh_res = res->heavy;
    gsh_result& rn_res = res->normal;
    auto join_heavy = [&]() -> gsh_status {
        if (!(nrh && nsh)) return GSH_OK;
        gsh_status js = ensure(x->wsh, gsh_workspace_bytes(nrh, nsh, &ch), s);
        if (js != GSH_OK) return js;
        return gsh_join(&Rh, &Sh, mode, mat ? &oh : nullptr, x->wsh.p, x->wsh.cap, &ch, s, &rh_res);
    };
    auto join_normal = [&]() -> gsh_status {
        gsh_output on{mat ? out->pairs + 2 * rh_res.written : nullptr, mat ? out->capacity - rh_res.written : 0};
        gsh_status js = ensure(x->wsn, gsh_workspace_bytes(nrn, nsn, &cn), s);
        if (js != GSH_OK) return js;
        return gsh_join(&Rn, &Sn, mode, mat ? &on : nullptr, x->wsn.p, x->wsn.cap, &cn, s, &rn_res);
    };

    std::vector<uint64_t> soff(G, 0), sbytes(G, 0), roff(G, 0), rbytes(G, 0);
    if (exch == GSH_EXCHANGE_P2P) {
        CK(c.barrier(c.ctx, s));   // every peer's stores into this rank's buffers are complete
        cudaEventRecord(x->ev[3], s);
        cudaEventRecord(x->ev[4], s);
        cudaEventRecord(x->ev[5], s);
        CK(join_heavy());
        cudaEventRecord(x->ev[6], s);
        CK(join_normal());
    } else {
        // skewed R: every rank's segment to every rank (in place in rh), on the compute stream
        for (int part = 0; part < 2; ++part) {
            const uint64_t base = part ? Lrh : 0;
            for (uint32_t g = 0; g < G; ++g) {
                soff[g] = 4 * (base + off_rh_me);
                sbytes[g] = g == me ? 0 : 4 * rc(me, G);
                roff[g] = 4 * (base + off_rh[g]);
                rbytes[g] = g == me ? 0 : 4 * rc(g, G);
            }
            CK(c.all_to_all_v(c.ctx, x->rh.p, soff.data(), sbytes.data(), x->rh.p, roff.data(), rbytes.data(), s));
        }
        cudaEventRecord(x->ev[3], s);
        // normal tuples on the exchange stream, beside the skewed-key join
        cudaStreamWaitEvent(x->xs, x->ev[2], 0);
        cudaEventRecord(x->ev[4], x->xs);
        uint64_t nrx = 0, nsx = 0;
        for (uint32_t d = 0; d < G; ++d)
            if (d != me) {
                nrx += rc(me, d);
                nsx += sc(me, d);
            }
        const uint64_t Lr = std::max<uint64_t>(nrx, 1), Ls = std::max<uint64_t>(nsx, 1);
        for (int rel = 0; rel < 2; ++rel) {
            for (int part = 0; part < 2; ++part) {
                uint64_t o = 0;
                for (uint32_t g = 0; g < G; ++g) {
                    const uint64_t cnt_out = g == me ? 0 : (rel ? sc(me, g) : rc(me, g));
                    soff[g] = 4 * ((part ? (rel ? Ls : Lr) : 0) + o);
                    sbytes[g] = 4 * cnt_out;
                    o += cnt_out;
                    const uint64_t cnt_in = g == me ? 0 : (rel ? sc(g, me) : rc(g, me));
                    // source g's run in my receive buffer starts at sum_{g' < g} count(g', me)
                    uint64_t ro = 0;
                    for (uint32_t h = 0; h < g; ++h) ro += rel ? sc(h, me) : rc(h, me);
                    roff[g] = 4 * ((part ? (rel ? Lsn : Lrn) : 0) + ro);
                    rbytes[g] = 4 * cnt_in;
                }
                CK(c.all_to_all_v(c.ctx, rel ? x->sx.p : x->rx.p, soff.data(), sbytes.data(), rel ? x->sn.p : x->rn.p,
                                  roff.data(), rbytes.data(), x->xs));
            }
        }
        cudaEventRecord(x->ev[5], x->xs);
        CK(join_heavy());
        cudaEventRecord(x->ev[6], s);
        cudaStreamWaitEvent(s, x->ev[5], 0);
        CK(join_normal());
    }
    cudaEventRecord(x->ev[7], s);
    launches += rh_res.launches + rn_res.launches;

    // ---- the global result
    uint64_t loc[2] = {rh_res.count + rn_res.count, rh_res.checksum + rn_res.checksum};
    CK(cuda_status(cudaMemcpyAsync(d_ctl, loc, 16, cudaMemcpyHostToDevice, s), "result"));
    CK(c.all_reduce_u64(c.ctx, d_ctl, 2, s));
    CK(cuda_status(cudaMemcpyAsync(loc, d_ctl, 16, cudaMemcpyDeviceToHost, s), "result"));
    cudaEventRecord(x->ev[8], s);
    CK(cuda_status(cudaStreamSynchronize(s), "result"));
    res->count = loc[0];
    res->checksum = loc[1];
    res->written = rh_res.written + rn_res.written;
    res->overflow = rh_res.overflow | rn_res.overflow;
    res->local_r = R->n;
    res->local_s = S->n;
    res->normal_r = nrn;
    res->normal_s = nsn;
    res->heavy_r = nrh;
    res->heavy_s = nsh;
    res->count_normal = rn_res.count;
    res->count_heavy = rh_res.count;
    res->exchange_bytes = xbytes;
    res->broadcast_bytes = bbytes;
    res->launches = launches;
    res->exchange = (uint32_t)exch;
    res->ms_agree = ms_between(x->ev[0], x->ev[1]);
    res->ms_route = ms_between(x->ev[1], x->ev[2]);
    res->ms_exchange = exch == GSH_EXCHANGE_P2P ? ms_between(x->ev[2], x->ev[3]) : ms_between(x->ev[4], x->ev[5]);
    res->ms_join_heavy = ms_between(exch == GSH_EXCHANGE_P2P ? x->ev[5] : x->ev[3], x->ev[6]);
    res->ms_join_normal = ms_between(x->ev[6], x->ev[7]);
    res->ms_reduce = ms_between(x->ev[7], x->ev[8]);
    res->ms_total = ms_between(x->ev[0], x->ev[8]);
    return GSH_OK;
#undef CK
}

}  // namespace

static gsh_status check_and_run(gsh_sharded* ctx, const gsh_relation* R, const gsh_relation* S, gsh_out_mode mode,
                                const gsh_output* out, const gsh_config* cfg, gsh_exchange exchange, void* stream,
                                gsh_sharded_result* res);

extern "C" {

gsh_status gsh_comm_nccl(void* nccl_comm, gsh_comm* out) {
    if (!nccl_comm || !out) return api_fail(GSH_ERR_INVALID, "NULL argument");
    if (!nccl_api().ok) return api_fail(GSH_ERR_NCCL, "libnccl.so.2 not found");
    NcclCtx* c = new (std::nothrow) NcclCtx;
    if (!c) return api_fail(GSH_ERR_NOMEM, "comm");
    c->comm = static_cast<ncclComm_t>(nccl_comm);
    c->owned = false;
    gsh_status st = fill_nccl(c, out);
    if (st != GSH_OK) delete c;
    return st;
}

gsh_status gsh_nccl_unique_id(void* id128) {
    if (!id128) return api_fail(GSH_ERR_INVALID, "NULL argument");
    const NcclApi& a = nccl_api();
    if (!a.ok) return api_fail(GSH_ERR_NCCL, "libnccl.so.2 not found");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    ncclUniqueId id;
    gsh_status st = nccl_status(a.GetUniqueId(&id), "ncclGetUniqueId");
    if (st == GSH_OK) std::memcpy(id128, &id, sizeof(id));
    return st;
}

gsh_status gsh_comm_nccl_init(const void* id128, uint32_t world, uint32_t rank, int device, gsh_comm* out) {
    if (!id128 || !out) return api_fail(GSH_ERR_INVALID, "NULL argument");
    if (world == 0 || rank >= world) return api_fail(GSH_ERR_INVALID, "bad world / rank");
    const NcclApi& a = nccl_api();
    if (!a.ok) return api_fail(GSH_ERR_NCCL, "libnccl.so.2 not found");
    gsh_status st = cuda_status(cudaSetDevice(device), "cudaSetDevice");
    if (st != GSH_OK) return st;
    ncclUniqueId id;
    std::memcpy(&id, id128, sizeof(id));
    NcclCtx* c = new (std::nothrow) NcclCtx;
    if (!c) return api_fail(GSH_ERR_NOMEM, "comm");
    st = nccl_status(a.CommInitRank(&c->comm, (int)world, id, (int)rank), "ncclCommInitRank");
    if (st != GSH_OK) {
        delete c;
        return st;
    }
    c->owned = true;
    st = fill_nccl(c, out);
    if (st != GSH_OK) {
        a.CommDestroy(c->comm);
        delete c;
    }
    return st;
}

gsh_status gsh_comm_destroy(gsh_comm* comm) {
    if (!comm || !comm->ctx) return GSH_OK;
    if (comm->all_reduce_u64 == nccl_all_reduce) {
        NcclCtx* c = static_cast<NcclCtx*>(comm->ctx);
        gsh_status st = GSH_OK;
        if (c->owned) st = nccl_status(nccl_api().CommDestroy(c->comm), "ncclCommDestroy");
        if (c->d_one) cudaFree(c->d_one);
        delete c;
        comm->ctx = nullptr;
        return st;
    }
    comm->ctx = nullptr;   // local world ranks: owned by the world
    return GSH_OK;
}

gsh_status gsh_local_world_create(uint32_t world, void** lw) {
    if (!lw || world == 0 || world > kMaxWorld) return api_fail(GSH_ERR_INVALID, "bad world (1..256) or NULL");
    LocalWorld* w = new (std::nothrow) LocalWorld;
    if (!w) return api_fail(GSH_ERR_NOMEM, "local world");
    w->G = world;
    w->slot.resize(world);
    w->ranks.resize(world);
    for (uint32_t r = 0; r < world; ++r) {
        w->ranks[r].w = w;
        w->ranks[r].rank = r;
    }
    *lw = w;
    return GSH_OK;
}

gsh_status gsh_comm_local(void* lw, uint32_t rank, gsh_comm* out) {
    LocalWorld* w = static_cast<LocalWorld*>(lw);
    if (!w || !out || rank >= w->G) return api_fail(GSH_ERR_INVALID, "NULL world or bad rank");
    std::memset(out, 0, sizeof(*out));
    out->rank = rank;
    out->world = w->G;
    out->same_process = 1;
    out->ctx = &w->ranks[rank];
    out->all_reduce_u64 = local_all_reduce;
    out->all_gather = local_all_gather;
    out->all_to_all_v = local_all_to_all_v;
    out->barrier = local_barrier;
    out->abort = local_abort;
    return GSH_OK;
}

gsh_status gsh_local_world_destroy(void* lw) {
    LocalWorld* w = static_cast<LocalWorld*>(lw);
    if (!w) return GSH_OK;
    for (LocalRank& r : w->ranks)
        if (r.tmp) cudaFree(r.tmp);
    delete w;
    return GSH_OK;
}

gsh_status gsh_sharded_create(const gsh_comm* comm, int device, gsh_sharded** ctx) {
    if (!comm || !ctx) return api_fail(GSH_ERR_INVALID, "NULL argument");
    if (comm->world == 0 || comm->world > kMaxWorld || (comm->world & (comm->world - 1)) || comm->rank >= comm->world)
        return api_fail(GSH_ERR_INVALID, "comm world must be a power of two <= 256, rank < world");
    if (!comm->all_reduce_u64 || !comm->all_gather || !comm->all_to_all_v || !comm->barrier)
        return api_fail(GSH_ERR_INVALID, "comm table incomplete");
    gsh_status st = cuda_status(cudaSetDevice(device), "cudaSetDevice");
    if (st != GSH_OK) return st;
    gsh_sharded* x = new (std::nothrow) gsh_sharded;
    if (!x) return api_fail(GSH_ERR_NOMEM, "driver state");
    x->c = *comm;
    x->dev = device;
    st = cuda_status(cudaStreamCreateWithFlags(&x->xs, cudaStreamNonBlocking), "exchange stream");
    for (int i = 0; i < 10 && st == GSH_OK; ++i) st = cuda_status(cudaEventCreate(&x->ev[i]), "driver events");
    if (st != GSH_OK) {
        gsh_sharded_destroy(x);
        return st;
    }
    *ctx = x;
    return GSH_OK;
}

gsh_status gsh_sharded_destroy(gsh_sharded* x) {
    if (!x) return GSH_OK;
    cudaSetDevice(x->dev);
    close_peers(x);
    for (gsh_sharded::Buf* b : {&x->ctl, &x->hist, &x->hloc, &x->cloc, &x->candws, &x->cand, &x->gathered, &x->agreews, &x->uni, &x->cnt,
                                &x->heavy, &x->set, &x->mat, &x->sh, &x->rx, &x->sx, &x->wsn, &x->wsh, &x->rn, &x->sn,
                                &x->rh})
        release(*b);
    for (cudaEvent_t& e : x->ev)
        if (e) cudaEventDestroy(e);
    if (x->xs) cudaStreamDestroy(x->xs);
    cudaGetLastError();
    delete x;
    return GSH_OK;
}

gsh_status gsh_join_sharded(gsh_sharded* ctx, const gsh_relation* R, const gsh_relation* S, gsh_out_mode mode,
                            const gsh_output* out, const gsh_config* cfg, gsh_exchange exchange, void* stream,
                            gsh_sharded_result* res) {
    if (!ctx) return api_fail(GSH_ERR_INVALID, "NULL argument");
    const gsh_status st = check_and_run(ctx, R, S, mode, out, cfg, exchange, stream, res);
    if (st != GSH_OK && ctx->c.abort) ctx->c.abort(ctx->c.ctx);   // release peers blocked in a collective
    return st;
}

}  // extern "C"

static gsh_status check_and_run(gsh_sharded* ctx, const gsh_relation* R, const gsh_relation* S, gsh_out_mode mode,
                                const gsh_output* out, const gsh_config* cfg, gsh_exchange exchange, void* stream,
                                gsh_sharded_result* res) {
    if (!R || !S || !res) return api_fail(GSH_ERR_INVALID, "NULL argument");
    std::memset(res, 0, sizeof(*res));
    if ((R->n && (!R->keys || !R->payloads)) || (S->n && (!S->keys || !S->payloads)))
        return api_fail(GSH_ERR_INVALID, "NULL relation arrays with n > 0");
    if (mode != GSH_OUT_COUNT && mode != GSH_OUT_MATERIALIZE) return api_fail(GSH_ERR_INVALID, "bad mode");
    if (mode == GSH_OUT_MATERIALIZE && (!out || (out->capacity && !out->pairs)))
        return api_fail(GSH_ERR_INVALID, "MATERIALIZE needs an output buffer");
    if (exchange != GSH_EXCHANGE_A2A && exchange != GSH_EXCHANGE_P2P) return api_fail(GSH_ERR_INVALID, "bad exchange");
    if (cfg && cfg->route_bits) return api_fail(GSH_ERR_INVALID, "cfg->route_bits must be 0 (the driver sets it)");
    if (cfg && cfg->input_side_only) return api_fail(GSH_ERR_INVALID, "input_side_only is a single-GPU hook");
    return run_sharded(ctx, R, S, mode, out, cfg, exchange, (cudaStream_t)stream, res);
}
