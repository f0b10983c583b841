// api.cu -- the C-ABI (include/gsh.h): argument checking, workspace carve-up and the host-side
// phase sequence of GSH (§IV-B) on one CUDA stream.
//
// Host synchronisation points: one after classification (number of large partitions, to size
// detection) and one after skewed-key selection (number of skewed keys, to size the split and
// the tile list); the final one fills gsh_result.  When no partition is large (uniform inputs,
// PAPER.md L166) the detect/split/skew phases are skipped entirely.
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "gsh_device.cuh"
#include "gsh_internal.h"

namespace gsh {
// defined in join.cu
uint32_t nm_table_slots(uint32_t rl);
}  // namespace gsh

using namespace gsh;

namespace {

thread_local std::string g_err;

gsh_status fail(gsh_status s, const std::string& msg) {
    g_err = msg;
    return s;
}

gsh_status cuda_fail(cudaError_t e, const char* where) {
    g_err = std::string(where) + ": " + cudaGetErrorString(e);
    return GSH_ERR_CUDA;
}

int device_sms() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return 148;
    static int cached[64] = {0};
    if (dev >= 0 && dev < 64 && cached[dev]) return cached[dev];
    int sms = 148;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) sms = 148;
    if (dev >= 0 && dev < 64) cached[dev] = sms;
    return sms;
}

uint64_t next_pow2_u64(uint64_t x) {
    uint64_t p = 1;
    while (p < x) p <<= 1;
    return p;
}

size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

struct Carver {
    unsigned char* base;
    size_t off = 0;
    template <class T>
    T* take(size_t count) {
        T* p = base ? reinterpret_cast<T*>(base + off) : nullptr;
        off = align256(off + count * sizeof(T));
        return p;
    }
};

bool validate_rel(const gsh_relation* r) {
    if (!r) return false;
    if (r->n >= (1ull << 32)) return false;
    if (r->n > 0 && (!r->keys || !r->payloads)) return false;
    return true;
}

}  // namespace

namespace gsh {

bool plan_build(Plan& p, uint64_t nR, uint64_t nS, const gsh_config* cfg_in, void* ws, int num_sms) {
    gsh_config cfg;
    gsh_config_default(&cfg);
    if (cfg_in) cfg = *cfg_in;
    p.n[0] = nR;
    p.n[1] = nS;
    p.num_sms = num_sms;
    const uint64_t nmax = nR > nS ? nR : nS;
    if (cfg.route_bits > 16) return false;
    p.route_bits = cfg.route_bits;
    // radix bits: mean partition ~2048 tuples ("shared memory sized partitions")
    if (cfg.pass_bits[0] >= 0 && cfg.pass_bits[1] >= 0) {
        if (cfg.pass_bits[0] > kMaxDigitBits || cfg.pass_bits[1] > kMaxDigitBits) return false;
        p.b1 = (uint32_t)cfg.pass_bits[0];
        p.b2 = (uint32_t)cfg.pass_bits[1];
    } else {
        uint32_t B = 0;
        while (B < (uint32_t)kMaxPartBits && (nmax >> B) > 2048) ++B;
        p.b1 = (B + 1) / 2;
        p.b2 = B / 2;
    }
    if (p.route_bits + p.b1 + p.b2 > 32) return false;
    p.F = 1u << (p.b1 + p.b2);
    // capacity C (power of two): large-partition threshold and NM build-table size (L107, L115)
    if (cfg.capacity) {
        uint64_t c = next_pow2_u64(cfg.capacity);
        if (c < 64 || c > kMaxCapacity) return false;
        p.C = (uint32_t)c;
    } else {
        uint64_t mean = (nmax + p.F - 1) / p.F;
        uint64_t c = next_pow2_u64(2 * mean);
        if (c < 4096) c = 4096;
        if (c > kMaxCapacity) c = kMaxCapacity;
        p.C = (uint32_t)c;
    }
    p.Th = cfg.heavy_threshold ? cfg.heavy_threshold : 64;
    if (cfg.large_threshold) {
        p.L = cfg.large_threshold;
    } else {
        const double mean = double(nmax) / double(p.F);
        uint64_t l = uint64_t(mean + 8.0 * std::sqrt(mean > 1.0 ? mean : 1.0)) + 1;
        p.L = (uint32_t)(l < 64 ? 64 : l);
    }
    p.force_normal = cfg.force_all_normal;
    p.input_only = cfg.input_side_only;
    p.detail = cfg.heavy_detail;
    p.force_heavy = cfg.force_all_heavy;
    p.timing = cfg.timing;
    if (cfg.nm_table < 0 || cfg.nm_table > 2) return false;
    p.nm_table = cfg.nm_table;
    if (cfg.detect_mode < 0 || cfg.detect_mode > 1) return false;
    p.detect_mode = cfg.detect_mode;
    p.sample_stride = cfg.sample_stride ? cfg.sample_stride : 100;
    p.top_k = cfg.top_k ? cfg.top_k : 3;
    if (p.top_k > 32) return false;
    if (p.force_normal && p.force_heavy) return false;
    if (cfg.hybrid < 0 || cfg.hybrid > 1) return false;
    p.hybrid = cfg.hybrid && !p.force_normal && !p.force_heavy;
    p.hyb_stride = cfg.hybrid_stride ? cfg.hybrid_stride : 100;
    p.hyb_min = cfg.hybrid_min ? cfg.hybrid_min : 3;
    if (cfg.hybrid_share > 256) return false;
    p.hyb_share = cfg.hybrid_share ? cfg.hybrid_share : 128;
    p.hist_grid = num_sms;  // one 1024-thread CTA (128 KB of counters) per SM
    uint64_t t = next_pow2_u64(2 * (nR + nS));
    if (t < 1024) t = 1024;
    if (t > (1ull << 25)) t = 1ull << 25;
    p.gt_cap_alloc = (uint32_t)t;
    if (p.force_heavy)
        p.h_max = p.gt_cap_alloc;
    else {
        // exact rule: a skewed key holds >= T_h tuples on one side; sampled rule (detect_mode 1):
        // up to top_k keys per large partition, whatever their counts
        uint64_t hm = (nR + nS) / (p.Th ? p.Th : 1) + 1;
        if (p.detect_mode == 1 && uint64_t(p.F) * p.top_k > hm) hm = uint64_t(p.F) * p.top_k;
        p.h_max = hm < p.gt_cap_alloc ? hm : p.gt_cap_alloc;
    }
    if (p.hybrid) p.h_max += kHybMaxKeys;   // the sampled keys come first in H
    // pass-1 units (= histogram slices): whole 16K-key chunks, about one unit per scatter CTA
    // (2 per SM) and at most kHistMaxUnitChunks chunks.  Pass-2 units: ranges of consecutive
    // slices of one pass-1 partition holding >= T tuples (planned on the device from the
    // histogram, largest partitions first), so a skewed pass-1 partition spreads over many CTAs.
    {
        const uint64_t nch0 = (p.n[0] + kScatterChunk - 1) / kScatterChunk, nch1 = (p.n[1] + kScatterChunk - 1) / kScatterChunk;
        uint64_t uc = (nch0 + nch1 + 2 * uint64_t(num_sms) - 1) / (2 * uint64_t(num_sms));
        if (uc < 1) uc = 1;
        if (uc > kHistMaxUnitChunks) uc = kHistMaxUnitChunks;
        p.unit_chunks = (uint32_t)uc;
        const uint64_t nch[2] = {nch0, nch1};
        for (int s = 0; s < 2; ++s) p.nu1[s] = (uint32_t)((nch[s] + uc - 1) / uc);
        if (p.nu1[0] > 4096 || p.nu1[1] > 4096) return false;   // k_hist_reduce stages <= 4096 slices
        uint64_t T = kGroupTuples >> p.b1;
        const uint64_t bal = (nR + nS) / (uint64_t(num_sms) * 8);   // >= 8 units per SM
        if (bal < T) T = bal;
        if (T < kPass2MinUnit) T = kPass2MinUnit;
        p.u2_target = (uint32_t)T;
        for (int s = 0; s < 2; ++s) p.u2_max[s] = (uint32_t)(p.n[s] / T + (1u << p.b1) + 1);
    }
    uint64_t scan_max = p.F + 1 > p.h_max + 1 ? p.F + 1 : p.h_max + 1;
    for (int s = 0; s < 2; ++s)
        if (uint64_t(p.nu1[s]) * 256 + 1 > scan_max) scan_max = uint64_t(p.nu1[s]) * 256 + 1;
    p.scan_scratch_elems = scan_max / 4096 + 2;
    {   // the histogram's four scans share one launch (launch_scan_u32_multi)
        const uint64_t m4 = (2 * (uint64_t(p.F) + 4095) + (uint64_t(p.nu1[0]) * 256 + 4095) +
                             (uint64_t(p.nu1[1]) * 256 + 4095)) / 4096 + 8;
        if (m4 > p.scan_scratch_elems) p.scan_scratch_elems = m4;
    }
    if (p.hybrid) {   // the hybrid key-major scans (kHybMaxKeys x slices per side)
        const uint64_t m = uint64_t(kHybMaxKeys) * (p.nu1[0] > p.nu1[1] ? p.nu1[0] : p.nu1[1]) + 1;
        if (m / 4096 + 2 > p.scan_scratch_elems) p.scan_scratch_elems = m / 4096 + 2;
    }

    Carver c{reinterpret_cast<unsigned char*>(ws)};
    const size_t F = p.F;
    p.st = c.take<DevState>(1);
    // side S starts 256-byte aligned so sector alignment of partition writes is index alignment
    const uint64_t nRp = (nR + 31) & ~uint64_t(31);
    uint2* a = c.take<uint2>(nRp + nS + 32);
    uint2* b = c.take<uint2>(nRp + nS + 32);
    uint32_t* hp = c.take<uint32_t>(nR + nS + 1);
    p.bufA[0] = a;
    p.bufA[1] = a ? a + nRp : nullptr;
    p.bufB[0] = b;
    p.bufB[1] = b ? b + nRp : nullptr;
    p.heavy_pay[0] = hp;
    p.heavy_pay[1] = hp ? hp + nR : nullptr;
    p.hist_partial = c.take<uint32_t>((size_t(p.nu1[0]) + p.nu1[1] + 1) * F);
    p.off2 = c.take<uint32_t>((size_t(p.u2_max[0]) + p.u2_max[1]) * (size_t(1) << p.b2));
    p.u2_info = c.take<uint4>(size_t(p.u2_max[0]) + p.u2_max[1]);
    p.c1cnt = c.take<uint32_t>((size_t(p.nu1[0]) + p.nu1[1]) * 256 + 1);
    p.slice_dom = c.take<uint32_t>(size_t(p.nu1[0]) + p.nu1[1] + 1);
    p.off1 = c.take<uint64_t>((size_t(p.nu1[0]) + p.nu1[1]) * 256 + 2);
    p.cnt = c.take<uint32_t>(2 * F);
    p.start = c.take<uint64_t>(2 * (F + 1));
    p.gt_key = c.take<unsigned long long>(p.gt_cap_alloc);
    p.gt_cnt = c.take<uint32_t>(size_t(2) * p.gt_cap_alloc);
    p.large_list = c.take<uint32_t>(F);
    p.large_idx = c.take<uint32_t>(F);
    p.part_heavy = c.take<uint32_t>(2 * F);
    p.det_prefix = c.take<uint64_t>(F + 1);
    p.det_prefix2 = c.take<uint64_t>(F + 1);
    p.item_cap = (nR + nS) / kDetectChunk + F + 1;        // bound on split items (any large set)
    p.item_cap2 = (nR + nS) / kDetectItem + F + 1;        // bound on exact-detect items
    p.item_li = c.take<uint32_t>(p.item_cap);
    p.item_li2 = c.take<uint32_t>(p.item_cap2);
    p.nrm_off = c.take<uint64_t>(2 * (F + 1));
    p.nrm_cur = c.take<uint32_t>(2 * F);
    p.H = c.take<HeavyKey>(p.h_max);
    p.h_off = c.take<uint64_t>(2 * (p.h_max + 1));
    p.h_tiles = c.take<uint64_t>(p.h_max + 1);
    p.h_chk = c.take<unsigned long long>(p.detail ? p.h_max : 0);
    p.h_cur = c.take<uint32_t>(2 * p.h_max);
    {   // the split's compact skewed-key table: load <= 1/2 at the list's capacity
        uint64_t hc = next_pow2_u64(2 * p.h_max);
        if (hc < 1024) hc = 1024;
        if (hc > (1ull << 26)) hc = 1ull << 26;
        p.htab_cap = (uint32_t)hc;
        p.htab = c.take<unsigned long long>(hc);
    }
    p.nm = c.take<NmPart>(F);
    p.nm_prefix = c.take<uint64_t>(F + 1);
    p.scan_scratch = c.take<uint64_t>(p.scan_scratch_elems);
    p.hyb_tab = reinterpret_cast<uint32_t*>(c.take<unsigned char>(kHybTabBytes));
    p.hyb_list = c.take<uint32_t>(kHybMaxKeys);
    p.hyb_cnt = c.take<uint32_t>(2 * kHybMaxKeys);
    {
        const size_t hs = p.hybrid ? (size_t(p.nu1[0]) + p.nu1[1]) * kHybMaxKeys : 0;
        p.hyb_slice = c.take<uint32_t>(hs);
        p.hyb_off = c.take<uint64_t>(hs + 2);
        p.hyb_ref = c.take<uint32_t>(p.hybrid ? size_t(p.nu1[0]) + p.nu1[1] : 0);
    }
    p.bytes = c.off;
    return true;
}

// Error helpers for the other C-ABI translation units (shard.cu): same thread-local message.
gsh_status api_fail(gsh_status st, const char* msg) { return fail(st, msg); }
gsh_status api_cuda(const char* where) {
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? GSH_OK : cuda_fail(e, where);
}

// The single-GPU rule's parameters for global sizes (multi-GPU skew agreement, gsh_shard_plan):
// partition bits B = b1 + b2, large-partition threshold L and skewed-key threshold T_h, exactly as
// plan_build derives them for one GPU holding the whole input.
bool shard_plan_params(uint64_t nR, uint64_t nS, const gsh_config* cfg, uint32_t* B, uint32_t* L, uint32_t* Th) {
    Plan p;
    if (!plan_build(p, nR, nS, cfg, nullptr, 148)) return false;
    *B = p.b1 + p.b2;
    *L = p.L;
    *Th = p.Th;
    return true;
}

}  // namespace gsh

namespace {

// Phase timing (gsh_config.timing): events come from a per-thread pool created once, so a timed
// call adds only cudaEventRecord / cudaEventElapsedTime on the host (a call is synchronous, so
// the pool is free again when the next call on this thread starts).
struct Timer {
    bool on;
    cudaStream_t s;
    int used, saved;
    static std::vector<cudaEvent_t>& pool() {
        static thread_local std::vector<cudaEvent_t> p;
        return p;
    }
    static int& top() {   // first free pool slot; nested timers (pre-pass sub-joins) stack above
        static thread_local int t = 0;
        return t;
    }
    explicit Timer(bool enable, cudaStream_t st) : on(enable), s(st), used(top()), saved(top()) {}
    ~Timer() { top() = saved; }
    int mark() {
        if (!on) return -1;
        auto& p = pool();
        if (used == (int)p.size()) {
            cudaEvent_t e;
            if (cudaEventCreate(&e) != cudaSuccess) return -1;
            p.push_back(e);
        }
        cudaEventRecord(p[used], s);
        top() = used + 1;
        return used++;
    }
    float ms(int a, int b) {
        if (!on || a < 0 || b < 0) return 0.f;
        float t = 0.f;
        cudaEventElapsedTime(&t, pool()[a], pool()[b]);
        return t;
    }
};

gsh_status check_launch(const char* where) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, where);
    return GSH_OK;
}

// Runs hist + scan + pass 1 + pass 2.  Returns kernels launched, or -1 after setting g_err.
// Skew detection over the large partitions (L107, L112): exact counts of every key (detect_mode
// 0), or the paper's sample + top-k per partition followed by exact counts of the chosen keys
// (detect_mode 1); then the threshold pass that builds H.
int run_detect(const Plan& p, uint32_t n_large, uint64_t large_tuples, uint32_t gcap, cudaStream_t s) {
    int l = launch_detect_prefix(p, n_large, large_tuples, s);
    if (p.detect_mode == 1) l += launch_sample_topk(p, n_large, gcap, s);
    l += launch_detect(p, n_large, gcap, s);
    l += launch_select(p, gcap, s);
    return l;
}

int run_partition(const Plan& p, const gsh_relation* R, const gsh_relation* S, cudaStream_t s) {
    int l = 0;
    l += launch_hist(p, R->keys, S->keys, s);
    l += launch_hist_reduce_scan(p, s);
    const uint32_t* keys[2] = {R->keys, S->keys};
    const uint32_t* pays[2] = {R->payloads, S->payloads};
    l += launch_scatter(p, 1, keys, pays, s);
    l += launch_scatter(p, 2, nullptr, nullptr, s);
    return l;
}

gsh_status prep(const gsh_relation* R, const gsh_relation* S, void* ws, size_t ws_bytes, const gsh_config* cfg,
                Plan& p) {
    if (!validate_rel(R) || !validate_rel(S)) return fail(GSH_ERR_INVALID, "invalid relation (NULL or n >= 2^32)");
    if (!plan_build(p, R->n, S->n, cfg, nullptr, device_sms()))
        return fail(GSH_ERR_INVALID, "invalid gsh_config");
    if (!ws || (reinterpret_cast<uintptr_t>(ws) & 255u)) return fail(GSH_ERR_INVALID, "workspace NULL or not 256-byte aligned");
    if (ws_bytes < p.bytes) return fail(GSH_ERR_INVALID, "workspace too small");
    plan_build(p, R->n, S->n, cfg, ws, device_sms());
    return GSH_OK;
}

}  // namespace

extern "C" {

void gsh_config_default(gsh_config* cfg) {
    if (!cfg) return;
    std::memset(cfg, 0, sizeof(*cfg));
    cfg->pass_bits[0] = -1;
    cfg->pass_bits[1] = -1;
}

static size_t direct_workspace_bytes(uint64_t n_r, uint64_t n_s, const gsh_config* cfg) {
    Plan p;
    if (!plan_build(p, n_r, n_s, cfg, nullptr, device_sms())) return 0;
    return p.bytes;
}

// Pre-partition pass bits (gsh_config.prepass_bits): auto = enough hash bits that each side's
// sub-problem is <= 2^28 tuples (the two radix passes then keep partitions within the NM ring).
// Returns -1 on a bad value.
static int prepass_bits_for(uint64_t n_r, uint64_t n_s, const gsh_config* cfg) {
    const int32_t want = cfg ? cfg->prepass_bits : 0;
    const uint32_t rb = cfg ? cfg->route_bits : 0;
    if (want < -1 || want > 8) return -1;
    int r = 0;
    if (want > 0) {
        r = want;
    } else if (want == 0) {
        const uint64_t nmax = n_r > n_s ? n_r : n_s;
        while (r < 8 && (nmax >> r) > (1ull << 28)) ++r;
    }
    if (r > 0 && rb + (uint32_t)r > 16) return want > 0 ? -1 : 0;
    return r;
}

// Sub-problem config: the pre-partition bits are consumed like routing bits; no further pre-pass.
static gsh_config sub_config(const gsh_config* cfg, int r) {
    gsh_config c;
    gsh_config_default(&c);
    if (cfg) c = *cfg;
    c.route_bits += (uint32_t)r;
    c.prepass_bits = -1;
    return c;
}

constexpr uint64_t kPrepassAlign = 64;   // tuples (256 B of u32)

struct Prepass {
    size_t sub_ws;        // workspace of one sub-problem's join (sized for the whole input)
    uint32_t* rk; uint32_t* rp; uint32_t* sk; uint32_t* sp;
    uint64_t* counts;     // [2][256]
    uint64_t* offs;       // [2][256]
    uint64_t* cur;        // [2][256]
    uint32_t* tile_cnt[2];   // rb <= 3: per-(bucket, tile) counts, bucket-major
    uint64_t* tpfx[2];       // their exclusive prefix
    uint64_t* scratch;       // scan scratch
    size_t bytes;
};

static Prepass prepass_layout(uint64_t n_r, uint64_t n_s, const gsh_config* sub, unsigned char* base) {
    Prepass q{};
    q.sub_ws = direct_workspace_bytes(n_r, n_s, sub);
    if (!q.sub_ws) return q;
    size_t off = align256(q.sub_ws);
    auto take = [&](size_t bytes) { unsigned char* p = base ? base + off : nullptr; off += align256(bytes); return p; };
    // each sub-problem starts 256-byte aligned (kPrepassAlign tuples): the radix passes' vector
    // and TMA bulk loads then see aligned inputs
    q.rk = reinterpret_cast<uint32_t*>(take((n_r + 256 * kPrepassAlign) * 4));
    q.rp = reinterpret_cast<uint32_t*>(take((n_r + 256 * kPrepassAlign) * 4));
    q.sk = reinterpret_cast<uint32_t*>(take((n_s + 256 * kPrepassAlign) * 4));
    q.sp = reinterpret_cast<uint32_t*>(take((n_s + 256 * kPrepassAlign) * 4));
    q.counts = reinterpret_cast<uint64_t*>(take(2 * 256 * 8));
    q.offs = reinterpret_cast<uint64_t*>(take(2 * 256 * 8));
    q.cur = reinterpret_cast<uint64_t*>(take(2 * 256 * 8));
    const uint64_t nt[2] = {8 * split_tiles(n_r), 8 * split_tiles(n_s)};
    for (int side = 0; side < 2; ++side) {
        q.tile_cnt[side] = reinterpret_cast<uint32_t*>(take(nt[side] * 4));
        q.tpfx[side] = reinterpret_cast<uint64_t*>(take((nt[side] + 1) * 8));
    }
    q.scratch = reinterpret_cast<uint64_t*>(take(((nt[0] > nt[1] ? nt[0] : nt[1]) / 4096 + 8) * 8));
    q.bytes = off;
    return q;
}

size_t gsh_workspace_bytes(uint64_t n_r, uint64_t n_s, const gsh_config* cfg) {
    const int r = prepass_bits_for(n_r, n_s, cfg);
    if (r < 0) return 0;
    if (r == 0) return direct_workspace_bytes(n_r, n_s, cfg);
    const gsh_config sub = sub_config(cfg, r);
    const Prepass q = prepass_layout(n_r, n_s, &sub, nullptr);
    return q.sub_ws ? q.bytes : 0;
}

static gsh_status join_direct(const gsh_relation* R, const gsh_relation* S, gsh_out_mode mode, const gsh_output* out,
                              void* workspace, size_t workspace_bytes, const gsh_config* cfg, void* stream,
                              gsh_result* res) {
    if (!res) return fail(GSH_ERR_INVALID, "res is NULL");
    std::memset(res, 0, sizeof(*res));
    if (mode != GSH_OUT_COUNT && mode != GSH_OUT_MATERIALIZE) return fail(GSH_ERR_INVALID, "bad mode");
    const bool mat = (mode == GSH_OUT_MATERIALIZE);
    if (mat && (!out || (!out->pairs && out->capacity > 0)))
        return fail(GSH_ERR_INVALID, "MATERIALIZE needs an output buffer");
    Plan p;
    gsh_status st = prep(R, S, workspace, workspace_bytes, cfg, p);
    if (st != GSH_OK) return st;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    res->pass_bits[0] = p.b1;
    res->pass_bits[1] = p.b2;
    res->capacity = p.C;
    res->heavy_threshold = p.Th;
    res->large_threshold = p.L;
    if (R->n == 0 || S->n == 0) return GSH_OK;

    uint32_t* pairs = mat ? out->pairs : nullptr;
    const uint64_t cap = mat ? out->capacity : 0;
    Timer tm(p.timing != 0, s);
    int launches = 0;
    cudaMemsetAsync(p.st, 0, sizeof(DevState), s);
    const int e0 = tm.mark();
    int es = e0;
    cudaError_t ce;
    if (p.hybrid) {   // CSH's sampling before partitioning (hybrid.cu): which keys pass 1 routes
        launches += launch_hybrid_sample(p, R->keys, S->keys, s);
        if ((st = check_launch("hybrid sample")) != GSH_OK) return st;
        uint32_t nh0 = 0;
        ce = cudaMemcpyAsync(&nh0, &p.st->n_h0, sizeof(nh0), cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "hybrid sample sync");
        if (nh0 > kHybMaxKeys) return fail(GSH_ERR_INTERNAL, "hybrid key list overflow");
        p.n_h0 = nh0;
        es = tm.mark();
    }
    launches += launch_hist(p, R->keys, S->keys, s);
    launches += launch_hist_reduce_scan(p, s);
    if (p.n_h0) {   // H's first entries with their exact counts; (key, unit) offsets for pass 1
        launches += launch_hybrid_fill(p, s);
        launches += launch_heavy_offsets(p, p.n_h0, s);
    }
    const int e1 = tm.mark();
    {
        const uint32_t* keys[2] = {R->keys, S->keys};
        const uint32_t* pays[2] = {R->payloads, S->payloads};
        launches += launch_scatter(p, 1, keys, pays, s);
    }
    const int e2 = tm.mark();
    launches += launch_scatter(p, 2, nullptr, nullptr, s);
    const int e3 = tm.mark();
    launches += launch_classify(p, s);
    if ((st = check_launch("partition")) != GSH_OK) return st;

    DevState hs;
    ce = cudaMemcpyAsync(&hs, p.st, sizeof(DevState), cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "classify sync");
    if (hs.route_mismatch)
        return fail(GSH_ERR_INVALID, "gsh_config.route_bits: the tuples do not all share the top route_bits of h");
    const uint32_t n_large = hs.n_large;
    uint32_t n_heavy = p.n_h0;   // hybrid keys first; the detection below appends
    p.nm_slots = nm_table_slots(hs.max_rlen < p.C ? (hs.max_rlen ? hs.max_rlen : 1) : p.C);
    int e4 = e3, e5 = e3;
    if (n_large > 0) {
        uint64_t gcap = next_pow2_u64(2 * (hs.large_tuples[0] + hs.large_tuples[1]));
        if (gcap < 1024) gcap = 1024;
        if (gcap > p.gt_cap_alloc) gcap = p.gt_cap_alloc;
        launches += run_detect(p, n_large, hs.large_tuples[0] + hs.large_tuples[1], (uint32_t)gcap, s);
        e4 = tm.mark();
        if ((st = check_launch("detect")) != GSH_OK) return st;
        ce = cudaMemcpyAsync(&hs, p.st, sizeof(DevState), cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "detect sync");
        n_heavy = hs.n_heavy;
        if (hs.heavy_overflow || n_heavy > p.h_max) return fail(GSH_ERR_INTERNAL, "skewed-key list overflow");
        launches += launch_heavy_prefix(p, n_heavy, n_large, s);
        launches += launch_split(p, n_large, n_heavy, s);
        e5 = tm.mark();
    }
    if (p.input_only) {   // measurement hook: stop after the input side
        ce = cudaMemcpyAsync(&hs, p.st, sizeof(DevState), cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "input-side sync");
        res->heavy_tuples_r = hs.heavy_tuples[0];
        res->heavy_tuples_s = hs.heavy_tuples[1];
        res->large_tuples = hs.large_tuples[0] + hs.large_tuples[1];
        res->skew_pairs = hs.skew_pairs;
        res->n_heavy = n_heavy;
        res->n_large = n_large;
        res->detect_overflow = hs.detect_overflow;
        res->launches = (uint32_t)launches;
        res->n_hybrid = p.n_h0;
        if (p.timing) {
            res->ms_sample = tm.ms(e0, es);
            res->ms_hist = tm.ms(es, e1);
            res->ms_pass1 = tm.ms(e1, e2);
            res->ms_pass2 = tm.ms(e2, e3);
            res->ms_detect = n_large ? tm.ms(e3, e4) : 0.f;
            res->ms_split = n_large ? tm.ms(e4, e5) : 0.f;
            res->ms_total = tm.ms(e0, e5);
        }
        return GSH_OK;
    }
    // Chained NM table (L115) when the partition digits fix the top 16 bits of h (the chain link
    // then lives there) and, in auto mode, no partition is large (no duplicated keys that would
    // serialise a chain walk; the CSR table flattens those across the warp).
    p.nm_chain = (p.route_bits + p.b1 + p.b2 >= 16) && p.nm_table != 1 && (p.nm_table == 2 || n_large == 0);
    res->nm_table = p.nm_chain ? 2 : 1;
    if (p.detail && n_heavy) cudaMemsetAsync(p.h_chk, 0, size_t(n_heavy) * 8, s);
    launches += launch_nm_setup(p, n_large, s);
    launches += launch_nmjoin(p, mat ? 1 : 0, pairs, cap, s);
    const int e6 = tm.mark();
    launches += launch_skewjoin(p, n_heavy, mat ? 1 : 0, pairs, cap, s);
    const int e7 = tm.mark();
    if ((st = check_launch("join")) != GSH_OK) return st;
    ce = cudaMemcpyAsync(&hs, p.st, sizeof(DevState), cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "join sync");

    res->count = hs.count + hs.nm_count;
    res->checksum = hs.checksum + hs.nm_checksum;
    res->normal_count = hs.nm_count;
    res->normal_checksum = hs.nm_checksum;
    res->written = mat ? (hs.cursor < cap ? hs.cursor : cap) : 0;
    res->overflow = mat ? (res->count > cap ? 1u : 0u) : 0u;  // items skip reserving once full
    res->heavy_tuples_r = hs.heavy_tuples[0];
    res->heavy_tuples_s = hs.heavy_tuples[1];
    res->large_tuples = hs.large_tuples[0] + hs.large_tuples[1];
    res->skew_pairs = hs.skew_pairs;
    res->n_heavy = n_heavy;
    res->n_large = n_large;
    res->detect_overflow = hs.detect_overflow;
    res->launches = (uint32_t)launches;
    res->n_hybrid = p.n_h0;
    if (p.timing) {
        res->ms_sample = tm.ms(e0, es);
        res->ms_hist = tm.ms(es, e1);
        res->ms_pass1 = tm.ms(e1, e2);
        res->ms_pass2 = tm.ms(e2, e3);
        res->ms_detect = n_large ? tm.ms(e3, e4) : 0.f;
        res->ms_split = n_large ? tm.ms(e4, e5) : 0.f;
        res->ms_nmjoin = tm.ms(e5, e6);
        res->ms_skewjoin = tm.ms(e6, e7);
        res->ms_total = tm.ms(e0, e7);
    }
    return GSH_OK;
}

// gsh_join: the direct path, or (beyond 2^28 tuples per side, or when forced) the pre-partition
// pass -- split R and S by `r` hash bits below route_bits (route.cu k_split_*), then join each
// of the 2^r sub-problems with the direct path.  Matches never cross sub-problems (equal keys,
// equal h); count / checksum add mod 2^64, MATERIALIZE pairs are appended.
gsh_status gsh_join(const gsh_relation* R, const gsh_relation* S, gsh_out_mode mode, const gsh_output* out,
                    void* workspace, size_t workspace_bytes, const gsh_config* cfg, void* stream, gsh_result* res) {
    if (!res) return fail(GSH_ERR_INVALID, "res is NULL");
    std::memset(res, 0, sizeof(*res));
    if (!validate_rel(R) || !validate_rel(S)) return fail(GSH_ERR_INVALID, "invalid relation (NULL or n >= 2^32)");
    const int r = prepass_bits_for(R->n, S->n, cfg);
    if (r < 0) return fail(GSH_ERR_INVALID, "invalid gsh_config (prepass_bits)");
    if (r == 0 || R->n == 0 || S->n == 0)
        return join_direct(R, S, mode, out, workspace, workspace_bytes, cfg, stream, res);
    if (cfg && cfg->heavy_detail) return fail(GSH_ERR_INVALID, "heavy_detail is not available with the pre-partition pass");
    if (mode != GSH_OUT_COUNT && mode != GSH_OUT_MATERIALIZE) return fail(GSH_ERR_INVALID, "bad mode");
    const bool mat = (mode == GSH_OUT_MATERIALIZE);
    if (mat && (!out || (!out->pairs && out->capacity > 0)))
        return fail(GSH_ERR_INVALID, "MATERIALIZE needs an output buffer");
    const gsh_config sub = sub_config(cfg, r);
    if (!workspace || (reinterpret_cast<uintptr_t>(workspace) & 255u))
        return fail(GSH_ERR_INVALID, "workspace NULL or not 256-byte aligned");
    const Prepass q = prepass_layout(R->n, S->n, &sub, reinterpret_cast<unsigned char*>(workspace));
    if (!q.sub_ws) return fail(GSH_ERR_INVALID, "invalid gsh_config");
    if (workspace_bytes < q.bytes) return fail(GSH_ERR_INVALID, "workspace too small");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const bool timing = cfg && cfg->timing;
    Timer tm(timing, s);
    const uint32_t G = 1u << r, skip = sub.route_bits - (uint32_t)r;
    const int e0 = tm.mark();
    cudaError_t ce = cudaMemsetAsync(q.counts, 0, 3 * align256(2 * 256 * 8), s);
    if (ce != cudaSuccess) return cuda_fail(ce, "prepass memset");
    int launches = 0;
    const bool tiled = r <= 3;   // atomic-free register-ranked kernels (G <= 8)
    if (tiled) {
        launches += launch_split_count_tiles(R->keys, R->n, skip, (uint32_t)r, q.tile_cnt[0], q.counts, s);
        launches += launch_split_count_tiles(S->keys, S->n, skip, (uint32_t)r, q.tile_cnt[1], q.counts + 256, s);
        launches += launch_split_tile_scan(q.tile_cnt[0], R->n, (uint32_t)r, q.tpfx[0], q.scratch, s);
        launches += launch_split_tile_scan(q.tile_cnt[1], S->n, (uint32_t)r, q.tpfx[1], q.scratch, s);
    } else {
        launches += launch_split_count(R->keys, R->n, skip, (uint32_t)r, q.counts, s);
        launches += launch_split_count(S->keys, S->n, skip, (uint32_t)r, q.counts + 256, s);
    }
    gsh_status st = check_launch("prepass count");
    if (st != GSH_OK) return st;
    uint64_t hc[512], ho[512];
    ce = cudaMemcpyAsync(hc, q.counts, sizeof(hc), cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "prepass counts");
    for (int side = 0; side < 2; ++side) {
        uint64_t acc = 0, tot = 0;
        for (uint32_t g = 0; g < 256; ++g) {
            ho[side * 256 + g] = acc;
            const uint64_t c = g < G ? hc[side * 256 + g] : 0;
            acc = (acc + c + kPrepassAlign - 1) & ~(kPrepassAlign - 1);
            tot += c;
        }
        if (tot != (side ? S->n : R->n)) return fail(GSH_ERR_INTERNAL, "prepass count mismatch");
    }
    ce = cudaMemcpyAsync(q.offs, ho, sizeof(ho), cudaMemcpyHostToDevice, s);
    if (ce != cudaSuccess) return cuda_fail(ce, "prepass offsets");
    if (tiled) {
        launches += launch_split_scatter_tiles(R->keys, R->payloads, R->n, skip, (uint32_t)r, q.offs, q.tpfx[0],
                                               q.rk, q.rp, s);
        launches += launch_split_scatter_tiles(S->keys, S->payloads, S->n, skip, (uint32_t)r, q.offs + 256,
                                               q.tpfx[1], q.sk, q.sp, s);
    } else {
        launches += launch_split_scatter(R->keys, R->payloads, R->n, skip, (uint32_t)r, q.offs, q.cur, q.rk, q.rp, s);
        launches += launch_split_scatter(S->keys, S->payloads, S->n, skip, (uint32_t)r, q.offs + 256, q.cur + 256,
                                         q.sk, q.sp, s);
    }
    const int e1 = tm.mark();
    if ((st = check_launch("prepass scatter")) != GSH_OK) return st;
    const uint64_t cap = mat ? out->capacity : 0;
    uint64_t written = 0;
    gsh_result acc;
    std::memset(&acc, 0, sizeof(acc));
    for (uint32_t g = 0; g < G; ++g) {
        const gsh_relation sR{q.rk + ho[g], q.rp + ho[g], hc[g]};
        const gsh_relation sS{q.sk + ho[256 + g], q.sp + ho[256 + g], hc[256 + g]};
        gsh_output so{mat && out->pairs ? out->pairs + 2 * written : nullptr, cap - written};
        gsh_result sr;
        st = join_direct(&sR, &sS, mode, mat ? &so : nullptr, workspace, q.sub_ws, &sub, stream, &sr);
        if (st != GSH_OK) return st;
        written += sr.written;
        acc.count += sr.count;
        acc.checksum += sr.checksum;
        acc.normal_count += sr.normal_count;
        acc.normal_checksum += sr.normal_checksum;
        acc.heavy_tuples_r += sr.heavy_tuples_r;
        acc.heavy_tuples_s += sr.heavy_tuples_s;
        acc.skew_pairs += sr.skew_pairs;
        acc.large_tuples += sr.large_tuples;
        acc.n_heavy += sr.n_heavy;
        acc.n_large += sr.n_large;
        acc.n_hybrid += sr.n_hybrid;
        acc.ms_sample += sr.ms_sample;
        acc.detect_overflow |= sr.detect_overflow;
        acc.launches += sr.launches;
        if (sR.n && sS.n) {   // parameters of a non-empty sub-problem
            acc.pass_bits[0] = sr.pass_bits[0];
            acc.pass_bits[1] = sr.pass_bits[1];
            acc.capacity = sr.capacity;
            acc.heavy_threshold = sr.heavy_threshold;
            acc.large_threshold = sr.large_threshold;
            acc.nm_table = sr.nm_table;
        }
        acc.ms_hist += sr.ms_hist;
        acc.ms_pass1 += sr.ms_pass1;
        acc.ms_pass2 += sr.ms_pass2;
        acc.ms_detect += sr.ms_detect;
        acc.ms_split += sr.ms_split;
        acc.ms_nmjoin += sr.ms_nmjoin;
        acc.ms_skewjoin += sr.ms_skewjoin;
    }
    const int e2 = tm.mark();
    acc.written = mat ? written : 0;
    acc.overflow = mat ? (acc.count > cap ? 1u : 0u) : 0u;
    acc.launches += (uint32_t)launches;
    acc.prepass_bits = (uint32_t)r;
    if (timing) {
        ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "prepass timing");
        acc.ms_prepass = tm.ms(e0, e1);
        acc.ms_total = tm.ms(e0, e2);
    }
    *res = acc;
    return GSH_OK;
}

size_t gsh_host_workspace_bytes(uint64_t n_r, uint64_t n_s, gsh_out_mode mode, uint64_t out_capacity,
                                const gsh_config* cfg) {
    size_t w = gsh_workspace_bytes(n_r, n_s, cfg);
    if (!w) return 0;
    w = align256(w);
    w += align256(n_r * 4) * 2 + align256(n_s * 4) * 2;
    if (mode == GSH_OUT_MATERIALIZE) w += align256(out_capacity * 8);
    return w;
}

gsh_status gsh_join_host(const gsh_relation* R, const gsh_relation* S, gsh_out_mode mode, const gsh_output* out,
                         void* workspace, size_t workspace_bytes, const gsh_config* cfg, void* stream,
                         gsh_result* res) {
    if (!res) return fail(GSH_ERR_INVALID, "res is NULL");
    std::memset(res, 0, sizeof(*res));
    if (!validate_rel(R) || !validate_rel(S)) return fail(GSH_ERR_INVALID, "invalid relation");
    const bool mat = (mode == GSH_OUT_MATERIALIZE);
    if (mat && (!out || (!out->pairs && out->capacity > 0)))
        return fail(GSH_ERR_INVALID, "MATERIALIZE needs an output buffer");
    const uint64_t cap = mat ? out->capacity : 0;
    const size_t need = gsh_host_workspace_bytes(R->n, S->n, mode, cap, cfg);
    if (!need) return fail(GSH_ERR_INVALID, "invalid gsh_config");
    if (!workspace || workspace_bytes < need || (reinterpret_cast<uintptr_t>(workspace) & 255u))
        return fail(GSH_ERR_INVALID, "workspace NULL, misaligned or too small");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const size_t jw = align256(gsh_workspace_bytes(R->n, S->n, cfg));
    unsigned char* base = reinterpret_cast<unsigned char*>(workspace);
    size_t off = jw;
    uint32_t* rk = reinterpret_cast<uint32_t*>(base + off); off += align256(R->n * 4);
    uint32_t* rp = reinterpret_cast<uint32_t*>(base + off); off += align256(R->n * 4);
    uint32_t* sk = reinterpret_cast<uint32_t*>(base + off); off += align256(S->n * 4);
    uint32_t* sp = reinterpret_cast<uint32_t*>(base + off); off += align256(S->n * 4);
    uint32_t* dp = mat ? reinterpret_cast<uint32_t*>(base + off) : nullptr;
    cudaError_t ce = cudaSuccess;
    if (R->n) {
        ce = cudaMemcpyAsync(rk, R->keys, R->n * 4, cudaMemcpyHostToDevice, s);
        if (ce == cudaSuccess) ce = cudaMemcpyAsync(rp, R->payloads, R->n * 4, cudaMemcpyHostToDevice, s);
    }
    if (ce == cudaSuccess && S->n) {
        ce = cudaMemcpyAsync(sk, S->keys, S->n * 4, cudaMemcpyHostToDevice, s);
        if (ce == cudaSuccess) ce = cudaMemcpyAsync(sp, S->payloads, S->n * 4, cudaMemcpyHostToDevice, s);
    }
    if (ce != cudaSuccess) return cuda_fail(ce, "H2D");
    gsh_relation dR{rk, rp, R->n}, dS{sk, sp, S->n};
    gsh_output dout{dp, cap};
    gsh_status st = gsh_join(&dR, &dS, mode, mat ? &dout : nullptr, workspace, jw, cfg, stream, res);
    if (st != GSH_OK) return st;
    if (mat && res->written) {
        ce = cudaMemcpyAsync(out->pairs, dp, res->written * 8, cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "D2H");
    }
    return GSH_OK;
}

gsh_status gsh_heavy_detail(uint64_t n_r, uint64_t n_s, const gsh_config* cfg, void* workspace, size_t workspace_bytes,
                            void* stream, uint32_t* h_keys, uint32_t* h_cnt_r, uint32_t* h_cnt_s, uint64_t* h_chk,
                            uint64_t cap, uint64_t* h_n) {
    if (!cfg || !cfg->heavy_detail || !h_n || (cap && (!h_keys || !h_cnt_r || !h_cnt_s || !h_chk)))
        return fail(GSH_ERR_INVALID, "heavy_detail config and output arrays required");
    if (prepass_bits_for(n_r, n_s, cfg) > 0) return fail(GSH_ERR_INVALID, "heavy_detail: pre-partition pass active");
    Plan p;
    if (!plan_build(p, n_r, n_s, cfg, nullptr, device_sms())) return fail(GSH_ERR_INVALID, "invalid gsh_config");
    if (!workspace || workspace_bytes < p.bytes || (reinterpret_cast<uintptr_t>(workspace) & 255u))
        return fail(GSH_ERR_INVALID, "workspace NULL, misaligned or too small");
    plan_build(p, n_r, n_s, cfg, workspace, device_sms());
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    DevState hs;
    cudaError_t ce = cudaMemcpyAsync(&hs, p.st, sizeof(DevState), cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "detail sync");
    const uint32_t nh = hs.n_heavy;   // hybrid keys (gsh_config.hybrid) + detected ones
    *h_n = nh;
    if (nh > cap) return fail(GSH_ERR_INVALID, "capacity too small (see *h_n)");
    if (nh) {
        std::vector<HeavyKey> hk(nh);
        std::vector<unsigned long long> ck(nh);
        ce = cudaMemcpyAsync(hk.data(), p.H, nh * sizeof(HeavyKey), cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaMemcpyAsync(ck.data(), p.h_chk, nh * 8, cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "detail copy");
        for (uint32_t i = 0; i < nh; ++i) {
            h_keys[i] = hk[i].h;
            h_cnt_r[i] = hk[i].cnt_r;
            h_cnt_s[i] = hk[i].cnt_s;
            h_chk[i] = ck[i];
        }
    }
    return GSH_OK;
}

gsh_status gsh_hash_keys(const uint32_t* d_keys, uint32_t* d_out, uint64_t n, void* stream) {
    if (n && (!d_keys || !d_out)) return fail(GSH_ERR_INVALID, "NULL pointer");
    launch_hash(d_keys, d_out, n, reinterpret_cast<cudaStream_t>(stream));
    return check_launch("hash");
}

gsh_status gsh_radix_histogram(const uint32_t* d_keys, uint64_t n, uint32_t hi_bits, uint32_t nbits,
                               uint64_t* d_hist, void* workspace, size_t workspace_bytes, void* stream) {
    (void)workspace;
    (void)workspace_bytes;
    if (nbits > 16 || hi_bits + nbits > 32) return fail(GSH_ERR_INVALID, "bad bit range");
    if (n && (!d_keys || !d_hist)) return fail(GSH_ERR_INVALID, "NULL pointer");
    launch_radix_hist(d_keys, n, hi_bits, nbits, d_hist, reinterpret_cast<cudaStream_t>(stream));
    return check_launch("radix_histogram");
}

gsh_status gsh_partition(const gsh_relation* R, const gsh_relation* S, const gsh_config* cfg, void* workspace,
                         size_t workspace_bytes, void* stream, uint32_t* d_part_r, uint32_t* d_part_s,
                         uint64_t* d_off_r, uint64_t* d_off_s, uint32_t* h_bits) {
    Plan p;
    gsh_status st = prep(R, S, workspace, workspace_bytes, cfg, p);
    if (st != GSH_OK) return st;
    if ((R->n && !d_part_r) || (S->n && !d_part_s) || !d_off_r || !d_off_s || !h_bits)
        return fail(GSH_ERR_INVALID, "NULL output");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    cudaMemsetAsync(p.st, 0, sizeof(DevState), s);
    run_partition(p, R, S, s);
    if ((st = check_launch("partition")) != GSH_OK) return st;
    if (R->n) cudaMemcpyAsync(d_part_r, p.bufB[0], R->n * 8, cudaMemcpyDeviceToDevice, s);
    if (S->n) cudaMemcpyAsync(d_part_s, p.bufB[1], S->n * 8, cudaMemcpyDeviceToDevice, s);
    cudaMemcpyAsync(d_off_r, p.start, (p.F + 1) * 8, cudaMemcpyDeviceToDevice, s);
    cudaMemcpyAsync(d_off_s, p.start + (p.F + 1), (p.F + 1) * 8, cudaMemcpyDeviceToDevice, s);
    cudaError_t ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "partition sync");
    h_bits[0] = p.b1;
    h_bits[1] = p.b2;
    return GSH_OK;
}

gsh_status gsh_detect(const gsh_relation* R, const gsh_relation* S, const gsh_config* cfg, void* workspace,
                      size_t workspace_bytes, void* stream, uint32_t* h_keys, uint32_t* h_cnt_r, uint32_t* h_cnt_s,
                      uint64_t cap, uint64_t* h_n, gsh_result* res) {
    Plan p;
    gsh_status st = prep(R, S, workspace, workspace_bytes, cfg, p);
    if (st != GSH_OK) return st;
    if (!h_n || (cap && (!h_keys || !h_cnt_r || !h_cnt_s))) return fail(GSH_ERR_INVALID, "NULL output");
    if (res) std::memset(res, 0, sizeof(*res));
    *h_n = 0;
    if (R->n == 0 || S->n == 0) return GSH_OK;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    cudaMemsetAsync(p.st, 0, sizeof(DevState), s);
    run_partition(p, R, S, s);
    launch_classify(p, s);
    if ((st = check_launch("partition")) != GSH_OK) return st;
    DevState hs;
    cudaError_t ce = cudaMemcpyAsync(&hs, p.st, sizeof(DevState), cudaMemcpyDeviceToHost, s);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
    if (ce != cudaSuccess) return cuda_fail(ce, "classify sync");
    if (hs.n_large) {
        uint64_t gcap = next_pow2_u64(2 * (hs.large_tuples[0] + hs.large_tuples[1]));
        if (gcap < 1024) gcap = 1024;
        if (gcap > p.gt_cap_alloc) gcap = p.gt_cap_alloc;
        run_detect(p, hs.n_large, hs.large_tuples[0] + hs.large_tuples[1], (uint32_t)gcap, s);
        if ((st = check_launch("detect")) != GSH_OK) return st;
        ce = cudaMemcpyAsync(&hs, p.st, sizeof(DevState), cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "detect sync");
        if (hs.heavy_overflow || hs.n_heavy > p.h_max) return fail(GSH_ERR_INTERNAL, "skewed-key list overflow");
    }
    if (res) {
        res->n_large = hs.n_large;
        res->n_heavy = hs.n_heavy;
        res->detect_overflow = hs.detect_overflow;
        res->pass_bits[0] = p.b1;
        res->pass_bits[1] = p.b2;
        res->capacity = p.C;
        res->heavy_threshold = p.Th;
        res->large_threshold = p.L;
        res->heavy_tuples_r = hs.heavy_tuples[0];
        res->heavy_tuples_s = hs.heavy_tuples[1];
        res->skew_pairs = hs.skew_pairs;
    }
    *h_n = hs.n_heavy;
    if (hs.n_heavy > cap) return fail(GSH_ERR_INVALID, "h_keys capacity too small");
    if (hs.n_heavy) {
        std::vector<HeavyKey> hk(hs.n_heavy);
        ce = cudaMemcpyAsync(hk.data(), p.H, hs.n_heavy * sizeof(HeavyKey), cudaMemcpyDeviceToHost, s);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) return cuda_fail(ce, "heavy copy");
        for (uint32_t i = 0; i < hs.n_heavy; ++i) {
            h_keys[i] = hk[i].h;
            h_cnt_r[i] = hk[i].cnt_r;
            h_cnt_s[i] = hk[i].cnt_s;
        }
    }
    return GSH_OK;
}

const char* gsh_status_string(gsh_status s) {
    switch (s) {
        case GSH_OK: return "GSH_OK";
        case GSH_ERR_INVALID: return "GSH_ERR_INVALID";
        case GSH_ERR_NOMEM: return "GSH_ERR_NOMEM";
        case GSH_ERR_CUDA: return "GSH_ERR_CUDA";
        case GSH_ERR_NCCL: return "GSH_ERR_NCCL";
        case GSH_ERR_INTERNAL: return "GSH_ERR_INTERNAL";
    }
    return "GSH_UNKNOWN";
}

const char* gsh_last_error(void) { return g_err.c_str(); }

int gsh_version(void) { return 1; }

int gsh_compiled_arch(void) { return 100; }

}  // extern "C"
