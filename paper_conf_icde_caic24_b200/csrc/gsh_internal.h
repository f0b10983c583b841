// gsh_internal.h -- host-side plan, workspace layout and kernel launchers (not part of the ABI).
#pragma once
#include <cstddef>
#include <cstdint>
#include <mutex>
#include <cuda_runtime.h>

#include "../../include/gsh.h"

namespace gsh {

// ----------------------------------------------------------------- fixed shapes --
#ifndef GSH_SCATTER_BLOCK
#define GSH_SCATTER_BLOCK 512
#endif
#ifndef GSH_SCATTER_IPT
#define GSH_SCATTER_IPT 12
#endif
constexpr int kScatterBlock = GSH_SCATTER_BLOCK;  // threads per partition-scatter CTA
constexpr int kScatterIpt = GSH_SCATTER_IPT;      // tuples per thread per tile
#ifndef GSH_SCATTER_IPT1
#define GSH_SCATTER_IPT1 20
#endif
constexpr int kScatterIpt1 = GSH_SCATTER_IPT1;    // pass 1: tuples per thread per tile
#ifndef GSH_SCATTER_BLOCK2
#define GSH_SCATTER_BLOCK2 448
#endif
constexpr int kScatterBlock2 = GSH_SCATTER_BLOCK2;  // pass 2: threads per CTA (tuples per thread: kScatterIpt)
constexpr int kScatterTile = kScatterBlock * kScatterIpt;  // TMA-store experiment tile
constexpr int kScatterChunk = 16384;               // keys: the histogram's load granule (unit lengths are multiples)
#ifndef GSH_SCATTER_BLOCK1
#define GSH_SCATTER_BLOCK1 256
#endif
constexpr int kScatterBlock1 = GSH_SCATTER_BLOCK1;  // pass 1: threads per CTA
#ifndef GSH_SCATTER_MINB
#define GSH_SCATTER_MINB 2
#endif
constexpr int kScatterMinBlocks = GSH_SCATTER_MINB;  // resident scatter CTAs per SM the register budget targets
static_assert(kScatterIpt1 % 4 == 0 && kScatterIpt % 2 == 0, "vector tile loads: uint4 = 4 keys / 2 tuples");
static_assert(kScatterBlock1 >= 256 && kScatterBlock2 >= 256 && kScatterBlock >= 256,
              "scatter CTAs keep one thread per bucket (2^kMaxDigitBits = 256)");
constexpr uint32_t kHistMaxUnitChunks = 64;      // a pass-1 unit (= histogram slice) is <= 64 chunks = 2^20 tuples
constexpr uint32_t kGroupTuples = 1u << 23;       // pass-2 unit target = kGroupTuples >> b1 (32K at b1 = 8)
constexpr uint32_t kPass2MinUnit = 4096;          // smallest pass-2 unit target (tuples)
constexpr int kMaxDigitBits = 8;                // radix bits per pass (256 buckets)
constexpr int kMaxPartBits = 16;                // b1 + b2 <= 16 (65536 partitions)
constexpr int kHistBlock = 1024;
constexpr int kNmBlock = 256;                   // NM-join CTA
constexpr uint32_t kMaxCapacity = 8192;         // largest NM build table (tuples)
constexpr uint32_t kNmSlice = 8192;             // S tuples probed per NM work item
// Streamed NM-join (nm_ring.cu): one producer warp + kRingGroups consumer groups of
// kRingGroupWarps warps; partition pairs staged by TMA in a shared-memory byte ring.
#ifndef GSH_RING_GROUPS
#define GSH_RING_GROUPS 2
#endif
#ifndef GSH_RING_GROUP_WARPS
#define GSH_RING_GROUP_WARPS 15
#endif
#ifndef GSH_RING_KB
#define GSH_RING_KB (kRingGroups == 1 ? 192u : 160u)
#endif
constexpr int kRingGroups = GSH_RING_GROUPS;
constexpr int kRingGroupWarps = GSH_RING_GROUP_WARPS;
constexpr int kRingThreads = 32 + kRingGroups * kRingGroupWarps * 32;
constexpr uint32_t kRingMaxR = 4096;            // largest staged R side = most CSR buckets
constexpr uint32_t kRingSeBytes = kRingGroups * 2 * kRingMaxR * 4;  // bucket (start, end) tables
constexpr uint32_t kRingBytes = GSH_RING_KB * 1024u;
// An item (R_p and S_p spans, 16-byte aligned) must fit the empty ring (every resident item is
// being joined or queued behind one that is, so the producer only ever waits for progress);
// half the ring keeps at least two in flight.
constexpr uint32_t kRingItemMax = kRingBytes / 2;
// The chained table (links are 16-bit byte offsets) stages R sides up to kRingMaxRChain tuples;
// the CSR table (packed-u16 bucket words) up to kRingMaxR.
constexpr uint32_t kRingMaxRChain = 8190;
__host__ __device__ __forceinline__ bool ring_eligible(uint32_t rl, uint32_t sl, bool chain) {
    return rl > 0 && sl > 0 && rl <= (chain ? kRingMaxRChain : kRingMaxR) &&
           (uint64_t(rl) + sl) * 8 + 32 + 48 <= kRingItemMax;   // + alignment + per-item slack
}
constexpr int kSkewBlock = 256;                 // skewed-key join CTA
constexpr int kSkewSpt = 4;                     // S payloads per thread (registers)
constexpr int kSkewTileS = kSkewBlock * kSkewSpt;  // 1024
constexpr int kSkewTileR = 64;                  // R payloads per tile (shared memory)
#ifndef GSH_SKEWSPLIT_BLOCK
#define GSH_SKEWSPLIT_BLOCK 256
#endif
constexpr int kSkewSplitBlock = GSH_SKEWSPLIT_BLOCK;   // split CTA (8 tuples per thread in registers)
constexpr uint32_t kDetectChunk = 8 * kSkewSplitBlock;   // tuples per split (and sampled-detect) work item
constexpr uint32_t kDetectItem = 16384;         // tuples per exact-detect work item
constexpr uint32_t kNoHeavy = 0xffffffffu;
constexpr int kDetectMaxProbe = 64;   // a full table degrades to "normal", never to a long probe
// Hybrid partition (gsh_config.hybrid, hybrid.cu): at most kHybMaxKeys sampled skewed keys, looked
// up in a kHybSlots-slot shared-memory copy of the table: u32 h per slot (kHybEmpty = empty; a key
// whose h is kHybEmpty is never chosen), then u16 key ids; load <= 1/4, so a miss usually ends at
// its first slot.
constexpr uint32_t kHybMaxKeys = 512;
constexpr uint32_t kHybSlots = 2048;
constexpr uint32_t kHybLogSlots = 11;
constexpr uint32_t kHybEmpty = 0xffffffffu;
constexpr size_t kHybTabBytes = size_t(kHybSlots) * 6;   // keys, then ids
constexpr int kScatterIptHyb = 16;               // pass-1 tile with the hybrid tables (two CTAs per SM)

// Device-resident counters and accumulators, zeroed once per call.
struct DevState {
    unsigned long long count, checksum, cursor;    // result accumulators (all phases)
    unsigned long long nm_count, nm_checksum;      // NM-join share
    unsigned long long large_tuples[2];            // tuples in large partitions (R, S)
    unsigned long long heavy_tuples[2];            // tuples of skewed keys (R, S)
    unsigned long long skew_pairs;                 // sum |R_k| |S_k|
    unsigned long long skew_tiles;                 // total dense tiles
    unsigned long long nm_items;                   // NM work items
    unsigned long long skew_claim;                 // tile claim counter
    unsigned int n_large, n_heavy, detect_overflow, max_rlen;  // max_rlen: largest |R_p| with |S_p| > 0
    unsigned int claim[8];                         // per-kernel work claim counters
    unsigned int route_mismatch;                   // route_bits > 0: tuples differ in the top route bits
    unsigned int u2_front, u2_back;                // pass-2 units at the front / back of the list
    unsigned int heavy_overflow;                   // more skewed keys than the list H holds
    unsigned int n_h0;                             // hybrid: sampled skewed keys selected
    unsigned int hyb_bins[33];                     // hybrid: sampled keys per floor(log2 count)
    unsigned long long hyb_mass[33];               // hybrid: their summed sample counts
};

// Per-(call site, device) one-time setup (kernel attributes): concurrent host threads wait until
// it has run; a process driving several devices runs it once on each.
constexpr int kMaxDevices = 64;
template <class Fn>
inline void once_per_device(std::once_flag (&flags)[kMaxDevices], Fn&& fn) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) {
        fn();
        return;
    }
    std::call_once(flags[dev], fn);
}

// Skewed-key side list entry H[k].
struct HeavyKey {
    uint32_t h, cnt_r, cnt_s, part;
};

// NM-join descriptor of one partition pair after the split (normal tuples only).
struct NmPart {
    const uint2* r;
    const uint2* s;
    uint32_t rlen, slen;
};

struct Plan {
    // sizes and parameters
    uint64_t n[2] = {0, 0};
    uint32_t b1 = 0, b2 = 0, route_bits = 0;
    uint32_t C = 4096, Th = 64, L = 4096;  // NM capacity, skew-key threshold, large-partition threshold
    uint32_t nm_slots = 0;          // NM build-table slots (set after classification; 0 = from C)
    uint32_t F = 1;                 // 1 << (b1 + b2)
    int force_normal = 0, force_heavy = 0, timing = 0, input_only = 0, detail = 0;
    int nm_table = 0;               // config: 0 auto, 1 CSR, 2 chained where possible
    int nm_chain = 0;               // chosen for this call (nm_ring.cu)
    int detect_mode = 0;            // 0 exact counts, 1 sampled top-k (L107, L112)
    uint32_t sample_stride = 100, top_k = 3;
    int hybrid = 0;                 // CSH-style hybrid partition (hybrid.cu)
    uint32_t hyb_stride = 100, hyb_min = 3, hyb_share = 128;
    uint32_t n_h0 = 0;              // hybrid keys selected (host copy, set after the sample)
    int num_sms = 148;
    int hist_grid = 148;            // histogram CTAs (1 per SM)
    uint32_t unit_chunks = 1;       // chunks per pass-1 unit (= histogram slice)
    uint32_t u2_target = 0;         // pass-2 unit size target T (tuples): units = slice ranges of a
                                    // pass-1 partition holding >= T tuples (the last one: any)
    uint32_t u2_max[2] = {0, 0};    // bound on pass-2 units per side: n / T + 2^b1 + 1
    uint32_t gt_cap_alloc = 0;      // detection table slots allocated
    uint64_t h_max = 0;             // skewed-key list capacity
    uint64_t scan_scratch_elems = 0;

    // workspace carve-up (device pointers)
    uint2* bufA[2] = {nullptr, nullptr};      // pass-1 output, later normal remainders
    uint2* bufB[2] = {nullptr, nullptr};      // final partitions
    uint32_t* heavy_pay[2] = {nullptr, nullptr};  // skewed-key payload arrays
    uint32_t* hist_partial = nullptr;         // [nu1[0] + nu1[1]][F] joint counts per pass-1 unit
    uint32_t nu1[2] = {0, 0};                 // pass-1 units per side
    uint32_t* c1cnt = nullptr;                // per side [256][nu1] pass-1 digit counts per unit
    uint32_t* slice_dom = nullptr;            // [nu1[0] + nu1[1]] dominant pass-1 digit per unit or ~0
    uint64_t* off1 = nullptr;                 // per side [256 * nu1 + 1] unit/bucket output offsets
    uint32_t* cnt = nullptr;                  // [2][F]
    uint64_t* start = nullptr;                // [2][F + 1]
    uint32_t* off2 = nullptr;                 // [u2_max[0] + u2_max[1]][2^b2] pass-2 unit offsets in
                                              // their final partitions (relative to its start)
    uint4* u2_info = nullptr;                 // [u2_max[0] + u2_max[1]] pass-2 units: (side << 8 | d1,
                                              // first slice, end slice, -); large rows' units at the front
    DevState* st = nullptr;
    unsigned long long* gt_key = nullptr;     // [gt_cap_alloc]  (1 << 32 | h), 0 = empty
    uint32_t* gt_cnt = nullptr;               // [2][gt_cap_alloc]
    uint32_t* large_list = nullptr;           // [F]
    uint32_t* large_idx = nullptr;            // [F] partition -> large index or kNoHeavy
    uint32_t* part_heavy = nullptr;           // [2][F]  skewed tuples per partition
    uint64_t* det_prefix = nullptr;           // [F + 1] split (and sampled-detect) items per large partition
    uint64_t* det_prefix2 = nullptr;          // [F + 1] exact-detect items per large partition
    uint32_t* item_li = nullptr;              // [item_cap]  split item -> large partition index
    uint32_t* item_li2 = nullptr;             // [item_cap2] exact-detect item -> large partition index
    uint64_t item_cap = 0, item_cap2 = 0;
    uint64_t* nrm_off = nullptr;              // [2][F + 1] normal remainder offsets (large idx)
    HeavyKey* H = nullptr;                    // [h_max]
    uint64_t* h_off = nullptr;                // [2][h_max + 1]
    uint64_t* h_tiles = nullptr;              // [h_max + 1]
    unsigned long long* h_chk = nullptr;      // [h_max] per skewed key checksum share (heavy_detail)
    uint32_t* h_cur = nullptr;                // [2][h_max] split cursors
    unsigned long long* htab = nullptr;       // [htab_cap] compact skewed-key table for the split:
                                              // (hid + 1) << 32 | h, 0 = empty (L2-resident size)
    uint32_t htab_cap = 0;
    uint32_t* nrm_cur = nullptr;              // [2][F]     split cursors (normal)
    NmPart* nm = nullptr;                     // [F]
    uint64_t* nm_prefix = nullptr;            // [F + 1]
    uint64_t* scan_scratch = nullptr;         // block sums for the generic scan
    uint32_t* hyb_tab = nullptr;              // hybrid lookup table: u32 h [kHybSlots], u16 id [kHybSlots]
    uint32_t* hyb_list = nullptr;             // [kHybMaxKeys] h of hybrid key hid
    uint32_t* hyb_cnt = nullptr;              // [2][kHybMaxKeys] exact counts (histogram pass)
    uint32_t* hyb_slice = nullptr;            // [nu1[0] + nu1[1]][kHybMaxKeys] counts per histogram slice
    uint64_t* hyb_off = nullptr;              // per side [kHybMaxKeys][nu1]: pass-1 unit's write offset
                                              // in heavy_pay (key-major scan of hyb_slice)
    uint32_t* hyb_ref = nullptr;              // [nu1[0] + nu1[1]] the slice's most frequent hybrid key or ~0
    size_t bytes = 0;
};

// Computes parameters and carves `ws` (may be nullptr to only size it).  Returns false on
// invalid configuration.
bool plan_build(Plan& p, uint64_t nR, uint64_t nS, const gsh_config* cfg, void* ws, int num_sms);
gsh_status api_fail(gsh_status st, const char* msg);   // api.cu: sets the thread-local message

// ------------------------------------------------------------------ launchers --
// Every launcher enqueues on `s` and returns the number of kernels it launched.
int launch_hash(const uint32_t* keys, uint32_t* out, uint64_t n, cudaStream_t s);
int launch_hist(const Plan& p, const uint32_t* k0, const uint32_t* k1, cudaStream_t s);
int launch_hist_reduce_scan(const Plan& p, cudaStream_t s);
int launch_scatter(const Plan& p, int pass, const uint32_t* const keys[2], const uint32_t* const pays[2],
                   cudaStream_t s);
int launch_classify(const Plan& p, cudaStream_t s);
int launch_detect_prefix(const Plan& p, uint32_t n_large, uint64_t large_tuples, cudaStream_t s);
int launch_detect(const Plan& p, uint32_t n_large, uint32_t gt_cap, cudaStream_t s);
int launch_sample_topk(const Plan& p, uint32_t n_large, uint32_t gt_cap, cudaStream_t s);
int launch_select(const Plan& p, uint32_t gt_cap, cudaStream_t s);
int launch_heavy_prefix(const Plan& p, uint32_t n_heavy, uint32_t n_large, cudaStream_t s);
int launch_heavy_offsets(const Plan& p, uint32_t n_heavy, cudaStream_t s);   // h_off / h_tiles only
// hybrid.cu: sample + select (n_h0 and hyb_tab on the device), then after the histogram pass the
// first n_h0 entries of H with their exact counts
int launch_hybrid_sample(const Plan& p, const uint32_t* k0, const uint32_t* k1, cudaStream_t s);
int launch_hybrid_fill(const Plan& p, cudaStream_t s);   // + the per-(key, unit) offsets
int launch_split(const Plan& p, uint32_t n_large, uint32_t n_heavy, cudaStream_t s);
int launch_nm_setup(const Plan& p, uint32_t n_large, cudaStream_t s);
int launch_nmjoin(const Plan& p, int materialize, uint32_t* pairs, uint64_t cap, cudaStream_t s);
int launch_nmjoin_ring(const Plan& p, int materialize, uint32_t* pairs, uint64_t cap, cudaStream_t s);
int launch_skewjoin(const Plan& p, uint32_t n_heavy, int materialize, uint32_t* pairs, uint64_t cap,
                    cudaStream_t s);   // p.detail: also per-key checksum shares into p.h_chk

// Routing (multi-GPU)
int launch_route_count(const uint32_t* keys, uint64_t n, uint32_t rb, const uint32_t* hk, uint64_t nh,
                       uint64_t* counts, cudaStream_t s);
int launch_route_scatter(const uint32_t* keys, const uint32_t* pays, uint64_t n, uint32_t rb,
                         const uint32_t* hk, uint64_t nh, const uint64_t* off, uint64_t* cur,
                         uint32_t* ok, uint32_t* op, cudaStream_t s);
int launch_split_count(const uint32_t* keys, uint64_t n, uint32_t skip, uint32_t rb, uint64_t* counts,
                       cudaStream_t s);
int launch_split_scatter(const uint32_t* keys, const uint32_t* pays, uint64_t n, uint32_t skip, uint32_t rb,
                         const uint64_t* off, uint64_t* cur, uint32_t* ok, uint32_t* op, cudaStream_t s);
uint64_t split_tiles(uint64_t n);
int launch_split_count_tiles(const uint32_t* keys, uint64_t n, uint32_t skip, uint32_t rb, uint32_t* tile_cnt,
                             uint64_t* counts, cudaStream_t s);
int launch_split_tile_scan(const uint32_t* tile_cnt, uint64_t n, uint32_t rb, uint64_t* tpfx, uint64_t* scratch,
                           cudaStream_t s);
int launch_split_scatter_tiles(const uint32_t* keys, const uint32_t* pays, uint64_t n, uint32_t skip, uint32_t rb,
                               const uint64_t* off, const uint64_t* tpfx, uint32_t* ok, uint32_t* op,
                               cudaStream_t s);
int launch_count_keys(const uint32_t* keys, uint64_t n, const uint32_t* q, uint64_t m, uint64_t* counts,
                      cudaStream_t s);
int launch_radix_hist(const uint32_t* keys, uint64_t n, uint32_t hi_bits, uint32_t nbits, uint64_t* hist,
                      cudaStream_t s);
// shard.cu: this rank's route counts without reading the keys again (native driver, route_bits <=
// part_bits): destination sums of the LOCAL partition histogram, minus the local counts of the
// skewed keys (exact: every skewed key lies in a large partition, where the local table counts
// every key), which go to destination G.  out = [R counts (G+1) | S counts (G+1)].
int launch_route_counts_from_hist(const uint64_t* hist_local, uint32_t part_bits, uint32_t route_bits,
                                  const uint32_t* uni, const uint64_t* cnt_global, const uint64_t* cnt_local,
                                  uint64_t m, uint32_t heavy_threshold, uint64_t* out, cudaStream_t s);

}  // namespace gsh
