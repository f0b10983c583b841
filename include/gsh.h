/*
 * gsh.h -- C-ABI of the B200-native GSH (GPU Skew-conscious Hash join) library, libgsh.so.
 *
 * Paper: Cai & Chen, "CPU and GPU Hash Joins on Skewed Data", ICDE 2024.
 * The operation (§III, §IV-B): an inner equi-join of two
 * GPU-resident tables R and S of (4 B key, 4 B payload) tuples (L49 "joining GPU-resident
 * data", L55 / L132 "a pair of 4B join key and 4B payload"), computed by GSH's phases
 *   (1) radix-partition R and S in two passes, count-then-partition (L106)
 *   (2) detect skewed keys in large partitions after partitioning (L107, L112)
 *   (3) divide large partitions into per-skewed-key arrays and a normal partition (L114)
 *   (4) NM-join: one thread block per normal partition pair, shared-memory table (L115)
 *   (5) skewed-key join spread over many thread blocks (L116).
 * Result: match count, an order-independent 64-bit checksum, optionally the pairs.
 *
 * Semantics:
 *   M = { (payload_R[i], payload_S[j]) : key_R[i] == key_S[j] }, multiset over row pairs.
 *   count    = |M|;
 *   checksum = sum_{(a,b) in M} fmix64(((u64)a << 32 | b) ^ 0x9E3779B97F4A7C15) mod 2^64;
 *   pairs    = (payload_R, payload_S) per match, unspecified order.
 *   Keys and payloads are opaque u32 bit patterns; every value (0, 0xFFFFFFFF, ...) is legal.
 *   n = 0 on either side gives count = checksum = written = 0.
 *
 * Conventions for every entry point:
 *   - Pointers named d_* / device are CUDA device pointers (cudaMalloc / torch CUDA storage);
 *     pointers named h_* / host are host pointers.  The caller owns all buffers; the library
 *     never allocates device memory (all scratch comes from the caller's `workspace`).
 *   - Inputs are read-only and never modified.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  All GPU
 *     work is enqueued on it; entry points that fill a host result synchronise it.
 *   - Errors are status codes; nothing is thrown across the ABI.  Argument errors are
 *     reported before any launch (GSH_ERR_INVALID).  After GSH_ERR_CUDA the contents of
 *     results and outputs are undefined.  gsh_last_error() gives a thread-local message.
 *   - Reentrant given distinct workspaces and streams.
 */
#ifndef GSH_H_
#define GSH_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define GSH_API __attribute__((visibility("default")))
#else
#define GSH_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    GSH_OK = 0,
    GSH_ERR_INVALID = 1,   /* bad argument (NULL with n > 0, workspace too small, ...) */
    GSH_ERR_NOMEM = 2,     /* host allocation failed */
    GSH_ERR_CUDA = 3,      /* a CUDA call or kernel failed */
    GSH_ERR_NCCL = 4,      /* reserved for collective failures (multi-GPU driver) */
    GSH_ERR_INTERNAL = 5   /* broken internal invariant */
} gsh_status;

typedef enum {
    GSH_OUT_COUNT = 0,        /* count + checksum only (output consumed) */
    GSH_OUT_MATERIALIZE = 1   /* also write (payload_R, payload_S) pairs */
} gsh_out_mode;

/* A relation in SoA layout: keys[i], payloads[i], i < n.  Device pointers for gsh_join,
 * host pointers for gsh_join_host.  n must be < 2^32 (payloads are row ids). */
typedef struct {
    const uint32_t *keys;
    const uint32_t *payloads;
    uint64_t n;
} gsh_relation;

/* Materialised output: pairs[2i] = payload_R, pairs[2i+1] = payload_S for i < written.
 * capacity is in pairs.  Device pointer for gsh_join, host pointer for gsh_join_host. */
typedef struct {
    uint32_t *pairs;
    uint64_t capacity;
} gsh_output;

/* Tuning / test hooks.  Initialise with gsh_config_default(); NULL means defaults. */
typedef struct {
    uint32_t capacity;         /* C: max R tuples per NM-join build table (L115).  0 = auto
                                  (max(4096, 2 * mean partition size), <= 8192). */
    int32_t pass_bits[2];      /* radix bits of pass 1 / pass 2 (L106).  -1 = auto so the
                                  mean partition holds ~2048 tuples (max 8 + 8 bits). */
    uint32_t heavy_threshold;  /* T_h: a key of a large partition is skewed iff
                                  max(cnt_R, cnt_S) >= T_h (L112 reading).  0 = 64. */
    uint32_t route_bits;       /* top bits of fmix32(key) already consumed by multi-GPU
                                  routing; partition digits start below them. */
    int32_t force_all_normal;  /* test hook: no skew detection; every key goes through the
                                  NM-join (chunked when a partition exceeds C). */
    int32_t force_all_heavy;   /* test hook: every partition is large and every key skewed. */
    int32_t timing;            /* 1 = record per-phase CUDA events into gsh_result.ms_* */
    uint32_t large_threshold;  /* L: a partition is large iff |R_p| > L or |S_p| > L (L107's
                                  "pre-defined threshold").  0 = auto: mean + 8 sqrt(mean),
                                  i.e. far beyond the binomial spread of a skew-free partition. */
    int32_t nm_table;          /* NM-join shared-memory table (L115: "chained hash table").
                                  0 = auto: chained when no partition is large and the partition
                                  digits cover the top 16 bits of fmix32(key), else bucketized
                                  CSR;  1 = always CSR;  2 = chained wherever possible.  The
                                  result never depends on it. */
    int32_t detect_mode;       /* skewed-key detection in large partitions (L107, L112):
                                  0 = exact counts of every key, skewed iff max(cnt_R, cnt_S) >= T_h
                                  (default, R3/R4);  1 = the paper's sampling: every
                                  sample_stride-th tuple of R_p ++ S_p goes into a linear-probing
                                  table, the top_k most frequent sampled keys are skewed.  The
                                  result never depends on it. */
    uint32_t sample_stride;    /* detect_mode 1: 1 tuple in sample_stride is sampled.  0 = 100 (1 %) */
    uint32_t top_k;            /* detect_mode 1: skewed keys per large partition.  0 = 3 (L112) */
    int32_t prepass_bits;      /* pre-partition pass: split R and S by this many
                                  hash bits below route_bits and join each of the 2^bits
                                  sub-problems separately, so partitions stay shared-memory
                                  sized beyond the 2^16-partition limit of the two radix passes
                                  (L106).  0 = auto (enough bits that each side's share is
                                  <= 2^28 tuples; none up to 2^28);  -1 = off;  1..8 = forced.
                                  The result never depends on it. */
    int32_t heavy_detail;      /* test hook: the skewed-key join also sums
                                  each skewed key's checksum share C_k into the workspace, read
                                  back with gsh_heavy_detail.  Not with the pre-partition pass. */
    int32_t input_side_only;   /* measurement hook: run the input side (partition, classify,
                                  detect, split) and stop before the NM-join and the skewed-key
                                  join; count / checksum / written are then 0.  Used to time the
                                  partition passes on inputs whose output takes minutes. */
    int32_t hybrid;            /* CSH's hybrid partition on the GPU (§IV-A;
                                  SURVEY §8(f) NEXT-1): 1 = before partitioning, every
                                  hybrid_stride-th key of R and of S is sampled into a
                                  linear-probing table; keys sampled more than hybrid_min - 1 times
                                  (L89: "exceeds the pre-defined threshold (e.g., 2)"), at most the
                                  512 most frequent, are skewed up front.  The histogram pass counts
                                  them exactly and pass 1 writes their R AND S tuples straight into
                                  the per-key arrays R_k / S_k (payloads), so they skip pass 2,
                                  detection and the split.  Skew left in the partitions is still
                                  detected after partitioning as usual.  0 = off (GSH, L104).
                                  Ignored with force_all_normal / force_all_heavy.  The result never
                                  depends on it. */
    uint32_t hybrid_stride;    /* hybrid: 1 key in hybrid_stride is sampled.  0 = 100 (1 %, L89) */
    uint32_t hybrid_min;       /* hybrid: sampled count a key needs.  0 = 3 (L89: "exceeds ... 2") */
    uint32_t hybrid_share;     /* hybrid: the chosen keys must hold >= hybrid_share / 256 of the sample,
                                  else the partition passes run without them (GSH).  0 = 128 (1/2: the
                                  hybrid passes pay off where the sampled keys hold most of the input,
                                  DESIGN.md R22). */
} gsh_config;

/* Per-call result (host struct). */
typedef struct {
    uint64_t count;            /* |M| (all pairs, even on overflow) */
    uint64_t checksum;         /* sum of pair_hash over M mod 2^64 */
    uint64_t written;          /* pairs written = min(count, capacity) (MATERIALIZE) */
    uint64_t normal_count;     /* share of count produced by the NM-join phase */
    uint64_t normal_checksum;  /* share of checksum produced by the NM-join phase */
    uint64_t heavy_tuples_r;   /* R tuples routed to skewed-key arrays */
    uint64_t heavy_tuples_s;   /* S tuples routed to skewed-key arrays */
    uint64_t skew_pairs;       /* |R_k| * |S_k| summed over skewed keys */
    uint32_t overflow;         /* 1 iff count > capacity (MATERIALIZE) */
    uint32_t n_heavy;          /* number of skewed keys detected */
    uint32_t n_large;          /* number of large partitions */
    uint32_t detect_overflow;  /* 1 iff the detection table filled (fallback used) */
    uint32_t pass_bits[2];     /* radix bits actually used */
    uint32_t capacity;         /* C actually used */
    uint32_t heavy_threshold;  /* T_h actually used */
    uint32_t launches;         /* kernels launched by this call */
    uint32_t large_threshold;  /* L actually used */
    int32_t nm_table;          /* NM-join table used by the streamed kernel: 1 = CSR, 2 = chained */
    float ms_hist, ms_pass1, ms_pass2, ms_detect, ms_split, ms_nmjoin, ms_skewjoin, ms_total;
    uint32_t prepass_bits;     /* pre-partition bits actually used (0 = none) */
    float ms_prepass;          /* pre-partition pass (count + scatter), included in ms_total */
    uint64_t large_tuples;     /* R + S tuples in large partitions (read by detect and split) */
    uint32_t n_hybrid;         /* skewed keys found by the hybrid sample (gsh_config.hybrid), the
                                  first n_hybrid of the n_heavy */
    float ms_sample;           /* hybrid sample + selection, included in ms_total */
} gsh_result;

/* Fill *cfg with defaults (all auto, no hooks, timing off). */
GSH_API void gsh_config_default(gsh_config *cfg);

/* Bytes of device workspace gsh_join needs for these sizes (independent of the data).
 * Roughly 20 B per input tuple plus O(fanout) tables, + 16 B per tuple when the pre-partition
 * pass runs (gsh_config.prepass_bits); see DESIGN.md §5. */
GSH_API size_t gsh_workspace_bytes(uint64_t n_r, uint64_t n_s, const gsh_config *cfg);

/*
 * gsh_join -- the GSH equi-join of device-resident R and S (§IV-B).
 *   R, S       : device SoA relations (host structs holding device pointers).
 *   mode       : GSH_OUT_COUNT or GSH_OUT_MATERIALIZE.
 *   out        : NULL iff mode == GSH_OUT_COUNT; else device pairs buffer + capacity.
 *                Exactly min(count, capacity) pairs are written, unspecified order and
 *                (on overflow) unspecified subset; count/checksum always cover all pairs.
 *   workspace  : device scratch of >= gsh_workspace_bytes(R->n, S->n, cfg) bytes,
 *                256-byte aligned.  Contents on entry are ignored.
 *   cfg        : NULL = defaults.
 *   stream     : cudaStream_t as void*.
 *   res        : host result, filled after the stream is synchronised.
 * Beyond 2^28 tuples per side (or with cfg->prepass_bits > 0) both relations are first split
 * by hash bits into 2^prepass_bits sub-problems (split copies in the workspace), which are
 * joined one after another on `stream`; count / checksum / written cover all of them.
 * Returns GSH_ERR_INVALID for NULL pointers with n > 0, MATERIALIZE without output,
 * a too-small or misaligned workspace, n >= 2^32, or bad config values.
 */
GSH_API gsh_status gsh_join(const gsh_relation *R, const gsh_relation *S, gsh_out_mode mode,
                    const gsh_output *out, void *workspace, size_t workspace_bytes,
                    const gsh_config *cfg, void *stream, gsh_result *res);

/*
 * gsh_join_gbase -- the paper's GPU comparison system "Gbase" (§II-B, §III
 * L78-L80), re-implemented on this GPU for the GSH-vs-Gbase measurement
 * (Table I), with no skew detection:
 *   partition: two passes into bucket-chained partitions (4096-tuple buckets allocated from a pool
 *   as partitions fill, linked per partition; tiles of 4 tuples per thread reordered in shared
 *   memory and written as coalesced runs, L70) -- GSH's fanout (R7);
 *   join: one thread block per (partition, R sub-list = one bucket) builds a chained
 *   shared-memory table and probes it with ALL of S's buckets of that partition (L71-L72), every
 *   thread advancing one chain element per round with a write bitmap and a block barrier per round
 *   (L79-L80).
 * Arguments, errors and result semantics as gsh_join (identical count, checksum and pair multiset);
 * the workspace is gsh_gbase_workspace_bytes (bucket pools: ~4x gsh_join's at 2^27 per side).
 * res: ms_pass1 / ms_pass2 = the partition passes, ms_nmjoin = the join phase, ms_total; skew
 * fields 0.  At most 2^28 tuples per side (GSH_ERR_INVALID beyond).
 */
GSH_API size_t gsh_gbase_workspace_bytes(uint64_t n_r, uint64_t n_s, const gsh_config *cfg);   /* 0: invalid */
GSH_API gsh_status gsh_join_gbase(const gsh_relation *R, const gsh_relation *S, gsh_out_mode mode,
                                  const gsh_output *out, void *workspace, size_t workspace_bytes,
                                  const gsh_config *cfg, void *stream, gsh_result *res);

/* Device workspace for gsh_join_host: gsh_workspace_bytes + device staging for the inputs
 * (8 B per tuple) and, for MATERIALIZE, for out_capacity pairs (8 B per pair). */
GSH_API size_t gsh_host_workspace_bytes(uint64_t n_r, uint64_t n_s, gsh_out_mode mode,
                                uint64_t out_capacity, const gsh_config *cfg);

/*
 * gsh_join_host -- end-to-end variant: R, S and out hold HOST pointers (pinned memory
 * gives full PCIe/C2C bandwidth; pageable works but is slower).  The inputs are copied
 * host->device into the workspace, joined with gsh_join, and (MATERIALIZE) the written
 * pairs copied device->host, all on `stream`.  res->written pairs land in out->pairs.
 */
GSH_API gsh_status gsh_join_host(const gsh_relation *R, const gsh_relation *S, gsh_out_mode mode,
                         const gsh_output *out, void *workspace, size_t workspace_bytes,
                         const gsh_config *cfg, void *stream, gsh_result *res);

/* Decomposition of the last gsh_join on this workspace (cfg->heavy_detail = 1, COUNT or
 * MATERIALIZE, no pre-partition pass): for every skewed key k (unspecified
 * order) h_keys[k] = fmix32(key), h_cnt_r / h_cnt_s = its tuple counts, h_chk[k] = C_k =
 * sum of pair_hash over R_k x S_k mod 2^64 (host arrays of cap entries); *h_n = number of
 * skewed keys.  With gsh_result.normal_count / normal_checksum this splits the result into the
 * NM-join's share and one term per skewed key: count = normal_count + sum cnt_r * cnt_s,
 * checksum = normal_checksum + sum C_k.  n_r, n_s and cfg must be those of the join.
 * GSH_ERR_INVALID if more than cap keys or the join did not run with heavy_detail. */
GSH_API gsh_status gsh_heavy_detail(uint64_t n_r, uint64_t n_s, const gsh_config *cfg,
                                    void *workspace, size_t workspace_bytes, void *stream,
                                    uint32_t *h_keys, uint32_t *h_cnt_r, uint32_t *h_cnt_s,
                                    uint64_t *h_chk, uint64_t cap, uint64_t *h_n);

/* ---------------------------------------------------------------- step entry points --
 * Individual phases exposed for per-kernel parity tests and the multi-GPU driver.
 * Each synchronises `stream` before returning when it fills host outputs.             */

/* d_out[i] = fmix32(d_keys[i]) (SURVEY §8 notation h).  Device arrays of length n. */
GSH_API gsh_status gsh_hash_keys(const uint32_t *d_keys, uint32_t *d_out, uint64_t n, void *stream);

/* Radix histogram, the "count" scan of L106: d_hist[d] += #{i : digit(i) == d} where
 * digit = bits [32 - hi_bits - nbits, 32 - hi_bits) of fmix32(key).  d_hist is a device
 * array of 2^nbits u64 that the caller zeroes; nbits <= 16, hi_bits + nbits <= 32. */
GSH_API gsh_status gsh_radix_histogram(const uint32_t *d_keys, uint64_t n, uint32_t hi_bits,
                               uint32_t nbits, uint64_t *d_hist, void *workspace,
                               size_t workspace_bytes, void *stream);

/* Run the partition phase (L106: histogram, scan, pass-1 scatter, pass-2 scatter) and copy
 * out the final partitioned relations.  d_part_r / d_part_s: device arrays of 2*n u32
 * receiving AoS (h = fmix32(key), payload) tuples grouped by partition; d_off_r / d_off_s:
 * device arrays of (2^(b1+b2) + 1) u64 partition start offsets; h_bits[2]: host, receives
 * (b1, b2).  The order of tuples inside a partition is unspecified. */
GSH_API gsh_status gsh_partition(const gsh_relation *R, const gsh_relation *S, const gsh_config *cfg,
                         void *workspace, size_t workspace_bytes, void *stream,
                         uint32_t *d_part_r, uint32_t *d_part_s, uint64_t *d_off_r,
                         uint64_t *d_off_s, uint32_t *h_bits);

/* Run partition + classify + skew detection (L107, L112) and copy out the skewed-key side
 * list H: h_keys[k] = fmix32(key), h_cnt_r[k], h_cnt_s[k] for k < *h_n (host arrays of
 * `cap` entries; unspecified order).  Returns GSH_ERR_INVALID if more than cap keys. */
GSH_API gsh_status gsh_detect(const gsh_relation *R, const gsh_relation *S, const gsh_config *cfg,
                      void *workspace, size_t workspace_bytes, void *stream,
                      uint32_t *h_keys, uint32_t *h_cnt_r, uint32_t *h_cnt_s, uint64_t cap,
                      uint64_t *h_n, gsh_result *res);

/* ------------------------------------------------------ multi-GPU hash sharding --
 * SURVEY.md §8(e), a north-star addition: the paper runs on one A100 (§V-A).
 * One process (or logical rank) per GPU; rank g holds any shard of R and S.  The driver
 * (paper_conf_icde_caic24_b200/sharded.py) calls these per-rank steps between collectives
 * (torch.distributed over NCCL, or an in-process exchange for the one-GPU test harness):
 *   1. gsh_shard_plan: the single-GPU rule's parameters for the GLOBAL sizes;
 *   2. gsh_shard_histogram -> all_reduce(sum) -> global partition sizes;
 *   3. gsh_shard_candidates: keys of globally large partitions (L107) whose LOCAL count
 *      max(cnt_R, cnt_S) reaches tau = ceil(T_h / G) (pigeonhole: a key whose global count
 *      reaches T_h reaches tau on some rank) -> all_gather;
 *   4. gsh_shard_agree: union of the gathered candidates + this rank's exact counts of each
 *      -> all_reduce(sum);  5. gsh_shard_select: skewed iff max(cnt_R, cnt_S) >= T_h (L112) --
 *      the single-GPU rule applied to the whole input, identical list on every rank;
 *   6. gsh_heavy_set_build + gsh_route_count / gsh_route_scatter: a normal tuple goes to rank
 *      top_route_bits(h), a tuple of a skewed key to the "heavy" destination G (S_k stays
 *      local, R_k is all-gathered), so no GPU receives a skewed key's full S.
 * Keys are identified by h = fmix32(key) throughout (a bijection, so h equality is key equality).
 */
typedef struct {
    uint32_t world;            /* G, a power of two <= 256 */
    uint32_t route_bits;       /* log2 G */
    uint32_t part_bits;        /* B: partition bits of the skew rule (top B bits of h) */
    uint32_t large_threshold;  /* L: a partition is large iff |R_p| > L or |S_p| > L (both > 0) */
    uint32_t heavy_threshold;  /* T_h: skewed iff max(cnt_R, cnt_S) >= T_h (global counts) */
    uint32_t cand_threshold;   /* tau = ceil(T_h / G): local candidate threshold */
    int32_t force_all_normal;  /* gsh_config hook: no partition is large, no skewed key */
} gsh_shard_params;

/* Parameters for global sizes n_r_global, n_s_global over `world` ranks; B, L and T_h are what
 * gsh_join would use on one GPU holding the whole input (cfg as for gsh_join; NULL = defaults).
 * Host-only (no CUDA call).  GSH_ERR_INVALID for a bad world or config. */
GSH_API gsh_status gsh_shard_plan(uint64_t n_r_global, uint64_t n_s_global, uint32_t world,
                                  const gsh_config *cfg, gsh_shard_params *out);

/* d_hist (device u64[2 << part_bits], overwritten): d_hist[d] = #{R tuples with top part_bits
 * of h == d}, d_hist[2^part_bits + d] the same for S (the L106 "count" of the local shard). */
GSH_API gsh_status gsh_shard_histogram(const gsh_relation *R, const gsh_relation *S,
                                       const gsh_shard_params *p, uint64_t *d_hist, void *stream);

/* Device workspace of gsh_shard_candidates for a local shard of n_r + n_s tuples (holds the
 * local count table reused by gsh_shard_agree; keep it alive between the two calls). */
GSH_API size_t gsh_shard_workspace_bytes(uint64_t n_r, uint64_t n_s);

/* Local skew candidates.  d_hist_global: device u64[2 << part_bits], the all-reduced histogram.
 * Counts every key of a globally large partition exactly (both sides) into a table in
 * `workspace`, then writes the h of every key with local max(cnt_R, cnt_S) >= cand_threshold
 * to d_cand (device u32[cap], unspecified order); *h_n = how many (host).  *h_overflow (host,
 * may be NULL) = 1 iff the count table filled: keys were dropped from the candidates, which
 * keeps the join exact (an unflagged skewed key is simply routed as a normal key) but loses
 * its skew handling.  GSH_ERR_INVALID if *h_n > cap (nothing beyond cap is written). */
GSH_API gsh_status gsh_shard_candidates(const gsh_relation *R, const gsh_relation *S,
                                        const gsh_shard_params *p, const uint64_t *d_hist_global,
                                        void *workspace, size_t workspace_bytes, void *stream,
                                        uint32_t *d_cand, uint64_t cap, uint64_t *h_n,
                                        uint32_t *h_overflow);

/* Device workspace of gsh_shard_agree for a gathered buffer of n_gathered slots (world x
 * stride); also enough for gsh_shard_select on m <= n_gathered union keys. */
GSH_API size_t gsh_shard_agree_workspace_bytes(uint64_t n_gathered);

/* Union of the all-gathered candidates.  d_gathered: device u32[world * stride], rank g's
 * h_sizes[g] (host u64[world]) candidates at [g * stride, g * stride + h_sizes[g]).  Writes
 * the distinct values to d_union (device u32[cap]) in order of FIRST occurrence in the
 * gathered buffer -- the same order on every rank, since every rank holds the same buffer --
 * and this rank's exact counts of each to d_counts (device u64[2 * cap], interleaved
 * cnt_R, cnt_S), looked up in the table cand_ws (the workspace of this rank's
 * gsh_shard_candidates call).  *h_n = number of distinct values (host).  world * stride < 2^32. */
GSH_API gsh_status gsh_shard_agree(const void *cand_ws, size_t cand_ws_bytes,
                                   const uint32_t *d_gathered, uint32_t world, uint64_t stride,
                                   const uint64_t *h_sizes, void *workspace, size_t workspace_bytes,
                                   void *stream, uint32_t *d_union, uint64_t *d_counts, uint64_t cap,
                                   uint64_t *h_n);

/* Skewed keys (L112 reading): d_heavy[i] (device u32[cap]) = the union keys with global
 * max(cnt_R, cnt_S) >= heavy_threshold, in union order (stable compaction: identical on every
 * rank).  d_counts: device u64[2 * m], the all-reduced interleaved counts.  *h_n (host). */
GSH_API gsh_status gsh_shard_select(const uint32_t *d_union, const uint64_t *d_counts, uint64_t m,
                                    const gsh_shard_params *p, void *workspace,
                                    size_t workspace_bytes, void *stream, uint32_t *d_heavy,
                                    uint64_t cap, uint64_t *h_n);

/* Bytes of the open-addressing set of n_heavy skewed keys (0 for an empty set). */
GSH_API size_t gsh_heavy_set_bytes(uint64_t n_heavy);

/* Build the set of the n skewed keys d_heavy (device u32 h values) in d_set (device,
 * 256-byte aligned, >= gsh_heavy_set_bytes(n) bytes).  Synchronises `stream`. */
GSH_API gsh_status gsh_heavy_set_build(const uint32_t *d_heavy, uint64_t n, void *d_set,
                                       size_t set_bytes, void *stream);

/* Tuples per destination: d_counts[0..G] (device u64[G + 1], overwritten), G = 2^route_bits;
 * destination d < G = top route_bits of h (normal key), d = G = skewed key (member of the
 * set d_set / set_bytes from gsh_heavy_set_build; NULL / 0 = no skewed keys).  route_bits <= 8. */
GSH_API gsh_status gsh_route_count(const uint32_t *d_keys, uint64_t n, uint32_t route_bits,
                                   const void *d_set, size_t set_bytes, uint64_t *d_counts,
                                   void *stream);

/* Scatter every tuple to its destination (as gsh_route_count).  d_dst: device
 * u64[2 (G + heavy_copies)]: d_dst[2d] / d_dst[2d + 1] = device addresses of destination d's
 * key / payload arrays (d < G: normal routes, d = G: the skewed tuples), each with room for its
 * count; heavy_copies >= 1 -- with more than one, every skewed tuple is also stored at the same
 * position in the arrays d_dst[2 (G + c)], d_dst[2 (G + c) + 1], c = 1 .. heavy_copies - 1 (the
 * all-gather of skewed R done by the scatter itself).  The addresses may be peer memory (another
 * GPU's buffer opened with gsh_ipc_open, or under peer access): the kernel then IS the exchange,
 * its stores travelling over NVLink.  d_cursor: device u64[G + 1] scratch (overwritten).  The
 * order of tuples inside a destination is unspecified. */
GSH_API gsh_status gsh_route_scatter(const uint32_t *d_keys, const uint32_t *d_payloads, uint64_t n,
                                     uint32_t route_bits, const void *d_set, size_t set_bytes,
                                     const uint64_t *d_dst, uint32_t heavy_copies, uint64_t *d_cursor,
                                     void *stream);

/* CUDA IPC for the peer-store exchange: *handle (host, 64 bytes) names the device allocation
 * holding d_ptr for other processes, d_ptr = that allocation's base + *offset; gsh_ipc_open maps
 * such a handle into this process (*d_ptr = the base, a device address usable by kernels: a peer
 * GPU's memory over NVLink, or the same GPU's memory from another process); gsh_ipc_close unmaps
 * it.  GSH_ERR_CUDA with the CUDA message on failure. */
GSH_API gsh_status gsh_ipc_handle(const void *d_ptr, void *handle, uint64_t *offset);
GSH_API gsh_status gsh_ipc_open(const void *handle, void **d_ptr);
GSH_API gsh_status gsh_ipc_close(void *d_ptr);

/* ------------------------------------------------- native multi-GPU driver --
 * gsh_join_sharded runs the whole per-rank protocol above (agreement, routing, exchange, the two
 * local joins, the result reduction) in the library, over a communicator given as a table of
 * collectives.  SURVEY.md §8(b) "gsh_join_sharded(..., ncclComm_t)", §8(e).  Three communicators
 * are provided: an existing ncclComm_t (e.g. the one a torch.distributed NCCL process group
 * owns), a new NCCL communicator from a unique id, and an in-process "local world" in which G
 * host threads act as G ranks on any devices (the one-GPU multi-rank test harness).
 * Every callback enqueues on / synchronises `stream` and returns a gsh_status. */
typedef struct gsh_comm {
    uint32_t rank, world;      /* this rank, number of ranks */
    uint32_t same_process;     /* 1: every rank lives in this process (device pointers are valid
                                  across ranks); 0: ranks are processes (buffers shared via CUDA IPC) */
    uint32_t reserved;
    void *ctx;                 /* the implementation's state */
    /* d_buf[0..n) (device u64) := sum over ranks mod 2^64, in place */
    gsh_status (*all_reduce_u64)(void *ctx, uint64_t *d_buf, uint64_t n, void *stream);
    /* d_recv[g * bytes .. +bytes) := rank g's d_send[0..bytes) (device buffers) */
    gsh_status (*all_gather)(void *ctx, const void *d_send, void *d_recv, uint64_t bytes, void *stream);
    /* variable all-to-all of bytes: rank g receives h_send_bytes[g] bytes from d_send + h_send_off[g]
       of every rank at d_recv + h_recv_off[src] (its h_recv_bytes[src] must match; host arrays of
       world entries; zero-byte pairs are skipped) */
    gsh_status (*all_to_all_v)(void *ctx, const void *d_send, const uint64_t *h_send_off,
                               const uint64_t *h_send_bytes, void *d_recv, const uint64_t *h_recv_off,
                               const uint64_t *h_recv_bytes, void *stream);
    /* returns once every rank's work enqueued on its stream before the call is complete */
    gsh_status (*barrier)(void *ctx, void *stream);
    /* optional (may be NULL): release ranks blocked in a collective after this rank failed */
    void (*abort)(void *ctx);
} gsh_comm;

/* NCCL communicators (libnccl.so.2 is looked up at run time: the copy already loaded in the
 * process, e.g. torch's, else the system one; GSH_ERR_NCCL if none).  gsh_comm_nccl wraps an
 * existing ncclComm_t (passed as void*, not owned); gsh_nccl_unique_id fills 128 bytes on one
 * rank, which every rank passes to gsh_comm_nccl_init (collective over the world's ranks, with
 * `device` current) to create an owned communicator.  gsh_comm_destroy frees what the
 * constructor allocated (an owned NCCL communicator, or nothing). */
GSH_API gsh_status gsh_comm_nccl(void *nccl_comm, gsh_comm *out);
GSH_API gsh_status gsh_nccl_unique_id(void *id128);
GSH_API gsh_status gsh_comm_nccl_init(const void *id128, uint32_t world, uint32_t rank, int device,
                                      gsh_comm *out);
GSH_API gsh_status gsh_comm_destroy(gsh_comm *comm);

/* In-process world of `world` ranks (one host thread each): collectives are device copies
 * between the ranks' buffers behind host barriers.  gsh_comm_local fills rank r's table; the
 * world outlives every use of its tables. */
GSH_API gsh_status gsh_local_world_create(uint32_t world, void **lw);
GSH_API gsh_status gsh_comm_local(void *lw, uint32_t rank, gsh_comm *out);
GSH_API gsh_status gsh_local_world_destroy(void *lw);

/* Per-rank driver state: the comm table (copied), the device, and the grow-only device buffers of
 * the protocol (receive / send buffers, the two local joins' workspaces, IPC mappings of the
 * peers' receive buffers).  The receive sizes depend on the data, so -- unlike gsh_join -- the
 * driver allocates (cudaMalloc) and keeps its buffers across calls; gsh_sharded_destroy frees
 * them (call it on every rank after the last join, no collective involved). */
typedef struct gsh_sharded gsh_sharded;
GSH_API gsh_status gsh_sharded_create(const gsh_comm *comm, int device, gsh_sharded **ctx);
GSH_API gsh_status gsh_sharded_destroy(gsh_sharded *ctx);

typedef enum {
    GSH_EXCHANGE_A2A = 0,      /* route into send buffers, then all_to_all_v of normal tuples and an
                                  all-gather of skewed R; the normal exchange runs on a second stream
                                  while the skewed-key join computes */
    GSH_EXCHANGE_P2P = 1       /* the route kernel stores every tuple straight into its destination
                                  rank's receive buffer (skewed R into every rank's): the scatter IS
                                  the exchange (NVLink peer stores), then one barrier */
} gsh_exchange;

typedef struct {
    uint64_t count;            /* GLOBAL |M| (identical on every rank) */
    uint64_t checksum;         /* GLOBAL checksum mod 2^64 */
    uint64_t written;          /* pairs written to this rank's out (MATERIALIZE) */
    uint32_t overflow;         /* this rank's out was too small */
    uint32_t n_heavy;          /* agreed skewed keys */
    uint32_t route_bits, part_bits, large_threshold, heavy_threshold, cand_threshold;
    uint32_t cand_overflow;    /* some rank's candidate table filled (exact, skew handling lost) */
    uint64_t n_candidates;     /* candidates gathered over all ranks */
    uint64_t n_union;          /* distinct candidates */
    uint64_t local_r, local_s; /* this rank's input shard */
    uint64_t normal_r, normal_s, heavy_r, heavy_s;   /* this rank's local join inputs */
    uint64_t count_normal, count_heavy;               /* this rank's share of count */
    uint64_t exchange_bytes;   /* bytes this rank moved to other ranks (a2a: normal tuples sent;
                                  p2p: every remote store, skewed-R copies included) */
    uint64_t broadcast_bytes;  /* a2a: skewed-R bytes received from the other ranks */
    uint32_t launches;         /* libgsh kernels this call launched (local joins included) */
    uint32_t exchange;         /* gsh_exchange used */
    float ms_agree, ms_route, ms_exchange, ms_join_heavy, ms_join_normal, ms_reduce, ms_total;
    gsh_result normal;         /* the local join of the routed normal shard */
    gsh_result heavy;          /* the local join of all ranks' skewed R x this rank's skewed S */
} gsh_sharded_result;

/*
 * gsh_join_sharded -- the hash-sharded GSH join; every rank calls it with its shards R, S (device
 * SoA, any positional split of the global relations).  Steps: gsh_shard_plan on the all-reduced
 * sizes, histogram -> all_reduce, candidates -> all_gather, agree -> all_reduce, select (the
 * single-GPU skew rule on the whole input), route counts -> all_gather (the G x 2(G+1) count
 * matrix fixes every buffer offset), route scatter + exchange (`exchange`), gsh_join of the
 * normal shard (cfg->route_bits := log2 G) and of all skewed R x local skewed S (route_bits 0),
 * all_reduce of (count, checksum).  The result equals gsh_join on the whole input bit-exactly.
 * cfg: NULL = defaults (route_bits must be 0).  out: NULL iff COUNT; this rank's pairs.
 * Returns GSH_ERR_INVALID for bad arguments (detected before any collective only when local), and
 * any status a collective returns; after an error the comm's abort (if any) has been called.
 */
GSH_API gsh_status gsh_join_sharded(gsh_sharded *ctx, const gsh_relation *R, const gsh_relation *S,
                                    gsh_out_mode mode, const gsh_output *out, const gsh_config *cfg,
                                    gsh_exchange exchange, void *stream, gsh_sharded_result *res);

/* ------------------------------------------------------------------- diagnostics -- */
GSH_API const char *gsh_status_string(gsh_status s);
GSH_API const char *gsh_last_error(void);
/* Library version and the SM architecture it was compiled for (e.g. 100 for sm_100a). */
GSH_API int gsh_version(void);
GSH_API int gsh_compiled_arch(void);

#ifdef __cplusplus
}
#endif

#endif /* GSH_H_ */
