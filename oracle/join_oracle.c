/*
 * oracle/join_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU equi-join used as the parity oracle for the
 * GSH (GPU Skew-conscious Hash join) CUDA path.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.  It shares
 * no code, header, table or constant generator with paper_conf_icde_caic24_b200/csrc.
 *
 * What it computes (the definition, not the paper's algorithm):
 *   GSH is an exact equi-join (§IV-B: skew detection, sampling,
 *   top-k and partition shapes change performance only; every matching R/S tuple pair
 *   is still produced, L55 "join output ... consumed by an upper level operator").
 *   Tuples are (4 B key, 4 B payload) (§III, §V-A).
 *   M = { (payload_R[i], payload_S[j]) : key_R[i] == key_S[j] }   (multiset over row pairs)
 *   count    = |M|
 *   checksum = sum over M of pair_hash(a, b)  mod 2^64         (reading #2)
 *   pair_hash(a, b) = fmix64(((u64)a << 32 | b) ^ 0x9E3779B97F4A7C15)
 *   fmix64 = MurmurHash3 64-bit finalizer.
 *
 * Plain implementation: a separately chained hash table (std::unordered_multimap
 * equivalent written out in C) built from R in one thread, probed with S in T parallel
 * chunks (read-only table), per-thread wrapping u64 sums added at the end.
 * MATERIALIZE: a counting pass per chunk, then a writing pass at exclusive-scan offsets.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

/* MurmurHash3 fmix32 (Appleby, SMHasher).  Used here only to spread keys over the
 * oracle's own chain buckets; any hash would do for the oracle. */
static inline uint32_t oracle_fmix32(uint32_t h) {
    h ^= h >> 16;
    h *= 0x85ebca6bu;
    h ^= h >> 13;
    h *= 0xc2b2ae35u;
    h ^= h >> 16;
    return h;
}

/* MurmurHash3 fmix64 (Appleby, SMHasher). */
static inline uint64_t oracle_fmix64(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return k;
}

/* pair_hash(a,b) = fmix64(((u64)a << 32 | b) ^ 0x9E3779B97F4A7C15). */
static inline uint64_t oracle_pair_hash(uint32_t a, uint32_t b) {
    return oracle_fmix64((((uint64_t)a << 32) | (uint64_t)b) ^ 0x9E3779B97F4A7C15ull);
}

/* Exported scalar versions so tests can pin them against published vectors. */
uint32_t oracle_fmix32_scalar(uint32_t h) { return oracle_fmix32(h); }
uint64_t oracle_fmix64_scalar(uint64_t k) { return oracle_fmix64(k); }
uint64_t oracle_pair_hash_scalar(uint32_t a, uint32_t b) { return oracle_pair_hash(a, b); }

/* ---------------------------------------------------------------- chained table -- */
typedef struct {
    uint64_t  nbuckets;   /* power of two */
    int64_t  *head;       /* bucket -> first entry index, -1 = empty */
    int64_t  *next;       /* entry -> next entry in chain, -1 = end */
    const uint32_t *key;  /* R keys (borrowed) */
    const uint32_t *pay;  /* R payloads (borrowed) */
} oracle_table;

static int table_build(oracle_table *t, const uint32_t *rk, const uint32_t *rp, uint64_t nr) {
    uint64_t nb = 1;
    while (nb < nr) nb <<= 1;
    t->nbuckets = nb;
    t->head = (int64_t *)malloc(nb * sizeof(int64_t));
    t->next = (int64_t *)malloc((nr ? nr : 1) * sizeof(int64_t));
    if (!t->head || !t->next) return -1;
    for (uint64_t b = 0; b < nb; ++b) t->head[b] = -1;
    t->key = rk;
    t->pay = rp;
    for (uint64_t i = 0; i < nr; ++i) {          /* insert R tuple i at its chain head */
        uint64_t b = oracle_fmix32(rk[i]) & (nb - 1);
        t->next[i] = t->head[b];
        t->head[b] = (int64_t)i;
    }
    return 0;
}

static void table_free(oracle_table *t) {
    free(t->head);
    free(t->next);
}

/* ------------------------------------------------------------------ probe task -- */
typedef struct {
    const oracle_table *t;
    const uint32_t *sk, *sp;
    uint64_t s_begin, s_end;
    uint64_t count, checksum;  /* outputs */
    uint32_t *pairs;           /* NULL = count only; else write count pairs here */
} probe_task;

static void *probe_worker(void *arg) {
    probe_task *task = (probe_task *)arg;
    const oracle_table *t = task->t;
    uint64_t count = 0, checksum = 0;
    for (uint64_t j = task->s_begin; j < task->s_end; ++j) {
        uint32_t k = task->sk[j];
        uint32_t b_pay = task->sp[j];
        for (int64_t e = t->head[oracle_fmix32(k) & (t->nbuckets - 1)]; e >= 0; e = t->next[e]) {
            if (t->key[e] != k) continue;          /* equality on the key itself */
            uint32_t a_pay = t->pay[e];
            if (task->pairs) {
                task->pairs[2 * count] = a_pay;
                task->pairs[2 * count + 1] = b_pay;
            }
            count += 1;
            checksum += oracle_pair_hash(a_pay, b_pay);  /* wraps mod 2^64 */
        }
    }
    task->count = count;
    task->checksum = checksum;
    return NULL;
}

static int run_probe(const oracle_table *t, const uint32_t *sk, const uint32_t *sp, uint64_t ns,
                     int nthreads, probe_task *tasks, uint32_t **pair_bufs) {
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    if (!th) return -1;
    for (int i = 0; i < nthreads; ++i) {
        tasks[i].t = t;
        tasks[i].sk = sk;
        tasks[i].sp = sp;
        tasks[i].s_begin = ns * (uint64_t)i / (uint64_t)nthreads;
        tasks[i].s_end = ns * (uint64_t)(i + 1) / (uint64_t)nthreads;
        tasks[i].pairs = pair_bufs ? pair_bufs[i] : NULL;
        if (nthreads == 1) probe_worker(&tasks[i]);
        else pthread_create(&th[i], NULL, probe_worker, &tasks[i]);
    }
    if (nthreads > 1)
        for (int i = 0; i < nthreads; ++i) pthread_join(th[i], NULL);
    free(th);
    return 0;
}

/*
 * oracle_join: count + checksum of R ⋈ S on key; optionally the pairs.
 *   rk/rp: R keys/payloads (host, length nr); sk/sp: S keys/payloads (host, length ns).
 *   nthreads >= 1: probe threads.
 *   pairs_out: NULL for count-only; else a host buffer of 2*pairs_cap u32 that receives
 *   (payload_R, payload_S) for every match if count <= pairs_cap (the return value 1
 *   signals count > pairs_cap and nothing written).
 * Returns 0 on success, -1 on allocation failure, 1 if pairs_cap was too small.
 */
int oracle_join(const uint32_t *rk, const uint32_t *rp, uint64_t nr,
                const uint32_t *sk, const uint32_t *sp, uint64_t ns,
                int nthreads, uint64_t *count_out, uint64_t *checksum_out,
                uint32_t *pairs_out, uint64_t pairs_cap) {
    if (nthreads < 1) nthreads = 1;
    oracle_table t;
    if (table_build(&t, rk, rp, nr) != 0) return -1;
    probe_task *tasks = (probe_task *)calloc((size_t)nthreads, sizeof(probe_task));
    if (!tasks) { table_free(&t); return -1; }

    /* pass 1: count + checksum per chunk */
    if (run_probe(&t, sk, sp, ns, nthreads, tasks, NULL) != 0) { free(tasks); table_free(&t); return -1; }
    uint64_t count = 0, checksum = 0;
    for (int i = 0; i < nthreads; ++i) { count += tasks[i].count; checksum += tasks[i].checksum; }
    *count_out = count;
    *checksum_out = checksum;

    int rc = 0;
    if (pairs_out) {
        if (count > pairs_cap) {
            rc = 1;
        } else {
            /* pass 2: each chunk writes at the exclusive scan of pass-1 chunk counts */
            uint32_t **bufs = (uint32_t **)malloc(sizeof(uint32_t *) * (size_t)nthreads);
            uint64_t off = 0;
            for (int i = 0; i < nthreads; ++i) { bufs[i] = pairs_out + 2 * off; off += tasks[i].count; }
            run_probe(&t, sk, sp, ns, nthreads, tasks, bufs);
            free(bufs);
        }
    }
    free(tasks);
    table_free(&t);
    return rc;
}

/* Vectorised helpers so numpy-side pins can check large arrays against the scalar
 * definitions without a Python loop. */
void oracle_fmix32_array(const uint32_t *in, uint32_t *out, uint64_t n) {
    for (uint64_t i = 0; i < n; ++i) out[i] = oracle_fmix32(in[i]);
}
void oracle_pair_hash_array(const uint32_t *a, const uint32_t *b, uint64_t *out, uint64_t n) {
    for (uint64_t i = 0; i < n; ++i) out[i] = oracle_pair_hash(a[i], b[i]);
}
