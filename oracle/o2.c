/*
 * oracle/o2.c -- ORACLE O2: plain multithreaded CPU TagMatch (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  The product (the CUDA library under
 * paper_conf_eurosys_rogorapkmcc17_b200/) never links, loads or calls it, and this
 * file shares no code, header or table with it.
 *
 * What it computes (sec. 2-3, cited per function):
 *   - the Bloom encoding of tag sets (m = 192, k = 7), with the
 *     hash functions fixed by DESIGN.md reading R1 (the paper does not name
 *     them): FNV-1a-64 of the tag bytes, then 7 SplitMix64 outputs seeded with
 *     that hash, each reduced to a position by (z * 192) >> 64;
 *   - brute-force matching: emit (q, key) for every DB entry whose signature is
 *     a bitwise subset of the query's;
 *   - the paper's CPU-side method: Algorithm 1 balanced partitioning
 *     (PAPER.md:120), the partition table PT[192] by leftmost one-bit and
 *     Algorithm 2 routing, then a linear scan of each routed
 *     partition (Alg. 3 semantics).
 *
 * Bit layout (reading R3): position p lives in 64-bit word p>>6 at
 * bit 63-(p&63); "leftmost" = lowest position.
 *
 * Parity status: encoder bits are pinned by published FNV-1a / SplitMix64 test
 * vectors and by the fn.3 false-positive statistics (tests/test_oracle_pins.py);
 * matching is pinned by brute-force exact-containment tests.
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

#define O2_M 192
#define O2_K 7

/* ------------------------------------------------------------- encoder --- */
/* FNV-1a 64-bit over the tag bytes (reading R1). */
uint64_t o2_fnv1a64(const uint8_t *p, uint64_t n) {
    uint64_t h = 0xcbf29ce484222325ULL;
    for (uint64_t i = 0; i < n; i++) {
        h ^= (uint64_t)p[i];
        h *= 0x100000001b3ULL;
    }
    return h;
}

/* SplitMix64 output function applied to state x (reading R1). */
uint64_t o2_splitmix_mix(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

/* The k = 7 hash positions of one tag: r-th SplitMix64 output seeded with h. */
void o2_tag_positions(const uint8_t *p, uint64_t n, uint32_t pos[O2_K]) {
    uint64_t h = o2_fnv1a64(p, n);
    for (int r = 0; r < O2_K; r++) {
        uint64_t z = o2_splitmix_mix(h + (uint64_t)(r + 1) * 0x9e3779b97f4a7c15ULL);
        pos[r] = (uint32_t)(((unsigned __int128)z * O2_M) >> 64);
    }
}

static void set_position(uint64_t sig[3], uint32_t p) { sig[p >> 6] |= 1ULL << (63 - (p & 63)); }

static void encode_set(const uint8_t *vocab, const uint64_t *voff, const uint32_t *tag_idx, uint64_t t0, uint64_t t1,
                       uint64_t sig[3]) {
    sig[0] = sig[1] = sig[2] = 0;
    for (uint64_t t = t0; t < t1; t++) {
        uint64_t v = tag_idx ? tag_idx[t] : t;
        uint32_t pos[O2_K];
        o2_tag_positions(vocab + voff[v], voff[v + 1] - voff[v], pos);
        for (int r = 0; r < O2_K; r++) set_position(sig, pos[r]);
    }
}

/* ------------------------------------------------------------- threads --- */
typedef void (*o2_range_fn)(void *ctx, uint64_t lo, uint64_t hi, int tid);
typedef struct {
    o2_range_fn fn;
    void *ctx;
    uint64_t lo, hi;
    int tid;
} o2_job;

static void *o2_job_main(void *a) {
    o2_job *j = (o2_job *)a;
    j->fn(j->ctx, j->lo, j->hi, j->tid);
    return NULL;
}

int o2_threads(int n) {
    if (n > 0) return n > 256 ? 256 : n;
    long c = sysconf(_SC_NPROCESSORS_ONLN);
    if (c < 1) c = 1;
    return c > 256 ? 256 : (int)c;
}

/* Static split of [0,n) in nthreads contiguous ranges (range t -> thread t). */
static void o2_parallel(uint64_t n, int nthreads, o2_range_fn fn, void *ctx) {
    pthread_t th[256];
    o2_job jobs[256];
    for (int t = 0; t < nthreads; t++) {
        jobs[t].fn = fn;
        jobs[t].ctx = ctx;
        jobs[t].lo = n * (uint64_t)t / (uint64_t)nthreads;
        jobs[t].hi = n * (uint64_t)(t + 1) / (uint64_t)nthreads;
        jobs[t].tid = t;
        pthread_create(&th[t], NULL, o2_job_main, &jobs[t]);
    }
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
}

typedef struct {
    const uint8_t *vocab;
    const uint64_t *voff;
    const uint32_t *tag_idx;
    const uint64_t *set_off;
    uint64_t *sig;
} enc_ctx;

static void enc_range(void *c, uint64_t lo, uint64_t hi, int tid) {
    (void)tid;
    enc_ctx *x = (enc_ctx *)c;
    for (uint64_t i = lo; i < hi; i++)
        encode_set(x->vocab, x->voff, x->tag_idx, x->set_off[i], x->set_off[i + 1], x->sig + 3 * i);
}

/* sig(T) = OR over tags of their 7 positions.  tag_idx may be
 * NULL (tag t of the CSR is vocabulary string t). */
void o2_encode(const uint8_t *vocab, const uint64_t *voff, const uint32_t *tag_idx, const uint64_t *set_off,
               uint64_t n_sets, uint64_t *sig_out, int nthreads) {
    enc_ctx x = {vocab, voff, tag_idx, set_off, sig_out};
    int nt = o2_threads(nthreads);
    if (n_sets < 1024) nt = 1;
    o2_parallel(n_sets, nt, enc_range, &x);
}

/* ---------------------------------------------------------------- results --- */
typedef struct {
    uint32_t *q, *k;
    uint64_t n, cap;
} o2_buf;

static void buf_push(o2_buf *b, uint32_t q, uint32_t k) {
    if (b->n == b->cap) {
        b->cap = b->cap ? b->cap * 2 : 1024;
        b->q = (uint32_t *)realloc(b->q, b->cap * sizeof(uint32_t));
        b->k = (uint32_t *)realloc(b->k, b->cap * sizeof(uint32_t));
    }
    b->q[b->n] = q;
    b->k[b->n] = k;
    b->n++;
}

typedef struct {
    uint64_t n;
    uint32_t *q, *k;
} o2_result;

static int cmp_u32(const void *a, const void *b) {
    uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
    return x < y ? -1 : x > y;
}

/* append query j's collected keys sorted (match) or sorted+unique (match-unique) */
static void flush_query(o2_buf *out, uint32_t j, uint32_t *keys, uint64_t n, int unique) {
    qsort(keys, n, sizeof(uint32_t), cmp_u32);
    for (uint64_t i = 0; i < n; i++) {
        if (unique && i > 0 && keys[i] == keys[i - 1]) continue;
        buf_push(out, j, keys[i]);
    }
}

static o2_result *concat(o2_buf *bufs, int nt) {
    o2_result *r = (o2_result *)calloc(1, sizeof(o2_result));
    for (int t = 0; t < nt; t++) r->n += bufs[t].n;
    r->q = (uint32_t *)malloc((r->n + 1) * sizeof(uint32_t));
    r->k = (uint32_t *)malloc((r->n + 1) * sizeof(uint32_t));
    uint64_t o = 0;
    for (int t = 0; t < nt; t++) {
        memcpy(r->q + o, bufs[t].q, bufs[t].n * sizeof(uint32_t));
        memcpy(r->k + o, bufs[t].k, bufs[t].n * sizeof(uint32_t));
        o += bufs[t].n;
        free(bufs[t].q);
        free(bufs[t].k);
    }
    return r;
}

uint64_t o2_result_n(const o2_result *r) { return r->n; }
void o2_result_copy(const o2_result *r, uint32_t *q, uint32_t *k) {
    memcpy(q, r->q, r->n * sizeof(uint32_t));
    memcpy(k, r->k, r->n * sizeof(uint32_t));
}
void o2_result_free(o2_result *r) {
    if (!r) return;
    free(r->q);
    free(r->k);
    free(r);
}

/* ------------------------------------------------------------ brute force --- */
typedef struct {
    const uint64_t *db, *key_off, *q;
    const uint32_t *keys;
    uint64_t n_sets;
    const uint32_t *qid; /* optional: output query ids */
    int unique;
    o2_buf *bufs;
} brute_ctx;

static void brute_range(void *c, uint64_t lo, uint64_t hi, int tid) {
    brute_ctx *x = (brute_ctx *)c;
    uint64_t cap = 1024, n;
    uint32_t *tmp = (uint32_t *)malloc(cap * sizeof(uint32_t));
    for (uint64_t j = lo; j < hi; j++) {
        const uint64_t *q = x->q + 3 * j;
        n = 0;
        for (uint64_t i = 0; i < x->n_sets; i++) {
            const uint64_t *s = x->db + 3 * i;
            /* sig(s) subset of sig(q): (s & ~q) == 0 in every block */
            if ((s[0] & ~q[0]) == 0 && (s[1] & ~q[1]) == 0 && (s[2] & ~q[2]) == 0) {
                for (uint64_t e = x->key_off[i]; e < x->key_off[i + 1]; e++) {
                    if (n == cap) {
                        cap *= 2;
                        tmp = (uint32_t *)realloc(tmp, cap * sizeof(uint32_t));
                    }
                    tmp[n++] = x->keys[e];
                }
            }
        }
        flush_query(&x->bufs[tid], x->qid ? x->qid[j] : (uint32_t)j, tmp, n, x->unique);
    }
    free(tmp);
}

/* Every (j, key) with sig(set) subset of sig(q_j), sorted by (j, key); unique
 * keeps one copy (match-unique), else multiplicity (match).  qid: optional
 * output id of each query (for sampled checks). */
o2_result *o2_match_brute(const uint64_t *db_sig, const uint64_t *key_off, const uint32_t *keys, uint64_t n_sets,
                          const uint64_t *q_sig, const uint32_t *qid, uint64_t n_q, int unique, int nthreads) {
    int nt = o2_threads(nthreads);
    if ((uint64_t)nt > n_q) nt = n_q ? (int)n_q : 1;
    o2_buf *bufs = (o2_buf *)calloc((size_t)nt, sizeof(o2_buf));
    brute_ctx x = {db_sig, key_off, q_sig, keys, n_sets, qid, unique, bufs};
    o2_parallel(n_q, nt, brute_range, &x);
    o2_result *r = concat(bufs, nt);
    free(bufs);
    return r;
}

/* ---------------------------------------------------------- Algorithm 1 --- */
/* One work-queue entry (mask -> P, used_bits). */
typedef struct {
    uint64_t mask[3], used[3];
    uint64_t *P; /* member indices */
    uint64_t n;
} o2_node;

typedef struct {
    uint64_t n_parts;
    uint64_t *masks;    /* 3 per partition */
    uint64_t *part_off; /* n_parts + 1 */
    uint64_t *members;  /* set indices, partition by partition */
    uint64_t cap_parts, n_members;
} o2_index;

static int has_pos(const uint64_t w[3], int p) { return (int)((w[p >> 6] >> (63 - (p & 63))) & 1ULL); }

static void index_add(o2_index *ix, const uint64_t mask[3], const uint64_t *P, uint64_t n) {
    if (ix->n_parts == ix->cap_parts) {
        ix->cap_parts = ix->cap_parts ? ix->cap_parts * 2 : 64;
        ix->masks = (uint64_t *)realloc(ix->masks, ix->cap_parts * 3 * sizeof(uint64_t));
        ix->part_off = (uint64_t *)realloc(ix->part_off, (ix->cap_parts + 1) * sizeof(uint64_t));
    }
    memcpy(ix->masks + 3 * ix->n_parts, mask, 3 * sizeof(uint64_t));
    memcpy(ix->members + ix->n_members, P, n * sizeof(uint64_t));
    ix->n_members += n;
    ix->n_parts++;
    ix->part_off[ix->n_parts] = ix->n_members;
}

/* Algorithm 1 with DESIGN.md reading R7:
 *   accept P when |P| <= MAX_P and mask != 0;
 *   otherwise pivot = unused bit with frequency closest to 50% among bits with
 *   0 < freq < |P| (ties -> lowest position); if there is no such bit all
 *   members share one signature sigma and P is accepted with mask sigma;
 *   empty P are dropped.
 * max_p == UINT32_MAX means "no partitioning": one partition, empty mask
 * (reading R8).  The queue is processed FIFO as written. */
o2_index *o2_alg1(const uint64_t *sig, uint64_t n_sets, uint32_t max_p) {
    o2_index *ix = (o2_index *)calloc(1, sizeof(o2_index));
    ix->members = (uint64_t *)malloc((n_sets + 1) * sizeof(uint64_t));
    ix->part_off = (uint64_t *)malloc(65 * sizeof(uint64_t));
    ix->masks = (uint64_t *)malloc(64 * 3 * sizeof(uint64_t));
    ix->cap_parts = 64;
    ix->part_off[0] = 0;
    if (n_sets == 0) return ix;
    uint64_t *all = (uint64_t *)malloc(n_sets * sizeof(uint64_t));
    for (uint64_t i = 0; i < n_sets; i++) all[i] = i;
    if (max_p == 0xFFFFFFFFu) {
        uint64_t zero[3] = {0, 0, 0};
        index_add(ix, zero, all, n_sets);
        free(all);
        return ix;
    }
    /* FIFO work queue */
    uint64_t qcap = 1024, qhead = 0, qtail = 0;
    o2_node *Q = (o2_node *)malloc(qcap * sizeof(o2_node));
    memset(&Q[0], 0, sizeof(o2_node));
    Q[0].P = all;
    Q[0].n = n_sets;
    qtail = 1;
    while (qhead < qtail) {
        o2_node nd = Q[qhead++];
        if (nd.n == 0) {
            free(nd.P);
            continue;
        }
        int mask_nonempty = (nd.mask[0] | nd.mask[1] | nd.mask[2]) != 0;
        if (nd.n <= (uint64_t)max_p && mask_nonempty) {
            index_add(ix, nd.mask, nd.P, nd.n);
            free(nd.P);
            continue;
        }
        /* frequencies of one-bits over the sets of P */
        uint64_t freq[O2_M];
        memset(freq, 0, sizeof(freq));
        for (uint64_t i = 0; i < nd.n; i++) {
            const uint64_t *s = sig + 3 * nd.P[i];
            for (int p = 0; p < O2_M; p++) freq[p] += (uint64_t)has_pos(s, p);
        }
        int pivot = -1;
        uint64_t best = 0;
        for (int p = 0; p < O2_M; p++) {
            if (has_pos(nd.used, p)) continue;
            if (freq[p] == 0 || freq[p] == nd.n) continue;
            uint64_t dist = 2 * freq[p] > nd.n ? 2 * freq[p] - nd.n : nd.n - 2 * freq[p];
            if (pivot < 0 || dist < best) {
                pivot = p;
                best = dist;
            }
        }
        if (pivot < 0) {
            /* every unused bit is constant; used bits are constant by construction:
               all members equal sigma = sig of any member (reading R7) */
            index_add(ix, sig + 3 * nd.P[0], nd.P, nd.n);
            free(nd.P);
            continue;
        }
        uint64_t *P0 = (uint64_t *)malloc((nd.n + 1) * sizeof(uint64_t));
        uint64_t *P1 = (uint64_t *)malloc((nd.n + 1) * sizeof(uint64_t));
        uint64_t n0 = 0, n1 = 0;
        for (uint64_t i = 0; i < nd.n; i++) {
            if (has_pos(sig + 3 * nd.P[i], pivot))
                P1[n1++] = nd.P[i];
            else
                P0[n0++] = nd.P[i];
        }
        free(nd.P);
        if (qtail + 2 > qcap) {
            /* compact the queue */
            memmove(Q, Q + qhead, (qtail - qhead) * sizeof(o2_node));
            qtail -= qhead;
            qhead = 0;
            if (qtail + 2 > qcap) {
                qcap *= 2;
                Q = (o2_node *)realloc(Q, qcap * sizeof(o2_node));
            }
        }
        o2_node a = nd, b = nd;
        a.used[pivot >> 6] |= 1ULL << (63 - (pivot & 63));
        b.used[pivot >> 6] |= 1ULL << (63 - (pivot & 63));
        b.mask[pivot >> 6] |= 1ULL << (63 - (pivot & 63));
        a.P = P0;
        a.n = n0;
        b.P = P1;
        b.n = n1;
        Q[qtail++] = a;
        Q[qtail++] = b;
    }
    free(Q);
    return ix;
}

uint64_t o2_index_n_parts(const o2_index *ix) { return ix->n_parts; }
void o2_index_copy(const o2_index *ix, uint64_t *masks, uint64_t *part_off, uint64_t *members) {
    memcpy(masks, ix->masks, ix->n_parts * 3 * sizeof(uint64_t));
    memcpy(part_off, ix->part_off, (ix->n_parts + 1) * sizeof(uint64_t));
    memcpy(members, ix->members, ix->n_members * sizeof(uint64_t));
}
void o2_index_free(o2_index *ix) {
    if (!ix) return;
    free(ix->masks);
    free(ix->part_off);
    free(ix->members);
    free(ix);
}

/* ------------------------------------------------- Algorithm 2 + scan --- */
/* PT[j] = partitions whose mask's leftmost one-bit is j; masks
 * with no one-bit go to an extra list that is forwarded to every query
 * (reading R9: the empty mask is a subset of every q). */
typedef struct {
    uint64_t *ids[O2_M + 1];
    uint64_t n[O2_M + 1];
} o2_pt;

static void pt_build(o2_pt *pt, const o2_index *ix) {
    memset(pt, 0, sizeof(*pt));
    for (uint64_t i = 0; i < ix->n_parts; i++) {
        const uint64_t *m = ix->masks + 3 * i;
        int j = O2_M;
        for (int p = 0; p < O2_M; p++)
            if (has_pos(m, p)) {
                j = p;
                break;
            }
        pt->ids[j] = (uint64_t *)realloc(pt->ids[j], (pt->n[j] + 1) * sizeof(uint64_t));
        pt->ids[j][pt->n[j]++] = i;
    }
}

static void pt_free(o2_pt *pt) {
    for (int j = 0; j <= O2_M; j++) free(pt->ids[j]);
}

typedef struct {
    const o2_index *ix;
    const o2_pt *pt;
    const uint64_t *db, *key_off, *q;
    const uint32_t *keys;
    const uint32_t *qid;
    int unique;
    o2_buf *bufs;
    uint64_t *routed; /* per thread: routed (q, partition) count */
    uint64_t *checked; /* per thread: pair checks */
} part_ctx;

static void part_range(void *c, uint64_t lo, uint64_t hi, int tid) {
    part_ctx *x = (part_ctx *)c;
    uint64_t cap = 1024, n;
    uint32_t *tmp = (uint32_t *)malloc(cap * sizeof(uint32_t));
    uint64_t routed = 0, checked = 0;
    for (uint64_t j = lo; j < hi; j++) {
        const uint64_t *q = x->q + 3 * j;
        n = 0;
        /* Algorithm 2: for each one-bit position of q, each mask in PT[pos]; plus empty masks */
        for (int pos = 0; pos <= O2_M; pos++) {
            if (pos < O2_M && !has_pos(q, pos)) continue;
            for (uint64_t t = 0; t < x->pt->n[pos]; t++) {
                uint64_t part = x->pt->ids[pos][t];
                const uint64_t *m = x->ix->masks + 3 * part;
                if ((m[0] & ~q[0]) || (m[1] & ~q[1]) || (m[2] & ~q[2])) continue; /* mask_i not subset of q */
                routed++;
                /* subset match within partition P_i: linear scan */
                for (uint64_t e = x->ix->part_off[part]; e < x->ix->part_off[part + 1]; e++) {
                    uint64_t i = x->ix->members[e];
                    const uint64_t *s = x->db + 3 * i;
                    checked++;
                    if ((s[0] & ~q[0]) == 0 && (s[1] & ~q[1]) == 0 && (s[2] & ~q[2]) == 0) {
                        for (uint64_t k = x->key_off[i]; k < x->key_off[i + 1]; k++) {
                            if (n == cap) {
                                cap *= 2;
                                tmp = (uint32_t *)realloc(tmp, cap * sizeof(uint32_t));
                            }
                            tmp[n++] = x->keys[k];
                        }
                    }
                }
            }
        }
        flush_query(&x->bufs[tid], x->qid ? x->qid[j] : (uint32_t)j, tmp, n, x->unique);
    }
    x->routed[tid] = routed;
    x->checked[tid] = checked;
    free(tmp);
}

/* stats_out (optional, 2 entries): routed (q, partition) pairs, pair checks. */
o2_result *o2_match_partitioned(const o2_index *ix, const uint64_t *db_sig, const uint64_t *key_off,
                                const uint32_t *keys, const uint64_t *q_sig, const uint32_t *qid, uint64_t n_q,
                                int unique, int nthreads, uint64_t *stats_out) {
    o2_pt pt;
    pt_build(&pt, ix);
    int nt = o2_threads(nthreads);
    if ((uint64_t)nt > n_q) nt = n_q ? (int)n_q : 1;
    o2_buf *bufs = (o2_buf *)calloc((size_t)nt, sizeof(o2_buf));
    uint64_t routed[256], checked[256];
    part_ctx x = {ix, &pt, db_sig, key_off, q_sig, keys, qid, unique, bufs, routed, checked};
    o2_parallel(n_q, nt, part_range, &x);
    if (stats_out) {
        stats_out[0] = stats_out[1] = 0;
        for (int t = 0; t < nt; t++) {
            stats_out[0] += routed[t];
            stats_out[1] += checked[t];
        }
    }
    o2_result *r = concat(bufs, nt);
    free(bufs);
    pt_free(&pt);
    return r;
}

/* ------------------------------------------------- Monte Carlo (fn. 3) --- */
/* False-positive rate of the encoder (PAPER.md:132 fn.3): S2 = s2 fresh tags,
 * S1 = d other fresh tags (S1 \ S2 has d elements); count trials where
 * sig(S1) subset of sig(S2).  Tags are the strings "mc<seed>_<trial>_<i>". */
static uint64_t mc_str(char *buf, uint64_t seed, uint64_t trial, int i) {
    /* tiny formatter without stdio */
    char tmp[64];
    int n = 0;
    uint64_t v[3] = {seed, trial, (uint64_t)i};
    buf[n++] = 'm';
    buf[n++] = 'c';
    for (int f = 0; f < 3; f++) {
        if (f) buf[n++] = '_';
        int m = 0;
        uint64_t x = v[f];
        do {
            tmp[m++] = (char)('0' + x % 10);
            x /= 10;
        } while (x);
        while (m) buf[n++] = tmp[--m];
    }
    return (uint64_t)n;
}

typedef struct {
    uint64_t seed;
    int s2, d;
    uint64_t *fp, *pop;
} mc_ctx;

static void mc_range(void *c, uint64_t lo, uint64_t hi, int tid) {
    mc_ctx *x = (mc_ctx *)c;
    char buf[96];
    uint64_t fp = 0, pop = 0;
    for (uint64_t t = lo; t < hi; t++) {
        uint64_t b2[3] = {0, 0, 0}, b1[3] = {0, 0, 0};
        uint32_t pos[O2_K];
        for (int i = 0; i < x->s2 + x->d; i++) {
            uint64_t n = mc_str(buf, x->seed, t, i);
            o2_tag_positions((const uint8_t *)buf, n, pos);
            for (int r = 0; r < O2_K; r++) set_position(i < x->s2 ? b2 : b1, pos[r]);
        }
        pop += (uint64_t)(__builtin_popcountll(b2[0]) + __builtin_popcountll(b2[1]) + __builtin_popcountll(b2[2]));
        if ((b1[0] & ~b2[0]) == 0 && (b1[1] & ~b2[1]) == 0 && (b1[2] & ~b2[2]) == 0) fp++;
    }
    x->fp[tid] = fp;
    x->pop[tid] = pop;
}

/* out[0] = false positives, out[1] = total popcount of sig(S2) over trials */
void o2_fp_montecarlo(uint64_t seed, int s2, int d, uint64_t trials, int nthreads, uint64_t *out) {
    int nt = o2_threads(nthreads);
    uint64_t fp[256], pop[256];
    mc_ctx x = {seed, s2, d, fp, pop};
    o2_parallel(trials, nt, mc_range, &x);
    out[0] = out[1] = 0;
    for (int t = 0; t < nt; t++) {
        out[0] += fp[t];
        out[1] += pop[t];
    }
}
