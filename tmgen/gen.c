/*
 * tmgen/gen.c -- seeded synthetic Twitter-like workload generator for TagMatch.
 *
 * This module is shared by the oracle side and the library side (it is the ONLY
 * code they share).  It holds none of the method's arithmetic: no Bloom
 * hashing, no signature encoding, no matching.  It only draws tag ids, keys and
 * queries with the shapes of the paper's workload:
 *
 *   - PAPER.md:262  300M users (keys) over 212M unique interest sets
 *                   -> keys per set = 1 + Poisson(0.415) (mean 300/212),
 *                      key ids ~ Zipf(1) over ceil(N*300/212) users.
 *   - PAPER.md:264  tags "translated" with a language prefix (fr_cat);
 *                   40% of users speak one language, 60% two.
 *   - PAPER.md:268  publisher id added as a tag for frequent writers (top 30%)
 *                   -> with probability 0.3 one tag is "u<id>", id ~ Zipf over
 *                      ceil(N*41.7/212) publishers.
 *   - PAPER.md:278  interests contain five tags on average
 *                   -> size = 1 + Poisson(4), clipped to [1, 20].
 *   - PAPER.md:282  each query = a database set + 2..4 extra tags
 *                   ("selected at random": read as popularity-weighted, from
 *                   the base set's language).
 *   - PAPER.md:290  broader range of query sizes (C5 sweep: total tags t).
 *
 * Recipe details are in DESIGN.md ("Input recipe").  Randomness is a
 * counter-based Philox-4x32-10 stream per (seed, domain, index), so the output
 * is identical for any thread count.
 *
 * Tag ids: id < 8*2^20 is a language tag, lang = id >> 20, rank = id & (2^20-1),
 * string "<lang>_t<rank>"; id >= 8*2^20 is a publisher tag "u<id - 8*2^20>".
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

#define TG_NLANG 8
#define TG_RANKS (1u << 20)
#define TG_PUB_BASE ((uint32_t)TG_NLANG * TG_RANKS)
#define TG_MAX_SET 20
#define TG_MAX_QUERY 64

static const char *TG_LANGS[TG_NLANG] = {"en", "ja", "pt", "es", "id", "ar", "fr", "tr"};

/* ------------------------------------------------------------------ RNG --- */
typedef struct {
    uint32_t key[2];
    uint32_t ctr[4];
    uint32_t buf[4];
    int pos;
} tg_rng;

static void philox10(const uint32_t in_ctr[4], const uint32_t in_key[2], uint32_t out[4]) {
    uint32_t c0 = in_ctr[0], c1 = in_ctr[1], c2 = in_ctr[2], c3 = in_ctr[3];
    uint32_t k0 = in_key[0], k1 = in_key[1];
    for (int r = 0; r < 10; r++) {
        uint64_t p0 = (uint64_t)0xD2511F53u * c0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * c2;
        uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
        uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
        uint32_t n0 = hi1 ^ c1 ^ k0, n1 = lo1, n2 = hi0 ^ c3 ^ k1, n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

static void rng_init(tg_rng *r, uint64_t seed, uint32_t domain, uint64_t index) {
    r->key[0] = (uint32_t)seed;
    r->key[1] = (uint32_t)(seed >> 32);
    r->ctr[0] = 0;
    r->ctr[1] = domain;
    r->ctr[2] = (uint32_t)index;
    r->ctr[3] = (uint32_t)(index >> 32);
    r->pos = 4;
}

static uint32_t rng_u32(tg_rng *r) {
    if (r->pos == 4) {
        philox10(r->ctr, r->key, r->buf);
        r->ctr[0]++;
        r->pos = 0;
    }
    return r->buf[r->pos++];
}

/* uniform double in [0,1) with 53 random bits */
static double rng_unif(tg_rng *r) {
    uint64_t a = rng_u32(r), b = rng_u32(r);
    uint64_t x = (a << 21) ^ (b >> 11);
    return (double)(x & ((1ULL << 53) - 1)) * (1.0 / 9007199254740992.0);
}

static uint64_t rng_below(tg_rng *r, uint64_t n) {
    uint64_t k = (uint64_t)(rng_unif(r) * (double)n);
    return k >= n ? n - 1 : k;
}

static int rng_poisson(tg_rng *r, double lambda) {
    double L = exp(-lambda), p = 1.0;
    int k = 0;
    do {
        k++;
        p *= rng_unif(r);
    } while (p > L);
    return k - 1;
}

/* Zipf(s = 1) over ranks {0..n-1}: rejection-inversion (Hormann & Derflinger). */
static uint64_t rng_zipf1(tg_rng *r, uint64_t n) {
    if (n <= 1) return 0;
    const double hx1 = log(1.5) - 1.0;
    const double hn = log((double)n + 0.5);
    const double s = 2.0 - exp(log(2.5) - 0.5);
    for (;;) {
        double u = hn + rng_unif(r) * (hx1 - hn);
        double x = exp(u);
        double kd = floor(x + 0.5);
        if (kd < 1.0) kd = 1.0;
        if (kd > (double)n) kd = (double)n;
        if (kd - x <= s || u >= log(kd + 0.5) - 1.0 / kd) return (uint64_t)kd - 1;
    }
}

/* language weights proportional to 1/(rank+1) (DESIGN.md input recipe) */
static int rng_lang(tg_rng *r) {
    double h = 0.0;
    for (int i = 0; i < TG_NLANG; i++) h += 1.0 / (i + 1);
    double u = rng_unif(r) * h, c = 0.0;
    for (int i = 0; i < TG_NLANG; i++) {
        c += 1.0 / (i + 1);
        if (u < c) return i;
    }
    return TG_NLANG - 1;
}

static int cmp_u32(const void *a, const void *b) {
    uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
    return x < y ? -1 : x > y;
}

static int contains_u32(const uint32_t *v, int n, uint32_t x) {
    for (int i = 0; i < n; i++)
        if (v[i] == x) return 1;
    return 0;
}

/* --------------------------------------------------------- DB candidates --- */
typedef struct {
    uint64_t n_pub, n_users;
} tg_params;

/* Draw candidate `idx`: fills tags (sorted), returns size; lang, keys too. */
static int gen_candidate(uint64_t seed, uint64_t idx, const tg_params *pp, uint32_t *tags, int *lang_out,
                         uint32_t *keys, int *nkeys_out) {
    tg_rng r;
    rng_init(&r, seed, 1u, idx);
    int nl = rng_unif(&r) < 0.4 ? 1 : 2;
    int l1 = rng_lang(&r), l2 = l1;
    if (nl == 2) {
        do { l2 = rng_lang(&r); } while (l2 == l1);
    }
    int lang = (nl == 1 || rng_unif(&r) < 0.5) ? l1 : l2;
    int size = 1 + rng_poisson(&r, 4.0);
    if (size > TG_MAX_SET) size = TG_MAX_SET;
    int k = 0;
    if (rng_unif(&r) < 0.3) tags[k++] = TG_PUB_BASE + (uint32_t)rng_zipf1(&r, pp->n_pub);
    while (k < size) {
        uint32_t t = (uint32_t)lang * TG_RANKS + (uint32_t)rng_zipf1(&r, TG_RANKS);
        if (!contains_u32(tags, k, t)) tags[k++] = t;
    }
    qsort(tags, (size_t)size, sizeof(uint32_t), cmp_u32);
    int nk = 1 + rng_poisson(&r, 0.415);
    if (nk > 16) nk = 16;
    if ((uint64_t)nk > pp->n_users) nk = (int)pp->n_users;
    int m = 0;
    while (m < nk) {
        uint32_t key = (uint32_t)rng_zipf1(&r, pp->n_users);
        if (!contains_u32(keys, m, key)) keys[m++] = key;
    }
    *lang_out = lang;
    *nkeys_out = nk;
    return size;
}

static uint64_t fmix64(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdULL;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ULL;
    k ^= k >> 33;
    return k;
}

static uint64_t set_fingerprint(const uint32_t *tags, int n) {
    uint64_t h = fmix64((uint64_t)n + 0x1234567ULL);
    for (int i = 0; i < n; i++) h = fmix64(h ^ ((uint64_t)tags[i] * 0x2545F4914F6CDD1DULL + (uint64_t)i));
    return h;
}

/* ------------------------------------------------------------- threads --- */
typedef void (*range_fn)(void *ctx, uint64_t lo, uint64_t hi);
typedef struct {
    range_fn fn;
    void *ctx;
    uint64_t lo, hi;
} tg_job;

static void *job_main(void *a) {
    tg_job *j = (tg_job *)a;
    j->fn(j->ctx, j->lo, j->hi);
    return NULL;
}

static int resolve_threads(int nthreads) {
    if (nthreads > 0) return nthreads;
    long n = sysconf(_SC_NPROCESSORS_ONLN);
    if (n < 1) n = 1;
    if (n > 256) n = 256;
    return (int)n;
}

static void parallel_for(uint64_t n, int nthreads, range_fn fn, void *ctx) {
    nthreads = resolve_threads(nthreads);
    if (n < 4096 || nthreads == 1) {
        fn(ctx, 0, n);
        return;
    }
    pthread_t th[256];
    tg_job jobs[256];
    for (int t = 0; t < nthreads; t++) {
        jobs[t].fn = fn;
        jobs[t].ctx = ctx;
        jobs[t].lo = n * (uint64_t)t / (uint64_t)nthreads;
        jobs[t].hi = n * (uint64_t)(t + 1) / (uint64_t)nthreads;
        pthread_create(&th[t], NULL, job_main, &jobs[t]);
    }
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
}

/* ------------------------------------------------------------ radix sort --- */
typedef struct {
    uint64_t fp;
    uint64_t idx;
} fp_pair;

static void radix_sort_fp(fp_pair *a, uint64_t n) {
    fp_pair *tmp = (fp_pair *)malloc(n * sizeof(fp_pair));
    uint64_t *cnt = (uint64_t *)malloc(65536 * sizeof(uint64_t));
    fp_pair *src = a, *dst = tmp;
    for (int pass = 0; pass < 4; pass++) {
        int sh = pass * 16;
        memset(cnt, 0, 65536 * sizeof(uint64_t));
        for (uint64_t i = 0; i < n; i++) cnt[(src[i].fp >> sh) & 0xffff]++;
        uint64_t s = 0;
        for (int d = 0; d < 65536; d++) {
            uint64_t c = cnt[d];
            cnt[d] = s;
            s += c;
        }
        for (uint64_t i = 0; i < n; i++) dst[cnt[(src[i].fp >> sh) & 0xffff]++] = src[i];
        fp_pair *t = src;
        src = dst;
        dst = t;
    }
    /* 4 passes: result back in a */
    free(tmp);
    free(cnt);
}

/* ------------------------------------------------------------------ DB --- */
typedef struct {
    uint64_t n_sets, n_tags, n_keys;
    uint64_t n_pub, n_users;
    uint64_t *set_off;
    uint32_t *tags;
    uint64_t *key_off;
    uint32_t *keys;
    uint8_t *lang;
    uint8_t *size;
} tg_db;

typedef struct {
    uint64_t seed;
    tg_params pp;
    fp_pair *fps;
    uint8_t *size;
    uint8_t *nkeys;
    uint8_t *lang;
    const uint64_t *cand; /* accepted candidate indices */
    tg_db *db;
} db_ctx;

static void db_fp_range(void *c, uint64_t lo, uint64_t hi) {
    db_ctx *x = (db_ctx *)c;
    uint32_t tags[TG_MAX_SET], keys[16];
    for (uint64_t i = lo; i < hi; i++) {
        int lang, nk;
        int n = gen_candidate(x->seed, i, &x->pp, tags, &lang, keys, &nk);
        x->fps[i].fp = set_fingerprint(tags, n);
        x->fps[i].idx = i;
    }
}

static void db_meta_range(void *c, uint64_t lo, uint64_t hi) {
    db_ctx *x = (db_ctx *)c;
    uint32_t tags[TG_MAX_SET], keys[16];
    for (uint64_t j = lo; j < hi; j++) {
        int lang, nk;
        int n = gen_candidate(x->seed, x->cand[j], &x->pp, tags, &lang, keys, &nk);
        x->size[j] = (uint8_t)n;
        x->nkeys[j] = (uint8_t)nk;
        x->lang[j] = (uint8_t)lang;
    }
}

static void db_fill_range(void *c, uint64_t lo, uint64_t hi) {
    db_ctx *x = (db_ctx *)c;
    tg_db *db = x->db;
    uint32_t tags[TG_MAX_SET], keys[16];
    for (uint64_t j = lo; j < hi; j++) {
        int lang, nk;
        int n = gen_candidate(x->seed, x->cand[j], &x->pp, tags, &lang, keys, &nk);
        memcpy(db->tags + db->set_off[j], tags, (size_t)n * sizeof(uint32_t));
        memcpy(db->keys + db->key_off[j], keys, (size_t)nk * sizeof(uint32_t));
    }
}

tg_db *tg_db_generate(uint64_t seed, uint64_t n_sets, int nthreads) {
    tg_db *db = (tg_db *)calloc(1, sizeof(tg_db));
    db_ctx x;
    memset(&x, 0, sizeof(x));
    x.seed = seed;
    x.pp.n_pub = (uint64_t)ceil((double)n_sets * 41.7 / 212.0);
    x.pp.n_users = (uint64_t)ceil((double)n_sets * 300.0 / 212.0);
    if (x.pp.n_pub < 1) x.pp.n_pub = 1;
    if (x.pp.n_users < 1) x.pp.n_users = 1;
    db->n_pub = x.pp.n_pub;
    db->n_users = x.pp.n_users;
    db->n_sets = n_sets;

    uint64_t *cand = (uint64_t *)malloc((n_sets ? n_sets : 1) * sizeof(uint64_t));
    if (n_sets > 0) {
        /* first n_sets distinct canonical sets in candidate-index order ("unique sets") */
        uint64_t M = n_sets + n_sets / 16 + 1024;
        for (;;) {
            x.fps = (fp_pair *)malloc(M * sizeof(fp_pair));
            parallel_for(M, nthreads, db_fp_range, &x);
            radix_sort_fp(x.fps, M); /* stable: within equal fp, idx ascending */
            uint8_t *acc = (uint8_t *)calloc(M, 1);
            uint64_t distinct = 0;
            for (uint64_t i = 0; i < M; i++) {
                if (i == 0 || x.fps[i].fp != x.fps[i - 1].fp) {
                    acc[x.fps[i].idx] = 1;
                    distinct++;
                }
            }
            free(x.fps);
            x.fps = NULL;
            if (distinct >= n_sets) {
                uint64_t j = 0;
                for (uint64_t i = 0; i < M && j < n_sets; i++)
                    if (acc[i]) cand[j++] = i;
                free(acc);
                break;
            }
            free(acc);
            M = M + M / 4 + 1024;
        }
    }
    x.cand = cand;
    x.size = (uint8_t *)malloc(n_sets + 1);
    x.nkeys = (uint8_t *)malloc(n_sets + 1);
    x.lang = (uint8_t *)malloc(n_sets + 1);
    parallel_for(n_sets, nthreads, db_meta_range, &x);
    db->set_off = (uint64_t *)malloc((n_sets + 1) * sizeof(uint64_t));
    db->key_off = (uint64_t *)malloc((n_sets + 1) * sizeof(uint64_t));
    db->set_off[0] = 0;
    db->key_off[0] = 0;
    for (uint64_t j = 0; j < n_sets; j++) {
        db->set_off[j + 1] = db->set_off[j] + x.size[j];
        db->key_off[j + 1] = db->key_off[j] + x.nkeys[j];
    }
    db->n_tags = db->set_off[n_sets];
    db->n_keys = db->key_off[n_sets];
    db->tags = (uint32_t *)malloc((db->n_tags + 1) * sizeof(uint32_t));
    db->keys = (uint32_t *)malloc((db->n_keys + 1) * sizeof(uint32_t));
    x.db = db;
    parallel_for(n_sets, nthreads, db_fill_range, &x);
    db->lang = x.lang;
    db->size = x.size;
    free(x.nkeys);
    free(cand);
    return db;
}

void tg_db_free(tg_db *db) {
    if (!db) return;
    free(db->set_off);
    free(db->tags);
    free(db->key_off);
    free(db->keys);
    free(db->lang);
    free(db->size);
    free(db);
}

uint64_t tg_db_n_sets(const tg_db *db) { return db->n_sets; }
uint64_t tg_db_n_tags(const tg_db *db) { return db->n_tags; }
uint64_t tg_db_n_keys(const tg_db *db) { return db->n_keys; }
uint64_t tg_db_n_users(const tg_db *db) { return db->n_users; }
void tg_db_copy(const tg_db *db, uint64_t *set_off, uint32_t *tags, uint64_t *key_off, uint32_t *keys,
                uint8_t *lang) {
    if (set_off) memcpy(set_off, db->set_off, (db->n_sets + 1) * sizeof(uint64_t));
    if (tags) memcpy(tags, db->tags, db->n_tags * sizeof(uint32_t));
    if (key_off) memcpy(key_off, db->key_off, (db->n_sets + 1) * sizeof(uint64_t));
    if (keys) memcpy(keys, db->keys, db->n_keys * sizeof(uint32_t));
    if (lang) memcpy(lang, db->lang, db->n_sets);
}

/* ------------------------------------------------------------- queries --- */
typedef struct {
    uint64_t n_q, n_tags;
    uint64_t *off;
    uint32_t *tags;
    uint64_t *base;
} tg_q;

typedef struct {
    const tg_db *db;
    uint64_t seed;
    int extra_min, extra_max, total;
    uint8_t *qsize;
    uint64_t *base;
    tg_q *q;
} q_ctx;

static int gen_query(const q_ctx *x, uint64_t j, uint32_t *out, uint64_t *base_out) {
    const tg_db *db = x->db;
    tg_rng r;
    rng_init(&r, x->seed, 2u, j);
    uint64_t base;
    int ne;
    if (x->total <= 0) {
        base = rng_below(&r, db->n_sets);
        ne = x->extra_min + (int)rng_below(&r, (uint64_t)(x->extra_max - x->extra_min + 1));
    } else {
        /* C5: base set with |s| <= t-1, then t-|s| extras */
        int tries = 0;
        do {
            base = rng_below(&r, db->n_sets);
            tries++;
        } while ((int)db->size[base] > x->total - 1 && tries < 100000);
        ne = x->total - (int)db->size[base];
        if (ne < 0) ne = 0;
    }
    int n = (int)(db->set_off[base + 1] - db->set_off[base]);
    memcpy(out, db->tags + db->set_off[base], (size_t)n * sizeof(uint32_t));
    int lang = db->lang[base];
    int want = n + ne;
    if (want > TG_MAX_QUERY) want = TG_MAX_QUERY;
    while (n < want) {
        uint32_t t = (uint32_t)lang * TG_RANKS + (uint32_t)rng_zipf1(&r, TG_RANKS);
        if (!contains_u32(out, n, t)) out[n++] = t;
    }
    qsort(out, (size_t)n, sizeof(uint32_t), cmp_u32);
    *base_out = base;
    return n;
}

static void q_size_range(void *c, uint64_t lo, uint64_t hi) {
    q_ctx *x = (q_ctx *)c;
    uint32_t tags[TG_MAX_QUERY];
    for (uint64_t j = lo; j < hi; j++) x->qsize[j] = (uint8_t)gen_query(x, j, tags, &x->base[j]);
}

static void q_fill_range(void *c, uint64_t lo, uint64_t hi) {
    q_ctx *x = (q_ctx *)c;
    uint32_t tags[TG_MAX_QUERY];
    uint64_t b;
    for (uint64_t j = lo; j < hi; j++) {
        int n = gen_query(x, j, tags, &b);
        memcpy(x->q->tags + x->q->off[j], tags, (size_t)n * sizeof(uint32_t));
    }
}

tg_q *tg_queries_generate(const tg_db *db, uint64_t seed, uint64_t n_q, int extra_min, int extra_max, int total,
                          int nthreads) {
    tg_q *q = (tg_q *)calloc(1, sizeof(tg_q));
    q->n_q = n_q;
    q->off = (uint64_t *)malloc((n_q + 1) * sizeof(uint64_t));
    q->base = (uint64_t *)malloc((n_q + 1) * sizeof(uint64_t));
    q->off[0] = 0;
    if (db->n_sets == 0) n_q = q->n_q = 0;
    q_ctx x;
    x.db = db;
    x.seed = seed;
    x.extra_min = extra_min;
    x.extra_max = extra_max < extra_min ? extra_min : extra_max;
    x.total = total;
    x.qsize = (uint8_t *)malloc(n_q + 1);
    x.base = q->base;
    x.q = q;
    parallel_for(n_q, nthreads, q_size_range, &x);
    for (uint64_t j = 0; j < n_q; j++) q->off[j + 1] = q->off[j] + x.qsize[j];
    q->n_tags = q->off[n_q];
    q->tags = (uint32_t *)malloc((q->n_tags + 1) * sizeof(uint32_t));
    parallel_for(n_q, nthreads, q_fill_range, &x);
    free(x.qsize);
    return q;
}

void tg_q_free(tg_q *q) {
    if (!q) return;
    free(q->off);
    free(q->tags);
    free(q->base);
    free(q);
}

uint64_t tg_q_n(const tg_q *q) { return q->n_q; }
uint64_t tg_q_n_tags(const tg_q *q) { return q->n_tags; }
void tg_q_copy(const tg_q *q, uint64_t *off, uint32_t *tags, uint64_t *base) {
    if (off) memcpy(off, q->off, (q->n_q + 1) * sizeof(uint64_t));
    if (tags) memcpy(tags, q->tags, q->n_tags * sizeof(uint32_t));
    if (base) memcpy(base, q->base, q->n_q * sizeof(uint64_t));
}

/* ------------------------------------------------------------- strings --- */
static int tag_string(uint32_t id, char *buf) {
    if (id < TG_PUB_BASE) return sprintf(buf, "%s_t%u", TG_LANGS[id >> 20], id & (TG_RANKS - 1));
    return sprintf(buf, "u%u", id - TG_PUB_BASE);
}

/* total bytes of the strings of ids[0..n) */
uint64_t tg_strings_size(const uint32_t *ids, uint64_t n) {
    char buf[64];
    uint64_t s = 0;
    for (uint64_t i = 0; i < n; i++) s += (uint64_t)tag_string(ids[i], buf);
    return s;
}

/* concatenated strings (no NUL) + n+1 offsets */
void tg_strings(const uint32_t *ids, uint64_t n, char *bytes, uint64_t *off) {
    char buf[64];
    uint64_t s = 0;
    off[0] = 0;
    for (uint64_t i = 0; i < n; i++) {
        int l = tag_string(ids[i], buf);
        memcpy(bytes + s, buf, (size_t)l);
        s += (uint64_t)l;
        off[i + 1] = s;
    }
}
