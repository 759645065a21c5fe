/*
 * tagmatch.h -- C ABI of the B200-native TagMatch subset-matching library.
 *
 * The library implements the data-parallel hot path of TagMatch (Rogora et al.,
 * "High-Throughput Subset Matching on Commodity GPU-Based Systems", EuroSys'17;
 * cited as PAPER.md:<line>):
 *
 *   tm_build        add-set(set, key)* followed by consolidate()  (Table 2)
 *                   = Bloom encoding + Algorithm 1 balanced
 *                   partitioning + lexicographic order
 *                   inside partitions + key table.
 *   tm_match_batch  match / match-unique of a batch of query sets
 *                   (Table 2): encode, route to
 *                   every partition whose mask is a subset of the query
 *                   (Algorithm 2), per-partition batches
 *                   (PAPER.md:144), tile prefix pre-filter (Algorithm 4,
 *                   PAPER.md:164-198), subset check sig(s) & ~sig(q) == 0
 *                   (Algorithm 3), compaction,
 *                   set-id -> key lookup and merge
 *                   (PAPER.md:236).  Every step runs in the library's CUDA
 *                   kernels on one B200 (sm_100a); there is no CPU fallback.
 *   tm_free         release a database.
 *
 * Result semantics (readings R10-R13): entry i of the
 * database is (set i, key) for every key in set i's key list.  For query j the
 * result holds (j, key) for every entry whose Bloom signature is a bitwise
 * subset of sig(q_j) -- Bloom false positives included --
 * once per matching entry (match) or once per distinct key (match-unique).
 * Pairs are returned sorted ascending by (query, key).
 *
 * Conventions for every call:
 *   - return TM_OK (0) on success or a negative tm_status; no exception or
 *     longjmp crosses the ABI; tm_last_error() gives a human-readable detail
 *     for the calling thread's last failure;
 *   - input arrays are borrowed for the duration of the call only, never
 *     retained and never written;
 *   - outputs are written only on TM_OK;
 *   - a tm_db handle is not re-entrant: serialize calls per handle (different
 *     handles may be used concurrently from different threads).
 */
#ifndef TAGMATCH_H
#define TAGMATCH_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define TM_ABI_VERSION 5u  /* 5: tm_tagsets.vocab_hash (pre-hashed vocabulary) */
/* Bloom filter width and number of hash functions. */
#define TM_SIG_BITS 192u
#define TM_SIG_WORDS 3u
#define TM_NUM_HASHES 7u
/* Default MAX_P (best throughput around 200K sets per partition). */
#define TM_DEFAULT_MAX_PARTITION 200000u
/* max_partition value meaning "no partitioning": one partition with the empty
 * mask, routed to every query (reading R8; BASELINE config C1). */
#define TM_NO_PARTITIONING 0xFFFFFFFFu
/* max_partition value meaning "choose MAX_P from the database size": clamp(n_sets / 30,000,
 * 5,000, 200,000) (reading R8b: the paper's optimum of ~200K
 * comes from its CPU pipeline's per-partition cost; with the bit-sliced GPU router the
 * measured optimum is much smaller: C2 (1M sets) and C3 (100M) at 5K, C4 (300M) at 10K). */
#define TM_AUTO_MAX_PARTITION 0xFFFFFFFEu

typedef struct tm_db tm_db; /* opaque, owned by the library */

typedef enum {
    TM_OK = 0,
    TM_EINVAL = -1, /* NULL pointer, non-monotone / out-of-range offsets, bad flag   */
    TM_ENOMEM = -2, /* host or device allocation failed                            */
    TM_ECUDA = -3,  /* CUDA runtime error (also: no CUDA device / no sm_100 device)  */
    TM_ENCCL = -4,  /* NCCL error (sharded mode)                                    */
    TM_ERANGE = -5, /* more than 2^32-1 sets, keys, tags or queries                 */
    TM_ESTATE = -6  /* call not valid in the handle's state                        */
} tm_status;

/*
 * A batch of tag sets in interned CSR form (tags are byte strings,
 * PAPER.md:80 "sets of string tags"; case-sensitive, any bytes, no NUL needed).
 *
 *   vocabulary string v = vocab_bytes[vocab_off[v] .. vocab_off[v+1])
 *   set i               = { string tag_idx[t] : set_off[i] <= t < set_off[i+1] }
 *
 * If tag_idx is NULL, tag t is vocabulary string t (n_tags == n_vocab).
 * Repeated tags in a set are allowed (a set is a set: they do not change its
 * signature).  Sizes are given explicitly so the same struct can describe
 * device-resident arrays (tm_match_batch_device):
 *   n_bytes = vocab_off[n_vocab], n_tags = set_off[n_sets], set_off[0] = 0,
 * offsets non-decreasing, tag_idx[t] < n_vocab.  tm_build and tm_encode
 * validate all of this on the host (TM_EINVAL).  The match calls check pointers,
 * sizes and the end points on the host and leave the O(n) checks (monotone
 * offsets, indices in range) to the query encoder kernels, which never read
 * out of bounds: a malformed batch fails with TM_EINVAL and no result, on both
 * tm_match_batch and tm_match_batch_device, and the handle stays usable.
 */
typedef struct {
    const uint8_t *vocab_bytes; /* n_bytes bytes (may be NULL if n_bytes == 0)  */
    const uint64_t *vocab_off;  /* n_vocab + 1 byte offsets                      */
    const uint32_t *tag_idx;    /* n_tags vocabulary indices, or NULL (identity) */
    const uint64_t *set_off;    /* n_sets + 1 offsets into the tag list          */
    uint64_t n_bytes;
    uint64_t n_vocab;
    uint64_t n_tags;
    uint64_t n_sets;
    /* Pre-hashed vocabulary (SURVEY 8(b) "n_tags pre-hashed tags"; 8(d): the throughput protocol
     * times pre-hashed query tags): NULL, or n_vocab values FNV-1a-64(bytes of string v) (DESIGN.md
     * reading R1, the hash tm_encode applies to the bytes).  When given, vocab_bytes must be NULL,
     * n_bytes 0 and vocab_off is ignored (may be NULL); with tag_idx NULL the hashes are the tags.
     * Accepted by the match calls (tm_match_batch*, tm_match_batch_sharded_device), tm_encode and a
     * config's plan_sample; calls that keep tag strings (tm_build, tm_add_sets, tm_stream_replay,
     * exact mode) fail with TM_EINVAL.  Device-resident on tm_match_batch_device. */
    const uint64_t *vocab_hash;
} tm_tagsets;

typedef struct {
    uint32_t max_partition; /* MAX_P; 0 -> TM_DEFAULT_MAX_PARTITION;
                               TM_NO_PARTITIONING -> one empty-mask partition        */
    int32_t device;         /* CUDA device ordinal; -1 -> the calling thread's current */
    uint32_t n_shards;      /* 0/1: this handle holds every partition; k > 1: it holds
                               only the partitions assigned to `shard` (sec. "Shards") */
    uint32_t shard;         /* 0 <= shard < n_shards                                   */
    uint32_t tile_filter;   /* 0 = Alg. 4 common prefix of each 32-set tile (default);
                               1 = AND of the tile's signatures (lossless strengthening);
                               2 = no pre-filter (plain Alg. 3 scan)                   */
    uint32_t row_order;     /* order of the sets inside a partition:
                               0 = lexicographic (default);
                               1 = Alg. 1's balanced splits continued inside the partition
                                   down to groups of <= 8 sets, depth-first (R18);
                                   requires tile_filter 1 or 2 (Alg. 4's first/last prefix
                                   is only sound for lexicographic order)            */
    uint32_t exact;         /* 1 = exact subset post-check ("the system ...
                               can perform an additional exact subset check"): a pair is
                               kept only if every tag string of the entry's set occurs in
                               the query, which removes Bloom false positives; 0 = the
                               Bloom result (default)                                  */
    uint32_t n_gpus;        /* in-process multi-GPU database (one process drives several GPUs,
                               no launcher needed; sec. "Multi-GPU"): 0/1 = one device
                               (`device`); k > 1 = k sub-databases on device_ids[0..k)  */
    uint32_t shard_mode;    /* how a multi-GPU database uses its GPUs (n_gpus > 1, or one process
                               per GPU with n_shards > 1): TM_SHARD_PARTITIONED (default) or
                               TM_SHARD_REPLICATED (see below)                          */
    uint32_t reserved;      /* must be 0                                               */
    const int32_t *device_ids; /* n_gpus device ordinals, or NULL for 0 .. n_gpus-1; a device may
                               repeat (several sub-databases on one GPU: functional testing) */
    const tm_tagsets *plan_sample; /* optional host query sample (e.g. 10K queries of the expected
                               stream) for the partition -> shard plan: partition p
                               weighs |P_p| x (sample queries routed to p); NULL: |P_p| x 4^-|mask_p| */
} tm_config;

/* shard_mode values.
 * TM_SHARD_PARTITIONED: the partitions are split into contiguous ranges of the partition table
 *   of ~equal estimated work, one per GPU ("partition an extremely large tagset
 *   table on multiple GPUs"); every GPU matches the whole batch against its partitions and the
 *   (query, key) pairs are exchanged so that GPU g holds the queries of owner range g
 *   (tm_owner_range), where they are merged (sorted / de-duplicated).
 * TM_SHARD_REPLICATED: every GPU holds the whole table and matches owner range g of the batch;
 *   no exchange ("maximal inter-GPU parallelism in the case of full replication"). */
#define TM_SHARD_PARTITIONED 0u
#define TM_SHARD_REPLICATED 1u

/* Result pairs in host memory, allocated by the library (pinned), released by
 * tm_pairs_free().  query[i] is a 0-based index into the call's query batch. */
typedef struct {
    uint64_t n;
    uint32_t *query;
    uint32_t *key;
    void *priv_; /* library bookkeeping; do not touch */
} tm_pairs;

/* Result as per-query key lists in host memory (match / match-unique
 * return, for each query, its keys), allocated by the library (pinned), released
 * by tm_csr_free().  Query j's keys are key[q_off[j] .. q_off[j+1]), ascending;
 * q_off[0] = 0 and q_off[n_queries] = n.  The same pairs as tm_pairs, in the
 * same order, with 4 B per pair + 8 B per query instead of 8 B per pair. */
typedef struct {
    uint64_t n_queries;
    uint64_t n;
    uint64_t *q_off; /* n_queries + 1 */
    uint32_t *key;   /* n */
    void *priv_;     /* library bookkeeping; do not touch */
} tm_csr;

/* Result pairs in device memory owned by the tm_db; valid until the next call
 * on the same handle or tm_free. */
typedef struct {
    uint64_t n;
    uint32_t *query; /* device pointer */
    uint32_t *key;   /* device pointer */
} tm_dev_pairs;

/* Build the database from n_sets tag sets with their keys (add-set* +
 * consolidate).
 *   sets    : host arrays, see tm_tagsets.
 *   key_off : host, n_sets + 1 non-decreasing offsets into keys (key_off[0] = 0)
 *             -- set i's keys are keys[key_off[i] .. key_off[i+1]) -- or NULL,
 *             meaning exactly one key per set, keys[i] (add-set semantics).
 *   keys    : host, uint32 keys ("a link to application data").
 *   cfg     : may be NULL (all defaults).
 *   out     : receives the new handle on TM_OK.
 * Sets with identical signatures share one row of the tagset table; their key
 * lists are concatenated (multiplicity kept; reading R10).
 * Errors: TM_EINVAL (NULL / inconsistent arrays, bad cfg), TM_ERANGE (more than
 * 2^32-1 sets, keys or queries), TM_ECUDA, TM_ENOMEM. */
tm_status tm_build(const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys, const tm_config *cfg,
                   tm_db **out);

/* match (unique = 0) or match-unique (unique = 1) of a batch of queries
 * (PAPER.md:94).  queries: host arrays.  On TM_OK *out owns the sorted pairs
 * (release with tm_pairs_free).  The call copies the queries to the GPU, runs
 * the whole path on the handle's stream, and copies the pairs back.
 * Errors: TM_EINVAL, TM_ERANGE, TM_ECUDA, TM_ENOMEM. */
tm_status tm_match_batch(tm_db *db, const tm_tagsets *queries, int unique, tm_pairs *out);

/* tm_match_batch with the result as per-query key lists (tm_csr): the query
 * offsets are found on the GPU (one binary search per query over the sorted
 * pairs) and only the keys and the offsets are copied back.
 * Errors: as tm_match_batch. */
tm_status tm_match_batch_csr(tm_db *db, const tm_tagsets *queries, int unique, tm_csr *out);

/* Same as tm_match_batch with the query arrays already resident in device
 * memory of the handle's device (pointers in *queries are device pointers;
 * the struct itself is host memory) and the result left in device memory.
 * stream: a cudaStream_t to run on, or NULL for the handle's own stream.
 * The call returns after the pair count is known (it synchronizes the stream). */
tm_status tm_match_batch_device(tm_db *db, const tm_tagsets *queries, int unique, tm_dev_pairs *out,
                                void *stream);

void tm_pairs_free(tm_pairs *p); /* NULL-safe; resets *p */
void tm_csr_free(tm_csr *c);     /* NULL-safe; resets *c */
void tm_free(tm_db *db);         /* NULL-safe */
const char *tm_strerror(tm_status s);
const char *tm_last_error(void); /* thread-local detail of the last failure ("" if none) */
uint32_t tm_abi_version(void);
/* Identifier of the library build: a hash of its CUDA/C++ sources, fixed at compile time
 * (lets measurement scripts tie a profile to the exact kernels it was taken on). */
const char *tm_build_id(void);

/* ------------------------------------------- add-set / remove-set / consolidate --- */
/*
 * The paper's interface (Table 2): add-set(set, key) and remove-set(set, key)
 * "are not immediately effective and instead are staged in a temporary index and become
 * effective only after a call to the consolidate function", which builds the partition and
 * tagset tables (Algorithm 1).  tm_create makes an empty, mutable database
 * (matches see the last consolidated state: initially empty); tm_build's handles are not
 * mutable (TM_ESTATE).  A set is given as n_tags tag strings bytes[tag_off[t] .. tag_off[t+1])
 * (tag_off[0] = 0); repeated tags do not count, order does not matter.  The database is a
 * multiset of (set, key) entries: add-set adds one instance; remove-set removes one instance
 * of an identical entry if there is one (else nothing; reading R20).  Staged
 * operations are applied in call order by tm_consolidate, which then rebuilds the GPU tables
 * (the same encode / sort / Alg. 1 / layout as tm_build; on failure the handle keeps its
 * tables and the operations stay staged).  The library keeps the entries on the host.
 */
tm_status tm_create(const tm_config *cfg, tm_db **out);
tm_status tm_add_set(tm_db *db, const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags, uint32_t key);
tm_status tm_remove_set(tm_db *db, const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags, uint32_t key);
/* add-set for every (set i, key) of a batch (key_off / keys as tm_build) */
tm_status tm_add_sets(tm_db *db, const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys);
tm_status tm_consolidate(tm_db *db);
/* staged operations and live entries (instances) of a mutable handle */
tm_status tm_pending(const tm_db *db, uint64_t *n_staged, uint64_t *n_live);

/* ---------------------------------------------------------- test hooks --- */

/* Bloom signatures of host tag sets computed on `device` (-1 = current):
 * sig_out (host) receives n_sets * 3 uint64 words, set i at [3i, 3i+3), with
 * position p (0..191) in word p>>6 at bit 63-(p&63) (reading R3).
 * The hash is DESIGN.md reading R1: FNV-1a-64 of the tag bytes, then the
 * first 7 SplitMix64 outputs seeded with it, each mapped to floor(z*192/2^64). */
tm_status tm_encode(const tm_tagsets *sets, uint64_t *sig_out, int device);

typedef struct {
    /* database (tm_build) */
    uint64_t n_sets;       /* input sets                                    */
    uint64_t n_entries;    /* (set, key) entries = keys                      */
    uint64_t n_unique;     /* distinct signatures = rows holding a set       */
    uint64_t n_rows;       /* rows incl. padding (each partition padded to 32) */
    uint64_t n_partitions; /* partitions held by this handle                 */
    uint64_t n_partitions_total; /* partitions of the whole database (all shards) */
    double build_ms;
    /* last match call */
    uint64_t n_queries;
    uint64_t routed;           /* (query, partition) pairs forwarded by Alg. 2       */
    uint64_t candidate_pairs;  /* sum over routed (q, p) of |P| (pairs Alg. 3 covers) */
    uint64_t tile_tests;       /* (32-set tile, query) pre-filter tests (Alg. 4)     */
    uint64_t pair_checks;      /* (set, query) subset checks after the pre-filter    */
    uint64_t matched_sets;     /* (set, query) matches                               */
    uint64_t emitted_pairs;    /* (query, key) pairs before merge                    */
    uint64_t result_pairs;     /* pairs returned                                     */
    uint64_t work_items;       /* (partition, set range, query chunk) items          */
    uint64_t retries;          /* capacity-overflow re-runs in the last call          */
    double encode_ms, route_ms, scan_ms, merge_ms, total_ms; /* CUDA-event stage times */
    uint32_t scan_launches;    /* scan-kernel launches in the last call               */
    uint32_t kernel_launches;  /* library kernel launches in the last call (CUB excluded) */
    uint64_t exact_checked;    /* exact mode: (query, entry) Bloom matches checked      */
    uint64_t exact_kept;       /* exact mode: ... that are exact subsets                  */
    uint32_t scan_variant;     /* scan-kernel variant of the last call */
    uint32_t tuning;           /* 1: the handle is still timing variants for batches of this size
                                  (ceil log2 class), so later calls may run other variants */
    /* shard exchange of the last sharded call (tm_match_batch_sharded_device; 0 otherwise) */
    uint64_t xchg_send_bytes;  /* (query, key) pair bytes this handle sent to other owners        */
    uint64_t xchg_recv_bytes;  /* ... and received from them                                      */
    double xchg_ms;            /* CUDA-event time of count all-gather + exchange + owner merge    */
    double local_ms;           /* CUDA-event time of the local S1-S8 part of a sharded call        */
    uint32_t max_partition;    /* MAX_P the database was partitioned with (TM_AUTO_MAX_PARTITION resolved) */
    uint32_t n_gpus;           /* GPUs behind the handle (1, or n_gpus of an in-process multi-GPU database) */
} tm_stats_t;

tm_status tm_stats(const tm_db *db, tm_stats_t *out);

/* Partition table of the handle in Algorithm 1's acceptance order
 * (FIFO work queue).  masks: n_partitions*3 words (layout as
 * tm_encode); sizes: n_partitions set counts (distinct signatures); either
 * may be NULL.  n_partitions via tm_stats. */
tm_status tm_partitions(const tm_db *db, uint64_t *masks, uint64_t *sizes);

/* Signatures (layout as tm_encode) of the distinct sets of partition p in
 * the tagset table's order (lexicographic). sig_out: sizes[p]*3. */
tm_status tm_partition_sigs(const tm_db *db, uint64_t p, uint64_t *sig_out);

/* ------------------------------------------------------------- shards --- */
/*
 * Partition sharding over G GPUs ("partition an extremely large
 * tagset table on multiple GPUs"), one process per GPU.  Every rank
 * calls tm_build on the same input with cfg.n_shards = G, cfg.shard = rank:
 * all ranks compute the same Alg. 1 table and each keeps the partitions the
 * deterministic plan (tm_shard_plan) assigns to it.  A call matches the whole
 * batch against the local partitions; the pairs are then exchanged so that
 * rank g owns queries [tm_owner_range(Q, G, g)) and returns that slice of the
 * global sorted result (for match-unique, de-duplicated across shards).
 * The exchange is NCCL (all-gather of counts + grouped send/recv over
 * NVLink); libnccl.so.2 is loaded at run time (TM_NCCL_LIB overrides the path).
 */

/* Query owner ranges: owner g holds queries [floor(Q*g/G), floor(Q*(g+1)/G)). Host only. */
tm_status tm_owner_range(uint64_t n_queries, uint32_t n_owners, uint32_t owner, uint64_t *lo, uint64_t *hi);

/* Partition -> shard plan (host only, deterministic): the partitions, in table
 * order, are cut into n_shards contiguous ranges of ~equal estimated work w_p = sizes[p] x
 * routed[p] (routed[p] = sample queries routed to p), or, with routed NULL or all zero,
 * w_p = sizes[p] x 4^-|mask_p| (a mask bit is in a query with probability ~1/4).  Partition p
 * goes to the shard whose share of the total work contains the middle of p's work.
 * masks: n_parts*3 words, sizes: n_parts set counts, routed: n_parts or NULL,
 * owner_out: n_parts shard ids (non-decreasing). */
tm_status tm_shard_plan(const uint64_t *masks, const uint64_t *sizes, const uint64_t *routed, uint64_t n_parts,
                        uint32_t n_shards, uint32_t *owner_out);

/* Exchange plan of one rank (host only): counts[s * n_ranks + d] = pairs rank s holds for owner
 * d (the all-gathered count matrix).  send_off[0..n_ranks]: where this rank's pairs for owner d
 * start in its sorted local result (prefix over d of counts[rank][d]); recv_off[0..n_ranks]:
 * where pairs from source s land in this rank's receive buffer (prefix over s of
 * counts[s][rank]); send_off[n_ranks] / recv_off[n_ranks] = totals. */
tm_status tm_exchange_plan(const uint64_t *counts, uint32_t n_ranks, uint32_t rank, uint64_t *send_off,
                           uint64_t *recv_off);

/* Algorithm 1 on the host (test hook, no GPU): signatures sigs[n*3] (any
 * order, duplicates allowed) are sorted and de-duplicated, then partitioned
 * (readings R7/R8).  Outputs, each with capacity for n entries:
 * masks_out[P*3], sizes_out[P], sigs_out[U*3] (may be NULL: the distinct
 * signatures partition by partition, lexicographic inside), *n_parts_out = P,
 * *n_unique_out = U. */
tm_status tm_partition_host(const uint64_t *sigs, uint64_t n, uint32_t max_partition, uint64_t *masks_out,
                            uint64_t *sizes_out, uint64_t *sigs_out, uint64_t *n_parts_out, uint64_t *n_unique_out);

/* The last call's merged local result as sorted (query << 32 | key) uint64 in
 * device memory (valid until the next call on the handle). */
tm_status tm_last_result(const tm_db *db, const uint64_t **pairs, uint64_t *n);

/* counts_out[g] (host) = pairs of the last local result owned by g, for
 * n_owners contiguous owner ranges of the last call's batch. */
tm_status tm_shard_counts(tm_db *db, uint32_t n_owners, uint64_t *counts_out);

/* Owner-side merge: sort n device pairs (query << 32 | key) received from all
 * shards, de-duplicate if unique, and return them split in device memory
 * owned by the handle.  n_queries = the batch size (sort width). */
tm_status tm_shard_merge(tm_db *db, const uint64_t *pairs, uint64_t n, uint64_t n_queries, int unique,
                         tm_dev_pairs *out, void *stream);

/* In-process multi-GPU databases (tm_config.n_gpus > 1).  tm_build builds one sub-database per
 * device (in parallel, one host thread each); tm_match_batch / tm_match_batch_csr run the batch
 * on all of them and return one result, sorted by (query, key) as always.  The exchange of a
 * partitioned database is fused into the scan: each GPU's scan kernel stores every (query, key)
 * pair straight into the query owner's receive region for that GPU (peer memory over NVLink;
 * peer access is enabled at build), and each owner compacts and merges its regions on its GPU.
 * Without peer access between some pair of GPUs, for more than 8 GPUs, in exact mode, or with
 * TM_NO_FUSED_EXCHANGE=1 in the environment, each GPU merges locally and the owners pull their
 * pieces with peer copies (cudaMemcpyPeerAsync).
 * tm_stats sums the counters and takes the maximum of the times over the GPUs.  Calls taking
 * device pointers (tm_match_batch_device, the shard hooks) return TM_ESTATE on such a handle.
 * tm_group_size: number of sub-databases (1 for a single-GPU handle); tm_group_member: the
 * read-only sub-database g (for tm_stats / tm_partitions; owned by the group). */
tm_status tm_group_size(const tm_db *db, uint32_t *n);
tm_status tm_group_member(const tm_db *db, uint32_t g, const tm_db **sub);

/* NCCL communicator of a shard handle.  id: 128 bytes from tm_nccl_unique_id
 * on one rank, distributed by the caller (e.g. torch.distributed). */
tm_status tm_nccl_unique_id(void *id_out, uint64_t len);
tm_status tm_comm_init(tm_db *db, const void *id, uint64_t len, int nranks, int rank);

/* match / match-unique of a batch resident in device memory (the same batch on
 * every rank) against this rank's partitions, exchanged over NCCL: *out holds
 * this rank's owner slice of the global sorted result (query ids global).
 * shard_mode TM_SHARD_REPLICATED (every rank holds the whole table): the rank matches
 * only its owner range of the batch, no exchange and no communicator needed. */
tm_status tm_match_batch_sharded_device(tm_db *db, const tm_tagsets *queries, int unique, tm_dev_pairs *out,
                                        void *stream);

/* ----------------------------------------------------------- streaming --- */
/*
 * Streaming front-end with batch timeout: queries are
 * submitted one at a time; a dispatcher thread closes the open batch when it
 * holds max_batch queries or its oldest query has waited timeout_us (0 = no
 * timeout), runs it through tm_match_batch while the next batch fills, and
 * publishes per-batch results.  One stream per tm_db; the stream owns the
 * handle's calls while open (do not call tm_match_batch* concurrently).
 */
typedef struct tm_stream tm_stream;

typedef struct {
    uint32_t max_batch;  /* dispatch when this many queries are waiting (> 0)        */
    uint32_t timeout_us; /* dispatch when the oldest has waited this long (0 = never) */
    int32_t unique;      /* 0 = match, 1 = match-unique                               */
    uint32_t reserved;   /* must be 0                                                 */
} tm_stream_config;

/* One dispatched batch: query i of the batch has ticket tickets[i] and keys
 * keys[key_off[i] .. key_off[i+1]) (sorted); times are steady-clock ns.
 * Owned by the library until tm_stream_result_free. */
typedef struct {
    uint64_t n_queries;
    const uint64_t *tickets;
    const uint64_t *submit_ns;
    const uint64_t *key_off;
    const uint32_t *keys;
    uint64_t dispatch_ns, done_ns;
    void *priv_;
} tm_stream_result;

tm_status tm_stream_open(tm_db *db, const tm_stream_config *cfg, tm_stream **out);
/* one query: n_tags tag strings bytes[tag_off[t] .. tag_off[t+1]); *ticket = its id */
tm_status tm_stream_submit(tm_stream *st, const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags,
                           uint64_t *ticket);
/* next completed batch (n_queries = 0 if none); wait = 1 blocks until one is ready
 * or nothing is in flight.  Errors of a failed batch are returned here. */
tm_status tm_stream_poll(tm_stream *st, int wait, tm_stream_result *out);
void tm_stream_result_free(tm_stream_result *r);
/* dispatch the open batch now and wait until every submitted query is published */
tm_status tm_stream_flush(tm_stream *st);
/* open-loop load generator (test / experiment hook): submits query i of q (host
 * arrays) at arrival_ns[i] after the call starts; returns when all are submitted */
tm_status tm_stream_replay(tm_stream *st, const tm_tagsets *q, const uint64_t *arrival_ns);
void tm_stream_close(tm_stream *st); /* dispatches what is open, joins the thread, frees */

#ifdef __cplusplus
}
#endif
#endif /* TAGMATCH_H */
