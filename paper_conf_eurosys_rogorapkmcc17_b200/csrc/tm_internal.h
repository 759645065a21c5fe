// tm_internal.h -- internal declarations of the TagMatch B200 library (not part of the ABI).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "tagmatch.h"

namespace tmb {

// ---------------------------------------------------------------- layout --
// Signatures are 3 x 64-bit words; position p is word p>>6, bit 63-(p&63)
// (reading R3).  In HBM they live as three SoA planes so that a warp
// reading 32 consecutive rows issues fully coalesced 256-B loads per plane.
constexpr int kWords = 3;
constexpr int kBits = 192;
constexpr int kHashes = 7;
constexpr int kTile = 32;  // rows per warp tile (= one warp, Alg. 4 "thread block")

// Scan-kernel geometry.
constexpr int kScanWarps = 4;      // warps per CTA
constexpr uint32_t kUnitTarget = 8; // filtered path: items of fewer blocks are split to this many units
constexpr int kMaxOwners = 8;       // fused exchange: GPUs of an in-process group the scan can emit to
#ifndef TM_CHUNK
#define TM_CHUNK 640
#endif
constexpr int kChunk = TM_CHUNK;   // queries per work item (per-partition batch); 640 fits 7 CTAs/SM of shared memory and measured 1.3% faster than 512 (profiles/r1v34_ab.txt)
constexpr int kSmallBatch = 8;     // partition batches up to this size take the unfiltered streaming path
constexpr int kRangeRows = 8192;    // default rows per work item (multiple of 256; TM_RANGE_ROWS)
constexpr int kScanVariants = 19;    // k_scan variants (TM_SCAN_VARIANT)
constexpr int kTune[] = {14, 8};  // variants the handle times on its first calls (first = default)
constexpr int kTuneN = 2;
constexpr int kTuneDense[] = {13, 9};  // tables without a pre-filter (tile_filter = 2): the dense scan
// partitions of at most kSmallPMax sets (the auto MAX_P of large tables): 128-row level-A blocks
// (C3 at 5K: scan 190.1 vs 194.3 ms; C4 at 10K 390.1 vs 397.6; C3 at 200K 285.9 vs 276.4: 256 rows
// stay for large partitions; profiles/r3u_*)
constexpr int kTuneSmallP[] = {17, 18};
constexpr uint32_t kSmallPMax = 50000;
constexpr int kTuneMinQ = 4096;     // smaller calls are not tuned (default variant kTune[0])

struct DevCounters {            // zeroed at the start of every match call
    unsigned long long n_out;   // (q,key) pairs emitted (may exceed capacity)
    unsigned long long n_items; // work items (written by the work-list kernel)
    unsigned long long item_ctr;// persistent-kernel work counter
    unsigned long long tile_tests;
    unsigned long long pair_checks;
    unsigned long long matched_sets;
    unsigned long long routed;      // R = routed (q, p) pairs
    unsigned long long candidates;  // sum |P| over routed pairs
    unsigned int input_err;         // malformed query CSR seen by the encoder (zeroed before it)
    unsigned int pad_;
};

struct ScanParams {
    const uint64_t *w0, *w1, *w2;     // db planes [rows]
    const uint64_t *t0, *t1, *t2;     // AND of each 32-row tile's real rows [rows / 32]
    const uint32_t *key_off;          // [rows+1]
    const uint32_t *keys;             // [K]
    const uint32_t *part_row;         // [P+1] padded row offsets
    const uint32_t *part_n;           // [P] real rows
    const uint64_t *q0, *q1, *q2;     // query planes [Q]
    const uint32_t *qidx;             // routed query ids, partition-major [R]
    unsigned long long qcap;          // capacity of qidx (scan is skipped if R > qcap)
    const unsigned long long *qoff;   // [P+1] offsets into qidx
    const unsigned long long *item_off; // [P+1]
    uint32_t n_parts;
    uint64_t *out;                    // (q<<32 | key) [cap]
    unsigned long long cap;
    DevCounters *ctr;
    uint32_t filter;                  // 0 prefix, 1 AND, 2 none
    const uint8_t *wsel;              // [rows] pre-check word per row (variant 5)
    const uint2 *wwords;              // [rows] the two pre-check words themselves (variant 14)
    uint32_t unit_target;             // filtered path: split items of fewer blocks to this many units
    uint32_t range_rows;              // rows per work item (multiple of 256)
    uint32_t one;                     // 1 (a run-time operand, so the FMA-pipe accumulate stays an IMAD)
    // fused exchange (n_owners > 1): pairs of query q go to xout[owner(q)] (owner(q) = last g with
    // xstart[g] <= q), reserved on the local counter xcnt[owner], at most xcap pairs per region
    uint32_t n_owners;
    uint32_t xstart[kMaxOwners];
    uint64_t *xout[kMaxOwners];
    unsigned long long *xcnt;
    unsigned long long xcap;
};

// ------------------------------------------------------------ launchers --
// All launchers are asynchronous on `s` and return the launch error.
// hashes: NULL, or the pre-hashed vocabulary (tm_tagsets.vocab_hash; bytes / off then unused)
cudaError_t launch_hash_vocab(const uint8_t *bytes, const uint64_t *off, const uint64_t *hashes, uint64_t n_vocab,
                              uint64_t n_bytes, uint64_t *vsig, unsigned int *err, cudaStream_t s);
cudaError_t launch_encode_sets(const uint64_t *vsig, const uint32_t *tag_idx, const uint64_t *set_off,
                               uint64_t n_sets, uint64_t n_tags, uint64_t n_vocab, uint64_t *w0, uint64_t *w1,
                               uint64_t *w2, unsigned int *err, cudaStream_t s);
// S2, bit-sliced Alg. 2 in two passes: pass 0 writes counts[p * NB + blk] (NB = route_blocks(n_q)),
// pass 1 scatters query ids at the scanned offsets off[p * NB + blk] into qidx (capacity cap).
uint64_t route_blocks(uint64_t n_q);
cudaError_t launch_route(int pass, const uint64_t *masks, uint32_t n_parts, const uint64_t *q0, const uint64_t *q1,
                         const uint64_t *q2, uint64_t n_q, uint32_t *counts, const unsigned long long *off,
                         uint32_t *qidx, unsigned long long cap, cudaStream_t s, uint32_t qbase = 0);
cudaError_t launch_items(const unsigned long long *word_off, uint64_t qw, const uint32_t *part_row,
                         const uint32_t *part_n, uint32_t n_parts, unsigned long long *qoff,
                         unsigned long long *item_cnt, DevCounters *ctr, uint32_t range_rows, cudaStream_t s);
uint32_t range_rows_env(uint64_t n_rows);  // TM_RANGE_ROWS (multiple of 256), else by table size
uint32_t unit_target_env();                // TM_UNIT_TARGET, else kUnitTarget
cudaError_t launch_scan(const ScanParams &p, int grid, cudaStream_t s, int variant);
void scan_debug_dump(int variant);  // variant 16: pre-check pass statistics to stderr
int scan_grid(int device, int variant);
int scan_variant_env();  // -1 = auto-tune
cudaError_t launch_word_select(const uint64_t *planes, const uint64_t *tand, uint64_t rows, uint8_t *wsel,
                               uint2 *wwords, cudaStream_t s);
cudaError_t launch_split(const uint64_t *pairs, uint64_t n, uint32_t *q, uint32_t *k, cudaStream_t s);
// q_off[i] = base + (first pair of query qlo + i), i < nq; q_off[nq] = base + n
cudaError_t launch_query_offsets(const uint64_t *pairs, uint64_t n, uint64_t qlo, uint64_t nq, uint64_t base,
                                 uint64_t *q_off, cudaStream_t s);
cudaError_t launch_gather_planes(const uint64_t *src0, const uint64_t *src1, const uint64_t *src2,
                                 const uint32_t *idx, uint64_t n, uint64_t *d0, uint64_t *d1, uint64_t *d2,
                                 cudaStream_t s);
cudaError_t launch_gather_u64(const uint64_t *src, const uint32_t *idx, uint64_t n, uint64_t *dst,
                              cudaStream_t s);
cudaError_t launch_iota(uint32_t *v, uint64_t n, cudaStream_t s);

// CUB wrappers (temp storage managed by the caller through `tmp`/`tmp_bytes`).
cudaError_t cub_exclusive_scan_u32_u64(const uint32_t *in, unsigned long long *out, uint64_t n, void *tmp,
                                      size_t *tmp_bytes, cudaStream_t s);
cudaError_t cub_exclusive_scan_u64(const unsigned long long *in, unsigned long long *out, uint64_t n, void *tmp,
                                   size_t *tmp_bytes, cudaStream_t s);
cudaError_t cub_sort_pairs_u64_u32(const uint64_t *kin, uint64_t *kout, const uint32_t *vin, uint32_t *vout,
                                   uint64_t n, void *tmp, size_t *tmp_bytes, cudaStream_t s);
cudaError_t cub_sort_keys_u64(uint64_t *k, uint64_t *kalt, uint64_t n, int end_bit, int *sel, void *tmp,
                              size_t *tmp_bytes, cudaStream_t s);
cudaError_t cub_unique_u64(const uint64_t *in, uint64_t *out, unsigned long long *n_out, uint64_t n, void *tmp,
                           size_t *tmp_bytes, cudaStream_t s);

// ---------------------------------------------------------- host build --
struct Sig {
    uint64_t w[3];
};

struct Partition {
    Sig mask;
    uint64_t begin, end;  // range in the unique-signature order produced by alg1
};

// Algorithm 1 over `n` distinct signatures given in lexicographic order.
// Writes `order` (a stable permutation: members of each partition contiguous,
// lexicographic inside) and the partitions in FIFO acceptance order.
void alg1_partition(const Sig *sigs, uint64_t n, uint32_t max_p, std::vector<uint32_t> &order,
                    std::vector<Partition> &parts);

// Reading R18: inside every partition, continue Alg. 1's balanced splits (pivot =
// unused bit with frequency closest to 50%) depth-first down to groups of <= leaf
// sets, rewriting `order` within each partition's range (P0 before P1; members
// of a group stay lexicographic).  Rows sharing a deep path share many bits,
// which strengthens the tile AND masks.
void refine_order(const Sig *sigs, std::vector<uint32_t> &order, const std::vector<Partition> &parts,
                  uint32_t leaf);

void set_error(const std::string &msg);

}  // namespace tmb
