// tm_db.h -- the database handle and host-side error plumbing (internal).
#pragma once

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <functional>
#include <new>
#include <string>
#include <vector>

#include "tm_internal.h"

namespace tmb {

struct Store;  // add-set / remove-set staging of a mutable handle (tm_store.cpp)

struct CudaFail {
    cudaError_t e;
    const char *what;
    int line;
};

#define TMCK(call)                                                       \
    do {                                                                 \
        cudaError_t _e = (call);                                         \
        if (_e != cudaSuccess) throw ::tmb::CudaFail{_e, #call, __LINE__}; \
    } while (0)

struct StatusFail {
    tm_status s;
    std::string msg;
};

[[noreturn]] inline void fail(tm_status s, const std::string &m) { throw StatusFail{s, m}; }

// Device buffer owned by one object: move-only, freed by its destructor (or release()), so no
// member of a handle can be missed on tm_free (res_off leaked).
struct DevBuf {
    void *p = nullptr;
    size_t cap = 0;
    DevBuf() = default;
    DevBuf(const DevBuf &) = delete;
    DevBuf &operator=(const DevBuf &) = delete;
    DevBuf(DevBuf &&o) noexcept : p(o.p), cap(o.cap) {
        o.p = nullptr;
        o.cap = 0;
    }
    DevBuf &operator=(DevBuf &&o) noexcept {
        if (this != &o) {
            release();
            p = o.p;
            cap = o.cap;
            o.p = nullptr;
            o.cap = 0;
        }
        return *this;
    }
    ~DevBuf() { release(); }
    template <class T>
    T *as() const { return static_cast<T *>(p); }
    // grows (never shrinks); the caller guarantees the stream is idle w.r.t. the old contents
    void ensure(size_t bytes) {
        if (bytes <= cap) return;
        if (p) TMCK(cudaFree(p));
        p = nullptr;
        cap = 0;
        size_t want = std::max<size_t>(bytes + bytes / 4, 256);
        cudaError_t e = cudaMalloc(&p, want);
        if (e != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
            if (e == cudaErrorMemoryAllocation) fail(TM_ENOMEM, "device allocation of " + std::to_string(want) + " bytes failed");
            throw CudaFail{e, "cudaMalloc", __LINE__};
        }
        cap = want;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        cap = 0;
    }
};

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (dev >= 0 && dev != prev) TMCK(cudaSetDevice(dev));
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

extern thread_local std::string g_err;

// NVTX range for the duration of a scope (stage names in nsys / ncu timelines; free when no
// tool is attached).
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

}  // namespace tmb

using namespace tmb;

struct tm_db {
    int device = 0;
    cudaStream_t stream = nullptr;
    cudaEvent_t ev[6] = {};
    tm_config cfg{};
    int scan_grid = 0;
    // scan-kernel variant: forced by TM_SCAN_VARIANT, else tuned per batch-size class
    // (floor(log2 Q): the best variant depends on how many queries share a partition) on the
    // first calls of that class, by kernel ns per decision (filter tests + pair checks) among kTune
    static constexpr int kClasses = 33;
    int variant[kClasses], tune_calls[kClasses] = {};
    double tune_cost[kClasses][kScanVariants] = {};
    const int *tune = kTune;      // the candidates of this table (kTune, or kTuneDense without a pre-filter)
    int call_variant = kTune[0];  // the variant the last call launched
    int call_class = 0;           // the batch-size class of the last call
    bool call_tunes = false;      // the last call is a tuning sample
    tm_db() {
        for (int &v : variant) v = kTune[0];
    }
    void set_tune(const int *t) {
        tune = t;
        call_variant = t[0];
        for (int &v : variant) v = t[0];
    }
    int grid_of[kScanVariants] = {};
    // database (device)
    uint64_t n_sets = 0, n_entries = 0, n_unique = 0, n_rows = 0, n_parts = 0, n_parts_total = 0;
    DevBuf planes;   // 3 x rows u64
    DevBuf tand;     // 3 x (rows / 32) u64: AND of each tile's real rows
    DevBuf wsel;     // rows u8: pre-check word per row (scan variant 5), made on first use
    DevBuf wwords;   // rows x uint2: those two words (scan variant 14)
    bool wsel_ok = false;
    DevBuf key_off;  // rows + 1 u32
    DevBuf keys;     // K u32
    DevBuf masks;    // P x 3 u64
    DevBuf part_row; // P + 1 u32
    DevBuf part_n;   // P u32
    std::vector<uint64_t> h_masks, h_sizes;
    std::vector<uint32_t> h_part_row;
    double build_ms = 0;
    // per-call workspace
    DevBuf in_bytes, in_voff, in_tidx, in_soff, in_vhash;  // host-API staging of the queries
    DevBuf vsig, qplanes, bm, word_off, qidx, qoff, item_cnt, item_off, out, out_alt, res_q, res_k, res_off, tmp, ctr;
    // pipelined tm_match_batch_csr: the D2H of query range k overlaps the GPU work of range k + 1
    cudaStream_t xstream = nullptr;  // copy stream (created on first use)
    cudaEvent_t xev[3] = {};         // [0], [1]: copy of the key buffer res_k / res_kb done; [2]: range matched
    DevBuf res_kb, res_qb;           // the second key / query buffers
    uint64_t pipe_pairs_hint = 0;    // pairs of the largest pipelined result so far: sizes its pinned block
    DevCounters *h_ctr = nullptr;  // pinned
    unsigned long long *h_nuniq = nullptr;
    unsigned long long cap_qidx = 0, cap_out = 0;
    // last call's merged result before the split (sorted (q<<32|key)), for the shard exchange
    uint64_t *last_sorted = nullptr;
    uint64_t last_n = 0, last_Q = 0;
    uint64_t last_qlo = 0, last_qn = 0;  // the query range the last call matched
    // shard layer (tm_shard.cu)
    uint64_t *merged = nullptr;  // merge_pairs: the owner's sorted (q<<32|key) pairs (mq/mk split)
    uint64_t merged_n = 0;
    // in-process multi-GPU database (tm_group.cu): sub-databases, one per device
    std::vector<tm_db *> subs;
    bool fused_ok = false;  // group: every pair of its GPUs has peer access (the fused exchange)
    uint64_t fx_cap = 0;    // group: receive-region capacity of the last call (pairs)
    // a sub-database's fused-exchange target for the current call (G = 0: none)
    struct {
        uint32_t G = 0;
        uint32_t xstart[kMaxOwners] = {};
        uint64_t *xout[kMaxOwners] = {};
        unsigned long long xcap = 0;
        uint64_t counts[kMaxOwners] = {};  // pairs this GPU wrote to each owner in the last call
    } fx;
    DevBuf xfcnt, xfin;  // fused exchange: counters per owner; an owner's compacted receive buffer
    unsigned long long *h_fx = nullptr;  // pinned copy of xfcnt
    // mutable handle (tm_create; tm_store.cpp): the entry multiset + staged operations
    Store *store = nullptr;
    std::vector<int32_t> store_devices;
    void *nccl_comm = nullptr;
    int nranks = 1, rank = 0;
    DevBuf xcounts, xall, xrecv, xalt, mq, mk;
    // exact mode (tm_exact.cu)
    uint64_t x_nvocab = 0;
    DevBuf xv_bytes, xv_off, xv_hash, xv_pos, xv_canon, xs_off, xs_ids, xk_off, xk_keys;
    DevBuf xq_canon, xq_ids, xflag, xcnt, xkoff, xkcnt;
    tm_stats_t st{};
};

namespace tmb {
void *cub_tmp(tm_db *db, size_t bytes);
// encoded: the handle's query planes already hold this batch's signatures (an earlier query range
// of the same call): S1 is skipped
uint64_t match_core(tm_db *db, const tm_tagsets *q, int unique, cudaStream_t s, uint64_t qlo = 0,
                    uint64_t qn = ~0ULL, bool encoded = false);
void finish_timing(tm_db *db, cudaStream_t s);
tm_status translate(const CudaFail &f);
int check_device(int dev);
void check_tagsets_device(const tm_tagsets *t);
void check_tagsets_host(const tm_tagsets *t, const char *what);
void require_strings(const tm_tagsets *t, const char *what);  // TM_EINVAL for a pre-hashed vocabulary
int bits_for(uint64_t n);
// partition -> shard plan of the handle's config (tm_shard.cu): contiguous ranges of ~equal
// estimated work; one shard: all 0; replicated: all = this handle's shard (it keeps everything)
std::vector<uint32_t> plan_shards(tm_db *db, const std::vector<Partition> &parts);
std::vector<uint32_t> plan_ranges(const std::vector<double> &w, uint32_t n_shards);
std::vector<double> model_weights(const std::vector<Partition> &parts);
void exchange_plan(const uint64_t *counts, uint32_t G, uint32_t r, uint64_t *send_off, uint64_t *recv_off);
inline uint64_t owner_start(uint64_t Q, uint32_t G, uint32_t g) { return (Q * g) / G; }
// sorts / de-duplicates n received (q<<32|key) pairs into db->mq / db->mk (db->merged: the sorted
// u64 pairs); synchronous
uint64_t merge_pairs(tm_db *db, uint64_t *in, uint64_t n, uint64_t Q, int unique, cudaStream_t s);
// db->xcounts[g] = pairs of the last local result owned by g (G owner ranges of the last batch)
void owner_counts(tm_db *db, uint32_t G, cudaStream_t s);
tm_tagsets upload_queries(tm_db *db, const tm_tagsets *q, cudaStream_t s);
// pinned host result blocks (cached; tm_api.cu)
struct PinnedBlock {
    void *p;
    size_t cap;
};
PinnedBlock *pinned_get(size_t bytes);
void pinned_put(PinnedBlock *b);
// in-process multi-GPU databases (tm_group.cu)
void group_build(tm_db *top, const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys,
                 const tm_config *cfg);
void group_match(tm_db *top, const tm_tagsets *q, int unique, tm_pairs *pout, tm_csr *cout);
void group_stats(const tm_db *top, tm_stats_t *out);
tm_db *build_db(const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys, const tm_config *cfg);
// consolidate(): rebuild the handle's tables in place from sets / keys (one key per set)
void rebuild(tm_db *db, const tm_tagsets *sets, const uint32_t *keys, const tm_config *cfg);
void store_destroy(tm_db *db);
void destroy_db(tm_db *db);
void shard_destroy(tm_db *db);
// exact subset post-check (tm_exact.cu)
void exact_build(tm_db *db, const uint8_t *d_bytes, uint64_t n_bytes, const uint64_t *d_voff, uint64_t V,
                 const uint32_t *d_tidx, const uint64_t *d_soff, uint64_t N, uint64_t n_tags,
                 const uint64_t *h_key_off, const uint32_t *h_keys);
uint64_t exact_filter(tm_db *db, const tm_tagsets *q, uint64_t n, cudaStream_t s);
// consolidate() on the GPU (tm_build.cu): distinct signatures, Alg. 1, row order, table, masks, keys
void build_gpu(tm_db *db, uint64_t N, const uint64_t *s0, const uint64_t *s1, const uint64_t *s2,
               const uint32_t *idx, const uint64_t *h_key_off, const uint32_t *h_keys,
               const std::function<void(const char *)> &mark);
}  // namespace tmb

#define TM_API_BEGIN \
    try {            \
        tmb::set_error("");
#define TM_API_END                                                   \
    }                                                                \
    catch (const tmb::StatusFail &f) {                                \
        tmb::set_error(f.msg);                                        \
        return f.s;                                                  \
    }                                                                \
    catch (const tmb::CudaFail &f) {                                  \
        return tmb::translate(f);                                     \
    }                                                                \
    catch (const std::bad_alloc &) {                                 \
        tmb::set_error("host allocation failed");                    \
        return TM_ENOMEM;                                            \
    }                                                                \
    catch (...) {                                                    \
        tmb::set_error("unexpected exception");                      \
        return TM_ESTATE;                                            \
    }

