// tm_shard.cu -- S9: partition sharding over GPUs ("partition an extremely
// large tagset table on multiple GPUs") and the result exchange over NCCL.
//
// Protocol, one process per GPU, rank g of G:
//   1. every rank builds the same Alg. 1 table and keeps the partitions the
//      deterministic plan assigns to it (tm_config.n_shards / shard);
//   2. a call matches the whole query batch against the local partitions
//      (S1-S8 on this GPU) -> pairs sorted by (query, key);
//   3. query owner ranges are contiguous: owner(q) = g with
//      floor(Q*g/G) <= q < floor(Q*(g+1)/G);  the sorted local pairs are cut at
//      the owner boundaries (binary search on the GPU);
//   4. ncclAllGather of the G x G count matrix, then grouped ncclSend/ncclRecv
//      (all-to-all-v over NVLink/NVSwitch) of the (q<<32|key) pairs to owners;
//   5. each owner re-sorts what it received (and de-duplicates for
//      match-unique), yielding its slice of the global sorted result.
// NCCL is loaded at run time (dlopen), so the library loads without it.
#include <dlfcn.h>

#include <cmath>
#include <cstring>
#include <mutex>

#include "nccl.h"
#include "tm_db.h"

namespace tmb {
namespace {

struct NcclApi {
    bool ok = false;
    std::string err;
    decltype(&ncclGetUniqueId) getUniqueId = nullptr;
    decltype(&ncclCommInitRank) commInitRank = nullptr;
    decltype(&ncclCommDestroy) commDestroy = nullptr;
    decltype(&ncclAllGather) allGather = nullptr;
    decltype(&ncclSend) send = nullptr;
    decltype(&ncclRecv) recv = nullptr;
    decltype(&ncclGroupStart) groupStart = nullptr;
    decltype(&ncclGroupEnd) groupEnd = nullptr;
    decltype(&ncclGetErrorString) errorString = nullptr;
};

NcclApi load_nccl() {
    NcclApi a;
    const char *env = getenv("TM_NCCL_LIB");
    const char *cands[] = {env, "libnccl.so.2",
                           "/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/lib/libnccl.so.2"};
    void *h = nullptr;
    for (const char *c : cands)
        if (c && (h = dlopen(c, RTLD_NOW | RTLD_GLOBAL))) break;
    if (!h) {
        a.err = "libnccl.so.2 not found (set TM_NCCL_LIB)";
        return a;
    }
#define TM_SYM(field, name)                                           \
    a.field = reinterpret_cast<decltype(a.field)>(dlsym(h, name));    \
    if (!a.field) {                                                   \
        a.err = std::string("NCCL symbol missing: ") + name;          \
        return a;                                                     \
    }
    TM_SYM(getUniqueId, "ncclGetUniqueId");
    TM_SYM(commInitRank, "ncclCommInitRank");
    TM_SYM(commDestroy, "ncclCommDestroy");
    TM_SYM(allGather, "ncclAllGather");
    TM_SYM(send, "ncclSend");
    TM_SYM(recv, "ncclRecv");
    TM_SYM(groupStart, "ncclGroupStart");
    TM_SYM(groupEnd, "ncclGroupEnd");
    TM_SYM(errorString, "ncclGetErrorString");
#undef TM_SYM
    a.ok = true;
    return a;
}

NcclApi &nccl() {
    static std::once_flag once;
    static NcclApi api;
    std::call_once(once, [] { api = load_nccl(); });
    if (!api.ok) fail(TM_ENCCL, api.err);
    return api;
}

#define TMNC(call)                                                                                  \
    do {                                                                                            \
        ncclResult_t _r = (call);                                                                   \
        if (_r != ncclSuccess) fail(TM_ENCCL, std::string("NCCL: ") + nccl().errorString(_r) + " in " #call); \
    } while (0)

// counts[g] = number of sorted (q<<32|key) pairs with owner(q) == g (one thread per owner)
__global__ void k_owner_counts(const uint64_t *__restrict__ sorted, uint64_t n, uint64_t Q, uint32_t G,
                               unsigned long long *__restrict__ counts) {
    const uint32_t g = blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= G) return;
    auto lower = [&](uint64_t key) {
        uint64_t lo = 0, hi = n;
        while (lo < hi) {
            const uint64_t mid = (lo + hi) >> 1;
            if (sorted[mid] < key) lo = mid + 1; else hi = mid;
        }
        return lo;
    };
    const uint64_t a = lower((Q * g / G) << 32);
    const uint64_t b = (g + 1 == G) ? n : lower((Q * (g + 1) / G) << 32);
    counts[g] = b - a;
}

}  // namespace

// Sort (query, key) pairs received by this owner, de-duplicate for match-unique,
// split into db->mq / db->mk.  `in` may alias db->xrecv.
uint64_t merge_pairs(tm_db *db, uint64_t *in, uint64_t n, uint64_t Q, int unique, cudaStream_t s) {
    db->xalt.ensure(std::max<uint64_t>(n, 1) * 8);
    uint64_t *sorted = in;
    size_t tb = 0;
    if (n > 1) {
        int sel = 0;
        const int end_bit = 32 + bits_for(Q);
        TMCK(cub_sort_keys_u64(in, db->xalt.as<uint64_t>(), n, end_bit, &sel, nullptr, &tb, s));
        TMCK(cub_sort_keys_u64(in, db->xalt.as<uint64_t>(), n, end_bit, &sel, cub_tmp(db, tb), &tb, s));
        sorted = sel ? db->xalt.as<uint64_t>() : in;
    }
    if (unique && n > 1) {
        uint64_t *dst = (sorted == in) ? db->xalt.as<uint64_t>() : in;
        db->xcounts.ensure(8 * 2);
        unsigned long long *d_n = db->xcounts.as<unsigned long long>();
        tb = 0;
        TMCK(cub_unique_u64(sorted, dst, d_n, n, nullptr, &tb, s));
        TMCK(cub_unique_u64(sorted, dst, d_n, n, cub_tmp(db, tb), &tb, s));
        TMCK(cudaMemcpyAsync(db->h_nuniq, d_n, 8, cudaMemcpyDeviceToHost, s));
        TMCK(cudaStreamSynchronize(s));
        n = *db->h_nuniq;
        sorted = dst;
    }
    db->mq.ensure(std::max<uint64_t>(n, 1) * 4);
    db->mk.ensure(std::max<uint64_t>(n, 1) * 4);
    TMCK(launch_split(sorted, n, db->mq.as<uint32_t>(), db->mk.as<uint32_t>(), s));
    TMCK(cudaStreamSynchronize(s));
    db->merged = sorted;
    db->merged_n = n;
    return n;
}

void owner_counts(tm_db *db, uint32_t G, cudaStream_t s) {
    db->xcounts.ensure(std::max<uint64_t>(G, 2) * 8);
    if (db->last_n == 0) {
        TMCK(cudaMemsetAsync(db->xcounts.p, 0, G * 8, s));
        return;
    }
    k_owner_counts<<<(G + 63) / 64, 64, 0, s>>>(db->last_sorted, db->last_n, db->last_Q, G,
                                                db->xcounts.as<unsigned long long>());
    TMCK(cudaGetLastError());
}

// ---------------------------------------------------------------- plan ---
// Contiguous ranges of the partition table with ~equal work: partition i goes to
// the shard whose 1/G share of the total work contains the middle of partition i's work.
std::vector<uint32_t> plan_ranges(const std::vector<double> &w, uint32_t G) {
    const size_t P = w.size();
    std::vector<uint32_t> owner(P, 0);
    if (G <= 1 || P == 0) return owner;
    double W = 0;
    for (double x : w) W += x;
    double acc = 0;
    for (size_t i = 0; i < P; ++i) {
        const double mid = W > 0 ? (acc + 0.5 * w[i]) / W : (i + 0.5) / (double)P;
        acc += w[i];
        owner[i] = std::min<uint32_t>(G - 1, (uint32_t)(mid * G));
    }
    return owner;
}

// |P| x 4^-|mask|: the chance that a query contains a mask of |mask| bits when ~1/4 of a query's
// positions are set (an 8-tag query sets ~49 of 192 bits, fn.3 / PAPER.md:132)
std::vector<double> model_weights(const std::vector<Partition> &parts) {
    std::vector<double> w(parts.size());
    for (size_t i = 0; i < parts.size(); ++i) {
        const int pc = __builtin_popcountll(parts[i].mask.w[0]) + __builtin_popcountll(parts[i].mask.w[1]) +
                       __builtin_popcountll(parts[i].mask.w[2]);
        w[i] = (double)(parts[i].end - parts[i].begin) * std::pow(0.25, pc);
    }
    return w;
}

namespace {
// queries of the config's plan sample routed to each partition (Alg. 2 on the GPU: the library's
// encoder and bit-sliced router, pass 0)
std::vector<uint64_t> sample_routes(tm_db *db, const std::vector<Partition> &parts, cudaStream_t s) {
    const tm_tagsets *smp = db->cfg.plan_sample;
    const uint64_t P = parts.size(), Qs = smp ? smp->n_sets : 0;
    std::vector<uint64_t> routed(P, 0);
    if (!Qs || !P) return routed;
    const tm_tagsets dq = upload_queries(db, smp, s);
    DevBuf vsig, planes, masks, counts;
    vsig.ensure(std::max<uint64_t>(dq.n_vocab, 1) * 24);
    planes.ensure(Qs * 24);
    uint64_t *q0 = planes.as<uint64_t>(), *q1 = q0 + Qs, *q2 = q1 + Qs;
    TMCK(launch_hash_vocab(dq.vocab_bytes, dq.vocab_off, dq.vocab_hash, dq.n_vocab, dq.n_bytes, vsig.as<uint64_t>(), nullptr, s));
    TMCK(launch_encode_sets(vsig.as<uint64_t>(), dq.n_tags ? dq.tag_idx : nullptr, dq.set_off, Qs, dq.n_tags,
                            dq.n_vocab, q0, q1, q2, nullptr, s));
    std::vector<uint64_t> hm(3 * P);
    for (uint64_t i = 0; i < P; ++i)
        for (int w = 0; w < 3; ++w) hm[3 * i + w] = parts[i].mask.w[w];
    masks.ensure(P * 24);
    TMCK(cudaMemcpyAsync(masks.p, hm.data(), P * 24, cudaMemcpyHostToDevice, s));
    const uint64_t NB = route_blocks(Qs);
    counts.ensure(P * NB * 4);
    TMCK(launch_route(0, masks.as<uint64_t>(), (uint32_t)P, q0, q1, q2, Qs, counts.as<uint32_t>(), nullptr, nullptr, 0,
                      s));
    std::vector<uint32_t> hc(P * NB);
    TMCK(cudaMemcpyAsync(hc.data(), counts.p, P * NB * 4, cudaMemcpyDeviceToHost, s));
    TMCK(cudaStreamSynchronize(s));
    for (uint64_t i = 0; i < P; ++i)
        for (uint64_t b = 0; b < NB; ++b) routed[i] += hc[i * NB + b];
    return routed;
}
}  // namespace

std::vector<uint32_t> plan_shards(tm_db *db, const std::vector<Partition> &parts) {
    const uint32_t G = std::max(1u, db->cfg.n_shards);
    if (G <= 1) return std::vector<uint32_t>(parts.size(), 0);
    // replicated: this handle keeps every partition
    if (db->cfg.shard_mode == TM_SHARD_REPLICATED) return std::vector<uint32_t>(parts.size(), db->cfg.shard);
    const std::vector<uint64_t> routed = sample_routes(db, parts, db->stream);
    std::vector<double> w(parts.size(), 0.0);
    double W = 0;
    for (size_t i = 0; i < parts.size(); ++i) W += (w[i] = (double)(parts[i].end - parts[i].begin) * routed[i]);
    if (W <= 0) w = model_weights(parts);
    return plan_ranges(w, G);
}

void exchange_plan(const uint64_t *counts, uint32_t G, uint32_t r, uint64_t *send_off, uint64_t *recv_off) {
    send_off[0] = recv_off[0] = 0;
    for (uint32_t p = 0; p < G; ++p) {
        send_off[p + 1] = send_off[p] + counts[(size_t)r * G + p];
        recv_off[p + 1] = recv_off[p] + counts[(size_t)p * G + r];
    }
}

void shard_destroy(tm_db *db) {
    if (db && db->nccl_comm) {
        NcclApi &a = nccl();
        a.commDestroy(static_cast<ncclComm_t>(db->nccl_comm));
        db->nccl_comm = nullptr;
    }
}

}  // namespace tmb

extern "C" {

tm_status tm_owner_range(uint64_t n_queries, uint32_t n_owners, uint32_t owner, uint64_t *lo, uint64_t *hi) {
    TM_API_BEGIN
    if (!lo || !hi || n_owners == 0 || owner >= n_owners) fail(TM_EINVAL, "bad owner range arguments");
    *lo = tmb::owner_start(n_queries, n_owners, owner);
    *hi = tmb::owner_start(n_queries, n_owners, owner + 1);
    return TM_OK;
    TM_API_END
}

tm_status tm_shard_plan(const uint64_t *masks, const uint64_t *sizes, const uint64_t *routed, uint64_t n_parts,
                        uint32_t n_shards, uint32_t *owner_out) {
    TM_API_BEGIN
    if ((n_parts && (!masks || !sizes || !owner_out)) || n_shards == 0) fail(TM_EINVAL, "bad shard plan arguments");
    std::vector<Partition> parts(n_parts);
    uint64_t b = 0;
    for (uint64_t i = 0; i < n_parts; ++i) {
        for (int w = 0; w < 3; ++w) parts[i].mask.w[w] = masks[3 * i + w];
        parts[i].begin = b;
        b += sizes[i];
        parts[i].end = b;
    }
    std::vector<double> w(n_parts, 0.0);
    double W = 0;
    if (routed)
        for (uint64_t i = 0; i < n_parts; ++i) W += (w[i] = (double)sizes[i] * (double)routed[i]);
    if (W <= 0) w = model_weights(parts);
    const std::vector<uint32_t> own = plan_ranges(w, n_shards);
    if (n_parts) std::memcpy(owner_out, own.data(), own.size() * 4);
    return TM_OK;
    TM_API_END
}

tm_status tm_exchange_plan(const uint64_t *counts, uint32_t n_ranks, uint32_t rank, uint64_t *send_off,
                           uint64_t *recv_off) {
    TM_API_BEGIN
    if (!counts || !send_off || !recv_off || n_ranks == 0 || rank >= n_ranks) fail(TM_EINVAL, "bad exchange plan arguments");
    tmb::exchange_plan(counts, n_ranks, rank, send_off, recv_off);
    return TM_OK;
    TM_API_END
}

tm_status tm_partition_host(const uint64_t *sigs, uint64_t n, uint32_t max_partition, uint64_t *masks_out,
                            uint64_t *sizes_out, uint64_t *sigs_out, uint64_t *n_parts_out, uint64_t *n_unique_out) {
    TM_API_BEGIN
    if ((n && !sigs) || !masks_out || !sizes_out || !n_parts_out || !n_unique_out) fail(TM_EINVAL, "NULL argument");
    if (max_partition == 0) max_partition = TM_DEFAULT_MAX_PARTITION;
    if (max_partition == TM_AUTO_MAX_PARTITION)  // reading R8b, as tm_build
        max_partition = (uint32_t)std::min<uint64_t>(200000, std::max<uint64_t>(5000, n / 30000));
    std::vector<Sig> v(n);
    for (uint64_t i = 0; i < n; ++i) v[i] = Sig{{sigs[3 * i], sigs[3 * i + 1], sigs[3 * i + 2]}};
    auto lt = [](const Sig &a, const Sig &b) {
        if (a.w[0] != b.w[0]) return a.w[0] < b.w[0];
        if (a.w[1] != b.w[1]) return a.w[1] < b.w[1];
        return a.w[2] < b.w[2];
    };
    std::sort(v.begin(), v.end(), lt);
    v.erase(std::unique(v.begin(), v.end(),
                        [](const Sig &a, const Sig &b) { return !std::memcmp(a.w, b.w, sizeof a.w); }),
            v.end());
    std::vector<uint32_t> order;
    std::vector<Partition> parts;
    alg1_partition(v.data(), v.size(), max_partition, order, parts);
    uint64_t k = 0;
    for (size_t i = 0; i < parts.size(); ++i) {
        for (int w = 0; w < 3; ++w) masks_out[3 * i + w] = parts[i].mask.w[w];
        sizes_out[i] = parts[i].end - parts[i].begin;
        if (sigs_out)
            for (uint64_t m = parts[i].begin; m < parts[i].end; ++m, ++k)
                for (int w = 0; w < 3; ++w) sigs_out[3 * k + w] = v[order[m]].w[w];
    }
    *n_parts_out = parts.size();
    *n_unique_out = v.size();
    return TM_OK;
    TM_API_END
}

tm_status tm_last_result(const tm_db *db, const uint64_t **pairs, uint64_t *n) {
    TM_API_BEGIN
    if (!db || !pairs || !n) fail(TM_EINVAL, "NULL argument");
    if (!db->subs.empty()) fail(TM_ESTATE, "not available on an in-process multi-GPU handle");
    *pairs = db->last_sorted;
    *n = db->last_n;
    return TM_OK;
    TM_API_END
}

tm_status tm_shard_counts(tm_db *db, uint32_t n_owners, uint64_t *counts_out) {
    TM_API_BEGIN
    if (!db || !counts_out || n_owners == 0) fail(TM_EINVAL, "bad arguments");
    if (!db->subs.empty()) fail(TM_ESTATE, "not available on an in-process multi-GPU handle");
    DeviceGuard g(db->device);
    owner_counts(db, n_owners, db->stream);
    TMCK(cudaMemcpyAsync(counts_out, db->xcounts.p, n_owners * 8, cudaMemcpyDeviceToHost, db->stream));
    TMCK(cudaStreamSynchronize(db->stream));
    return TM_OK;
    TM_API_END
}

tm_status tm_shard_merge(tm_db *db, const uint64_t *pairs, uint64_t n, uint64_t n_queries, int unique,
                         tm_dev_pairs *out, void *stream) {
    TM_API_BEGIN
    if (!db || !out || (n && !pairs)) fail(TM_EINVAL, "bad arguments");
    if (!db->subs.empty()) fail(TM_ESTATE, "not available on an in-process multi-GPU handle");
    DeviceGuard g(db->device);
    cudaStream_t s = stream ? static_cast<cudaStream_t>(stream) : db->stream;
    db->xrecv.ensure(std::max<uint64_t>(n, 1) * 8);
    if (n) TMCK(cudaMemcpyAsync(db->xrecv.p, pairs, n * 8, cudaMemcpyDeviceToDevice, s));
    const uint64_t m = merge_pairs(db, db->xrecv.as<uint64_t>(), n, n_queries, unique, s);
    out->n = m;
    out->query = db->mq.as<uint32_t>();
    out->key = db->mk.as<uint32_t>();
    return TM_OK;
    TM_API_END
}

tm_status tm_nccl_unique_id(void *id_out, uint64_t len) {
    TM_API_BEGIN
    if (!id_out || len < sizeof(ncclUniqueId)) fail(TM_EINVAL, "id buffer must hold 128 bytes");
    ncclUniqueId id;
    TMNC(nccl().getUniqueId(&id));
    std::memcpy(id_out, &id, sizeof id);
    return TM_OK;
    TM_API_END
}

tm_status tm_comm_init(tm_db *db, const void *id, uint64_t len, int nranks, int rank) {
    TM_API_BEGIN
    if (!db || !id || len < sizeof(ncclUniqueId) || nranks < 1 || rank < 0 || rank >= nranks)
        fail(TM_EINVAL, "bad communicator arguments");
    if (!db->subs.empty()) fail(TM_ESTATE, "not available on an in-process multi-GPU handle");
    if (db->cfg.n_shards != (uint32_t)nranks || db->cfg.shard != (uint32_t)rank)
        fail(TM_ESTATE, "the handle must be built with n_shards == nranks and shard == rank");
    DeviceGuard g(db->device);
    shard_destroy(db);
    ncclUniqueId uid;
    std::memcpy(&uid, id, sizeof uid);
    ncclComm_t comm;
    TMNC(nccl().commInitRank(&comm, nranks, uid, rank));
    db->nccl_comm = comm;
    db->nranks = nranks;
    db->rank = rank;
    return TM_OK;
    TM_API_END
}

tm_status tm_match_batch_sharded_device(tm_db *db, const tm_tagsets *q, int unique, tm_dev_pairs *out,
                                        void *stream) {
    TM_API_BEGIN
    if (!db || !out) fail(TM_EINVAL, "db or out is NULL");
    if (!db->subs.empty()) fail(TM_ESTATE, "not available on an in-process multi-GPU handle");
    if (unique != 0 && unique != 1) fail(TM_EINVAL, "unique must be 0 or 1");
    check_tagsets_device(q);
    DeviceGuard g(db->device);
    cudaStream_t s = stream ? static_cast<cudaStream_t>(stream) : db->stream;
    tm_tagsets dq = *q;
    if (!dq.n_tags) dq.tag_idx = nullptr;
    if (db->cfg.shard_mode == TM_SHARD_REPLICATED) {
        // the whole table on every rank: match this rank's owner range only, no exchange
        const uint32_t G = std::max(1u, db->cfg.n_shards);
        const uint64_t lo = owner_start(q->n_sets, G, db->cfg.shard), hi = owner_start(q->n_sets, G, db->cfg.shard + 1);
        const uint64_t n = match_core(db, &dq, unique, s, lo, hi - lo);
        finish_timing(db, s);
        db->st.local_ms = db->st.total_ms;
        db->st.xchg_ms = 0;
        db->st.xchg_send_bytes = db->st.xchg_recv_bytes = 0;
        out->n = n;
        out->query = db->res_q.as<uint32_t>();
        out->key = db->res_k.as<uint32_t>();
        return TM_OK;
    }
    if (!db->nccl_comm) fail(TM_ESTATE, "tm_comm_init was not called");
    // S1-S8 against the local partitions
    match_core(db, &dq, unique, s);
    finish_timing(db, s);
    db->st.local_ms = db->st.total_ms;
    TMCK(cudaEventRecord(db->ev[5], s));
    const uint32_t G = (uint32_t)db->nranks;
    const int r = db->rank;
    ncclComm_t comm = static_cast<ncclComm_t>(db->nccl_comm);
    NcclApi &a = nccl();
    NvtxRange nv_x("tm_exchange");
    // S9: counts per owner, all-gathered
    owner_counts(db, G, s);
    db->xall.ensure((uint64_t)G * G * 8);
    TMNC(a.allGather(db->xcounts.p, db->xall.p, G, ncclUint64, comm, s));
    std::vector<uint64_t> all((size_t)G * G);
    TMCK(cudaMemcpyAsync(all.data(), db->xall.p, (size_t)G * G * 8, cudaMemcpyDeviceToHost, s));
    TMCK(cudaStreamSynchronize(s));
    std::vector<uint64_t> soff(G + 1, 0), roff(G + 1, 0);
    exchange_plan(all.data(), G, (uint32_t)r, soff.data(), roff.data());
    db->xrecv.ensure(std::max<uint64_t>(roff[G], 1) * 8);
    // all-to-all-v of (q<<32|key) pairs to query owners
    TMNC(a.groupStart());
    for (uint32_t p = 0; p < G; ++p) {
        const uint64_t sc = soff[p + 1] - soff[p], rc = roff[p + 1] - roff[p];
        if (sc) TMNC(a.send(db->last_sorted + soff[p], sc, ncclUint64, (int)p, comm, s));
        if (rc) TMNC(a.recv(db->xrecv.as<uint64_t>() + roff[p], rc, ncclUint64, (int)p, comm, s));
    }
    TMNC(a.groupEnd());
    const uint64_t m = merge_pairs(db, db->xrecv.as<uint64_t>(), roff[G], q->n_sets, unique, s);
    TMCK(cudaEventRecord(db->ev[4], s));
    TMCK(cudaEventSynchronize(db->ev[4]));
    float xms = 0;
    TMCK(cudaEventElapsedTime(&xms, db->ev[5], db->ev[4]));
    db->st.xchg_ms = xms;
    db->st.xchg_send_bytes = 8 * (soff[G] - (soff[r + 1] - soff[r]));
    db->st.xchg_recv_bytes = 8 * (roff[G] - (roff[r + 1] - roff[r]));
    out->n = m;
    out->query = db->mq.as<uint32_t>();
    out->key = db->mk.as<uint32_t>();
    return TM_OK;
    TM_API_END
}

}  // extern "C"
