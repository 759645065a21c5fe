// tm_group.cu -- in-process multi-GPU databases (tm_config.n_gpus > 1; include/tagmatch.h
// "In-process multi-GPU databases"): one process drives several GPUs, so the C ABI needs no
// launcher.  One sub-database per device, built and matched by one host thread each.
//
//   TM_SHARD_PARTITIONED ("partition an extremely large tagset table on multiple
//   GPUs"): sub g keeps the contiguous partition range the plan assigns to g, matches
//   the whole batch (S1-S8 on its GPU), its sorted pairs are cut at the query-owner boundaries,
//   each owner pulls its pieces from every GPU with peer copies (cudaMemcpyPeerAsync: NVLink /
//   NVSwitch with peer access enabled) and merges them on its GPU (sort / de-duplicate).
//   TM_SHARD_REPLICATED ("maximal inter-GPU parallelism in the case of full
//   replication"): every sub holds the whole table and matches owner range g; no exchange.
// The owner slices are query ranges in order, so the result is their concatenation.
#include <chrono>
#include <cstring>
#include <thread>

#include "tm_db.h"

namespace tmb {
namespace {

struct WorkerError {
    bool failed = false;
    tm_status s = TM_OK;
    std::string msg;
};

// Runs f(g) on one host thread per sub-database with that sub's device current; rethrows the
// first failure on the calling thread (errors are thread-local in the workers).
template <class F>
void on_each(const std::vector<tm_db *> &subs, F f) {
    const size_t G = subs.size();
    std::vector<WorkerError> err(G);
    std::vector<std::thread> th;
    th.reserve(G);
    for (size_t g = 0; g < G; ++g)
        th.emplace_back([&, g] {
            try {
                DeviceGuard dg(subs[g] ? subs[g]->device : -1);
                f(g);
            } catch (const StatusFail &e) {
                err[g] = {true, e.s, e.msg};
            } catch (const CudaFail &e) {
                const tm_status s = translate(e);
                err[g] = {true, s, g_err};
            } catch (const std::bad_alloc &) {
                err[g] = {true, TM_ENOMEM, "host allocation failed"};
            } catch (...) {
                err[g] = {true, TM_ESTATE, "unexpected exception"};
            }
        });
    for (auto &t : th) t.join();
    for (size_t g = 0; g < G; ++g)
        if (err[g].failed) fail(err[g].s, "GPU " + std::to_string(g) + ": " + err[g].msg);
}

// Enables peer access between every pair of distinct devices; returns whether every pair has it
// (the fused exchange stores into peer memory from the scan kernel).
bool enable_peers(const std::vector<int> &dev) {
    bool all = true;
    for (int a : dev)
        for (int b : dev) {
            if (a == b) continue;
            int ok = 0;
            if (cudaDeviceCanAccessPeer(&ok, a, b) != cudaSuccess || !ok) {
                cudaGetLastError();
                all = false;
                continue;  // cudaMemcpyPeerAsync still works (staged by the driver)
            }
            DeviceGuard g(a);
            const cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
            if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) throw CudaFail{e, "cudaDeviceEnablePeerAccess", __LINE__};
            cudaGetLastError();
        }
    return all;
}

}  // namespace

void group_build(tm_db *top, const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys,
                 const tm_config *cfg) {
    const uint32_t G = cfg->n_gpus;
    if (G > 64) fail(TM_EINVAL, "n_gpus > 64");
    if (cfg->n_shards > 1) fail(TM_EINVAL, "n_gpus > 1 and n_shards > 1 cannot be combined");
    if (cfg->shard_mode > 1) fail(TM_EINVAL, "shard_mode must be TM_SHARD_PARTITIONED or TM_SHARD_REPLICATED");
    int visible = 0;
    if (cudaGetDeviceCount(&visible) != cudaSuccess || visible == 0) {
        cudaGetLastError();
        fail(TM_ECUDA, "no CUDA device available (the library has no CPU fallback)");
    }
    std::vector<int> dev(G);
    for (uint32_t g = 0; g < G; ++g) {
        dev[g] = cfg->device_ids ? cfg->device_ids[g] : (int)g;
        if (dev[g] < 0 || dev[g] >= visible) fail(TM_EINVAL, "device_ids[" + std::to_string(g) + "] is not a visible device");
        check_device(dev[g]);
    }
    // the fused exchange needs peer stores between every pair of GPUs, at most kMaxOwners of them,
    // and the Bloom result (exact mode post-checks candidates on the GPU that found them);
    // TM_NO_FUSED_EXCHANGE=1 selects the pull exchange (peer copies after a local merge)
    top->fused_ok = enable_peers(dev) && G <= (uint32_t)kMaxOwners && !cfg->exact &&
                    !getenv("TM_NO_FUSED_EXCHANGE");
    top->device = dev[0];
    top->cfg.device_ids = nullptr;
    top->cfg.plan_sample = nullptr;
    top->subs.assign(G, nullptr);
    std::vector<tm_config> sc(G, *cfg);
    for (uint32_t g = 0; g < G; ++g) {
        sc[g].n_gpus = 0;
        sc[g].device = dev[g];
        sc[g].device_ids = nullptr;
        sc[g].n_shards = cfg->shard_mode == TM_SHARD_REPLICATED ? 1 : G;
        sc[g].shard = cfg->shard_mode == TM_SHARD_REPLICATED ? 0 : g;
    }
    const auto t0 = std::chrono::steady_clock::now();
    std::vector<tm_db *> none(G, nullptr);
    std::vector<tm_db *> built(G, nullptr);
    try {
        on_each(none, [&](size_t g) {
            DeviceGuard dg(dev[g]);
            built[g] = build_db(sets, key_off, keys, &sc[g]);
        });
    } catch (...) {
        for (tm_db *b : built) destroy_db(b);
        top->subs.clear();
        throw;
    }
    top->subs = built;
    top->n_sets = built[0]->n_sets;
    top->cfg.max_partition = built[0]->cfg.max_partition;
    top->build_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

// tm_match_batch (pout) or tm_match_batch_csr (cout) of a group handle.
void group_match(tm_db *top, const tm_tagsets *q, int unique, tm_pairs *pout, tm_csr *cout) {
    NvtxRange nv("tm_group_match");
    std::vector<tm_db *> &subs = top->subs;
    const uint32_t G = (uint32_t)subs.size();
    const uint64_t Q = q->n_sets;
    const bool repl = top->cfg.shard_mode == TM_SHARD_REPLICATED;
    std::vector<uint64_t> lo(G), hi(G);
    for (uint32_t g = 0; g < G; ++g) {
        lo[g] = owner_start(Q, G, g);
        hi[g] = owner_start(Q, G, g + 1);
    }
    const auto t0 = std::chrono::steady_clock::now();
    std::vector<uint64_t> counts((size_t)G * G, 0);
    std::vector<const uint64_t *> res(G, nullptr);  // owner g's sorted (q<<32|key) pairs
    std::vector<uint64_t> n(G, 0);
    std::vector<uint64_t> sent(G, 0), recvd(G, 0);
    std::chrono::steady_clock::time_point t1, t2;
    if (!repl && top->fused_ok && G > 1) {
        // ---- fused exchange: every GPU's scan stores each pair straight into its query owner's
        // receive region for that GPU (peer memory over NVLink); no local sort, no copy step
        uint64_t xcap = top->fx_cap ? top->fx_cap : std::max<uint64_t>(1 << 16, 8 * Q / G + 1024);
        if (const char *e = getenv("TM_FUSED_XCAP"))  // tests: start small to exercise the retry
            if (!top->fx_cap && atoll(e) > 0) xcap = (uint64_t)atoll(e);
        for (int attempt = 0;; ++attempt) {
            for (uint32_t d = 0; d < G; ++d) {
                DeviceGuard dg(subs[d]->device);
                subs[d]->xrecv.ensure((uint64_t)G * xcap * 8);
            }
            for (uint32_t g = 0; g < G; ++g) {
                auto &fx = subs[g]->fx;
                fx.G = G;
                fx.xcap = xcap;
                for (uint32_t d = 0; d < G; ++d) {
                    fx.xstart[d] = (uint32_t)lo[d];
                    fx.xout[d] = subs[d]->xrecv.as<uint64_t>() + (uint64_t)g * xcap;
                }
            }
            try {
                on_each(subs, [&](size_t g) {
                    tm_db *db = subs[g];
                    const tm_tagsets dq = upload_queries(db, q, db->stream);
                    match_core(db, &dq, unique, db->stream);
                    finish_timing(db, db->stream);
                    for (uint32_t d = 0; d < G; ++d) counts[(size_t)g * G + d] = db->fx.counts[d];
                });
            } catch (...) {
                for (tm_db *db : subs) db->fx.G = 0;
                throw;
            }
            uint64_t mx = 0;
            for (uint64_t c : counts) mx = std::max(mx, c);
            if (mx <= xcap) break;
            if (attempt >= 4) {
                for (tm_db *db : subs) db->fx.G = 0;
                fail(TM_ESTATE, "fused exchange: capacity retry did not converge");
            }
            xcap = mx + mx / 4;  // a region overflowed (the stores past xcap were dropped): again
        }
        for (tm_db *db : subs) db->fx.G = 0;
        top->fx_cap = xcap;
        t1 = std::chrono::steady_clock::now();
        // each owner compacts its G regions and merges them (sort / de-duplicate)
        on_each(subs, [&](size_t d) {
            tm_db *db = subs[d];
            cudaStream_t s = db->stream;
            uint64_t total = 0;
            for (uint32_t g = 0; g < G; ++g) total += counts[(size_t)g * G + d];
            db->xfin.ensure(std::max<uint64_t>(total, 1) * 8);
            uint64_t o = 0;
            for (uint32_t g = 0; g < G; ++g) {
                const uint64_t c = counts[(size_t)g * G + d];
                if (c)
                    TMCK(cudaMemcpyAsync(db->xfin.as<uint64_t>() + o, db->xrecv.as<uint64_t>() + (uint64_t)g * xcap,
                                         c * 8, cudaMemcpyDeviceToDevice, s));
                if (g != d) recvd[d] += c * 8;
                o += c;
            }
            n[d] = merge_pairs(db, db->xfin.as<uint64_t>(), total, Q, unique, s);
            res[d] = db->merged;
            for (uint32_t dd = 0; dd < G; ++dd)
                if (dd != d) sent[d] += 8 * counts[(size_t)d * G + dd];
        });
        t2 = std::chrono::steady_clock::now();
    } else {
    // phase 1: every GPU runs S1-S8 (partitioned: the whole batch against its partitions;
    // replicated: its owner range against the whole table)
    on_each(subs, [&](size_t g) {
        tm_db *db = subs[g];
        const tm_tagsets dq = upload_queries(db, q, db->stream);
        if (repl) {
            match_core(db, &dq, unique, db->stream, lo[g], hi[g] - lo[g]);
            finish_timing(db, db->stream);
        } else {
            match_core(db, &dq, unique, db->stream);
            finish_timing(db, db->stream);
            owner_counts(db, G, db->stream);
            TMCK(cudaMemcpyAsync(counts.data() + (size_t)g * G, db->xcounts.p, (size_t)G * 8, cudaMemcpyDeviceToHost,
                                 db->stream));
            TMCK(cudaStreamSynchronize(db->stream));
        }
    });
    t1 = std::chrono::steady_clock::now();
    // phase 2 (partitioned): each owner pulls its pieces from every GPU and merges them
    if (repl) {
        for (uint32_t g = 0; g < G; ++g) {
            res[g] = subs[g]->last_sorted;
            n[g] = subs[g]->last_n;
        }
    } else {
        std::vector<std::vector<uint64_t>> soff(G, std::vector<uint64_t>(G + 1)), roff(G, std::vector<uint64_t>(G + 1));
        for (uint32_t g = 0; g < G; ++g) exchange_plan(counts.data(), G, g, soff[g].data(), roff[g].data());
        on_each(subs, [&](size_t d) {
            tm_db *db = subs[d];
            cudaStream_t s = db->stream;
            const uint64_t total = roff[d][G];
            db->xrecv.ensure(std::max<uint64_t>(total, 1) * 8);
            for (uint32_t src = 0; src < G; ++src) {
                const uint64_t c = counts[(size_t)src * G + d];
                if (!c) continue;
                TMCK(cudaMemcpyPeerAsync(db->xrecv.as<uint64_t>() + roff[d][src], db->device,
                                         subs[src]->last_sorted + soff[src][d], subs[src]->device, c * 8, s));
                if (src != d) recvd[d] += c * 8;
            }
            n[d] = merge_pairs(db, db->xrecv.as<uint64_t>(), total, Q, unique, s);
            res[d] = db->merged;
            sent[d] = 8 * (soff[d][G] - (soff[d][d + 1] - soff[d][d]));
        });
    }
    t2 = std::chrono::steady_clock::now();
    }
    std::vector<uint64_t> base(G + 1, 0);
    for (uint32_t g = 0; g < G; ++g) base[g + 1] = base[g] + n[g];
    const uint64_t N = base[G];
    // results to host: owner slices in query order
    PinnedBlock *blk = nullptr;
    try {
        if (pout) {
            blk = pinned_get(std::max<uint64_t>(N, 1) * 8);
            uint32_t *hq = static_cast<uint32_t *>(blk->p), *hk = hq + N;
            on_each(subs, [&](size_t g) {
                tm_db *db = subs[g];
                if (!n[g]) return;
                const uint32_t *dq = repl ? db->res_q.as<uint32_t>() : db->mq.as<uint32_t>();
                const uint32_t *dk = repl ? db->res_k.as<uint32_t>() : db->mk.as<uint32_t>();
                TMCK(cudaMemcpyAsync(hq + base[g], dq, n[g] * 4, cudaMemcpyDeviceToHost, db->stream));
                TMCK(cudaMemcpyAsync(hk + base[g], dk, n[g] * 4, cudaMemcpyDeviceToHost, db->stream));
                TMCK(cudaStreamSynchronize(db->stream));
            });
            pout->n = N;
            pout->query = hq;
            pout->key = hk;
            pout->priv_ = blk;
        } else {
            blk = pinned_get((Q + 1) * 8 + std::max<uint64_t>(N, 1) * 4);
            uint64_t *hoff = static_cast<uint64_t *>(blk->p);
            uint32_t *hk = reinterpret_cast<uint32_t *>(hoff + Q + 1);
            on_each(subs, [&](size_t g) {
                tm_db *db = subs[g];
                const uint64_t nq = hi[g] - lo[g];
                db->res_off.ensure((nq + 1) * 8);
                TMCK(launch_query_offsets(res[g], n[g], lo[g], nq, base[g], db->res_off.as<uint64_t>(), db->stream));
                // owner g writes q_off[lo, hi); the last owner also q_off[Q] = N
                TMCK(cudaMemcpyAsync(hoff + lo[g], db->res_off.p, (nq + (g + 1 == G ? 1 : 0)) * 8,
                                     cudaMemcpyDeviceToHost, db->stream));
                const uint32_t *dk = repl ? db->res_k.as<uint32_t>() : db->mk.as<uint32_t>();
                if (n[g]) TMCK(cudaMemcpyAsync(hk + base[g], dk, n[g] * 4, cudaMemcpyDeviceToHost, db->stream));
                TMCK(cudaStreamSynchronize(db->stream));
            });
            if (Q == 0) hoff[0] = 0;
            cout->n_queries = Q;
            cout->n = N;
            cout->q_off = hoff;
            cout->key = hk;
            cout->priv_ = blk;
        }
    } catch (...) {
        pinned_put(blk);
        throw;
    }
    // the group's statistics of this call
    tm_stats_t &st = top->st;
    std::memset(&st.n_queries, 0, sizeof(tm_stats_t) - offsetof(tm_stats_t, n_queries));
    st.n_queries = Q;
    st.result_pairs = N;
    for (uint32_t g = 0; g < G; ++g) {
        st.xchg_send_bytes += sent[g];
        st.xchg_recv_bytes += recvd[g];
    }
    st.local_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
    st.xchg_ms = std::chrono::duration<double, std::milli>(t2 - t1).count();
}

void group_stats(const tm_db *top, tm_stats_t *out) {
    const std::vector<tm_db *> &subs = top->subs;
    const bool repl = top->cfg.shard_mode == TM_SHARD_REPLICATED;
    std::vector<tm_stats_t> ss(subs.size());
    for (size_t g = 0; g < subs.size(); ++g) {
        tm_db *d = subs[g];
        ss[g] = d->st;
        ss[g].n_sets = d->n_sets;
        ss[g].n_entries = d->n_entries;
        ss[g].n_unique = d->n_unique;
        ss[g].n_rows = d->n_rows;
        ss[g].n_partitions = d->n_parts;
        ss[g].n_partitions_total = d->n_parts_total;
    }
    tm_stats_t o = top->st;  // n_queries, result_pairs, exchange of the last call
    const tm_stats_t &a = ss[0];
    o.n_sets = a.n_sets;
    o.n_partitions_total = a.n_partitions_total;
    o.build_ms = top->build_ms;
    o.n_entries = o.n_unique = o.n_rows = o.n_partitions = 0;
    o.routed = o.candidate_pairs = o.tile_tests = o.pair_checks = o.matched_sets = o.emitted_pairs = 0;
    o.work_items = o.retries = o.exact_checked = o.exact_kept = 0;
    o.encode_ms = o.route_ms = o.scan_ms = o.merge_ms = o.total_ms = 0;
    o.scan_launches = o.kernel_launches = 0;
    o.tuning = 0;
    for (const tm_stats_t &x : ss) {
        if (!repl || &x == &ss[0]) {
            o.n_entries += x.n_entries;
            o.n_unique += x.n_unique;
            o.n_rows += x.n_rows;
            o.n_partitions += x.n_partitions;
        }
        o.routed += x.routed;
        o.candidate_pairs += x.candidate_pairs;
        o.tile_tests += x.tile_tests;
        o.pair_checks += x.pair_checks;
        o.matched_sets += x.matched_sets;
        o.emitted_pairs += x.emitted_pairs;
        o.work_items += x.work_items;
        o.retries += x.retries;
        o.exact_checked += x.exact_checked;
        o.exact_kept += x.exact_kept;
        o.encode_ms = std::max(o.encode_ms, x.encode_ms);
        o.route_ms = std::max(o.route_ms, x.route_ms);
        o.scan_ms = std::max(o.scan_ms, x.scan_ms);
        o.merge_ms = std::max(o.merge_ms, x.merge_ms);
        o.total_ms = std::max(o.total_ms, x.total_ms);
        o.scan_launches += x.scan_launches;
        o.kernel_launches += x.kernel_launches;
        o.tuning |= x.tuning;
    }
    o.scan_variant = a.scan_variant;
    o.max_partition = top->cfg.max_partition;
    o.n_gpus = (uint32_t)subs.size();
    *out = o;
}

}  // namespace tmb

extern "C" {

tm_status tm_group_size(const tm_db *db, uint32_t *n) {
    TM_API_BEGIN
    if (!db || !n) fail(TM_EINVAL, "NULL argument");
    *n = db->subs.empty() ? 1u : (uint32_t)db->subs.size();
    return TM_OK;
    TM_API_END
}

tm_status tm_group_member(const tm_db *db, uint32_t g, const tm_db **sub) {
    TM_API_BEGIN
    if (!db || !sub) fail(TM_EINVAL, "NULL argument");
    if (db->subs.empty()) {
        if (g != 0) fail(TM_EINVAL, "member index out of range");
        *sub = db;
        return TM_OK;
    }
    if (g >= db->subs.size()) fail(TM_EINVAL, "member index out of range");
    *sub = db->subs[g];
    return TM_OK;
    TM_API_END
}

}  // extern "C"
