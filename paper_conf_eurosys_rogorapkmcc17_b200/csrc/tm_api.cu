// tm_api.cu -- the C ABI (include/tagmatch.h): tm_build, tm_match_batch, tm_free, hooks.
//
// Host code only orchestrates: it validates arguments, owns device buffers and
// the stream, launches the stage kernels (tm_kernels.cu) and reads back one
// small counter block per call.  Every step of the matching path runs on the GPU.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstddef>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <numeric>
#include <string>
#include <vector>

#include "tm_db.h"

namespace tmb {

thread_local std::string g_err;
void set_error(const std::string &msg) { g_err = msg; }



// -------------------------------------------- pinned host result blocks --
std::mutex g_pin_mu;
std::multimap<size_t, void *> g_pin_cache;
size_t g_pin_cached = 0;

PinnedBlock *pinned_get(size_t bytes) {
    {
        std::lock_guard<std::mutex> lk(g_pin_mu);
        auto it = g_pin_cache.lower_bound(bytes);
        if (it != g_pin_cache.end() && it->first <= 2 * bytes + (1 << 20)) {
            PinnedBlock *b = new PinnedBlock{it->second, it->first};
            g_pin_cached -= it->first;
            g_pin_cache.erase(it);
            return b;
        }
    }
    void *p = nullptr;
    size_t cap = std::max<size_t>(bytes, 4096);
    cudaError_t e = cudaMallocHost(&p, cap);
    if (e != cudaSuccess) {
        cudaGetLastError();
        fail(TM_ENOMEM, "pinned host allocation failed");
    }
    return new PinnedBlock{p, cap};
}

void pinned_put(PinnedBlock *b) {
    if (!b) return;
    {
        std::lock_guard<std::mutex> lk(g_pin_mu);
        if (g_pin_cached + b->cap <= (size_t(4) << 30)) {
            g_pin_cache.emplace(b->cap, b->p);
            g_pin_cached += b->cap;
            delete b;
            return;
        }
    }
    cudaFreeHost(b->p);
    delete b;
}

// ------------------------------------------------------------ validation --
// a pre-hashed vocabulary (tm_tagsets.vocab_hash) comes without strings
static void check_hashed(const tm_tagsets *t, const std::string &w) {
    if (t->vocab_bytes || t->n_bytes) fail(TM_EINVAL, w + ": vocab_hash given together with vocab_bytes / n_bytes");
    if (t->n_vocab > 0xFFFFFFFFull) fail(TM_ERANGE, w + ": more than 2^32-1 vocabulary strings");
    if (t->n_tags > 0 && t->tag_idx == nullptr && t->n_tags != t->n_vocab)
        fail(TM_EINVAL, w + ": tag_idx NULL requires n_tags == n_vocab");
    if (t->n_tags > 0 && t->n_vocab == 0) fail(TM_EINVAL, w + ": tags without a vocabulary");
}

void require_strings(const tm_tagsets *t, const char *what) {
    if (t && t->vocab_hash)
        fail(TM_EINVAL, std::string(what) + ": this call needs tag strings (vocab_hash is accepted by the match calls, "
                                            "tm_encode and plan_sample only)");
}

void check_tagsets_host(const tm_tagsets *t, const char *what) {
    const std::string w(what);
    if (!t) fail(TM_EINVAL, w + ": NULL tagsets");
    if (t->n_sets > 0xFFFFFFFFull) fail(TM_ERANGE, w + ": more than 2^32-1 sets");
    if (!t->set_off) fail(TM_EINVAL, w + ": set_off is NULL");
    if (t->vocab_hash) {
        check_hashed(t, w);
        if (t->set_off[0] != 0 || t->set_off[t->n_sets] != t->n_tags)
            fail(TM_EINVAL, w + ": set_off[0] != 0 or set_off[n_sets] != n_tags");
        for (uint64_t i = 0; i < t->n_sets; ++i)
            if (t->set_off[i + 1] < t->set_off[i]) fail(TM_EINVAL, w + ": set_off not non-decreasing");
        if (t->tag_idx)
            for (uint64_t i = 0; i < t->n_tags; ++i)
                if (t->tag_idx[i] >= t->n_vocab) fail(TM_EINVAL, w + ": tag_idx out of range");
        return;
    }
    if (t->n_vocab > 0 && !t->vocab_off) fail(TM_EINVAL, w + ": vocab_off is NULL");
    if (t->n_bytes > 0 && !t->vocab_bytes) fail(TM_EINVAL, w + ": vocab_bytes is NULL");
    if (t->n_tags > 0 && t->tag_idx == nullptr && t->n_tags != t->n_vocab)
        fail(TM_EINVAL, w + ": tag_idx NULL requires n_tags == n_vocab");
    if (t->n_vocab > 0xFFFFFFFFull) fail(TM_ERANGE, w + ": more than 2^32-1 vocabulary strings");
    if (t->set_off[0] != 0 || t->set_off[t->n_sets] != t->n_tags) fail(TM_EINVAL, w + ": set_off[0] != 0 or set_off[n_sets] != n_tags");
    for (uint64_t i = 0; i < t->n_sets; ++i)
        if (t->set_off[i + 1] < t->set_off[i]) fail(TM_EINVAL, w + ": set_off not non-decreasing");
    if (t->n_vocab > 0) {
        if (t->vocab_off[0] != 0 || t->vocab_off[t->n_vocab] != t->n_bytes)
            fail(TM_EINVAL, w + ": vocab_off[0] != 0 or vocab_off[n_vocab] != n_bytes");
        for (uint64_t i = 0; i < t->n_vocab; ++i)
            if (t->vocab_off[i + 1] < t->vocab_off[i]) fail(TM_EINVAL, w + ": vocab_off not non-decreasing");
    } else if (t->n_tags > 0) {
        fail(TM_EINVAL, w + ": tags without a vocabulary");
    }
    if (t->tag_idx)
        for (uint64_t i = 0; i < t->n_tags; ++i)
            if (t->tag_idx[i] >= t->n_vocab) fail(TM_EINVAL, w + ": tag_idx out of range");
}

// O(1) checks of host query arrays (pointers, sizes, end points); the O(n) monotonicity and range
// checks run inside the encoder kernels (match_core)
void check_tagsets_shape(const tm_tagsets *t, const char *what) {
    const std::string w(what);
    if (!t) fail(TM_EINVAL, w + ": NULL tagsets");
    if (t->n_sets > 0xFFFFFFFFull) fail(TM_ERANGE, w + ": more than 2^32-1 sets");
    if (!t->set_off) fail(TM_EINVAL, w + ": set_off is NULL");
    if (t->vocab_hash) {
        check_hashed(t, w);
        if (t->set_off[0] != 0 || t->set_off[t->n_sets] != t->n_tags)
            fail(TM_EINVAL, w + ": set_off[0] != 0 or set_off[n_sets] != n_tags");
        return;
    }
    if (t->n_vocab > 0 && !t->vocab_off) fail(TM_EINVAL, w + ": vocab_off is NULL");
    if (t->n_bytes > 0 && !t->vocab_bytes) fail(TM_EINVAL, w + ": vocab_bytes is NULL");
    if (t->n_tags > 0 && t->tag_idx == nullptr && t->n_tags != t->n_vocab)
        fail(TM_EINVAL, w + ": tag_idx NULL requires n_tags == n_vocab");
    if (t->n_vocab > 0xFFFFFFFFull) fail(TM_ERANGE, w + ": more than 2^32-1 vocabulary strings");
    if (t->set_off[0] != 0 || t->set_off[t->n_sets] != t->n_tags) fail(TM_EINVAL, w + ": set_off[0] != 0 or set_off[n_sets] != n_tags");
    if (t->n_vocab > 0) {
        if (t->vocab_off[0] != 0 || t->vocab_off[t->n_vocab] != t->n_bytes)
            fail(TM_EINVAL, w + ": vocab_off[0] != 0 or vocab_off[n_vocab] != n_bytes");
    } else if (t->n_tags > 0) {
        fail(TM_EINVAL, w + ": tags without a vocabulary");
    }
}

void check_tagsets_device(const tm_tagsets *t) {
    if (!t) fail(TM_EINVAL, "queries: NULL tagsets");
    if (t->n_sets > 0xFFFFFFFFull) fail(TM_ERANGE, "queries: more than 2^32-1 sets");
    if (t->n_sets > 0 && !t->set_off) fail(TM_EINVAL, "queries: set_off is NULL");
    if (t->vocab_hash) {
        check_hashed(t, "queries");
        return;
    }
    if (t->n_vocab > 0 && !t->vocab_off) fail(TM_EINVAL, "queries: vocab_off is NULL");
    if (t->n_bytes > 0 && !t->vocab_bytes) fail(TM_EINVAL, "queries: vocab_bytes is NULL");
    if (t->n_tags > 0 && t->tag_idx == nullptr && t->n_tags != t->n_vocab)
        fail(TM_EINVAL, "queries: tag_idx NULL requires n_tags == n_vocab");
    if (t->n_tags > 0 && t->n_vocab == 0) fail(TM_EINVAL, "queries: tags without a vocabulary");
}

int bits_for(uint64_t n) {  // bits needed to represent values < n
    int b = 0;
    while (b < 64 && (1ULL << b) < n) ++b;
    return b;
}

}  // namespace tmb

using namespace tmb;

// ================================================================== tm_db ==

namespace tmb {

void *cub_tmp(tm_db *db, size_t bytes) {
    db->tmp.ensure(bytes);
    return db->tmp.p;
}

// Run the whole path for device-resident queries; leaves n results in db->res_q/res_k.
// Every query of the batch is encoded; queries [qlo, qlo + qn) are matched (the share of one GPU
// of a replicated multi-GPU database; default: all), with their batch-global indices.
uint64_t match_core(tm_db *db, const tm_tagsets *q, int unique, cudaStream_t s, uint64_t qlo, uint64_t qn,
                    bool encoded) {
    NvtxRange nv_call("tm_match");
    if (db->cfg.exact && q->vocab_hash)  // the exact check compares tag strings
        fail(TM_EINVAL, "queries: exact mode needs tag strings, not vocab_hash");
    tm_stats_t &st = db->st;
    const uint64_t Qall = q->n_sets;
    if (qlo > Qall) qlo = Qall;
    if (qn > Qall - qlo) qn = Qall - qlo;
    const uint64_t Qm = qn;                        // queries matched
    const uint32_t P = (uint32_t)db->n_parts;
    std::memset(&st.n_queries, 0, sizeof(tm_stats_t) - offsetof(tm_stats_t, n_queries));
    st.n_queries = Qm;
    db->last_sorted = nullptr;
    db->last_n = 0;
    db->last_Q = Qall;
    db->last_qlo = qlo;
    db->last_qn = Qm;
    for (uint64_t &c : db->fx.counts) c = 0;  // fused exchange: nothing sent yet
    if (Qm == 0 || P == 0) return 0;
    const uint64_t Q = Qall;                       // encoded (and the sort width)
    const uint64_t NB = route_blocks(Qm);          // route blocks of 384 queries
    const uint64_t n_words = (uint64_t)P * NB;    // (partition, route block) counts
    uint32_t launches = 0, cub_calls = 0;

    db->ctr.ensure(sizeof(DevCounters));
    DevCounters *ctr = db->ctr.as<DevCounters>();
    if (!db->wsel_ok) {  // pre-check word per row (scan variant 5), once per database
        db->wsel.ensure(std::max<uint64_t>(db->n_rows, 1));
        db->wwords.ensure(std::max<uint64_t>(db->n_rows, 1) * 8);
        TMCK(launch_word_select(db->planes.as<uint64_t>(), db->tand.as<uint64_t>(), db->n_rows,
                                db->wsel.as<uint8_t>(), db->wwords.as<uint2>(), s));
        db->wsel_ok = true;
    }
    TMCK(cudaEventRecord(db->ev[0], s));

    // S1: encode
    if (!encoded) {
        db->vsig.ensure(std::max<uint64_t>(q->n_vocab, 1) * 24);
        db->qplanes.ensure(Q * 24);
    }
    uint64_t *q0 = db->qplanes.as<uint64_t>(), *q1 = q0 + Q, *q2 = q1 + Q;
    if (!encoded) {
        // the query CSR is validated by the encoder kernels themselves (input_err, checked below with
        // the scan counters): no O(n) host pass over the batch on the call's critical path
        TMCK(cudaMemsetAsync(&ctr->input_err, 0, sizeof(ctr->input_err), s));
        TMCK(launch_hash_vocab(q->vocab_bytes, q->vocab_off, q->vocab_hash, q->n_vocab, q->n_bytes,
                               db->vsig.as<uint64_t>(), &ctr->input_err, s));
        TMCK(launch_encode_sets(db->vsig.as<uint64_t>(), q->tag_idx, q->set_off, Q, q->n_tags, q->n_vocab, q0, q1,
                                q2, &ctr->input_err, s));
        launches += 2;
    }
    TMCK(cudaEventRecord(db->ev[1], s));

    // S2: route (Alg. 2, bit-sliced): per (partition, route block) counts, scanned to the
    // offsets of a partition-major CSR of ascending query ids
    db->bm.ensure(n_words * 4);
    db->word_off.ensure((n_words + 1) * 8);
    TMCK(launch_route(0, db->masks.as<uint64_t>(), P, q0 + qlo, q1 + qlo, q2 + qlo, Qm, db->bm.as<uint32_t>(), nullptr,
                      nullptr, 0, s));
    launches++;
    size_t tb = 0;
    TMCK(cub_exclusive_scan_u32_u64(db->bm.as<uint32_t>(), db->word_off.as<unsigned long long>(), n_words, nullptr,
                                    &tb, s));
    TMCK(cub_exclusive_scan_u32_u64(db->bm.as<uint32_t>(), db->word_off.as<unsigned long long>(), n_words,
                                    cub_tmp(db, tb), &tb, s));
    cub_calls++;
    db->qoff.ensure((uint64_t)(P + 1) * 8);
    db->item_cnt.ensure((uint64_t)(P + 1) * 8);
    db->item_off.ensure((uint64_t)(P + 1) * 8);
    if (db->cap_qidx == 0) db->cap_qidx = std::max<unsigned long long>(Qm * 32, 1 << 16);
    if (db->cap_out == 0) db->cap_out = std::max<unsigned long long>(Qm * 32, 1 << 16);

    for (int attempt = 0;; ++attempt) {
        db->qidx.ensure(db->cap_qidx * 4);
        db->out.ensure(db->cap_out * 8);
        TMCK(cudaMemsetAsync(ctr, 0, offsetof(DevCounters, input_err), s));
        TMCK(launch_route(1, db->masks.as<uint64_t>(), P, q0 + qlo, q1 + qlo, q2 + qlo, Qm, nullptr,
                          db->word_off.as<unsigned long long>(), db->qidx.as<uint32_t>(), db->cap_qidx, s,
                          (uint32_t)qlo));
        // S3: per-partition batches -> work items
        const uint32_t range_rows = range_rows_env(db->n_rows);
        TMCK(launch_items(db->word_off.as<unsigned long long>(), NB, db->part_row.as<uint32_t>(),
                          db->part_n.as<uint32_t>(), P, db->qoff.as<unsigned long long>(),
                          db->item_cnt.as<unsigned long long>(), ctr, range_rows, s));
        launches += 2;
        tb = 0;
        TMCK(cub_exclusive_scan_u64(db->item_cnt.as<unsigned long long>(), db->item_off.as<unsigned long long>(),
                                    P + 1, nullptr, &tb, s));
        TMCK(cub_exclusive_scan_u64(db->item_cnt.as<unsigned long long>(), db->item_off.as<unsigned long long>(),
                                    P + 1, cub_tmp(db, tb), &tb, s));
        cub_calls++;
        TMCK(cudaEventRecord(db->ev[2], s));
        // S4-S7: subset scan
        ScanParams sp;
        sp.w0 = db->planes.as<uint64_t>();
        sp.w1 = sp.w0 + db->n_rows;
        sp.w2 = sp.w1 + db->n_rows;
        sp.t0 = db->tand.as<uint64_t>();
        sp.t1 = sp.t0 + db->n_rows / kTile;
        sp.t2 = sp.t1 + db->n_rows / kTile;
        sp.key_off = db->key_off.as<uint32_t>();
        sp.keys = db->keys.as<uint32_t>();
        sp.part_row = db->part_row.as<uint32_t>();
        sp.part_n = db->part_n.as<uint32_t>();
        sp.q0 = q0;
        sp.q1 = q1;
        sp.q2 = q2;
        sp.qidx = db->qidx.as<uint32_t>();
        sp.qcap = db->cap_qidx;
        sp.qoff = db->qoff.as<unsigned long long>();
        sp.item_off = db->item_off.as<unsigned long long>();
        sp.n_parts = P;
        sp.out = db->out.as<uint64_t>();
        sp.cap = db->cap_out;
        sp.ctr = ctr;
        sp.filter = db->cfg.tile_filter;
        sp.wsel = db->wsel.as<uint8_t>();
        sp.wwords = db->wwords.as<uint2>();
        sp.range_rows = range_rows;
        sp.one = 1;
        sp.unit_target = unit_target_env();
        // fused exchange (in-process multi-GPU group, tm_group.cu): emit to the owners' regions
        sp.n_owners = db->fx.G > 1 ? db->fx.G : 0;
        sp.xcap = db->fx.xcap;
        sp.xcnt = nullptr;
        for (int g = 0; g < kMaxOwners; ++g) {
            sp.xstart[g] = db->fx.xstart[g];
            sp.xout[g] = db->fx.xout[g];
        }
        if (sp.n_owners) {
            db->xfcnt.ensure(kMaxOwners * 8);
            sp.xcnt = db->xfcnt.as<unsigned long long>();
            TMCK(cudaMemsetAsync(sp.xcnt, 0, kMaxOwners * 8, s));
        }
        // variant: TM_SCAN_VARIANT if set; else a call whose partition batches are all small
        // (Q <= kSmallBatch) takes the streaming path only, in the streaming-only kernels (small
        // shared memory: 8 CTAs/SM) -- up to four queries checked directly (variant 6), 5-8
        // through the two-word pre-check (variant 7; scripts/hbm_sweep.py) -- and is not a
        // tuning sample (the candidates differ only in the filtered path); other calls cycle
        // through the candidates on the handle's first qualifying calls, then keep the cheapest
        const int forced = scan_variant_env();
        int var = forced;
        // the streaming-only kernels cannot take a filtered batch: a forced 6 / 7 maps to 0 / 5 then
        if ((var == 6 || var == 7) && Qm > (uint64_t)kSmallBatch) var = var == 6 ? 0 : 5;
        db->call_tunes = false;
        if (var < 0) {
            if (Qm <= (uint64_t)kSmallBatch) {
                var = Qm <= 4 ? 6 : 7;
            } else {
                const int c = 63 - __builtin_clzll(Qm);
                db->call_class = c;
                // batches below kTuneMinQ queries keep the default variant: a tuning round there
                // would put slow candidates into a latency-bound stream for little gain
                if (Qm >= (uint64_t)kTuneMinQ && db->tune_calls[c] < 2 * kTuneN) {
                    var = db->tune[db->tune_calls[c] % kTuneN];
                    db->call_tunes = true;
                } else {
                    var = db->variant[c];
                }
            }
        }
        if (!db->grid_of[var]) db->grid_of[var] = scan_grid(db->device, var);
        db->call_variant = var;
        st.scan_variant = (uint32_t)var;
        TMCK(launch_scan(sp, db->grid_of[var], s, var));
        launches++;
        st.scan_launches++;
        TMCK(cudaEventRecord(db->ev[3], s));
        TMCK(cudaMemcpyAsync(db->h_ctr, ctr, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
        if (sp.n_owners) TMCK(cudaMemcpyAsync(db->h_fx, sp.xcnt, kMaxOwners * 8, cudaMemcpyDeviceToHost, s));
        TMCK(cudaStreamSynchronize(s));
        scan_debug_dump(var);
        const DevCounters c = *db->h_ctr;
        if (c.input_err)
            fail(TM_EINVAL, std::string("queries: malformed CSR found by the encoder (") +
                                ((c.input_err & 1u) ? "vocab_off " : "") + ((c.input_err & 2u) ? "set_off " : "") +
                                ((c.input_err & 4u) ? "tag_idx out of range" : "") + ")");
        bool retry = false;
        if (c.routed > db->cap_qidx) {
            db->cap_qidx = c.routed + c.routed / 4;
            retry = true;
        }
        if (!retry && c.n_out > db->cap_out) {
            db->cap_out = c.n_out + c.n_out / 8;
            retry = true;
        }
        if (retry) {
            st.retries++;
            if (attempt > 4) fail(TM_ESTATE, "capacity retry loop did not converge");
            continue;
        }
        st.routed = c.routed;
        st.candidate_pairs = c.candidates;
        st.tile_tests = c.tile_tests;
        st.pair_checks = c.pair_checks;
        st.matched_sets = c.matched_sets;
        st.emitted_pairs = c.n_out;
        st.work_items = c.n_items;
        break;
    }
    if (db->fx.G > 1) {  // fused exchange: the pairs are in the owners' regions; they merge them
        st.emitted_pairs = 0;
        for (uint32_t g = 0; g < db->fx.G; ++g) {
            db->fx.counts[g] = db->h_fx[g];
            st.emitted_pairs += db->h_fx[g];
        }
        TMCK(cudaEventRecord(db->ev[4], s));
        st.kernel_launches = launches;
        return 0;
    }
    uint64_t n = st.emitted_pairs;
    if (db->cfg.exact) {  // S7': exact subset check of the (query, set) candidates, then keys
        n = exact_filter(db, q, n, s);
        launches += 5;
    }
    // S8: canonical order (sort by (query, key)), merge (unique for match-unique)
    db->out_alt.ensure(std::max<uint64_t>(n, 1) * 8);
    uint64_t *sorted = db->out.as<uint64_t>();
    if (n > 1) {
        int sel = 0;
        const int end_bit = 32 + bits_for(Q);
        tb = 0;
        TMCK(cub_sort_keys_u64(db->out.as<uint64_t>(), db->out_alt.as<uint64_t>(), n, end_bit, &sel, nullptr, &tb, s));
        TMCK(cub_sort_keys_u64(db->out.as<uint64_t>(), db->out_alt.as<uint64_t>(), n, end_bit, &sel,
                               cub_tmp(db, tb), &tb, s));
        cub_calls++;
        sorted = sel ? db->out_alt.as<uint64_t>() : db->out.as<uint64_t>();
    }
    if (unique && n > 1) {
        uint64_t *dst = (sorted == db->out.as<uint64_t>()) ? db->out_alt.as<uint64_t>() : db->out.as<uint64_t>();
        unsigned long long *d_n = &ctr->item_ctr;  // reuse a counter slot
        tb = 0;
        TMCK(cub_unique_u64(sorted, dst, d_n, n, nullptr, &tb, s));
        TMCK(cub_unique_u64(sorted, dst, d_n, n, cub_tmp(db, tb), &tb, s));
        cub_calls++;
        TMCK(cudaMemcpyAsync(db->h_nuniq, d_n, 8, cudaMemcpyDeviceToHost, s));
        TMCK(cudaStreamSynchronize(s));
        n = *db->h_nuniq;
        sorted = dst;
    }
    db->last_sorted = sorted;
    db->last_n = n;
    db->last_Q = Q;
    db->res_q.ensure(std::max<uint64_t>(n, 1) * 4);
    db->res_k.ensure(std::max<uint64_t>(n, 1) * 4);
    TMCK(launch_split(sorted, n, db->res_q.as<uint32_t>(), db->res_k.as<uint32_t>(), s));
    launches++;
    TMCK(cudaEventRecord(db->ev[4], s));
    st.result_pairs = n;
    st.kernel_launches = launches;
    (void)cub_calls;
    return n;
}

void finish_timing(tm_db *db, cudaStream_t s) {
    TMCK(cudaStreamSynchronize(s));
    float ms = 0;
    tm_stats_t &st = db->st;
    if (st.n_queries == 0 || db->n_parts == 0) return;
    TMCK(cudaEventElapsedTime(&ms, db->ev[0], db->ev[1]));
    st.encode_ms = ms;
    TMCK(cudaEventElapsedTime(&ms, db->ev[1], db->ev[2]));
    st.route_ms = ms;
    TMCK(cudaEventElapsedTime(&ms, db->ev[2], db->ev[3]));
    st.scan_ms = ms;
    // variant tuning: qualifying calls 0 .. 2N-1 cycle through the N candidates kTune; the
    // second round (warm: module loaded, buffers grown) is timed as kernel ns per decision;
    // the cheapest is kept
    const double dec = (double)(st.tile_tests + st.pair_checks);
    if (db->call_tunes && dec > 1e6 && st.retries == 0) {
        const int c = db->call_class;
        if (db->tune_calls[c] >= kTuneN) db->tune_cost[c][db->call_variant] = ms * 1e6 / dec;
        if (++db->tune_calls[c] == 2 * kTuneN) {
            int best = db->tune[0];
            for (int i = 1; i < kTuneN; ++i)
                if (db->tune_cost[c][db->tune[i]] < db->tune_cost[c][best]) best = db->tune[i];
            db->variant[c] = best;
        }
    }
    if (db->call_tunes) st.tuning = db->tune_calls[db->call_class] < 2 * kTuneN ? 1u : 0u;
    TMCK(cudaEventElapsedTime(&ms, db->ev[3], db->ev[4]));
    st.merge_ms = ms;
    TMCK(cudaEventElapsedTime(&ms, db->ev[0], db->ev[4]));
    st.total_ms = ms;
}

tm_status translate(const CudaFail &f) {
    char buf[512];
    snprintf(buf, sizeof buf, "CUDA error %d (%s) at tm_api.cu:%d in %s", (int)f.e, cudaGetErrorString(f.e), f.line,
             f.what);
    set_error(buf);
    cudaGetLastError();
    if (f.e == cudaErrorMemoryAllocation) return TM_ENOMEM;
    return TM_ECUDA;
}

void build_impl(tm_db *db, const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys) {
    NvtxRange nv_build("tm_build");
    auto t0 = std::chrono::steady_clock::now();
    const bool trace = getenv("TM_TRACE_BUILD") != nullptr;
    auto mark = [&](const char *what) {
        if (trace)
            fprintf(stderr, "[tm_build] %-28s %9.1f ms\n", what,
                    std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    };
    cudaStream_t s = db->stream;
    const uint64_t N = sets->n_sets;
    // keys
    std::vector<uint64_t> koff_default;
    if (!key_off) {
        koff_default.resize(N + 1);
        for (uint64_t i = 0; i <= N; ++i) koff_default[i] = i;
        key_off = koff_default.data();
    } else {
        if (key_off[0] != 0) fail(TM_EINVAL, "key_off[0] != 0");
        for (uint64_t i = 0; i < N; ++i)
            if (key_off[i + 1] < key_off[i]) fail(TM_EINVAL, "key_off not non-decreasing");
    }
    const uint64_t K = key_off[N];
    if (K > 0xFFFFFFFFull) fail(TM_ERANGE, "more than 2^32-1 keys");
    if (K > 0 && !keys) fail(TM_EINVAL, "keys is NULL");
    db->n_sets = N;
    db->n_entries = K;
    if (db->cfg.max_partition == TM_AUTO_MAX_PARTITION)  // reading R8b: MAX_P = N / 3*10^4 (measured)
        db->cfg.max_partition = (uint32_t)std::min<uint64_t>(200000, std::max<uint64_t>(5000, N / 30000));
    if (db->cfg.tile_filter != 2 && db->cfg.max_partition <= kSmallPMax) db->set_tune(kTuneSmallP);

    // S0a: encode every set on the GPU
    DevBuf d_bytes, d_voff, d_tidx, d_soff, d_vsig, d_planes, d_sorted, d_idx, d_idx2, d_key, d_key2;
    struct Releaser {
        std::vector<DevBuf *> v;
        ~Releaser() {
            for (auto *b : v) b->release();
        }
    } rel{{&d_bytes, &d_voff, &d_tidx, &d_soff, &d_vsig, &d_planes, &d_sorted, &d_idx, &d_idx2, &d_key, &d_key2}};
    std::vector<Sig> usig;            // distinct signatures, lexicographic
    std::vector<uint64_t> ustart;     // group starts into the sorted entry order
    std::vector<uint32_t> h_idx(N);   // sorted order of sets
    if (N > 0) {
        d_bytes.ensure(std::max<uint64_t>(sets->n_bytes, 1));
        d_voff.ensure((sets->n_vocab + 1) * 8);
        d_soff.ensure((N + 1) * 8);
        if (sets->n_bytes) TMCK(cudaMemcpyAsync(d_bytes.p, sets->vocab_bytes, sets->n_bytes, cudaMemcpyHostToDevice, s));
        if (sets->n_vocab) TMCK(cudaMemcpyAsync(d_voff.p, sets->vocab_off, (sets->n_vocab + 1) * 8, cudaMemcpyHostToDevice, s));
        TMCK(cudaMemcpyAsync(d_soff.p, sets->set_off, (N + 1) * 8, cudaMemcpyHostToDevice, s));
        if (sets->tag_idx && sets->n_tags) {
            d_tidx.ensure(sets->n_tags * 4);
            TMCK(cudaMemcpyAsync(d_tidx.p, sets->tag_idx, sets->n_tags * 4, cudaMemcpyHostToDevice, s));
        }
        d_vsig.ensure(std::max<uint64_t>(sets->n_vocab, 1) * 24);
        d_planes.ensure(N * 24);
        uint64_t *w0 = d_planes.as<uint64_t>(), *w1 = w0 + N, *w2 = w1 + N;
        TMCK(launch_hash_vocab(d_bytes.as<uint8_t>(), d_voff.as<uint64_t>(), nullptr, sets->n_vocab, sets->n_bytes,
                               d_vsig.as<uint64_t>(), nullptr, s));
        TMCK(launch_encode_sets(d_vsig.as<uint64_t>(), (sets->tag_idx && sets->n_tags) ? d_tidx.as<uint32_t>() : nullptr,
                                d_soff.as<uint64_t>(), N, sets->n_tags, sets->n_vocab, w0, w1, w2, nullptr, s));
        // S0b: lexicographic sort of the signatures (LSD: word 2, then 1, then 0; stable)
        d_idx.ensure(N * 4);
        d_idx2.ensure(N * 4);
        d_key.ensure(N * 8);
        d_key2.ensure(N * 8);
        TMCK(launch_iota(d_idx.as<uint32_t>(), N, s));
        const uint64_t *planes[3] = {w0, w1, w2};
        for (int w = 2; w >= 0; --w) {
            TMCK(launch_gather_u64(planes[w], d_idx.as<uint32_t>(), N, d_key.as<uint64_t>(), s));
            size_t tb = 0;
            TMCK(cub_sort_pairs_u64_u32(d_key.as<uint64_t>(), d_key2.as<uint64_t>(), d_idx.as<uint32_t>(),
                                        d_idx2.as<uint32_t>(), N, nullptr, &tb, s));
            TMCK(cub_sort_pairs_u64_u32(d_key.as<uint64_t>(), d_key2.as<uint64_t>(), d_idx.as<uint32_t>(),
                                        d_idx2.as<uint32_t>(), N, cub_tmp(db, tb), &tb, s));
            std::swap(d_idx, d_idx2);
        }
        d_sorted.ensure(N * 24);
        uint64_t *s0 = d_sorted.as<uint64_t>(), *s1 = s0 + N, *s2 = s1 + N;
        TMCK(launch_gather_planes(w0, w1, w2, d_idx.as<uint32_t>(), N, s0, s1, s2, s));
        if (!getenv("TM_BUILD_HOST") || db->cfg.exact) {  // consolidate on the GPU (default)
            d_planes.release();
            build_gpu(db, N, s0, s1, s2, d_idx.as<uint32_t>(), key_off, keys, mark);
            if (db->cfg.exact) {
                exact_build(db, d_bytes.as<uint8_t>(), sets->n_bytes, d_voff.as<uint64_t>(), sets->n_vocab,
                            (sets->tag_idx && sets->n_tags) ? d_tidx.as<uint32_t>() : nullptr, d_soff.as<uint64_t>(),
                            N, sets->n_tags, key_off, keys);
                mark("exact tables");
            }
            mark("done");
            db->build_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
            return;
        }
        std::vector<uint64_t> hs(3 * N);
        TMCK(cudaMemcpyAsync(hs.data(), d_sorted.p, N * 24, cudaMemcpyDeviceToHost, s));
        TMCK(cudaMemcpyAsync(h_idx.data(), d_idx.p, N * 4, cudaMemcpyDeviceToHost, s));
        TMCK(cudaStreamSynchronize(s));
        // distinct signatures (reading R10: identical signatures share a row)
        usig.reserve(N);
        ustart.reserve(N + 1);
        for (uint64_t i = 0; i < N; ++i) {
            Sig g{{hs[i], hs[N + i], hs[2 * N + i]}};
            if (i == 0 || g.w[0] != usig.back().w[0] || g.w[1] != usig.back().w[1] || g.w[2] != usig.back().w[2]) {
                usig.push_back(g);
                ustart.push_back(i);
            }
        }
        ustart.push_back(N);
    }
    const uint64_t U = usig.size();
    db->n_unique = U;

    mark("encode+sort+unique");
    // S0c: Algorithm 1 over the distinct signatures
    std::vector<uint32_t> order;
    std::vector<Partition> parts;
    alg1_partition(usig.data(), U, db->cfg.max_partition, order, parts);
    mark("alg1");
    if (db->cfg.row_order == 1) refine_order(usig.data(), order, parts, 8);
    mark("row order");
    db->n_parts_total = parts.size();
    const std::vector<uint32_t> owner = plan_shards(db, parts);

    // S0d: layout -- kept partitions in acceptance order, each padded to 32 rows
    std::vector<uint32_t> keep;
    for (uint32_t i = 0; i < parts.size(); ++i)
        if (owner[i] == db->cfg.shard) keep.push_back(i);
    const uint64_t P = keep.size();
    uint64_t rows = 0;
    for (uint32_t i : keep) rows += ((parts[i].end - parts[i].begin) + kTile - 1) / kTile * kTile;
    if (rows > 0xFFFFFFF0ull) fail(TM_ERANGE, "more than 2^32 rows");
    db->n_parts = P;
    db->n_rows = rows;
    std::vector<uint64_t> hp(3 * std::max<uint64_t>(rows, 1), ~0ULL);
    std::vector<uint32_t> hko(rows + 1, 0), hkeys;
    hkeys.reserve(K);
    db->h_masks.assign(3 * P, 0);
    db->h_sizes.assign(P, 0);
    db->h_part_row.assign(P + 1, 0);
    std::vector<uint32_t> hpn(std::max<uint64_t>(P, 1), 0);
    uint64_t r = 0;
    for (uint64_t pi = 0; pi < P; ++pi) {
        const Partition &pt = parts[keep[pi]];
        db->h_part_row[pi] = (uint32_t)r;
        const uint64_t np = pt.end - pt.begin;
        db->h_sizes[pi] = np;
        hpn[pi] = (uint32_t)np;
        for (int w = 0; w < 3; ++w) db->h_masks[3 * pi + w] = pt.mask.w[w];
        for (uint64_t m = 0; m < np; ++m, ++r) {
            const uint32_t u = order[pt.begin + m];
            hp[r] = usig[u].w[0];
            hp[rows + r] = usig[u].w[1];
            hp[2 * rows + r] = usig[u].w[2];
            for (uint64_t e = ustart[u]; e < ustart[u + 1]; ++e) {  // entries with this signature, set order
                const uint32_t set = h_idx[e];
                for (uint64_t k = key_off[set]; k < key_off[set + 1]; ++k) hkeys.push_back(keys[k]);
            }
            hko[r + 1] = (uint32_t)hkeys.size();
        }
        const uint64_t padded = (np + kTile - 1) / kTile * kTile;
        for (uint64_t m = np; m < padded; ++m, ++r) hko[r + 1] = (uint32_t)hkeys.size();  // padding rows: no keys
    }
    db->h_part_row[P] = (uint32_t)r;
    db->n_entries = hkeys.size();
    // per-tile AND of the real rows (the lossless strengthening of Alg. 4's prefix)
    const uint64_t ntiles = rows / kTile;
    std::vector<uint64_t> ht(3 * std::max<uint64_t>(ntiles, 1), ~0ULL);
    for (uint64_t pi = 0; pi < P; ++pi) {
        const uint64_t r0 = db->h_part_row[pi], r1 = r0 + db->h_sizes[pi];
        for (uint64_t rr = r0; rr < r1; ++rr)
            for (int w = 0; w < 3; ++w) ht[w * ntiles + rr / kTile] &= hp[w * rows + rr];
    }

    mark("layout");
    db->planes.ensure(std::max<uint64_t>(rows, 1) * 24);
    db->tand.ensure(std::max<uint64_t>(ntiles, 1) * 24);
    if (ntiles) TMCK(cudaMemcpyAsync(db->tand.p, ht.data(), ntiles * 24, cudaMemcpyHostToDevice, s));
    db->key_off.ensure((rows + 1) * 4);
    db->keys.ensure(std::max<uint64_t>(hkeys.size(), 1) * 4);
    db->masks.ensure(std::max<uint64_t>(P, 1) * 24);
    db->part_row.ensure((P + 1) * 4);
    db->part_n.ensure(std::max<uint64_t>(P, 1) * 4);
    if (rows) TMCK(cudaMemcpyAsync(db->planes.p, hp.data(), rows * 24, cudaMemcpyHostToDevice, s));
    TMCK(cudaMemcpyAsync(db->key_off.p, hko.data(), (rows + 1) * 4, cudaMemcpyHostToDevice, s));
    if (!hkeys.empty()) TMCK(cudaMemcpyAsync(db->keys.p, hkeys.data(), hkeys.size() * 4, cudaMemcpyHostToDevice, s));
    if (P) {
        TMCK(cudaMemcpyAsync(db->masks.p, db->h_masks.data(), P * 24, cudaMemcpyHostToDevice, s));
        TMCK(cudaMemcpyAsync(db->part_n.p, hpn.data(), P * 4, cudaMemcpyHostToDevice, s));
    }
    TMCK(cudaMemcpyAsync(db->part_row.p, db->h_part_row.data(), (P + 1) * 4, cudaMemcpyHostToDevice, s));
    TMCK(cudaStreamSynchronize(s));
    mark("upload");
    db->build_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

tm_db *new_db(const tm_config *cfg) {
    tm_db *db = new tm_db();
    if (cfg) db->cfg = *cfg;
    if (db->cfg.max_partition == 0) db->cfg.max_partition = TM_DEFAULT_MAX_PARTITION;
    if (db->cfg.n_shards == 0) db->cfg.n_shards = 1;
    if (db->cfg.tile_filter == 2) db->set_tune(kTuneDense);  // no pre-filter: the dense scan
    return db;
}

void destroy_db(tm_db *db) {
    if (!db) return;
    store_destroy(db);
    for (tm_db *sub : db->subs) destroy_db(sub);
    db->subs.clear();
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(db->device);
    if (db->stream) cudaStreamSynchronize(db->stream);
    try {
        shard_destroy(db);
    } catch (...) {
    }
    for (DevBuf *b : {&db->xfcnt, &db->xfin, &db->planes, &db->tand, &db->wsel, &db->wwords, &db->key_off, &db->keys, &db->masks, &db->part_row, &db->part_n, &db->in_bytes,
                      &db->in_voff, &db->in_tidx, &db->in_soff, &db->vsig, &db->qplanes, &db->bm, &db->word_off,
                      &db->qidx, &db->qoff, &db->item_cnt, &db->item_off, &db->out, &db->out_alt, &db->res_q,
                      &db->res_k, &db->res_off, &db->tmp, &db->ctr, &db->xcounts, &db->xall, &db->xrecv, &db->xalt, &db->mq,
                      &db->mk, &db->xv_bytes, &db->xv_off, &db->xv_hash, &db->xv_pos, &db->xv_canon, &db->xs_off,
                      &db->xs_ids, &db->xk_off, &db->xk_keys, &db->xq_canon, &db->xq_ids, &db->xflag, &db->xcnt,
                      &db->xkoff, &db->xkcnt, &db->res_kb, &db->res_qb})
        b->release();
    for (auto &e : db->ev)
        if (e) cudaEventDestroy(e);
    if (db->h_ctr) cudaFreeHost(db->h_ctr);
    if (db->h_nuniq) cudaFreeHost(db->h_nuniq);
    if (db->h_fx) cudaFreeHost(db->h_fx);
    for (auto &e : db->xev)
        if (e) cudaEventDestroy(e);
    if (db->xstream) cudaStreamDestroy(db->xstream);
    if (db->stream) cudaStreamDestroy(db->stream);
    if (prev >= 0) cudaSetDevice(prev);
    delete db;
}

int check_device(int dev) {
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0) {
        cudaGetLastError();
        fail(TM_ECUDA, "no CUDA device available (the library has no CPU fallback)");
    }
    if (dev < 0) TMCK(cudaGetDevice(&dev));
    if (dev >= n) fail(TM_EINVAL, "device ordinal out of range");
    cudaDeviceProp prop;
    TMCK(cudaGetDeviceProperties(&prop, dev));
    if (prop.major != 10) fail(TM_ECUDA, std::string("device is not sm_100 (Blackwell B200): ") + prop.name);
    return dev;
}

}  // namespace tmb

// ==================================================================== ABI ==
extern "C" {

uint32_t tm_abi_version(void) { return TM_ABI_VERSION; }

#ifndef TM_BUILD_ID
#define TM_BUILD_ID "unknown"
#endif
const char *tm_build_id(void) { return TM_BUILD_ID; }

const char *tm_strerror(tm_status s) {
    switch (s) {
        case TM_OK: return "ok";
        case TM_EINVAL: return "invalid argument";
        case TM_ENOMEM: return "out of memory";
        case TM_ECUDA: return "CUDA error";
        case TM_ENCCL: return "NCCL error";
        case TM_ERANGE: return "size out of range";
        case TM_ESTATE: return "invalid state";
    }
    return "unknown status";
}

const char *tm_last_error(void) { return tmb::g_err.c_str(); }

}  // extern "C"

namespace tmb {
// Validates the config and builds a single-GPU database (throws; the caller owns the result).
tm_db *build_db(const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys, const tm_config *cfg) {
    if (cfg) {
        if (cfg->n_shards > 1 && cfg->shard >= cfg->n_shards) fail(TM_EINVAL, "shard >= n_shards");
        if (cfg->tile_filter > 2) fail(TM_EINVAL, "tile_filter must be 0, 1 or 2");
        if (cfg->row_order > 1) fail(TM_EINVAL, "row_order must be 0 or 1");
        if (cfg->row_order == 1 && cfg->tile_filter == 0)
            fail(TM_EINVAL, "row_order 1 needs tile_filter 1 or 2 (the first/last prefix needs lexicographic order)");
        if (cfg->exact > 1) fail(TM_EINVAL, "exact must be 0 or 1");
        if (cfg->shard_mode > 1) fail(TM_EINVAL, "shard_mode must be TM_SHARD_PARTITIONED or TM_SHARD_REPLICATED");
        if (cfg->reserved) fail(TM_EINVAL, "reserved fields must be 0");
        if (cfg->plan_sample) check_tagsets_host(cfg->plan_sample, "plan_sample");
    }
    const int dev = check_device(cfg ? cfg->device : -1);
    DeviceGuard g(dev);
    tm_db *db = new_db(cfg);
    try {
        db->device = dev;
        TMCK(cudaStreamCreateWithFlags(&db->stream, cudaStreamNonBlocking));
        for (auto &e : db->ev) TMCK(cudaEventCreate(&e));
        TMCK(cudaMallocHost((void **)&db->h_ctr, sizeof(DevCounters)));
        TMCK(cudaMallocHost((void **)&db->h_nuniq, 8));
        TMCK(cudaMallocHost((void **)&db->h_fx, kMaxOwners * 8));
        db->scan_grid = 0;
        build_impl(db, sets, key_off, keys);
        // load every scan-kernel variant now (lazy module loading would otherwise put ~10-30 ms into
        // the first call that picks a variant: a latency spike inside a stream, profiles/r1v46_stream_*)
        for (int v = 0; v < kScanVariants; ++v) db->grid_of[v] = scan_grid(db->device, v);
        db->st.n_sets = db->n_sets;
        db->cfg.plan_sample = nullptr;  // borrowed for the build only
        db->cfg.device_ids = nullptr;
    } catch (...) {
        destroy_db(db);
        throw;
    }
    return db;
}
}  // namespace tmb

namespace tmb {
// H2D of a host query batch into the handle's input buffers; returns the device-side tagsets.
tm_tagsets upload_queries(tm_db *db, const tm_tagsets *q, cudaStream_t s) {
    tm_tagsets dq = *q;
    dq.vocab_bytes = nullptr;
    dq.vocab_off = nullptr;
    db->in_soff.ensure((q->n_sets + 1) * 8);
    TMCK(cudaMemcpyAsync(db->in_soff.p, q->set_off, (q->n_sets + 1) * 8, cudaMemcpyHostToDevice, s));
    dq.set_off = db->in_soff.as<uint64_t>();
    if (q->vocab_hash && q->n_vocab) {  // pre-hashed vocabulary: the hashes instead of the strings
        db->in_vhash.ensure(q->n_vocab * 8);
        TMCK(cudaMemcpyAsync(db->in_vhash.p, q->vocab_hash, q->n_vocab * 8, cudaMemcpyHostToDevice, s));
        dq.vocab_hash = db->in_vhash.as<uint64_t>();
    }
    if (q->n_bytes) {
        db->in_bytes.ensure(q->n_bytes);
        TMCK(cudaMemcpyAsync(db->in_bytes.p, q->vocab_bytes, q->n_bytes, cudaMemcpyHostToDevice, s));
        dq.vocab_bytes = db->in_bytes.as<uint8_t>();
    }
    if (q->n_vocab && !q->vocab_hash) {
        db->in_voff.ensure((q->n_vocab + 1) * 8);
        TMCK(cudaMemcpyAsync(db->in_voff.p, q->vocab_off, (q->n_vocab + 1) * 8, cudaMemcpyHostToDevice, s));
        dq.vocab_off = db->in_voff.as<uint64_t>();
    }
    if (q->tag_idx && q->n_tags) {
        db->in_tidx.ensure(q->n_tags * 4);
        TMCK(cudaMemcpyAsync(db->in_tidx.p, q->tag_idx, q->n_tags * 4, cudaMemcpyHostToDevice, s));
        dq.tag_idx = db->in_tidx.as<uint32_t>();
    } else {
        dq.tag_idx = nullptr;
    }
    return dq;
}
// consolidate() of a mutable handle: a fresh database is built from the live entries and swapped
// into the handle (the caller's pointer stays valid); the old tables are freed.
void rebuild(tm_db *db, const tm_tagsets *sets, const uint32_t *keys, const tm_config *cfg) {
    tm_db *fresh = nullptr;
    if (cfg->n_gpus > 1) {
        fresh = new_db(cfg);
        try {
            group_build(fresh, sets, nullptr, keys, cfg);
        } catch (...) {
            destroy_db(fresh);
            throw;
        }
    } else {
        fresh = build_db(sets, nullptr, keys, cfg);
    }
    Store *st = db->store;
    std::vector<int32_t> devs = std::move(db->store_devices);
    void *comm = db->nccl_comm;
    const int nr = db->nranks, rk = db->rank;
    db->store = nullptr;
    db->nccl_comm = nullptr;
    std::swap(*db, *fresh);
    db->store = st;
    db->store_devices = std::move(devs);
    db->nccl_comm = comm;
    db->nranks = nr;
    db->rank = rk;
    fresh->nccl_comm = nullptr;
    destroy_db(fresh);
}
// Query ranges of a pipelined tm_match_batch_csr / tm_match_batch: the result's device-to-host copy
// (4 or 8 B per pair, ~0.85 GB at C3, PCIe-bound) of range k runs on a copy stream while the GPU matches range k + 1,
// so only the last range's copy stays on the critical path.  TM_PIPELINE=n forces n ranges (1 = off).
uint32_t pipeline_ranges(uint64_t Q) {
    const char *e = getenv("TM_PIPELINE");
    const long forced = e ? atol(e) : 0;
    if (forced >= 1) return (uint32_t)std::min<long>(forced, 64);
    // ranges of >= 250K queries: smaller ones leave few routed queries per partition, which the item
    // planner cuts into quarter row ranges (C3 at 8 ranges of 125K: 284 instead of 229 ms per step)
    return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(4, Q / 250000));
}

// Pipelined tm_match_batch_csr (cout) / tm_match_batch (pout): S query ranges matched in order
// on the handle's stream; range k's result (keys and its slice of the query offsets, or its query
// and key arrays) is copied to the pinned result block on a copy stream while range k + 1 runs.
// Result buffers are double-buffered (res_k / res_kb, res_q / res_qb), each reused only after the
// copy that read it; the pinned block holds [Q + 1 offsets | cap keys] or [cap queries | cap keys].
void match_pipelined(tm_db *db, const tm_tagsets *dq, int unique, uint32_t S, tm_csr *cout, tm_pairs *pout) {
    cudaStream_t s = db->stream;
    const uint64_t Q = dq->n_sets;
    const bool csr = cout != nullptr;
    if (!db->xstream) {
        TMCK(cudaStreamCreateWithFlags(&db->xstream, cudaStreamNonBlocking));
        for (auto &e : db->xev) TMCK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    cudaStream_t x = db->xstream;
    if (csr) db->res_off.ensure((Q + 1) * 8);
    const uint64_t head = csr ? (Q + 1) * 8 : 0;  // bytes before the first result array
    PinnedBlock *blk = nullptr;
    uint64_t cap = 0, total = 0;  // pairs the pinned block holds (per array) / pairs copied so far
    struct Guard {  // on an error: no copy in flight into a block that is handed back
        tm_db *db;
        PinnedBlock **blk;
        ~Guard() {
            if (*blk) {
                cudaStreamSynchronize(db->xstream);
                pinned_put(*blk);
            }
        }
    } guard{db, &blk};
    auto q_arr = [&](void *base) { return reinterpret_cast<uint32_t *>(static_cast<char *>(base) + head); };
    auto k_arr = [&](void *base, uint64_t c) { return q_arr(base) + (csr ? 0 : c); };
    tm_stats_t acc = db->st;
    double enc = 0, route = 0, scan = 0, merge = 0, tot = 0;
    uint64_t sums[11] = {};
    uint32_t launches = 0, scans = 0;
    for (uint32_t k = 0; k < S; ++k) {
        const uint64_t qlo = Q * k / S, qn = Q * (k + 1) / S - qlo;
        if (k) {  // range k writes result buffers k & 1
            std::swap(db->res_k, db->res_kb);
            std::swap(db->res_q, db->res_qb);
        }
        // the copy of range k - 2 read these buffers
        if (k >= 2) TMCK(cudaStreamWaitEvent(s, db->xev[k & 1], 0));
        const uint64_t n = match_core(db, dq, unique, s, qlo, qn, k > 0);
        if (csr) {
            const uint64_t *sorted = n ? db->last_sorted : nullptr;
            TMCK(launch_query_offsets(sorted, n, qlo, qn, total, db->res_off.as<uint64_t>() + qlo, s));
        }
        TMCK(cudaEventRecord(db->xev[2], s));
        finish_timing(db, s);
        const tm_stats_t &st = db->st;
        enc += st.encode_ms;
        route += st.route_ms;
        scan += st.scan_ms;
        merge += st.merge_ms;
        tot += st.total_ms;
        const uint64_t v[11] = {st.routed, st.candidate_pairs, st.tile_tests, st.pair_checks, st.matched_sets,
                                st.emitted_pairs, st.result_pairs, st.work_items, st.retries, st.exact_checked,
                                st.exact_kept};
        for (int i = 0; i < 11; ++i) sums[i] += v[i];
        launches += st.kernel_launches + (csr ? 1 : 0);
        scans += st.scan_launches;
        acc.scan_variant = st.scan_variant;
        acc.tuning = st.tuning;
        if (total + n > cap) {  // the pinned result block: sized by the first range and the largest earlier
                                // result, so a repeated batch size reuses one cached block; grown if short
            const uint64_t want = std::max<uint64_t>(std::max<uint64_t>((total + n) + (total + n) / 4,
                                                                        (n + 1) * S + (n + 1) * S / 4),
                                                     db->pipe_pairs_hint + db->pipe_pairs_hint / 16);
            PinnedBlock *nb = pinned_get(head + want * 4 * (csr ? 1 : 2));
            if (blk) {
                TMCK(cudaStreamSynchronize(x));
                memcpy(nb->p, blk->p, head + total * 4);  // offsets + keys, or the queries
                if (!csr) memcpy(k_arr(nb->p, want), k_arr(blk->p, cap), total * 4);
                pinned_put(blk);
            }
            blk = nb;
            cap = want;
        }
        TMCK(cudaStreamWaitEvent(x, db->xev[2], 0));
        if (csr)
            TMCK(cudaMemcpyAsync(static_cast<uint64_t *>(blk->p) + qlo, db->res_off.as<uint64_t>() + qlo, qn * 8,
                                 cudaMemcpyDeviceToHost, x));
        else if (n)
            TMCK(cudaMemcpyAsync(q_arr(blk->p) + total, db->res_q.p, n * 4, cudaMemcpyDeviceToHost, x));
        if (n) TMCK(cudaMemcpyAsync(k_arr(blk->p, cap) + total, db->res_k.p, n * 4, cudaMemcpyDeviceToHost, x));
        TMCK(cudaEventRecord(db->xev[k & 1], x));
        total += n;
    }
    TMCK(cudaStreamSynchronize(x));
    db->pipe_pairs_hint = std::max(db->pipe_pairs_hint, total);
    // the call's statistics: sums over the ranges (stage times are the ranges' CUDA-event times)
    acc.n_queries = Q;
    uint64_t *dst[11] = {&acc.routed, &acc.candidate_pairs, &acc.tile_tests, &acc.pair_checks, &acc.matched_sets,
                         &acc.emitted_pairs, &acc.result_pairs, &acc.work_items, &acc.retries, &acc.exact_checked,
                         &acc.exact_kept};
    for (int i = 0; i < 11; ++i) *dst[i] = sums[i];
    acc.encode_ms = enc;
    acc.route_ms = route;
    acc.scan_ms = scan;
    acc.merge_ms = merge;
    acc.total_ms = tot;
    acc.kernel_launches = launches;
    acc.scan_launches = scans;
    db->st = acc;
    db->last_sorted = nullptr;  // the pairs of the last range only: not a whole-call result
    db->last_n = 0;
    if (csr) {
        uint64_t *hoff = static_cast<uint64_t *>(blk->p);
        hoff[Q] = total;
        cout->n_queries = Q;
        cout->n = total;
        cout->q_off = hoff;
        cout->key = k_arr(blk->p, cap);
        cout->priv_ = blk;
    } else {
        pout->n = total;
        pout->query = q_arr(blk->p);
        pout->key = k_arr(blk->p, cap);
        pout->priv_ = blk;
    }
    blk = nullptr;  // handed to the caller (tm_csr_free / tm_pairs_free)
}
}  // namespace tmb

extern "C" {

tm_status tm_build(const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys, const tm_config *cfg,
                   tm_db **out) {
    TM_API_BEGIN
    if (!out) fail(TM_EINVAL, "out is NULL");
    check_tagsets_host(sets, "sets");
    require_strings(sets, "sets");
    if (cfg && cfg->n_gpus > 1) {  // in-process multi-GPU database (tm_group.cu)
        tm_db *top = new_db(cfg);
        try {
            group_build(top, sets, key_off, keys, cfg);
        } catch (...) {
            destroy_db(top);
            throw;
        }
        *out = top;
        return TM_OK;
    }
    *out = build_db(sets, key_off, keys, cfg);
    return TM_OK;
    TM_API_END
}



tm_status tm_match_batch(tm_db *db, const tm_tagsets *q, int unique, tm_pairs *out) {
    TM_API_BEGIN
    if (!db || !out) fail(TM_EINVAL, "db or out is NULL");
    if (unique != 0 && unique != 1) fail(TM_EINVAL, "unique must be 0 or 1");
    check_tagsets_shape(q, "queries");
    if (!db->subs.empty()) {
        group_match(db, q, unique, out, nullptr);
        return TM_OK;
    }
    DeviceGuard g(db->device);
    cudaStream_t s = db->stream;
    const tm_tagsets dq = upload_queries(db, q, s);  // one H2D copy of the query batch
    const uint32_t S = pipeline_ranges(q->n_sets);
    if (S > 1) {  // query ranges, each range's D2H under the next range's GPU work
        match_pipelined(db, &dq, unique, S, nullptr, out);
        return TM_OK;
    }
    const uint64_t n = match_core(db, &dq, unique, s);
    PinnedBlock *blk = pinned_get(std::max<uint64_t>(n, 1) * 8);
    uint32_t *hq = static_cast<uint32_t *>(blk->p), *hk = hq + n;
    if (n) {
        cudaError_t e1 = cudaMemcpyAsync(hq, db->res_q.p, n * 4, cudaMemcpyDeviceToHost, s);
        cudaError_t e2 = cudaMemcpyAsync(hk, db->res_k.p, n * 4, cudaMemcpyDeviceToHost, s);
        if (e1 != cudaSuccess || e2 != cudaSuccess) {
            pinned_put(blk);
            throw CudaFail{e1 != cudaSuccess ? e1 : e2, "cudaMemcpyAsync(D2H results)", __LINE__};
        }
    }
    try {
        finish_timing(db, s);
    } catch (...) {
        pinned_put(blk);
        throw;
    }
    out->n = n;
    out->query = hq;
    out->key = hk;
    out->priv_ = blk;
    return TM_OK;
    TM_API_END
}

tm_status tm_match_batch_csr(tm_db *db, const tm_tagsets *q, int unique, tm_csr *out) {
    TM_API_BEGIN
    if (!db || !out) fail(TM_EINVAL, "db or out is NULL");
    if (unique != 0 && unique != 1) fail(TM_EINVAL, "unique must be 0 or 1");
    check_tagsets_shape(q, "queries");
    if (!db->subs.empty()) {
        group_match(db, q, unique, nullptr, out);
        return TM_OK;
    }
    DeviceGuard g(db->device);
    cudaStream_t s = db->stream;
    const tm_tagsets dq = upload_queries(db, q, s);
    const uint64_t Q = q->n_sets;
    const uint32_t S = pipeline_ranges(Q);
    if (S > 1) {
        match_pipelined(db, &dq, unique, S, out, nullptr);
        return TM_OK;
    }
    const uint64_t n = match_core(db, &dq, unique, s);
    db->res_off.ensure((Q + 1) * 8);
    const uint64_t *sorted = n ? db->last_sorted : nullptr;
    TMCK(launch_query_offsets(sorted, n, 0, Q, 0, db->res_off.as<uint64_t>(), s));
    PinnedBlock *blk = pinned_get((Q + 1) * 8 + std::max<uint64_t>(n, 1) * 4);
    uint64_t *hoff = static_cast<uint64_t *>(blk->p);
    uint32_t *hk = reinterpret_cast<uint32_t *>(hoff + Q + 1);
    cudaError_t e1 = cudaMemcpyAsync(hoff, db->res_off.p, (Q + 1) * 8, cudaMemcpyDeviceToHost, s);
    cudaError_t e2 = n ? cudaMemcpyAsync(hk, db->res_k.p, n * 4, cudaMemcpyDeviceToHost, s) : cudaSuccess;
    if (e1 != cudaSuccess || e2 != cudaSuccess) {
        pinned_put(blk);
        throw CudaFail{e1 != cudaSuccess ? e1 : e2, "cudaMemcpyAsync(D2H results)", __LINE__};
    }
    try {
        finish_timing(db, s);
    } catch (...) {
        pinned_put(blk);
        throw;
    }
    out->n_queries = Q;
    out->n = n;
    out->q_off = hoff;
    out->key = hk;
    out->priv_ = blk;
    return TM_OK;
    TM_API_END
}

tm_status tm_match_batch_device(tm_db *db, const tm_tagsets *q, int unique, tm_dev_pairs *out, void *stream) {
    TM_API_BEGIN
    if (!db || !out) fail(TM_EINVAL, "db or out is NULL");
    if (!db->subs.empty()) fail(TM_ESTATE, "device-pointer calls are not available on an in-process multi-GPU handle");
    if (unique != 0 && unique != 1) fail(TM_EINVAL, "unique must be 0 or 1");
    check_tagsets_device(q);
    DeviceGuard g(db->device);
    cudaStream_t s = stream ? static_cast<cudaStream_t>(stream) : db->stream;
    tm_tagsets dq = *q;
    if (!dq.n_tags) dq.tag_idx = nullptr;
    const uint64_t n = match_core(db, &dq, unique, s);
    finish_timing(db, s);
    out->n = n;
    out->query = db->res_q.as<uint32_t>();
    out->key = db->res_k.as<uint32_t>();
    return TM_OK;
    TM_API_END
}

void tm_csr_free(tm_csr *c) {
    if (!c) return;
    if (c->priv_) tmb::pinned_put(static_cast<tmb::PinnedBlock *>(c->priv_));
    c->n_queries = 0;
    c->n = 0;
    c->q_off = nullptr;
    c->key = nullptr;
    c->priv_ = nullptr;
}

void tm_pairs_free(tm_pairs *p) {
    if (!p) return;
    if (p->priv_) tmb::pinned_put(static_cast<tmb::PinnedBlock *>(p->priv_));
    p->n = 0;
    p->query = nullptr;
    p->key = nullptr;
    p->priv_ = nullptr;
}

void tm_free(tm_db *db) { tmb::destroy_db(db); }

tm_status tm_encode(const tm_tagsets *sets, uint64_t *sig_out, int device) {
    TM_API_BEGIN
    check_tagsets_host(sets, "sets");
    if (sets->n_sets && !sig_out) fail(TM_EINVAL, "sig_out is NULL");
    const int dev = check_device(device);
    DeviceGuard g(dev);
    const uint64_t N = sets->n_sets;
    if (!N) return TM_OK;
    cudaStream_t s;
    TMCK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    DevBuf b, vo, ti, so, vs, pl, vh;
    struct Rel {
        std::vector<DevBuf *> v;
        cudaStream_t s;
        ~Rel() {
            cudaStreamSynchronize(s);
            for (auto *x : v) x->release();
            cudaStreamDestroy(s);
        }
    } rel{{&b, &vo, &ti, &so, &vs, &pl, &vh}, s};
    b.ensure(std::max<uint64_t>(sets->n_bytes, 1));
    vo.ensure((sets->n_vocab + 1) * 8);
    so.ensure((N + 1) * 8);
    vs.ensure(std::max<uint64_t>(sets->n_vocab, 1) * 24);
    pl.ensure(N * 24);
    if (sets->n_bytes) TMCK(cudaMemcpyAsync(b.p, sets->vocab_bytes, sets->n_bytes, cudaMemcpyHostToDevice, s));
    const uint64_t *dvh = nullptr;
    if (sets->vocab_hash) {
        if (sets->n_vocab) {
            vh.ensure(sets->n_vocab * 8);
            TMCK(cudaMemcpyAsync(vh.p, sets->vocab_hash, sets->n_vocab * 8, cudaMemcpyHostToDevice, s));
        }
        dvh = vh.as<uint64_t>();
    } else if (sets->n_vocab) {
        TMCK(cudaMemcpyAsync(vo.p, sets->vocab_off, (sets->n_vocab + 1) * 8, cudaMemcpyHostToDevice, s));
    }
    TMCK(cudaMemcpyAsync(so.p, sets->set_off, (N + 1) * 8, cudaMemcpyHostToDevice, s));
    const uint32_t *dti = nullptr;
    if (sets->tag_idx && sets->n_tags) {
        ti.ensure(sets->n_tags * 4);
        TMCK(cudaMemcpyAsync(ti.p, sets->tag_idx, sets->n_tags * 4, cudaMemcpyHostToDevice, s));
        dti = ti.as<uint32_t>();
    }
    uint64_t *w0 = pl.as<uint64_t>(), *w1 = w0 + N, *w2 = w1 + N;
    TMCK(launch_hash_vocab(b.as<uint8_t>(), vo.as<uint64_t>(), dvh, sets->n_vocab, sets->n_bytes, vs.as<uint64_t>(),
                           nullptr, s));
    TMCK(launch_encode_sets(vs.as<uint64_t>(), dti, so.as<uint64_t>(), N, sets->n_tags, sets->n_vocab, w0, w1, w2,
                            nullptr, s));
    std::vector<uint64_t> h(3 * N);
    TMCK(cudaMemcpyAsync(h.data(), pl.p, N * 24, cudaMemcpyDeviceToHost, s));
    TMCK(cudaStreamSynchronize(s));
    for (uint64_t i = 0; i < N; ++i) {
        sig_out[3 * i] = h[i];
        sig_out[3 * i + 1] = h[N + i];
        sig_out[3 * i + 2] = h[2 * N + i];
    }
    return TM_OK;
    TM_API_END
}

tm_status tm_stats(const tm_db *db, tm_stats_t *out) {
    TM_API_BEGIN
    if (!db || !out) fail(TM_EINVAL, "db or out is NULL");
    if (!db->subs.empty()) {
        group_stats(db, out);
        return TM_OK;
    }
    *out = db->st;
    out->n_sets = db->n_sets;
    out->n_entries = db->n_entries;
    out->n_unique = db->n_unique;
    out->n_rows = db->n_rows;
    out->n_partitions = db->n_parts;
    out->n_partitions_total = db->n_parts_total;
    out->build_ms = db->build_ms;
    out->max_partition = db->cfg.max_partition;
    out->n_gpus = 1;
    return TM_OK;
    TM_API_END
}

tm_status tm_partitions(const tm_db *db, uint64_t *masks, uint64_t *sizes) {
    TM_API_BEGIN
    if (!db) fail(TM_EINVAL, "db is NULL");
    if (!db->subs.empty()) fail(TM_ESTATE, "use tm_group_member on an in-process multi-GPU handle");
    if (masks && !db->h_masks.empty()) std::memcpy(masks, db->h_masks.data(), db->h_masks.size() * 8);
    if (sizes && !db->h_sizes.empty()) std::memcpy(sizes, db->h_sizes.data(), db->h_sizes.size() * 8);
    return TM_OK;
    TM_API_END
}

tm_status tm_partition_sigs(const tm_db *db, uint64_t p, uint64_t *sig_out) {
    TM_API_BEGIN
    if (!db || !sig_out) fail(TM_EINVAL, "db or sig_out is NULL");
    if (!db->subs.empty()) fail(TM_ESTATE, "use tm_group_member on an in-process multi-GPU handle");
    if (p >= db->n_parts) fail(TM_EINVAL, "partition index out of range");
    DeviceGuard g(db->device);
    const uint64_t r0 = db->h_part_row[p], n = db->h_sizes[p];
    std::vector<uint64_t> h(3 * n);
    const uint64_t *d = db->planes.as<uint64_t>();
    for (int w = 0; w < 3; ++w)
        if (n) TMCK(cudaMemcpy(h.data() + w * n, d + w * db->n_rows + r0, n * 8, cudaMemcpyDeviceToHost));
    for (uint64_t i = 0; i < n; ++i)
        for (int w = 0; w < 3; ++w) sig_out[3 * i + w] = h[w * n + i];
    return TM_OK;
    TM_API_END
}

}  // extern "C"
