// tm_stream.cpp -- streaming front-end with batch timeout ("TagMatch
// batches queries ... uses a configurable timeout period after which it
// automatically processes batches even if they are not full"; Fig. 6).
//
// Queries are submitted one at a time; a dispatcher thread closes the open batch
// when it holds max_batch queries or when its oldest query has waited timeout_us,
// runs it through the whole GPU path (tm_match_batch) while the next batch keeps
// filling, and publishes per-batch results with timestamps.  On the B200 one
// batch covers every partition (one kernel chain), so there is one queue rather
// than one per partition as in the paper's CPU/GPU pipeline.
#include <chrono>
#include <condition_variable>
#include <cstring>
#include <deque>
#include <mutex>
#include <thread>

#include "tm_db.h"

namespace tmb {
namespace {

uint64_t now_ns() {
    return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
               std::chrono::steady_clock::now().time_since_epoch())
        .count();
}

struct Batch {
    std::vector<uint8_t> bytes;
    std::vector<uint64_t> tag_off{0};   // byte offsets of tag strings
    std::vector<uint64_t> set_off{0};   // tag offsets of queries
    std::vector<uint64_t> tickets, submit_ns;
    void clear() {
        bytes.clear();
        tag_off.assign(1, 0);
        set_off.assign(1, 0);
        tickets.clear();
        submit_ns.clear();
    }
    size_t size() const { return tickets.size(); }
};

// move the first n queries of src into dst (dst cleared), rebasing src's offsets
void take_front(Batch &src, size_t n, Batch &dst) {
    dst.clear();
    if (n >= src.size()) {
        std::swap(dst, src);
        src.clear();
        return;
    }
    const uint64_t ntag = src.set_off[n], nbyte = src.tag_off[ntag];
    dst.bytes.assign(src.bytes.begin(), src.bytes.begin() + nbyte);
    dst.tag_off.assign(src.tag_off.begin(), src.tag_off.begin() + ntag + 1);
    dst.set_off.assign(src.set_off.begin(), src.set_off.begin() + n + 1);
    dst.tickets.assign(src.tickets.begin(), src.tickets.begin() + n);
    dst.submit_ns.assign(src.submit_ns.begin(), src.submit_ns.begin() + n);
    Batch rest;
    rest.bytes.assign(src.bytes.begin() + nbyte, src.bytes.end());
    rest.tag_off.clear();
    for (size_t i = ntag; i < src.tag_off.size(); ++i) rest.tag_off.push_back(src.tag_off[i] - nbyte);
    rest.set_off.clear();
    for (size_t i = n; i < src.set_off.size(); ++i) rest.set_off.push_back(src.set_off[i] - ntag);
    rest.tickets.assign(src.tickets.begin() + n, src.tickets.end());
    rest.submit_ns.assign(src.submit_ns.begin() + n, src.submit_ns.end());
    std::swap(src, rest);
}

struct Result {
    std::vector<uint64_t> tickets, submit_ns, key_off;
    std::vector<uint32_t> keys;
    uint64_t dispatch_ns = 0, done_ns = 0;
    tm_status status = TM_OK;
};

}  // namespace
}  // namespace tmb

struct tm_stream {
    tm_db *db = nullptr;
    tm_stream_config cfg{};
    std::mutex mu;
    std::condition_variable cv_submit, cv_done;
    tmb::Batch open;
    std::deque<tmb::Result *> done;
    uint64_t next_ticket = 0;
    uint64_t inflight = 0;  // submitted but not yet published
    bool closing = false;
    bool force = false;  // tm_stream_flush: dispatch the open batch now
    std::thread worker;
};

namespace tmb {
namespace {

void dispatcher(tm_stream *st) {
    Batch work;
    for (;;) {
        {
            std::unique_lock<std::mutex> lk(st->mu);
            for (;;) {
                if (st->open.size() >= st->cfg.max_batch) break;
                if (st->open.size() && (st->closing || st->force)) break;
                if (!st->open.size()) {
                    if (st->closing) return;
                    st->cv_submit.wait(lk);
                    continue;
                }
                const uint64_t deadline = st->open.submit_ns[0] + (uint64_t)st->cfg.timeout_us * 1000ULL;
                const uint64_t t = now_ns();
                if (st->cfg.timeout_us && t >= deadline) break;
                if (st->cfg.timeout_us)
                    st->cv_submit.wait_for(lk, std::chrono::nanoseconds(deadline - t));
                else
                    st->cv_submit.wait(lk);
            }
            // at most max_batch queries; the rest (and new arrivals) fill the next batch
            take_front(st->open, st->cfg.max_batch, work);
            if (!st->open.size()) st->force = false;
        }
        Result *r = new Result();
        r->dispatch_ns = now_ns();
        tm_tagsets q{};
        q.vocab_bytes = work.bytes.data();
        q.vocab_off = work.tag_off.data();
        q.tag_idx = nullptr;
        q.set_off = work.set_off.data();
        q.n_bytes = work.bytes.size();
        q.n_vocab = work.tag_off.size() - 1;
        q.n_tags = q.n_vocab;
        q.n_sets = work.size();
        tm_pairs pairs{};
        r->status = tm_match_batch(st->db, &q, st->cfg.unique, &pairs);
        r->tickets = work.tickets;
        r->submit_ns = work.submit_ns;
        r->key_off.assign(work.size() + 1, 0);
        if (r->status == TM_OK) {
            for (uint64_t i = 0; i < pairs.n; ++i) r->key_off[pairs.query[i] + 1]++;
            for (size_t i = 0; i < work.size(); ++i) r->key_off[i + 1] += r->key_off[i];
            r->keys.assign(pairs.key, pairs.key + pairs.n);  // pairs are sorted by (query, key)
            tm_pairs_free(&pairs);
        }
        r->done_ns = now_ns();
        {
            std::lock_guard<std::mutex> lk(st->mu);
            st->inflight -= work.size();
            st->done.push_back(r);
        }
        st->cv_done.notify_all();
        work.clear();
    }
}

}  // namespace
}  // namespace tmb

extern "C" {

tm_status tm_stream_open(tm_db *db, const tm_stream_config *cfg, tm_stream **out) {
    TM_API_BEGIN
    if (!db || !cfg || !out) fail(TM_EINVAL, "NULL argument");
    if (cfg->max_batch == 0) fail(TM_EINVAL, "max_batch must be > 0");
    if (cfg->unique != 0 && cfg->unique != 1) fail(TM_EINVAL, "unique must be 0 or 1");
    tm_stream *st = new tm_stream();
    st->db = db;
    st->cfg = *cfg;
    st->worker = std::thread(tmb::dispatcher, st);
    *out = st;
    return TM_OK;
    TM_API_END
}

tm_status tm_stream_submit(tm_stream *st, const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags,
                           uint64_t *ticket) {
    TM_API_BEGIN
    if (!st || !ticket || (n_tags && !tag_off)) fail(TM_EINVAL, "NULL argument");
    if (n_tags && tag_off[0] != 0) fail(TM_EINVAL, "tag_off[0] != 0");
    for (uint64_t i = 0; i < n_tags; ++i)
        if (tag_off[i + 1] < tag_off[i]) fail(TM_EINVAL, "tag_off not non-decreasing");
    const uint64_t nb = n_tags ? tag_off[n_tags] : 0;
    if (nb && !bytes) fail(TM_EINVAL, "bytes is NULL");
    bool wake = false;
    {
        std::lock_guard<std::mutex> lk(st->mu);
        if (st->closing) fail(TM_ESTATE, "stream is closing");
        tmb::Batch &b = st->open;
        const uint64_t base = b.bytes.size();
        b.bytes.insert(b.bytes.end(), bytes, bytes + nb);
        for (uint64_t i = 1; i <= n_tags; ++i) b.tag_off.push_back(base + tag_off[i]);
        b.set_off.push_back(b.tag_off.size() - 1);
        *ticket = st->next_ticket++;
        b.tickets.push_back(*ticket);
        b.submit_ns.push_back(tmb::now_ns());
        st->inflight++;
        // wake the dispatcher only when its decision can change: the batch became
        // non-empty (its timeout clock starts) or reached max_batch
        wake = b.size() == 1 || b.size() >= st->cfg.max_batch;
    }
    if (wake) st->cv_submit.notify_one();
    return TM_OK;
    TM_API_END
}

tm_status tm_stream_poll(tm_stream *st, int wait, tm_stream_result *out) {
    TM_API_BEGIN
    if (!st || !out) fail(TM_EINVAL, "NULL argument");
    std::memset(out, 0, sizeof *out);
    tmb::Result *r = nullptr;
    {
        std::unique_lock<std::mutex> lk(st->mu);
        if (wait)
            st->cv_done.wait(lk, [&] { return !st->done.empty() || st->inflight == 0; });
        if (st->done.empty()) return TM_OK;  // n_queries = 0: nothing ready
        r = st->done.front();
        st->done.pop_front();
    }
    if (r->status != TM_OK) {
        const tm_status s = r->status;
        delete r;
        fail(s, "batch failed on the GPU path");
    }
    out->n_queries = r->tickets.size();
    out->tickets = r->tickets.data();
    out->submit_ns = r->submit_ns.data();
    out->key_off = r->key_off.data();
    out->keys = r->keys.data();
    out->dispatch_ns = r->dispatch_ns;
    out->done_ns = r->done_ns;
    out->priv_ = r;
    return TM_OK;
    TM_API_END
}

void tm_stream_result_free(tm_stream_result *r) {
    if (!r) return;
    delete static_cast<tmb::Result *>(r->priv_);
    std::memset(r, 0, sizeof *r);
}

tm_status tm_stream_flush(tm_stream *st) {
    TM_API_BEGIN
    if (!st) fail(TM_EINVAL, "NULL stream");
    std::unique_lock<std::mutex> lk(st->mu);
    while (st->inflight > 0) {
        if (st->open.size()) {
            st->force = true;
            st->cv_submit.notify_one();
        }
        st->cv_done.wait_for(lk, std::chrono::milliseconds(1));
    }
    return TM_OK;
    TM_API_END
}

tm_status tm_stream_replay(tm_stream *st, const tm_tagsets *q, const uint64_t *arrival_ns) {
    TM_API_BEGIN
    if (!st || !q || !arrival_ns) fail(TM_EINVAL, "NULL argument");
    if (q->n_sets && (!q->set_off || (q->n_vocab && !q->vocab_off))) fail(TM_EINVAL, "bad tag sets");
    const uint64_t t0 = tmb::now_ns();
    for (uint64_t i = 0; i < q->n_sets; ++i) {
        const uint64_t due = t0 + arrival_ns[i];
        while (tmb::now_ns() < due) {
        }
        bool wake = false;
        {
            std::lock_guard<std::mutex> lk(st->mu);
            if (st->closing) fail(TM_ESTATE, "stream is closing");
            tmb::Batch &b = st->open;
            for (uint64_t t = q->set_off[i]; t < q->set_off[i + 1]; ++t) {
                const uint64_t v = q->tag_idx ? q->tag_idx[t] : t;
                if (v >= q->n_vocab) fail(TM_EINVAL, "tag_idx out of range");
                const uint64_t a = q->vocab_off[v], e = q->vocab_off[v + 1];
                b.bytes.insert(b.bytes.end(), q->vocab_bytes + a, q->vocab_bytes + e);
                b.tag_off.push_back(b.bytes.size());
            }
            b.set_off.push_back(b.tag_off.size() - 1);
            b.tickets.push_back(st->next_ticket++);
            b.submit_ns.push_back(tmb::now_ns());
            st->inflight++;
            wake = b.size() == 1 || b.size() >= st->cfg.max_batch;
        }
        if (wake) st->cv_submit.notify_one();
    }
    return TM_OK;
    TM_API_END
}

void tm_stream_close(tm_stream *st) {
    if (!st) return;
    {
        std::lock_guard<std::mutex> lk(st->mu);
        st->closing = true;
    }
    st->cv_submit.notify_all();
    if (st->worker.joinable()) st->worker.join();
    for (auto *r : st->done) delete r;
    delete st;
}

}  // extern "C"
