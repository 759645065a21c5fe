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

// One submitted query (its own tag strings), queued until a batch takes it.
struct Query {
    std::vector<uint8_t> bytes;
    std::vector<uint64_t> tag_off{0};  // byte offsets of its tag strings
    uint64_t ticket = 0, submit_ns = 0;
};

// A dispatched batch in the tm_tagsets CSR form (vocabulary = the batch's tag strings).
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
    void append(const Query &q) {
        const uint64_t base = bytes.size();
        bytes.insert(bytes.end(), q.bytes.begin(), q.bytes.end());
        for (size_t i = 1; i < q.tag_off.size(); ++i) tag_off.push_back(base + q.tag_off[i]);
        set_off.push_back(tag_off.size() - 1);
        tickets.push_back(q.ticket);
        submit_ns.push_back(q.submit_ns);
    }
};

// move the first n queued queries into dst (dst cleared): O(n), the rest of the queue stays put
void take_front(std::deque<Query> &src, size_t n, Batch &dst) {
    dst.clear();
    for (size_t i = 0; i < n && !src.empty(); ++i) {
        dst.append(src.front());
        src.pop_front();
    }
}

struct Result {
    std::vector<uint64_t> tickets, submit_ns, key_off;
    std::vector<uint32_t> keys;
    uint64_t dispatch_ns = 0, done_ns = 0;
    tm_status status = TM_OK;
    std::string error;  // tm_last_error() of the failed batch (the dispatcher thread's detail)
};

}  // namespace
}  // namespace tmb

struct tm_stream {
    tm_db *db = nullptr;
    tm_stream_config cfg{};
    std::mutex mu;
    std::condition_variable cv_submit, cv_done;
    std::deque<tmb::Query> open;  // submitted, not yet dispatched
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
                const uint64_t deadline = st->open.front().submit_ns + (uint64_t)st->cfg.timeout_us * 1000ULL;
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
        if (r->status != TM_OK) r->error = tm_last_error();  // thread-local: copy it for the poller
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
    if (cfg->reserved) fail(TM_EINVAL, "reserved must be 0");
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
    tmb::Query q;  // built outside the lock, queued only once complete
    q.bytes.assign(bytes, bytes + nb);
    q.tag_off.assign(tag_off, tag_off + (n_tags ? n_tags + 1 : 1));
    bool wake = false;
    {
        std::lock_guard<std::mutex> lk(st->mu);
        if (st->closing) fail(TM_ESTATE, "stream is closing");
        q.ticket = *ticket = st->next_ticket++;
        q.submit_ns = tmb::now_ns();
        st->open.push_back(std::move(q));
        st->inflight++;
        // wake the dispatcher only when its decision can change: the queue became
        // non-empty (its timeout clock starts) or reached max_batch
        wake = st->open.size() == 1 || st->open.size() >= st->cfg.max_batch;
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
        const std::string msg = "batch failed on the GPU path: " + r->error;
        delete r;
        fail(s, msg);
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
    // the whole batch is validated before the first query is queued (offsets monotone and in
    // range, tag indices < n_vocab): a malformed batch queues nothing
    tmb::check_tagsets_host(q, "queries");
    tmb::require_strings(q, "queries");
    const uint64_t t0 = tmb::now_ns();
    for (uint64_t i = 0; i < q->n_sets; ++i) {
        tmb::Query one;
        for (uint64_t t = q->set_off[i]; t < q->set_off[i + 1]; ++t) {
            const uint64_t v = q->tag_idx ? q->tag_idx[t] : t;
            const uint64_t a = q->vocab_off[v], e = q->vocab_off[v + 1];
            one.bytes.insert(one.bytes.end(), q->vocab_bytes + a, q->vocab_bytes + e);
            one.tag_off.push_back(one.bytes.size());
        }
        const uint64_t due = t0 + arrival_ns[i];
        while (tmb::now_ns() < due) {
        }
        bool wake = false;
        {
            std::lock_guard<std::mutex> lk(st->mu);
            if (st->closing) fail(TM_ESTATE, "stream is closing");
            one.ticket = st->next_ticket++;
            one.submit_ns = tmb::now_ns();
            st->open.push_back(std::move(one));
            st->inflight++;
            wake = st->open.size() == 1 || st->open.size() >= st->cfg.max_batch;
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
