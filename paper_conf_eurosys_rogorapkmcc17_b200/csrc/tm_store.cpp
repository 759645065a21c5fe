// tm_store.cpp -- add-set / remove-set / consolidate (Table 2; sec. 4.3.6):
// "The add-set and remove-set functions add and remove a set with an associated key ... These
// changes are not immediately effective and instead are staged in a temporary index and become
// effective only after a call to the consolidate function", which builds the partition and
// tagset tables (Algorithm 1).
//
// A handle made by tm_create is mutable: it keeps the database as a multiset of (tag set, key)
// entries on the host -- tag strings interned to ids, a set = its sorted distinct ids -- plus the
// staged operations in call order.  tm_consolidate applies the staged operations to the multiset
// (remove-set removes one instance of the entry if present, reading R20) and rebuilds the GPU
// tables from it with the same code as tm_build (encode, Alg. 1, layout: consolidate() on the
// GPU, tm_build.cu).  Until then matches see the last consolidated database.
#include <algorithm>
#include <cstring>
#include <map>
#include <string>
#include <unordered_map>
#include <vector>

#include "tm_db.h"

namespace tmb {

struct VecHash {
    size_t operator()(const std::vector<uint32_t> &v) const {
        uint64_t h = 0x9e3779b97f4a7c15ULL ^ v.size();
        for (uint32_t x : v) h = (h ^ x) * 0x100000001b3ULL;
        return (size_t)(h ^ (h >> 29));
    }
};

struct Store {
    std::unordered_map<std::string, uint32_t> vocab_id;  // tag string -> id
    std::vector<std::string> vocab;                       // id -> tag string
    std::unordered_map<std::vector<uint32_t>, uint32_t, VecHash> set_id;  // canonical set -> set id
    std::vector<const std::vector<uint32_t> *> sets;      // set id -> canonical set (owned by set_id)
    std::unordered_map<uint64_t, uint64_t> live;          // (set id << 32 | key) -> multiplicity
    struct Op {
        bool add;
        uint32_t set;
        uint32_t key;
    };
    std::vector<Op> staged;  // the temporary index, in call order
    tm_config cfg{};
    bool consolidated = false;

    uint32_t intern_set(const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags) {
        std::vector<uint32_t> ids;
        ids.reserve(n_tags);
        for (uint64_t t = 0; t < n_tags; ++t) {
            std::string s(reinterpret_cast<const char *>(bytes) + tag_off[t], tag_off[t + 1] - tag_off[t]);
            auto it = vocab_id.find(s);
            if (it == vocab_id.end()) {
                it = vocab_id.emplace(s, (uint32_t)vocab.size()).first;
                vocab.push_back(s);
            }
            ids.push_back(it->second);
        }
        std::sort(ids.begin(), ids.end());
        ids.erase(std::unique(ids.begin(), ids.end()), ids.end());  // a set is a set (repeats do not count)
        auto it = set_id.find(ids);
        if (it == set_id.end()) {
            it = set_id.emplace(std::move(ids), (uint32_t)sets.size()).first;
            sets.push_back(&it->first);
        }
        return it->second;
    }
};

void store_destroy(tm_db *db) {
    delete db->store;
    db->store = nullptr;
}

namespace {

void check_tags(const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags) {
    if (n_tags && !tag_off) fail(TM_EINVAL, "tag_off is NULL");
    if (n_tags && tag_off[0] != 0) fail(TM_EINVAL, "tag_off[0] != 0");
    for (uint64_t i = 0; i < n_tags; ++i)
        if (tag_off[i + 1] < tag_off[i]) fail(TM_EINVAL, "tag_off not non-decreasing");
    if (n_tags && tag_off[n_tags] && !bytes) fail(TM_EINVAL, "bytes is NULL");
}

Store &mutable_store(tm_db *db) {
    if (!db) fail(TM_EINVAL, "db is NULL");
    if (!db->store) fail(TM_ESTATE, "the handle is not mutable (made by tm_build; use tm_create for add-set / remove-set)");
    return *db->store;
}

// the live multiset as tm_build input: vocabulary = every interned string, one set per entry
// instance (a (set, key) of multiplicity m appears m times), keys one per set
void live_input(const Store &st, std::vector<uint8_t> &vb, std::vector<uint64_t> &vo, std::vector<uint32_t> &tidx,
                std::vector<uint64_t> &soff, std::vector<uint32_t> &keys) {
    vo.assign(1, 0);
    for (const std::string &s : st.vocab) {
        vb.insert(vb.end(), s.begin(), s.end());
        vo.push_back(vb.size());
    }
    soff.assign(1, 0);
    // entries in (set id, key) order: a deterministic table for a given multiset
    std::vector<std::pair<uint64_t, uint64_t>> ent(st.live.begin(), st.live.end());
    std::sort(ent.begin(), ent.end());
    for (const auto &e : ent) {
        const std::vector<uint32_t> &ids = *st.sets[e.first >> 32];
        for (uint64_t m = 0; m < e.second; ++m) {
            tidx.insert(tidx.end(), ids.begin(), ids.end());
            soff.push_back(tidx.size());
            keys.push_back((uint32_t)e.first);
        }
    }
}

}  // namespace
}  // namespace tmb

extern "C" {

tm_status tm_create(const tm_config *cfg, tm_db **out) {
    TM_API_BEGIN
    if (!out) fail(TM_EINVAL, "out is NULL");
    // an empty database (consolidated from no entries) so that matches work before the first
    // consolidate; the same config checks as tm_build
    const uint8_t none = 0;
    const uint64_t zero = 0;
    tm_tagsets empty{&none, &zero, nullptr, &zero, 0, 0, 0, 0};
    tm_db *db = nullptr;
    const tm_status s = tm_build(&empty, nullptr, nullptr, cfg, &db);
    if (s != TM_OK) return s;
    db->store = new tmb::Store();
    if (cfg) db->store->cfg = *cfg;
    db->store->cfg.device_ids = nullptr;
    db->store->cfg.plan_sample = nullptr;
    if (cfg && cfg->n_gpus > 1 && cfg->device_ids) {  // keep the device list for group rebuilds
        db->store_devices.assign(cfg->device_ids, cfg->device_ids + cfg->n_gpus);
    }
    *out = db;
    return TM_OK;
    TM_API_END
}

tm_status tm_add_set(tm_db *db, const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags, uint32_t key) {
    TM_API_BEGIN
    tmb::Store &st = tmb::mutable_store(db);
    tmb::check_tags(bytes, tag_off, n_tags);
    st.staged.push_back({true, st.intern_set(bytes, tag_off, n_tags), key});
    return TM_OK;
    TM_API_END
}

tm_status tm_remove_set(tm_db *db, const uint8_t *bytes, const uint64_t *tag_off, uint64_t n_tags, uint32_t key) {
    TM_API_BEGIN
    tmb::Store &st = tmb::mutable_store(db);
    tmb::check_tags(bytes, tag_off, n_tags);
    st.staged.push_back({false, st.intern_set(bytes, tag_off, n_tags), key});
    return TM_OK;
    TM_API_END
}

tm_status tm_add_sets(tm_db *db, const tm_tagsets *sets, const uint64_t *key_off, const uint32_t *keys) {
    TM_API_BEGIN
    tmb::Store &st = tmb::mutable_store(db);
    tmb::check_tagsets_host(sets, "sets");
    tmb::require_strings(sets, "sets");
    const uint64_t N = sets->n_sets;
    if (key_off) {
        if (key_off[0] != 0) fail(TM_EINVAL, "key_off[0] != 0");
        for (uint64_t i = 0; i < N; ++i)
            if (key_off[i + 1] < key_off[i]) fail(TM_EINVAL, "key_off not non-decreasing");
    }
    const uint64_t K = key_off ? key_off[N] : N;
    if (K && !keys) fail(TM_EINVAL, "keys is NULL");
    std::vector<uint64_t> toff;
    for (uint64_t i = 0; i < N; ++i) {
        // set i's tag strings as (bytes, offsets) relative to the vocabulary
        toff.assign(1, 0);
        std::vector<uint8_t> b;
        for (uint64_t t = sets->set_off[i]; t < sets->set_off[i + 1]; ++t) {
            const uint64_t v = sets->tag_idx ? sets->tag_idx[t] : t;
            b.insert(b.end(), sets->vocab_bytes + sets->vocab_off[v], sets->vocab_bytes + sets->vocab_off[v + 1]);
            toff.push_back(b.size());
        }
        const uint32_t sid = st.intern_set(b.data(), toff.data(), toff.size() - 1);
        const uint64_t k0 = key_off ? key_off[i] : i, k1 = key_off ? key_off[i + 1] : i + 1;
        for (uint64_t k = k0; k < k1; ++k) st.staged.push_back({true, sid, keys[k]});
    }
    return TM_OK;
    TM_API_END
}

tm_status tm_pending(const tm_db *db, uint64_t *n_staged, uint64_t *n_live) {
    TM_API_BEGIN
    if (!db || !n_staged || !n_live) fail(TM_EINVAL, "NULL argument");
    if (!db->store) fail(TM_ESTATE, "the handle is not mutable");
    *n_staged = db->store->staged.size();
    uint64_t n = 0;
    for (const auto &e : db->store->live) n += e.second;
    *n_live = n;
    return TM_OK;
    TM_API_END
}

tm_status tm_consolidate(tm_db *db) {
    TM_API_BEGIN
    tmb::Store &st = tmb::mutable_store(db);
    // apply the temporary index in call order to a copy (the handle is unchanged on failure)
    auto live = st.live;
    for (const tmb::Store::Op &op : st.staged) {
        const uint64_t k = (uint64_t)op.set << 32 | op.key;
        if (op.add) {
            ++live[k];
        } else {
            auto it = live.find(k);
            if (it != live.end() && --it->second == 0) live.erase(it);  // reading R20: one instance, if present
        }
    }
    std::swap(st.live, live);
    std::vector<uint8_t> vb;
    std::vector<uint64_t> vo, soff;
    std::vector<uint32_t> tidx, keys;
    try {
        tmb::live_input(st, vb, vo, tidx, soff, keys);
        static const uint8_t none = 0;
        static const uint32_t no_idx = 0;  // any valid pointer: n_tags may be 0 with a non-empty vocabulary
        tm_tagsets in{vb.empty() ? &none : vb.data(), vo.data(), tidx.empty() ? &no_idx : tidx.data(), soff.data(),
                      vb.size(), vo.size() - 1, tidx.size(), soff.size() - 1};
        tm_config cfg = st.cfg;
        if (cfg.n_gpus > 1 && !db->store_devices.empty()) cfg.device_ids = db->store_devices.data();
        tmb::rebuild(db, &in, keys.empty() ? nullptr : keys.data(), &cfg);
    } catch (...) {
        std::swap(st.live, live);  // restore the multiset; the staged operations stay staged
        throw;
    }
    st.staged.clear();
    st.consolidated = true;
    return TM_OK;
    TM_API_END
}

}  // extern "C"
