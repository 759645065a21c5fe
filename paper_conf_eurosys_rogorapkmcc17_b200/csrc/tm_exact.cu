// tm_exact.cu -- exact subset post-check ("In cases where false
// positives are absolutely unacceptable, the system or the application can
// perform an additional exact subset check"; NEXT-4 in SURVEY 8f).
//
// Build: every distinct tag string of the database gets a canonical id (the
// smallest vocabulary index with the same bytes; strings are found through
// their FNV-1a-64 hash, sorted, with byte comparison inside a hash run), and
// every set keeps its sorted canonical ids.  In exact mode the tagset table's
// rows list the *sets* of their signature instead of keys, so the scan emits
// (query, set) candidates.  Match: each query tag string is looked up in the
// sorted hash array (absent -> no id), the query's ids are sorted, every
// candidate is checked by a two-pointer merge (set ids subset of query ids), the
// survivors are compacted and expanded to (query, key) pairs.
#include <cub/cub.cuh>

#include "tm_db.h"

namespace tmb {
namespace {

constexpr uint32_t kNoId = 0xFFFFFFFFu;

inline unsigned gridx(uint64_t n, unsigned bs) { return (unsigned)std::max<uint64_t>(1, (n + bs - 1) / bs); }

__device__ __forceinline__ uint64_t fnv(const uint8_t *b, uint64_t n) {
    uint64_t h = 0xcbf29ce484222325ULL;
    for (uint64_t i = 0; i < n; ++i) {
        h ^= (uint64_t)b[i];
        h *= 0x100000001b3ULL;
    }
    return h;
}

__device__ __forceinline__ bool same_bytes(const uint8_t *a, uint64_t na, const uint8_t *b, uint64_t nb) {
    if (na != nb) return false;
    for (uint64_t i = 0; i < na; ++i)
        if (a[i] != b[i]) return false;
    return true;
}

__global__ void k_vocab_hash(const uint8_t *__restrict__ bytes, const uint64_t *__restrict__ off, uint64_t n,
                             uint64_t *__restrict__ h, uint32_t *__restrict__ pos) {
    uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v >= n) return;
    h[v] = fnv(bytes + off[v], off[v + 1] - off[v]);
    pos[v] = (uint32_t)v;
}

__device__ __forceinline__ uint64_t lower_bound_u64(const uint64_t *a, uint64_t n, uint64_t x) {
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (a[mid] < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// canonical id of the string at sorted position i: first position of its hash run with equal bytes
__global__ void k_vocab_canon(const uint8_t *__restrict__ bytes, const uint64_t *__restrict__ off,
                              const uint64_t *__restrict__ sh, const uint32_t *__restrict__ spos, uint64_t n,
                              uint32_t *__restrict__ canon) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t v = spos[i];
    const uint64_t a = off[v], la = off[v + 1] - a;
    uint64_t j = lower_bound_u64(sh, n, sh[i]);
    for (; j < i; ++j) {
        const uint32_t w = spos[j];
        if (same_bytes(bytes + a, la, bytes + off[w], off[w + 1] - off[w])) break;
    }
    canon[v] = spos[j];
}

// query vocabulary string -> canonical database id (kNoId if the database never uses it)
__global__ void k_query_canon(const uint8_t *__restrict__ qb, const uint64_t *__restrict__ qoff, uint64_t nq,
                              const uint8_t *__restrict__ dbb, const uint64_t *__restrict__ dboff,
                              const uint64_t *__restrict__ sh, const uint32_t *__restrict__ spos,
                              const uint32_t *__restrict__ canon, uint64_t n, uint32_t *__restrict__ out) {
    uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v >= nq) return;
    const uint8_t *b = qb + qoff[v];
    const uint64_t len = qoff[v + 1] - qoff[v];
    const uint64_t h = fnv(b, len);
    uint32_t id = kNoId;
    for (uint64_t j = lower_bound_u64(sh, n, h); j < n && sh[j] == h; ++j) {
        const uint32_t w = spos[j];
        if (same_bytes(b, len, dbb + dboff[w], dboff[w + 1] - dboff[w])) {
            id = canon[w];
            break;
        }
    }
    out[v] = id;
}

// ids of set i (tags [off[i], off[i+1])) <- canon of each tag, sorted ascending (insertion sort:
// sets are small; correct for any size)
__global__ void k_set_ids(const uint32_t *__restrict__ tag_idx, const uint64_t *__restrict__ off, uint64_t n,
                          const uint32_t *__restrict__ canon, uint32_t *__restrict__ ids) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t a = off[i], e = off[i + 1];
    for (uint64_t t = a; t < e; ++t) {
        const uint32_t x = canon[tag_idx ? tag_idx[t] : t];
        uint64_t k = t;
        while (k > a && ids[k - 1] > x) {
            ids[k] = ids[k - 1];
            --k;
        }
        ids[k] = x;
    }
}

// flag[i] = the set of candidate i is an exact subset of its query
__global__ void k_exact_check(const uint64_t *__restrict__ pairs, uint64_t n, const uint64_t *__restrict__ soff,
                              const uint32_t *__restrict__ sids, const uint64_t *__restrict__ qoff,
                              const uint32_t *__restrict__ qids, uint8_t *__restrict__ flag) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t q = (uint32_t)(pairs[i] >> 32), s = (uint32_t)pairs[i];
    uint64_t a = soff[s];
    const uint64_t ae = soff[s + 1];
    uint64_t b = qoff[q];
    const uint64_t be = qoff[q + 1];
    bool ok = true;
    for (; a < ae; ++a) {
        const uint32_t x = sids[a];
        while (b < be && qids[b] < x) ++b;
        if (b == be || qids[b] != x) {
            ok = false;
            break;
        }
    }
    flag[i] = ok;
}

__global__ void k_pair_key_count(const uint64_t *__restrict__ pairs, uint64_t n, const uint64_t *__restrict__ koff,
                                 unsigned long long *__restrict__ cnt) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i > n) return;
    if (i == n) {
        cnt[i] = 0;
        return;
    }
    const uint32_t s = (uint32_t)pairs[i];
    cnt[i] = koff[s + 1] - koff[s];
}

__global__ void k_pair_key_scatter(const uint64_t *__restrict__ pairs, uint64_t n,
                                   const unsigned long long *__restrict__ off, const uint64_t *__restrict__ koff,
                                   const uint32_t *__restrict__ keys, uint64_t *__restrict__ out) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t hi = pairs[i] & 0xFFFFFFFF00000000ULL;
    const uint32_t s = (uint32_t)pairs[i];
    unsigned long long o = off[i];
    for (uint64_t k = koff[s]; k < koff[s + 1]; ++k) out[o++] = hi | keys[k];
}

template <class T>
T readback(const T *d, cudaStream_t s) {
    T v;
    TMCK(cudaMemcpyAsync(&v, d, sizeof(T), cudaMemcpyDeviceToHost, s));
    TMCK(cudaStreamSynchronize(s));
    return v;
}

}  // namespace

void exact_build(tm_db *db, const uint8_t *d_bytes, uint64_t n_bytes, const uint64_t *d_voff, uint64_t V,
                 const uint32_t *d_tidx, const uint64_t *d_soff, uint64_t N, uint64_t n_tags,
                 const uint64_t *h_key_off, const uint32_t *h_keys) {
    cudaStream_t s = db->stream;
    const uint64_t K = h_key_off[N];
    db->x_nvocab = V;
    // database vocabulary (kept for byte comparisons at query time)
    db->xv_bytes.ensure(std::max<uint64_t>(n_bytes, 1));
    db->xv_off.ensure((V + 1) * 8);
    if (n_bytes) TMCK(cudaMemcpyAsync(db->xv_bytes.p, d_bytes, n_bytes, cudaMemcpyDeviceToDevice, s));
    TMCK(cudaMemcpyAsync(db->xv_off.p, d_voff, (V + 1) * 8, cudaMemcpyDeviceToDevice, s));
    // sorted hashes -> canonical ids
    DevBuf h, pos;
    db->xv_hash.ensure(std::max<uint64_t>(V, 1) * 8);
    db->xv_pos.ensure(std::max<uint64_t>(V, 1) * 4);
    db->xv_canon.ensure(std::max<uint64_t>(V, 1) * 4);
    if (V) {
        h.ensure(V * 8);
        pos.ensure(V * 4);
        k_vocab_hash<<<gridx(V, 256), 256, 0, s>>>(db->xv_bytes.as<uint8_t>(), db->xv_off.as<uint64_t>(), V,
                                                   h.as<uint64_t>(), pos.as<uint32_t>());
        TMCK(cudaGetLastError());
        size_t tb = 0;
        TMCK(cub_sort_pairs_u64_u32(h.as<uint64_t>(), db->xv_hash.as<uint64_t>(), pos.as<uint32_t>(),
                                    db->xv_pos.as<uint32_t>(), V, nullptr, &tb, s));
        TMCK(cub_sort_pairs_u64_u32(h.as<uint64_t>(), db->xv_hash.as<uint64_t>(), pos.as<uint32_t>(),
                                    db->xv_pos.as<uint32_t>(), V, cub_tmp(db, tb), &tb, s));
        k_vocab_canon<<<gridx(V, 256), 256, 0, s>>>(db->xv_bytes.as<uint8_t>(), db->xv_off.as<uint64_t>(),
                                                    db->xv_hash.as<uint64_t>(), db->xv_pos.as<uint32_t>(), V,
                                                    db->xv_canon.as<uint32_t>());
        TMCK(cudaGetLastError());
    }
    // per-set sorted canonical ids
    db->xs_off.ensure((N + 1) * 8);
    db->xs_ids.ensure(std::max<uint64_t>(n_tags, 1) * 4);
    TMCK(cudaMemcpyAsync(db->xs_off.p, d_soff, (N + 1) * 8, cudaMemcpyDeviceToDevice, s));
    if (N) {
        k_set_ids<<<gridx(N, 256), 256, 0, s>>>(d_tidx, d_soff, N, db->xv_canon.as<uint32_t>(),
                                                db->xs_ids.as<uint32_t>());
        TMCK(cudaGetLastError());
    }
    // key table of the sets (rows list sets in exact mode)
    db->xk_off.ensure((N + 1) * 8);
    db->xk_keys.ensure(std::max<uint64_t>(K, 1) * 4);
    TMCK(cudaMemcpyAsync(db->xk_off.p, h_key_off, (N + 1) * 8, cudaMemcpyHostToDevice, s));
    if (K) TMCK(cudaMemcpyAsync(db->xk_keys.p, h_keys, K * 4, cudaMemcpyHostToDevice, s));
    TMCK(cudaStreamSynchronize(s));
    h.release();
    pos.release();
}

uint64_t exact_filter(tm_db *db, const tm_tagsets *q, uint64_t n, cudaStream_t s) {
    const uint64_t Q = q->n_sets, Vq = q->n_vocab, T = q->n_tags;
    db->st.exact_checked = n;
    // query tags -> canonical ids, sorted per query
    db->xq_canon.ensure(std::max<uint64_t>(Vq, 1) * 4);
    db->xq_ids.ensure(std::max<uint64_t>(T, 1) * 4);
    if (Vq) {
        k_query_canon<<<gridx(Vq, 256), 256, 0, s>>>(q->vocab_bytes, q->vocab_off, Vq, db->xv_bytes.as<uint8_t>(),
                                                     db->xv_off.as<uint64_t>(), db->xv_hash.as<uint64_t>(),
                                                     db->xv_pos.as<uint32_t>(), db->xv_canon.as<uint32_t>(),
                                                     db->x_nvocab, db->xq_canon.as<uint32_t>());
        TMCK(cudaGetLastError());
    }
    if (Q) {
        k_set_ids<<<gridx(Q, 256), 256, 0, s>>>(q->tag_idx, q->set_off, Q, db->xq_canon.as<uint32_t>(),
                                                db->xq_ids.as<uint32_t>());
        TMCK(cudaGetLastError());
    }
    if (n == 0) {
        db->st.exact_kept = 0;
        return 0;
    }
    // check, compact into out_alt, expand sets to keys into out
    db->xflag.ensure(n);
    k_exact_check<<<gridx(n, 256), 256, 0, s>>>(db->out.as<uint64_t>(), n, db->xs_off.as<uint64_t>(),
                                                db->xs_ids.as<uint32_t>(), q->set_off, db->xq_ids.as<uint32_t>(),
                                                db->xflag.as<uint8_t>());
    TMCK(cudaGetLastError());
    db->out_alt.ensure(n * 8);
    db->xcnt.ensure(16);
    size_t tb = 0;
    TMCK(cub::DeviceSelect::Flagged(nullptr, tb, db->out.as<uint64_t>(), db->xflag.as<uint8_t>(),
                                    db->out_alt.as<uint64_t>(), db->xcnt.as<unsigned long long>(), (int64_t)n, s));
    TMCK(cub::DeviceSelect::Flagged(cub_tmp(db, tb), tb, db->out.as<uint64_t>(), db->xflag.as<uint8_t>(),
                                    db->out_alt.as<uint64_t>(), db->xcnt.as<unsigned long long>(), (int64_t)n, s));
    const uint64_t m = readback(db->xcnt.as<unsigned long long>(), s);
    db->st.exact_kept = m;
    if (m == 0) return 0;
    db->xkoff.ensure((m + 1) * 8);
    db->xkcnt.ensure((m + 1) * 8);
    k_pair_key_count<<<gridx(m + 1, 256), 256, 0, s>>>(db->out_alt.as<uint64_t>(), m, db->xk_off.as<uint64_t>(),
                                                       db->xkcnt.as<unsigned long long>());
    TMCK(cudaGetLastError());
    tb = 0;
    TMCK(cub::DeviceScan::ExclusiveSum(nullptr, tb, db->xkcnt.as<unsigned long long>(),
                                       db->xkoff.as<unsigned long long>(), (int64_t)(m + 1), s));
    TMCK(cub::DeviceScan::ExclusiveSum(cub_tmp(db, tb), tb, db->xkcnt.as<unsigned long long>(),
                                       db->xkoff.as<unsigned long long>(), (int64_t)(m + 1), s));
    const uint64_t nk = readback(db->xkoff.as<unsigned long long>() + m, s);
    if (nk > db->cap_out) {
        db->cap_out = nk + nk / 8;
        db->out.ensure(db->cap_out * 8);
    }
    k_pair_key_scatter<<<gridx(m, 256), 256, 0, s>>>(db->out_alt.as<uint64_t>(), m,
                                                     db->xkoff.as<unsigned long long>(), db->xk_off.as<uint64_t>(),
                                                     db->xk_keys.as<uint32_t>(), db->out.as<uint64_t>());
    TMCK(cudaGetLastError());
    return nk;
}

}  // namespace tmb
