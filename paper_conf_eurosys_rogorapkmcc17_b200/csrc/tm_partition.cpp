// tm_partition.cpp -- Algorithm 1 (balanced partitioning) for tm_build.
//
// Runs once per build, off the matching path ("done off-line
// within the consolidate() function").  Input: the distinct signatures in
// lexicographic order.  The work queue is processed FIFO exactly as written
// in Alg. 1; every node is a contiguous range of a permutation that is split
// stably, so the members of each accepted partition stay in lexicographic
// order (what Alg. 4 needs).  Readings R7/R8 fix
// the cases the paper leaves open.
#include <algorithm>
#include <atomic>
#include <cstring>
#include <deque>
#include <thread>

#include "tm_internal.h"

namespace tmb {

namespace {

inline bool pos_set(const Sig &s, int p) { return (s.w[p >> 6] >> (63 - (p & 63))) & 1ULL; }
inline void pos_add(Sig &s, int p) { s.w[p >> 6] |= 1ULL << (63 - (p & 63)); }

unsigned hw_threads() {
    unsigned t = std::thread::hardware_concurrency();
    return t ? std::min(t, 64u) : 1u;
}

void histogram_range(const Sig *sigs, const uint32_t *idx, uint64_t n, uint64_t *freq) {
    for (uint64_t i = 0; i < n; ++i) {
        const Sig &s = sigs[idx[i]];
        for (int w = 0; w < 3; ++w) {
            uint64_t x = s.w[w];
            while (x) {
                const int c = __builtin_clzll(x);  // bit 63-c of word w = position 64w + c
                freq[64 * w + c]++;
                x &= ~(1ULL << (63 - c));
            }
        }
    }
}

void histogram(const Sig *sigs, const uint32_t *idx, uint64_t n, uint64_t *freq) {
    std::memset(freq, 0, sizeof(uint64_t) * kBits);
    const unsigned T = hw_threads();
    if (n < (1u << 18) || T == 1) {
        histogram_range(sigs, idx, n, freq);
        return;
    }
    std::vector<uint64_t> part((size_t)T * kBits, 0);
    std::vector<std::thread> th;
    for (unsigned t = 0; t < T; ++t) {
        const uint64_t lo = n * t / T, hi = n * (t + 1) / T;
        th.emplace_back(histogram_range, sigs, idx + lo, hi - lo, part.data() + (size_t)t * kBits);
    }
    for (auto &x : th) x.join();
    for (unsigned t = 0; t < T; ++t)
        for (int p = 0; p < kBits; ++p) freq[p] += part[(size_t)t * kBits + p];
}

// stable split of idx[0..n) by position `pivot`: zeros first; returns #zeros
uint64_t stable_split(const Sig *sigs, uint32_t *idx, uint64_t n, int pivot, uint32_t *scratch) {
    const unsigned T = (n < (1u << 18)) ? 1 : hw_threads();
    std::vector<uint64_t> zeros(T + 1, 0), ones(T + 1, 0);
    auto count = [&](unsigned t) {
        const uint64_t lo = n * t / T, hi = n * (t + 1) / T;
        uint64_t z = 0;
        for (uint64_t i = lo; i < hi; ++i) z += !pos_set(sigs[idx[i]], pivot);
        zeros[t + 1] = z;
        ones[t + 1] = (hi - lo) - z;
    };
    auto place = [&](unsigned t, uint64_t zbase, uint64_t obase) {
        const uint64_t lo = n * t / T, hi = n * (t + 1) / T;
        for (uint64_t i = lo; i < hi; ++i) {
            if (pos_set(sigs[idx[i]], pivot)) scratch[obase++] = idx[i];
            else scratch[zbase++] = idx[i];
        }
    };
    if (T == 1) {
        count(0);
        place(0, 0, zeros[1]);
    } else {
        std::vector<std::thread> th;
        for (unsigned t = 0; t < T; ++t) th.emplace_back(count, t);
        for (auto &x : th) x.join();
        th.clear();
        for (unsigned t = 0; t < T; ++t) {
            zeros[t + 1] += zeros[t];
            ones[t + 1] += ones[t];
        }
        const uint64_t nz = zeros[T];
        for (unsigned t = 0; t < T; ++t) th.emplace_back(place, t, zeros[t], nz + ones[t]);
        for (auto &x : th) x.join();
    }
    std::memcpy(idx, scratch, n * sizeof(uint32_t));
    return zeros[T];
}

struct Node {
    uint64_t lo, hi;
    Sig mask, used;
};

}  // namespace

void alg1_partition(const Sig *sigs, uint64_t n, uint32_t max_p, std::vector<uint32_t> &order,
                    std::vector<Partition> &parts) {
    order.resize(n);
    for (uint64_t i = 0; i < n; ++i) order[i] = (uint32_t)i;
    parts.clear();
    if (n == 0) return;
    const Sig zero{{0, 0, 0}};
    if (max_p == TM_NO_PARTITIONING) {  // reading R8: one partition, empty mask
        parts.push_back({zero, 0, n});
        return;
    }
    std::vector<uint32_t> scratch(n);
    std::deque<Node> Q;  // the work queue of Alg. 1, FIFO
    Q.push_back({0, n, zero, zero});
    uint64_t freq[kBits];
    while (!Q.empty()) {
        Node nd = Q.front();
        Q.pop_front();
        const uint64_t cnt = nd.hi - nd.lo;
        if (cnt == 0) continue;  // reading R7: empty P dropped
        const bool mask_nonempty = (nd.mask.w[0] | nd.mask.w[1] | nd.mask.w[2]) != 0;
        if (cnt <= max_p && mask_nonempty) {  // |P| <= MAX_P and mask != 0: accept
            parts.push_back({nd.mask, nd.lo, nd.hi});
            continue;
        }
        histogram(sigs, order.data() + nd.lo, cnt, freq);
        int pivot = -1;
        uint64_t best = 0;
        for (int p = 0; p < kBits; ++p) {
            if (pos_set(nd.used, p) || freq[p] == 0 || freq[p] == cnt) continue;
            const uint64_t d = 2 * freq[p] > cnt ? 2 * freq[p] - cnt : cnt - 2 * freq[p];
            if (pivot < 0 || d < best) {  // closest to 50%, ties -> lowest position
                pivot = p;
                best = d;
            }
        }
        if (pivot < 0) {  // reading R7: all members share one signature sigma
            parts.push_back({sigs[order[nd.lo]], nd.lo, nd.hi});
            continue;
        }
        const uint64_t n0 = stable_split(sigs, order.data() + nd.lo, cnt, pivot, scratch.data());
        Node a = nd, b = nd;
        pos_add(a.used, pivot);
        pos_add(b.used, pivot);
        pos_add(b.mask, pivot);
        a.hi = nd.lo + n0;
        b.lo = nd.lo + n0;
        Q.push_back(a);  // (mask -> P0, used_bits)
        Q.push_back(b);  // (mask u {pivot} -> P1, used_bits)
    }
}

namespace {

// DFS refinement of one partition's range [lo, hi) of `order` (single thread).
void refine_range(const Sig *sigs, uint32_t *idx, uint64_t n, uint32_t leaf, uint32_t *scratch) {
    struct R {
        uint64_t lo, hi;
    };
    std::vector<R> st;
    st.push_back({0, n});
    uint64_t freq[kBits];
    while (!st.empty()) {
        const R r = st.back();
        st.pop_back();
        const uint64_t cnt = r.hi - r.lo;
        if (cnt <= leaf) continue;
        std::memset(freq, 0, sizeof freq);
        histogram_range(sigs, idx + r.lo, cnt, freq);
        int pivot = -1;
        uint64_t best = 0;
        for (int p = 0; p < kBits; ++p) {
            if (freq[p] == 0 || freq[p] == cnt) continue;
            const uint64_t d = 2 * freq[p] > cnt ? 2 * freq[p] - cnt : cnt - 2 * freq[p];
            if (pivot < 0 || d < best) {
                pivot = p;
                best = d;
            }
        }
        if (pivot < 0) continue;  // identical signatures
        uint64_t n0 = 0;
        for (uint64_t i = r.lo; i < r.hi; ++i)
            if (!pos_set(sigs[idx[i]], pivot)) scratch[n0++] = idx[i];
        uint64_t k = n0;
        for (uint64_t i = r.lo; i < r.hi; ++i)
            if (pos_set(sigs[idx[i]], pivot)) scratch[k++] = idx[i];
        std::memcpy(idx + r.lo, scratch, cnt * sizeof(uint32_t));
        st.push_back({r.lo + n0, r.hi});  // P1 after P0 (stack: push P1 first)
        st.push_back({r.lo, r.lo + n0});
    }
}

}  // namespace

void refine_order(const Sig *sigs, std::vector<uint32_t> &order, const std::vector<Partition> &parts,
                  uint32_t leaf) {
    const unsigned T = hw_threads();
    std::atomic<size_t> next{0};
    auto work = [&]() {
        std::vector<uint32_t> scratch;
        for (;;) {
            const size_t i = next.fetch_add(1);
            if (i >= parts.size()) break;
            const uint64_t n = parts[i].end - parts[i].begin;
            if (scratch.size() < n) scratch.resize(n);
            refine_range(sigs, order.data() + parts[i].begin, n, leaf, scratch.data());
        }
    };
    std::vector<std::thread> th;
    for (unsigned t = 0; t < T; ++t) th.emplace_back(work);
    for (auto &x : th) x.join();
}

}  // namespace tmb
