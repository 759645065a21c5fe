// tm_build.cu -- consolidate() on the GPU (the off-line partitioning of
// the database; NEXT-3 in SURVEY 8f): distinct signatures, Algorithm 1, the row
// order inside partitions (R18), the padded tagset table, tile masks and key CSR,
// all built in HBM.  The host only drives the level loop (one small read-back per
// level) and computes the shard plan.
//
// Algorithm 1 is processed level by level: the FIFO queue of PAPER.md:120 visits
// the nodes of each tree depth in order, children pushed as (P0, P1), so
// processing a whole depth at once accepts partitions in exactly the FIFO order
// (the tests compare it with a literal FIFO implementation).  Each node is a
// contiguous range of a permutation that is split stably, so members stay in
// lexicographic order unless the row-order refinement reorders them.
#include <cub/cub.cuh>

#include <cstring>
#include <functional>

#include "tm_db.h"

namespace tmb {
namespace {

constexpr uint32_t kChunkElems = 4096;  // elements per CTA in the level kernels
constexpr uint32_t kNone = 0xFFFFFFFFu;

inline unsigned gridn(uint64_t n, unsigned bs) { return (unsigned)std::max<uint64_t>(1, (n + bs - 1) / bs); }

__device__ __forceinline__ bool pos_bit(uint64_t w0, uint64_t w1, uint64_t w2, uint32_t p) {
    const uint64_t w = p < 64 ? w0 : (p < 128 ? w1 : w2);
    return (w >> (63 - (p & 63))) & 1ULL;
}

// ------------------------------------------------------------- unique ---
__global__ void k_uflags(const uint64_t *__restrict__ s0, const uint64_t *__restrict__ s1,
                         const uint64_t *__restrict__ s2, uint64_t n, uint32_t *__restrict__ f) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    f[i] = (i == 0 || s0[i] != s0[i - 1] || s1[i] != s1[i - 1] || s2[i] != s2[i - 1]) ? 1u : 0u;
}

// distinct signature u: planes us*, first sorted entry ustart[u]; ustart[U] = n
__global__ void k_ucompact(const uint64_t *__restrict__ s0, const uint64_t *__restrict__ s1,
                           const uint64_t *__restrict__ s2, const uint32_t *__restrict__ f,
                           const uint32_t *__restrict__ fs, uint64_t n, uint64_t *__restrict__ u0,
                           uint64_t *__restrict__ u1, uint64_t *__restrict__ u2, uint32_t *__restrict__ ustart) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    if (f[i]) {
        const uint32_t u = fs[i];
        u0[u] = s0[i];
        u1[u] = s1[i];
        u2[u] = s2[i];
        ustart[u] = (uint32_t)i;
    }
    if (i == n - 1) ustart[fs[i] + f[i]] = (uint32_t)n;
}

// keys per sorted entry (entry e is set idx[e])
__global__ void k_entry_keys(const uint32_t *__restrict__ idx, const uint64_t *__restrict__ key_off, uint64_t n,
                             uint32_t *__restrict__ kc) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t s = idx[i];
    kc[i] = (uint32_t)(key_off[s + 1] - key_off[s]);
}

// ------------------------------------------------------------- levels ---
struct Nodes {  // one tree depth
    uint32_t *lo, *hi;
    uint64_t *mask, *used;  // 3 words per node
};

// chunk count of node i (0 when the node needs no work at this level)
__global__ void k_node_need(const uint32_t *__restrict__ lo, const uint32_t *__restrict__ hi,
                            const uint64_t *__restrict__ mask, uint32_t M, int phase, uint32_t max_p, uint32_t leaf,
                            uint32_t *__restrict__ nchunk) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i > M) return;
    if (i == M) {
        nchunk[i] = 0;
        return;
    }
    const uint32_t n = hi[i] - lo[i];
    bool need;
    if (phase == 0) {  // Alg. 1: accepted nodes (|P| <= MAX_P and mask != 0) need no histogram
        const bool nonempty = (mask[3 * i] | mask[3 * i + 1] | mask[3 * i + 2]) != 0;
        need = !(n <= max_p && nonempty);
    } else {
        need = n > leaf;
    }
    nchunk[i] = need ? (n + kChunkElems - 1) / kChunkElems : 0;
}

__device__ __forceinline__ uint32_t chunk_node(const uint32_t *__restrict__ choff, uint32_t M, uint32_t b) {
    uint32_t lo = 0, hi = M;  // last node with choff[node] <= b
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (choff[mid] <= b) lo = mid; else hi = mid;
    }
    return lo;
}

// Warp argmin over the 192 positions of a node's histogram ("pivot
// <- bit not in used_bits with freq. closest to 50%"; reading R7: candidates have
// 0 < freq < |P|, ties -> lowest position).  Returns kNone if there is none.
__device__ uint32_t warp_pivot(const uint32_t *cnt, uint32_t n, const uint64_t *used, int lane) {
    unsigned long long best = ~0ULL;
    for (int p = lane; p < kBits; p += 32) {
        const uint32_t f = cnt[p];
        const bool u = used ? pos_bit(used[0], used[1], used[2], p) : false;
        if (!u && f > 0 && f < n) {
            const uint32_t d = 2 * f > n ? 2 * f - n : n - 2 * f;
            const unsigned long long key = ((unsigned long long)d << 8) | (unsigned)p;
            best = key < best ? key : best;
        }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        const unsigned long long x = __shfl_xor_sync(0xffffffffu, best, o);
        best = x < best ? x : best;
    }
    return best == ~0ULL ? kNone : (uint32_t)(best & 0xFF);
}

// Histogram of one chunk (CTA of 128 threads): ballot counting, lane l owns
// positions l, l+32, ...; CTA reduction in SMEM.  Single-chunk nodes pick their
// pivot in place; multi-chunk nodes accumulate into hist[node][192].
__global__ void __launch_bounds__(128) k_node_hist(const uint64_t *__restrict__ u0, const uint64_t *__restrict__ u1,
                                                   const uint64_t *__restrict__ u2, const uint32_t *__restrict__ perm,
                                                   Nodes nd, const uint32_t *__restrict__ choff, uint32_t M,
                                                   const uint32_t *__restrict__ mc_off, uint32_t *__restrict__ hist,
                                                   uint32_t *__restrict__ pivot, uint32_t *__restrict__ cnt1,
                                                   int phase) {
    __shared__ uint32_t sh[kBits];
    const uint32_t b = blockIdx.x;
    const uint32_t node = chunk_node(choff, M, b);
    const uint32_t c = b - choff[node];
    const uint32_t lo = nd.lo[node], hi = nd.hi[node];
    const uint32_t a = lo + c * kChunkElems, e = min(hi, a + kChunkElems);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int p = threadIdx.x; p < kBits; p += blockDim.x) sh[p] = 0;
    __syncthreads();
    uint32_t acc[6] = {0, 0, 0, 0, 0, 0};
    for (uint32_t base = a + warp * 32; base < e; base += 128) {
        const uint32_t i = base + lane;
        uint64_t w[3] = {0, 0, 0};
        if (i < e) {
            const uint32_t u = perm[i];
            w[0] = u0[u];
            w[1] = u1[u];
            w[2] = u2[u];
        }
#pragma unroll
        for (int k = 0; k < 6; ++k) {
#pragma unroll
            for (int j = 0; j < 32; ++j) {
                const int p = k * 32 + j;
                const uint32_t bb = __ballot_sync(0xffffffffu, (w[p >> 6] >> (63 - (p & 63))) & 1ULL);
                if (lane == j) acc[k] += __popc(bb);
            }
        }
    }
#pragma unroll
    for (int k = 0; k < 6; ++k)
        if (acc[k]) atomicAdd(&sh[k * 32 + lane], acc[k]);
    __syncthreads();
    const bool single = (hi - lo) <= kChunkElems;
    if (single) {
        if (warp == 0) {
            const uint32_t pv = warp_pivot(sh, hi - lo, phase == 0 ? nd.used + 3 * node : nullptr, lane);
            if (lane == 0) {
                pivot[node] = pv;
                cnt1[node] = pv == kNone ? 0 : sh[pv];
            }
        }
    } else {
        for (int p = threadIdx.x; p < kBits; p += blockDim.x)
            if (sh[p]) atomicAdd(&hist[(uint64_t)mc_off[node] * kBits + p], sh[p]);
    }
}

// multi-chunk nodes get a global histogram slot: mc_flag -> scan -> mc_off, mc_list
__global__ void k_mc_flag(const uint32_t *__restrict__ nchunk, uint32_t M, uint32_t *__restrict__ flag) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i <= M) flag[i] = (i < M && nchunk[i] > 1) ? 1u : 0u;
}

__global__ void k_mc_list(const uint32_t *__restrict__ flag, const uint32_t *__restrict__ off, uint32_t M,
                          uint32_t *__restrict__ list) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < M && flag[i]) list[off[i]] = i;
}

// pivots of multi-chunk nodes (one warp per node)
__global__ void k_node_pivot(Nodes nd, const uint32_t *__restrict__ mc_list, uint32_t nmc,
                             const uint32_t *__restrict__ hist, uint32_t *__restrict__ pivot,
                             uint32_t *__restrict__ cnt1, int phase) {
    const uint32_t m = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const int lane = threadIdx.x & 31;
    if (m >= nmc) return;
    const uint32_t node = mc_list[m];
    const uint32_t *h = hist + (uint64_t)m * kBits;
    const uint32_t pv = warp_pivot(h, nd.hi[node] - nd.lo[node], phase == 0 ? nd.used + 3 * node : nullptr, lane);
    if (lane == 0) {
        pivot[node] = pv;
        cnt1[node] = pv == kNone ? 0 : h[pv];
    }
}

// status of every node: leaf (accepted / identical), split, or done
__global__ void k_node_status(Nodes nd, const uint32_t *__restrict__ nchunk, const uint32_t *__restrict__ pivot,
                              uint32_t M, int phase, uint32_t *__restrict__ is_leaf,
                              uint32_t *__restrict__ is_split) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i > M) return;
    if (i == M) {
        is_leaf[i] = is_split[i] = 0;
        return;
    }
    const bool worked = nchunk[i] > 0;
    const bool split = worked && pivot[i] != kNone;
    is_split[i] = split;
    is_leaf[i] = (phase == 0) ? !split : 0;  // phase 0: accepted or identical-signature leaf
}

// partitions of this depth, in node order (FIFO acceptance order)
__global__ void k_emit_leaves(Nodes nd, const uint32_t *__restrict__ nchunk, const uint32_t *__restrict__ is_leaf,
                              const uint32_t *__restrict__ leaf_off, uint32_t M, const uint64_t *__restrict__ u0,
                              const uint64_t *__restrict__ u1, const uint64_t *__restrict__ u2,
                              const uint32_t *__restrict__ perm, uint32_t pbase, uint32_t *__restrict__ plo,
                              uint32_t *__restrict__ phi, uint64_t *__restrict__ pmask) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= M || !is_leaf[i]) return;
    const uint32_t o = pbase + leaf_off[i];
    plo[o] = nd.lo[i];
    phi[o] = nd.hi[i];
    if (nchunk[i] == 0) {  // accepted: |P| <= MAX_P and mask != 0
        pmask[3 * o] = nd.mask[3 * i];
        pmask[3 * o + 1] = nd.mask[3 * i + 1];
        pmask[3 * o + 2] = nd.mask[3 * i + 2];
    } else {  // reading R7: no candidate bit -> all members share sigma
        const uint32_t u = perm[nd.lo[i]];
        pmask[3 * o] = u0[u];
        pmask[3 * o + 1] = u1[u];
        pmask[3 * o + 2] = u2[u];
    }
}

__device__ __forceinline__ void set_pos(uint64_t *w, uint32_t p) { w[p >> 6] |= 1ULL << (63 - (p & 63)); }

// children of split nodes: (mask -> P0, used u {pivot}), (mask u {pivot} -> P1, used u {pivot})
__global__ void k_make_children(Nodes nd, const uint32_t *__restrict__ is_split, const uint32_t *__restrict__ split_off,
                                const uint32_t *__restrict__ pivot, const uint32_t *__restrict__ cnt1, uint32_t M,
                                Nodes out) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= M || !is_split[i]) return;
    const uint32_t j = 2 * split_off[i];
    const uint32_t lo = nd.lo[i], hi = nd.hi[i], n0 = (hi - lo) - cnt1[i];
    uint64_t m[3] = {nd.mask[3 * i], nd.mask[3 * i + 1], nd.mask[3 * i + 2]};
    uint64_t u[3] = {nd.used[3 * i], nd.used[3 * i + 1], nd.used[3 * i + 2]};
    set_pos(u, pivot[i]);
    out.lo[j] = lo;
    out.hi[j] = lo + n0;
    out.lo[j + 1] = lo + n0;
    out.hi[j + 1] = hi;
    for (int w = 0; w < 3; ++w) {
        out.mask[3 * j + w] = m[w];
        out.used[3 * j + w] = u[w];
        out.used[3 * (j + 1) + w] = u[w];
    }
    set_pos(m, pivot[i]);
    for (int w = 0; w < 3; ++w) out.mask[3 * (j + 1) + w] = m[w];
}

// flag[e] = pivot bit of element e for positions inside split nodes
__global__ void __launch_bounds__(256) k_split_flags(const uint64_t *__restrict__ u0, const uint64_t *__restrict__ u1,
                                                     const uint64_t *__restrict__ u2, const uint32_t *__restrict__ perm,
                                                     Nodes nd, const uint32_t *__restrict__ choff, uint32_t M,
                                                     const uint32_t *__restrict__ is_split,
                                                     const uint32_t *__restrict__ pivot, uint32_t *__restrict__ flag) {
    const uint32_t node = chunk_node(choff, M, blockIdx.x);
    if (!is_split[node]) return;
    const uint32_t c = blockIdx.x - choff[node];
    const uint32_t a = nd.lo[node] + c * kChunkElems, e = min(nd.hi[node], a + kChunkElems);
    const uint32_t pv = pivot[node];
    for (uint32_t i = a + threadIdx.x; i < e; i += blockDim.x) {
        const uint32_t u = perm[i];
        flag[i] = pos_bit(u0[u], u1[u], u2[u], pv) ? 1u : 0u;
    }
}

// stable partition: P0 members first, then P1, both in their current order
__global__ void __launch_bounds__(256) k_split_scatter(const uint32_t *__restrict__ perm, Nodes nd,
                                                       const uint32_t *__restrict__ choff, uint32_t M,
                                                       const uint32_t *__restrict__ is_split,
                                                       const uint32_t *__restrict__ cnt1,
                                                       const uint32_t *__restrict__ flag,
                                                       const uint32_t *__restrict__ fscan, uint32_t *__restrict__ out) {
    const uint32_t node = chunk_node(choff, M, blockIdx.x);
    if (!is_split[node]) return;
    const uint32_t c = blockIdx.x - choff[node];
    const uint32_t lo = nd.lo[node], hi = nd.hi[node];
    const uint32_t a = lo + c * kChunkElems, e = min(hi, a + kChunkElems);
    const uint32_t n0 = (hi - lo) - cnt1[node], base = fscan[lo];
    for (uint32_t i = a + threadIdx.x; i < e; i += blockDim.x) {
        const uint32_t r1 = fscan[i] - base;
        const uint32_t dst = flag[i] ? lo + n0 + r1 : lo + (i - lo) - r1;
        out[dst] = perm[i];
    }
}

// ------------------------------------------------------------- layout ---
// row r of the table: partition p (binary search on row offsets), member i
__global__ void k_layout_rows(const uint32_t *__restrict__ row_off, const uint32_t *__restrict__ kp_lo,
                              const uint32_t *__restrict__ kp_n, uint32_t P, uint64_t rows,
                              const uint32_t *__restrict__ perm, const uint64_t *__restrict__ u0,
                              const uint64_t *__restrict__ u1, const uint64_t *__restrict__ u2,
                              const uint32_t *__restrict__ ustart, const uint64_t *__restrict__ ekscan,
                              uint64_t *__restrict__ w0, uint64_t *__restrict__ w1, uint64_t *__restrict__ w2,
                              uint32_t *__restrict__ row_u, uint32_t *__restrict__ row_kc, int exact) {
    uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (r >= rows) return;
    uint32_t lo = 0, hi = P;
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (row_off[mid] <= r) lo = mid; else hi = mid;
    }
    const uint32_t p = lo, i = (uint32_t)(r - row_off[p]);
    if (i < kp_n[p]) {
        const uint32_t u = perm[kp_lo[p] + i];
        w0[r] = u0[u];
        w1[r] = u1[u];
        w2[r] = u2[u];
        row_u[r] = u;
        // keys of the row's sets, or (exact mode) the sets themselves
        row_kc[r] = exact ? ustart[u + 1] - ustart[u] : (uint32_t)(ekscan[ustart[u + 1]] - ekscan[ustart[u]]);
    } else {  // padding row: all ones, no keys
        w0[r] = w1[r] = w2[r] = ~0ULL;
        row_u[r] = kNone;
        row_kc[r] = 0;
    }
}

// keys of row r = keys of every entry with its signature, in set order (reading R10)
__global__ void k_layout_keys(const uint32_t *__restrict__ row_u, const uint32_t *__restrict__ koff_rows,
                              uint64_t rows, const uint32_t *__restrict__ ustart, const uint32_t *__restrict__ idx,
                              const uint64_t *__restrict__ key_off, const uint32_t *__restrict__ keys,
                              uint32_t *__restrict__ out, int exact) {
    uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (r >= rows) return;
    const uint32_t u = row_u[r];
    if (u == kNone) return;
    uint32_t o = koff_rows[r];
    for (uint32_t e = ustart[u]; e < ustart[u + 1]; ++e) {
        const uint32_t s = idx[e];
        if (exact) {
            out[o++] = s;
            continue;
        }
        for (uint64_t k = key_off[s]; k < key_off[s + 1]; ++k) out[o++] = keys[k];
    }
}

// AND of each tile's real rows (padding rows are all ones)
__global__ void k_tile_and(const uint64_t *__restrict__ w0, const uint64_t *__restrict__ w1,
                           const uint64_t *__restrict__ w2, uint64_t ntiles, uint64_t *__restrict__ t0,
                           uint64_t *__restrict__ t1, uint64_t *__restrict__ t2) {
    uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (t >= ntiles) return;
    uint64_t a0 = ~0ULL, a1 = ~0ULL, a2 = ~0ULL;
    for (int j = 0; j < kTile; ++j) {
        a0 &= w0[t * kTile + j];
        a1 &= w1[t * kTile + j];
        a2 &= w2[t * kTile + j];
    }
    t0[t] = a0;
    t1[t] = a1;
    t2[t] = a2;
}

struct Widen {
    __device__ unsigned long long operator()(const uint32_t &x) const { return x; }
};

template <class T>
void scan_excl(tm_db *db, const T *in, T *out, uint64_t n, cudaStream_t s) {
    size_t tb = 0;
    TMCK(cub::DeviceScan::ExclusiveSum(nullptr, tb, in, out, (int64_t)n, s));
    TMCK(cub::DeviceScan::ExclusiveSum(cub_tmp(db, tb), tb, in, out, (int64_t)n, s));
}

template <class T>
T read1(const T *d, cudaStream_t s) {
    T v;
    TMCK(cudaMemcpyAsync(&v, d, sizeof(T), cudaMemcpyDeviceToHost, s));
    TMCK(cudaStreamSynchronize(s));
    return v;
}

struct Bufs {
    std::vector<DevBuf *> v;
    ~Bufs() {
        for (auto *b : v) b->release();
    }
};

// One depth-synchronous pass over the tree.  phase 0: Algorithm 1 (leaves appended
// to the partition arrays); phase 1: row-order refinement inside partitions.
struct LevelWork {
    DevBuf lo[2], hi[2], mask[2], used[2], nchunk, choff, hist, pivot, cnt1, is_leaf, is_split, leaf_off, split_off,
        flag, fscan, perm2, mcflag, mcoff, mclist;
    Nodes nodes(int k) {
        return Nodes{lo[k].as<uint32_t>(), hi[k].as<uint32_t>(), mask[k].as<uint64_t>(), used[k].as<uint64_t>()};
    }
    void ensure_nodes(int k, uint64_t M) {
        lo[k].ensure((M + 1) * 4);
        hi[k].ensure((M + 1) * 4);
        mask[k].ensure((M + 1) * 24);
        used[k].ensure((M + 1) * 24);
    }
    void release() {
        for (DevBuf *b : {&lo[0], &lo[1], &hi[0], &hi[1], &mask[0], &mask[1], &used[0], &used[1], &nchunk, &choff,
                          &hist, &pivot, &cnt1, &is_leaf, &is_split, &leaf_off, &split_off, &flag, &fscan, &perm2,
                          &mcflag, &mcoff, &mclist})
            b->release();
    }
};

}  // namespace

// Builds db's tables from the sorted signatures (planes s0..s2, N entries, sorted
// order idx -> set index), the host key CSR and the config.  Returns nothing;
// fills db->planes/tand/key_off/keys/masks/part_row/part_n and the host copies.
void build_gpu(tm_db *db, uint64_t N, const uint64_t *s0, const uint64_t *s1, const uint64_t *s2,
               const uint32_t *idx, const uint64_t *h_key_off, const uint32_t *h_keys,
               const std::function<void(const char *)> &mark) {
    cudaStream_t s = db->stream;
    const uint64_t K = h_key_off[N];
    DevBuf f, fs, us, ustart, dkoff, dkeys, ekscan, perm, plo, phi, pmask;
    Bufs rel{{&f, &fs, &us, &ustart, &dkoff, &dkeys, &ekscan, &perm, &plo, &phi, &pmask}};
    LevelWork L;
    struct LRel {
        LevelWork &l;
        ~LRel() { l.release(); }
    } lrel{L};

    // ---- distinct signatures (reading R10)
    f.ensure(N * 4);
    fs.ensure((N + 1) * 4);
    k_uflags<<<gridn(N, 256), 256, 0, s>>>(s0, s1, s2, N, f.as<uint32_t>());
    TMCK(cudaGetLastError());
    scan_excl(db, f.as<uint32_t>(), fs.as<uint32_t>(), N, s);
    const uint32_t U = read1(fs.as<uint32_t>() + N - 1, s) + read1(f.as<uint32_t>() + N - 1, s);
    us.ensure((uint64_t)U * 24);
    ustart.ensure(((uint64_t)U + 1) * 4);
    uint64_t *u0 = us.as<uint64_t>(), *u1 = u0 + U, *u2 = u1 + U;
    k_ucompact<<<gridn(N, 256), 256, 0, s>>>(s0, s1, s2, f.as<uint32_t>(), fs.as<uint32_t>(), N, u0, u1, u2,
                                            ustart.as<uint32_t>());
    TMCK(cudaGetLastError());
    db->n_unique = U;
    // keys per entry (sorted order) and their prefix sums
    dkoff.ensure((N + 1) * 8);
    dkeys.ensure(std::max<uint64_t>(K, 1) * 4);
    TMCK(cudaMemcpyAsync(dkoff.p, h_key_off, (N + 1) * 8, cudaMemcpyHostToDevice, s));
    if (K) TMCK(cudaMemcpyAsync(dkeys.p, h_keys, K * 4, cudaMemcpyHostToDevice, s));
    ekscan.ensure((N + 1) * 8);
    {
        // f <- 32-bit key counts per sorted entry, widened to 64-bit prefix sums
        k_entry_keys<<<gridn(N, 256), 256, 0, s>>>(idx, dkoff.as<uint64_t>(), N, f.as<uint32_t>());
        TMCK(cudaGetLastError());
        cub::TransformInputIterator<unsigned long long, Widen, const uint32_t *> it(f.as<uint32_t>(), Widen{});
        size_t tb = 0;
        TMCK(cub::DeviceScan::ExclusiveSum(nullptr, tb, it, ekscan.as<unsigned long long>(), (int64_t)N, s));
        TMCK(cub::DeviceScan::ExclusiveSum(cub_tmp(db, tb), tb, it, ekscan.as<unsigned long long>(), (int64_t)N, s));
        // ekscan[N] = K
        const unsigned long long Kv = K;
        TMCK(cudaMemcpyAsync(ekscan.as<unsigned long long>() + N, &Kv, 8, cudaMemcpyHostToDevice, s));
        TMCK(cudaStreamSynchronize(s));
    }
    mark("unique (gpu)");

    // ---- Algorithm 1, depth-synchronous (phase 0), then the row order (phase 1)
    perm.ensure(std::max<uint64_t>(U, 1) * 4);
    L.perm2.ensure(std::max<uint64_t>(U, 1) * 4);
    L.flag.ensure(((uint64_t)U + 1) * 4);
    L.fscan.ensure(((uint64_t)U + 1) * 4);
    TMCK(launch_iota(perm.as<uint32_t>(), U, s));
    uint64_t pcap = 1024;
    plo.ensure(pcap * 4);
    phi.ensure(pcap * 4);
    pmask.ensure(pcap * 24);
    uint32_t P = 0;
    const uint32_t max_p = db->cfg.max_partition;
    if (U > 0 && max_p == TM_NO_PARTITIONING) {  // reading R8
        const uint32_t z0 = 0;
        const uint64_t zm[3] = {0, 0, 0};
        TMCK(cudaMemcpyAsync(plo.p, &z0, 4, cudaMemcpyHostToDevice, s));
        TMCK(cudaMemcpyAsync(phi.p, &U, 4, cudaMemcpyHostToDevice, s));
        TMCK(cudaMemcpyAsync(pmask.p, zm, 24, cudaMemcpyHostToDevice, s));
        TMCK(cudaStreamSynchronize(s));
        P = 1;
    }
    for (int phase = 0; phase < 2; ++phase) {
        uint64_t M = 0;
        int cur = 0;
        if (phase == 0) {
            if (U > 0 && max_p != TM_NO_PARTITIONING) {
                M = 1;
                L.ensure_nodes(0, 1);
                const uint32_t z0 = 0;
                TMCK(cudaMemcpyAsync(L.lo[0].p, &z0, 4, cudaMemcpyHostToDevice, s));
                TMCK(cudaMemcpyAsync(L.hi[0].p, &U, 4, cudaMemcpyHostToDevice, s));
                TMCK(cudaMemsetAsync(L.mask[0].p, 0, 24, s));
                TMCK(cudaMemsetAsync(L.used[0].p, 0, 24, s));
            }
        } else {
            if (db->cfg.row_order != 1 || P == 0) break;
            M = P;  // every partition is a root of the refinement
            L.ensure_nodes(0, M);
            TMCK(cudaMemcpyAsync(L.lo[0].p, plo.p, M * 4, cudaMemcpyDeviceToDevice, s));
            TMCK(cudaMemcpyAsync(L.hi[0].p, phi.p, M * 4, cudaMemcpyDeviceToDevice, s));
            TMCK(cudaMemsetAsync(L.mask[0].p, 0, M * 24, s));
            TMCK(cudaMemsetAsync(L.used[0].p, 0, M * 24, s));
        }
        int depth = 0;
        while (M > 0) {
            if (++depth > 4096) fail(TM_ESTATE, "partitioning did not terminate");
            Nodes nd = L.nodes(cur);
            L.nchunk.ensure((M + 1) * 4);
            L.choff.ensure((M + 1) * 4);
            L.pivot.ensure(M * 4);
            L.cnt1.ensure(M * 4);
            L.is_leaf.ensure((M + 1) * 4);
            L.is_split.ensure((M + 1) * 4);
            L.leaf_off.ensure((M + 1) * 4);
            L.split_off.ensure((M + 1) * 4);
            k_node_need<<<gridn(M + 1, 256), 256, 0, s>>>(nd.lo, nd.hi, nd.mask, (uint32_t)M, phase, max_p, 8,
                                                        L.nchunk.as<uint32_t>());
            TMCK(cudaGetLastError());
            scan_excl(db, L.nchunk.as<uint32_t>(), L.choff.as<uint32_t>(), M + 1, s);
            const uint32_t nch = read1(L.choff.as<uint32_t>() + M, s);
            // pivots (nodes that need them)
            TMCK(cudaMemsetAsync(L.pivot.p, 0xFF, M * 4, s));
            if (nch) {
                // global histograms only for multi-chunk nodes (at most U / 4096 of them)
                L.mcflag.ensure((M + 1) * 4);
                L.mcoff.ensure((M + 1) * 4);
                k_mc_flag<<<gridn(M + 1, 256), 256, 0, s>>>(L.nchunk.as<uint32_t>(), (uint32_t)M,
                                                          L.mcflag.as<uint32_t>());
                TMCK(cudaGetLastError());
                scan_excl(db, L.mcflag.as<uint32_t>(), L.mcoff.as<uint32_t>(), M + 1, s);
                const uint32_t nmc = read1(L.mcoff.as<uint32_t>() + M, s);
                if (nmc) {
                    L.mclist.ensure((uint64_t)nmc * 4);
                    L.hist.ensure((uint64_t)nmc * kBits * 4);
                    TMCK(cudaMemsetAsync(L.hist.p, 0, (uint64_t)nmc * kBits * 4, s));
                    k_mc_list<<<gridn(M, 256), 256, 0, s>>>(L.mcflag.as<uint32_t>(), L.mcoff.as<uint32_t>(),
                                                          (uint32_t)M, L.mclist.as<uint32_t>());
                    TMCK(cudaGetLastError());
                }
                k_node_hist<<<nch, 128, 0, s>>>(u0, u1, u2, perm.as<uint32_t>(), nd, L.choff.as<uint32_t>(),
                                                (uint32_t)M, L.mcoff.as<uint32_t>(), L.hist.as<uint32_t>(),
                                                L.pivot.as<uint32_t>(), L.cnt1.as<uint32_t>(), phase);
                TMCK(cudaGetLastError());
                if (nmc) {
                    k_node_pivot<<<gridn(nmc, 8), 256, 0, s>>>(nd, L.mclist.as<uint32_t>(), nmc,
                                                               L.hist.as<uint32_t>(), L.pivot.as<uint32_t>(),
                                                               L.cnt1.as<uint32_t>(), phase);
                    TMCK(cudaGetLastError());
                }
            }
            k_node_status<<<gridn(M + 1, 256), 256, 0, s>>>(nd, L.nchunk.as<uint32_t>(), L.pivot.as<uint32_t>(),
                                                          (uint32_t)M, phase, L.is_leaf.as<uint32_t>(),
                                                          L.is_split.as<uint32_t>());
            TMCK(cudaGetLastError());
            scan_excl(db, L.is_leaf.as<uint32_t>(), L.leaf_off.as<uint32_t>(), M + 1, s);
            scan_excl(db, L.is_split.as<uint32_t>(), L.split_off.as<uint32_t>(), M + 1, s);
            const uint32_t nleaf = read1(L.leaf_off.as<uint32_t>() + M, s);
            const uint32_t nsplit = read1(L.split_off.as<uint32_t>() + M, s);
            if (phase == 0 && nleaf) {
                if (P + nleaf > pcap) {  // grow the partition arrays (keep contents)
                    uint64_t ncap = std::max<uint64_t>(pcap * 2, P + nleaf);
                    DevBuf a, b, c;
                    a.ensure(ncap * 4);
                    b.ensure(ncap * 4);
                    c.ensure(ncap * 24);
                    TMCK(cudaMemcpyAsync(a.p, plo.p, P * 4, cudaMemcpyDeviceToDevice, s));
                    TMCK(cudaMemcpyAsync(b.p, phi.p, P * 4, cudaMemcpyDeviceToDevice, s));
                    TMCK(cudaMemcpyAsync(c.p, pmask.p, (uint64_t)P * 24, cudaMemcpyDeviceToDevice, s));
                    TMCK(cudaStreamSynchronize(s));
                    std::swap(plo, a);
                    std::swap(phi, b);
                    std::swap(pmask, c);
                    a.release();
                    b.release();
                    c.release();
                    pcap = ncap;
                }
                k_emit_leaves<<<gridn(M, 256), 256, 0, s>>>(nd, L.nchunk.as<uint32_t>(), L.is_leaf.as<uint32_t>(),
                                                          L.leaf_off.as<uint32_t>(), (uint32_t)M, u0, u1, u2,
                                                          perm.as<uint32_t>(), P, plo.as<uint32_t>(),
                                                          phi.as<uint32_t>(), pmask.as<uint64_t>());
                TMCK(cudaGetLastError());
                P += nleaf;
            }
            if (nsplit) {
                // stable split of every splitting node's range
                TMCK(cudaMemsetAsync(L.flag.p, 0, ((uint64_t)U + 1) * 4, s));
                k_split_flags<<<nch, 256, 0, s>>>(u0, u1, u2, perm.as<uint32_t>(), nd, L.choff.as<uint32_t>(),
                                                  (uint32_t)M, L.is_split.as<uint32_t>(), L.pivot.as<uint32_t>(),
                                                  L.flag.as<uint32_t>());
                TMCK(cudaGetLastError());
                scan_excl(db, L.flag.as<uint32_t>(), L.fscan.as<uint32_t>(), (uint64_t)U + 1, s);
                TMCK(cudaMemcpyAsync(L.perm2.p, perm.p, (uint64_t)U * 4, cudaMemcpyDeviceToDevice, s));
                k_split_scatter<<<nch, 256, 0, s>>>(perm.as<uint32_t>(), nd, L.choff.as<uint32_t>(), (uint32_t)M,
                                                    L.is_split.as<uint32_t>(), L.cnt1.as<uint32_t>(),
                                                    L.flag.as<uint32_t>(), L.fscan.as<uint32_t>(),
                                                    L.perm2.as<uint32_t>());
                TMCK(cudaGetLastError());
                std::swap(perm, L.perm2);
                // children -> next depth
                L.ensure_nodes(cur ^ 1, 2 * (uint64_t)nsplit);
                k_make_children<<<gridn(M, 256), 256, 0, s>>>(nd, L.is_split.as<uint32_t>(),
                                                            L.split_off.as<uint32_t>(), L.pivot.as<uint32_t>(),
                                                            L.cnt1.as<uint32_t>(), (uint32_t)M, L.nodes(cur ^ 1));
                TMCK(cudaGetLastError());
                cur ^= 1;
            }
            M = 2 * (uint64_t)nsplit;
        }
        mark(phase == 0 ? "alg1 (gpu)" : "row order (gpu)");
    }
    db->n_parts_total = P;

    // ---- partitions to host (small), shard plan, kept partitions
    std::vector<uint32_t> h_lo(P), h_hi(P);
    std::vector<uint64_t> h_mask(3 * (size_t)P);
    if (P) {
        TMCK(cudaMemcpyAsync(h_lo.data(), plo.p, P * 4, cudaMemcpyDeviceToHost, s));
        TMCK(cudaMemcpyAsync(h_hi.data(), phi.p, P * 4, cudaMemcpyDeviceToHost, s));
        TMCK(cudaMemcpyAsync(h_mask.data(), pmask.p, (uint64_t)P * 24, cudaMemcpyDeviceToHost, s));
        TMCK(cudaStreamSynchronize(s));
    }
    std::vector<Partition> parts(P);
    for (uint32_t i = 0; i < P; ++i) {
        for (int w = 0; w < 3; ++w) parts[i].mask.w[w] = h_mask[3 * i + w];
        parts[i].begin = h_lo[i];
        parts[i].end = h_hi[i];
    }
    const std::vector<uint32_t> owner = plan_shards(db, parts);
    std::vector<uint32_t> keep;
    for (uint32_t i = 0; i < P; ++i)
        if (owner[i] == db->cfg.shard) keep.push_back(i);
    const uint32_t KP = (uint32_t)keep.size();
    std::vector<uint32_t> kp_lo(KP), kp_n(KP), row_off(KP + 1, 0);
    db->h_masks.assign(3 * (size_t)KP, 0);
    db->h_sizes.assign(KP, 0);
    uint64_t rows64 = 0;  // padded rows summed in 64 bits: the table is addressed with u32 row ids
    for (uint32_t j = 0; j < KP; ++j) {
        const Partition &pt = parts[keep[j]];
        kp_lo[j] = (uint32_t)pt.begin;
        kp_n[j] = (uint32_t)(pt.end - pt.begin);
        rows64 += ((uint64_t)kp_n[j] + kTile - 1) / kTile * kTile;
        if (rows64 > 0xFFFFFFF0ull) fail(TM_ERANGE, "more than 2^32 rows");
        row_off[j + 1] = (uint32_t)rows64;
        for (int w = 0; w < 3; ++w) db->h_masks[3 * j + w] = pt.mask.w[w];
        db->h_sizes[j] = kp_n[j];
    }
    const uint64_t rows = row_off[KP];
    db->n_parts = KP;
    db->n_rows = rows;
    db->h_part_row = row_off;

    // ---- the tagset table in HBM
    db->planes.ensure(std::max<uint64_t>(rows, 1) * 24);
    db->key_off.ensure((rows + 1) * 4);
    db->masks.ensure(std::max<uint64_t>(KP, 1) * 24);
    db->part_row.ensure(((uint64_t)KP + 1) * 4);
    db->part_n.ensure(std::max<uint64_t>(KP, 1) * 4);
    const uint64_t ntiles = rows / kTile;
    db->tand.ensure(std::max<uint64_t>(ntiles, 1) * 24);
    if (KP) {
        TMCK(cudaMemcpyAsync(db->masks.p, db->h_masks.data(), (uint64_t)KP * 24, cudaMemcpyHostToDevice, s));
        TMCK(cudaMemcpyAsync(db->part_n.p, kp_n.data(), (uint64_t)KP * 4, cudaMemcpyHostToDevice, s));
    }
    TMCK(cudaMemcpyAsync(db->part_row.p, row_off.data(), ((uint64_t)KP + 1) * 4, cudaMemcpyHostToDevice, s));
    uint64_t nkeys = 0;
    if (rows) {
        DevBuf dlo, rowu, rowkc;
        Bufs rel2{{&dlo, &rowu, &rowkc}};
        dlo.ensure((uint64_t)KP * 4);
        rowu.ensure(rows * 4);
        rowkc.ensure((rows + 1) * 4);
        TMCK(cudaMemcpyAsync(dlo.p, kp_lo.data(), (uint64_t)KP * 4, cudaMemcpyHostToDevice, s));
        uint64_t *w0 = db->planes.as<uint64_t>(), *w1 = w0 + rows, *w2 = w1 + rows;
        k_layout_rows<<<gridn(rows, 256), 256, 0, s>>>(db->part_row.as<uint32_t>(), dlo.as<uint32_t>(),
                                                       db->part_n.as<uint32_t>(), KP, rows, perm.as<uint32_t>(), u0,
                                                       u1, u2, ustart.as<uint32_t>(), ekscan.as<uint64_t>(), w0, w1,
                                                       w2, rowu.as<uint32_t>(), rowkc.as<uint32_t>(),
                                                       (int)db->cfg.exact);
        TMCK(cudaGetLastError());
        TMCK(cudaMemsetAsync(rowkc.as<uint32_t>() + rows, 0, 4, s));
        scan_excl(db, rowkc.as<uint32_t>(), db->key_off.as<uint32_t>(), rows + 1, s);
        nkeys = read1(db->key_off.as<uint32_t>() + rows, s);
        db->keys.ensure(std::max<uint64_t>(nkeys, 1) * 4);
        k_layout_keys<<<gridn(rows, 256), 256, 0, s>>>(rowu.as<uint32_t>(), db->key_off.as<uint32_t>(), rows,
                                                       ustart.as<uint32_t>(), idx, dkoff.as<uint64_t>(),
                                                       dkeys.as<uint32_t>(), db->keys.as<uint32_t>(),
                                                       (int)db->cfg.exact);
        TMCK(cudaGetLastError());
        uint64_t *t0 = db->tand.as<uint64_t>(), *t1 = t0 + ntiles, *t2 = t1 + ntiles;
        k_tile_and<<<gridn(ntiles, 256), 256, 0, s>>>(w0, w1, w2, ntiles, t0, t1, t2);
        TMCK(cudaGetLastError());
        TMCK(cudaStreamSynchronize(s));
    } else {
        const uint32_t z = 0;
        TMCK(cudaMemcpyAsync(db->key_off.p, &z, 4, cudaMemcpyHostToDevice, s));
        db->keys.ensure(4);
        TMCK(cudaStreamSynchronize(s));
    }
    db->n_entries = nkeys;
    mark("layout (gpu)");
}

}  // namespace tmb
