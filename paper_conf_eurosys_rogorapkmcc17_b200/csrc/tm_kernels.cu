// tm_kernels.cu -- sm_100a kernels of the TagMatch hot path.
//
// Stage map (sec. 3):
//   k_hash_vocab     S1  tag string -> 7 Bloom positions (reading R1)
//   k_encode_sets    S1  OR of a set's tag signatures
//   k_route_bitmap   S2  mask_p subset-of q for every (q, p) (Alg. 2)
//   k_route_scatter  S2  per-partition query lists (partition-major CSR)
//   k_items          S3  per-partition batches cut into work items
//   k_scan           S4-S7 persistent subset-scan: tile pre-filter (Alg. 4,
//                        PAPER.md:164-198), subset check (Alg. 3),
//                        warp-aggregated compaction fused with the
//                        set-id -> key lookup
//   k_split          S8  sorted (q<<32|key) -> query[], key[]
// plus CUB scans / radix sorts / unique (S2, S8) and small gather kernels used
// by tm_build.
#include <cub/cub.cuh>
#include <type_traits>

#include "tm_internal.h"

namespace tmb {

namespace {

constexpr uint64_t kFnvOffset = 0xcbf29ce484222325ULL;
constexpr uint64_t kFnvPrime = 0x100000001b3ULL;
constexpr uint64_t kGolden = 0x9e3779b97f4a7c15ULL;

__device__ __forceinline__ uint64_t splitmix_out(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

inline unsigned grid_for(uint64_t n, unsigned bs) {
    uint64_t g = (n + bs - 1) / bs;
    return (unsigned)(g ? g : 1);
}

// ------------------------------------------------------------------ S1 ---
// One thread per vocabulary string: FNV-1a-64 of the bytes, then positions
// floor(z*192/2^64) of the first 7 SplitMix64 outputs seeded with it.
// The CSR is validated on the device (non-decreasing offsets inside [0, n_bytes], end points):
// a malformed string sets *err and is hashed as empty, so nothing is read out of bounds.
// hashes != NULL: the vocabulary is given pre-hashed (tm_tagsets.vocab_hash): h = hashes[v].
__global__ void k_hash_vocab(const uint8_t *__restrict__ bytes, const uint64_t *__restrict__ off,
                             const uint64_t *__restrict__ hashes, uint64_t n, uint64_t n_bytes,
                             uint64_t *__restrict__ vsig, unsigned int *err) {
    uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v >= n) return;
    uint64_t h = kFnvOffset;
    if (hashes) {
        h = __ldg(hashes + v);
    } else {
        uint64_t b = off[v], e = off[v + 1];
        if (e < b || e > n_bytes || (v == 0 && b != 0) || (v == n - 1 && e != n_bytes)) {
            if (err) atomicOr(err, 1u);
            e = b = 0;
        }
        for (uint64_t i = b; i < e; ++i) {
            h ^= (uint64_t)__ldg(bytes + i);
            h *= kFnvPrime;
        }
    }
    uint64_t s[3] = {0, 0, 0};
    uint64_t state = h;
#pragma unroll
    for (int r = 0; r < kHashes; ++r) {
        state += kGolden;
        const uint64_t z = splitmix_out(state);
        const uint32_t p = (uint32_t)__umul64hi(z, (uint64_t)kBits);
        const uint64_t bit = 1ULL << (63 - (p & 63));
        s[0] |= (p < 64) ? bit : 0ULL;
        s[1] |= (p >= 64 && p < 128) ? bit : 0ULL;
        s[2] |= (p >= 128) ? bit : 0ULL;
    }
    vsig[3 * v + 0] = s[0];
    vsig[3 * v + 1] = s[1];
    vsig[3 * v + 2] = s[2];
}

// One thread per set; writes the three signature planes.
// Validated like k_hash_vocab: offsets non-decreasing inside [0, n_tags] with set_off[0] = 0 and
// set_off[n] = n_tags, tag indices < n_vocab; violations set *err and are skipped.
__global__ void k_encode_sets(const uint64_t *__restrict__ vsig, const uint32_t *__restrict__ tag_idx,
                              const uint64_t *__restrict__ set_off, uint64_t n, uint64_t n_tags, uint64_t n_vocab,
                              uint64_t *__restrict__ w0, uint64_t *__restrict__ w1, uint64_t *__restrict__ w2,
                              unsigned int *err) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    uint64_t b = set_off[i], e = set_off[i + 1];
    if (e < b || e > n_tags || (i == 0 && b != 0) || (i == n - 1 && e != n_tags)) {
        if (err) atomicOr(err, 2u);
        e = b = 0;
    }
    uint64_t a0 = 0, a1 = 0, a2 = 0;
    for (uint64_t t = b; t < e; ++t) {
        const uint64_t v = tag_idx ? (uint64_t)__ldg(tag_idx + t) : t;
        if (v >= n_vocab) {
            if (err) atomicOr(err, 4u);
            continue;
        }
        a0 |= __ldg(vsig + 3 * v + 0);
        a1 |= __ldg(vsig + 3 * v + 1);
        a2 |= __ldg(vsig + 3 * v + 2);
    }
    w0[i] = a0;
    w1[i] = a1;
    w2[i] = a2;
}

// ------------------------------------------------------------------ S2 ---
// Alg. 2 bit-sliced: partition p is routed to query q iff mask_p is a subset
// of sig(q), i.e. iff no one-bit of mask_p is a zero-bit of q.  A warp owns a route block of
// kRouteWB query words (32 queries each) and first transposes them into
//   Z[pos][i] = ballot over the 32 queries of word i of "bit pos of q is 0"   (pos = 64 w + j)
// in shared memory; then lane l takes partition p = g + l and ORs Z[pos] over the one-bits pos
// of its mask (a mask has ~2-5 bits): ~Z-OR is the 32-query routing word of (p, word i), for
// all kRouteWB words at once (three LDS.128 per mask bit).  Per (partition, 32 queries) that is
// a few instructions per LANE instead of a 6-op test per (partition, query): routing cost stays
// small when MAX_P is small and partitions are many.
// Two passes over the same function: count (per (partition, route block) counts, scanned into
// the partition-major CSR offsets) and scatter (ascending query ids per partition).  Scratch:
// 12 B per (partition, 384 queries) instead of a dense P x Q bitmap.
// Bank conflicts: lane l reads the Z row of its own mask bit, so the 8 lanes of an LDS.128 phase
// hit data-dependent rows.  With 16-word rows (64 B) every row started on one of two bank quads
// of a 128-B window (8 lanes on 2 quads: ~5-way conflicts, the router was LSU-bound: 10 ms at
// 40K partitions); 12-word rows (48 B) put consecutive rows on different quads (pos x 3 mod 8),
// so random rows spread over all 8.
constexpr int kRouteWB = 12;                 // query words per route block (one warp)
constexpr int kRouteBlockQ = 32 * kRouteWB;  // 384 queries
constexpr int kRouteWarps = 4;               // warps per CTA (36 KB of Z)

__device__ __forceinline__ void route_build_z(uint32_t *__restrict__ z, const uint64_t *__restrict__ q0,
                                              const uint64_t *__restrict__ q1, const uint64_t *__restrict__ q2,
                                              uint64_t qb, uint64_t n_q, int lane) {
    for (int i = 0; i < kRouteWB; ++i) {
        const uint64_t q = qb + (uint64_t)i * 32 + lane;
        uint64_t a[3] = {~0ULL, ~0ULL, ~0ULL};  // past the batch: all ones (no zero bits); masked by `valid`
        if (q < n_q) {
            a[0] = __ldg(q0 + q);
            a[1] = __ldg(q1 + q);
            a[2] = __ldg(q2 + q);
        }
#pragma unroll
        for (int w = 0; w < 3; ++w) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const uint32_t x = (uint32_t)(a[w] >> (32 * h));
                uint32_t mine = 0;
#pragma unroll
                for (int t = 0; t < 32; ++t) {
                    const uint32_t b = __ballot_sync(0xffffffffu, ((x >> t) & 1u) == 0u);
                    if (lane == t) mine = b;
                }
                z[(64 * w + 32 * h + lane) * kRouteWB + i] = mine;
            }
        }
    }
}

// PASS 0: counts[p * NB + blk] = routed queries of partition p in route block blk.
// PASS 1: scatter the routed query ids of (p, blk) at off[p * NB + blk] (ascending query order).
template <int PASS>
__global__ void __launch_bounds__(kRouteWarps * 32, 6) k_route(const uint64_t *__restrict__ masks, uint32_t n_parts,
                                                            const uint64_t *__restrict__ q0,
                                                            const uint64_t *__restrict__ q1,
                                                            const uint64_t *__restrict__ q2, uint64_t n_q,
                                                            uint64_t n_blocks, uint32_t *__restrict__ counts,
                                                            const unsigned long long *__restrict__ off,
                                                            uint32_t *__restrict__ qidx, unsigned long long cap,
                                                            uint32_t qbase, uint32_t n_slices) {
    extern __shared__ __align__(16) uint32_t zsm[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // warp -> (route block, partition slice): a small batch (few route blocks) has its partitions
    // cut into n_slices ranges of whole 32-partition groups, so the grid still fills the GPU
    const uint64_t li = (uint64_t)blockIdx.x * kRouteWarps + warp;
    if (li >= n_blocks * n_slices) return;  // warp-uniform; no CTA barrier below
    const uint64_t blk = li % n_blocks;
    const uint32_t slice = (uint32_t)(li / n_blocks);
    const uint32_t ngroups = (n_parts + 31) / 32;
    const uint32_t gps = (ngroups + n_slices - 1) / n_slices;
    const uint32_t g_lo = slice * gps * 32, g_hi = min(n_parts, (slice + 1) * gps * 32);
    uint32_t *z = zsm + warp * (192 * kRouteWB);
    const uint64_t qb = blk * kRouteBlockQ;
    route_build_z(z, q0, q1, q2, qb, n_q, lane);
    __syncwarp();
    // valid-query mask of each word of the block (warp-uniform)
    const uint64_t nvq = n_q - qb;  // > 0
    for (uint32_t g = g_lo; g < g_hi; g += 32) {
        const uint32_t p = g + lane;
        uint64_t m[3] = {0, 0, 0};
        if (p < n_parts) {
            m[0] = __ldg(masks + 3 * (uint64_t)p);
            m[1] = __ldg(masks + 3 * (uint64_t)p + 1);
            m[2] = __ldg(masks + 3 * (uint64_t)p + 2);
        }
        uint32_t acc[kRouteWB];
#pragma unroll
        for (int i = 0; i < kRouteWB; ++i) acc[i] = 0;
#pragma unroll
        for (int w = 0; w < 3; ++w) {
            uint64_t mw = m[w];
            while (mw) {
                const int j = __ffsll((long long)mw) - 1;
                mw &= mw - 1;
                const uint4 *zz = reinterpret_cast<const uint4 *>(z + (64 * w + j) * kRouteWB);
#pragma unroll
                for (int v = 0; v < kRouteWB / 4; ++v) {
                    const uint4 x = zz[v];
                    acc[4 * v + 0] |= x.x;
                    acc[4 * v + 1] |= x.y;
                    acc[4 * v + 2] |= x.z;
                    acc[4 * v + 3] |= x.w;
                }
            }
        }
        if (p >= n_parts) continue;
        if constexpr (PASS == 0) {
            uint32_t c = 0;
#pragma unroll
            for (int i = 0; i < kRouteWB; ++i) {
                const uint64_t lo = 32ULL * i;
                const uint32_t vm = nvq > lo ? (nvq - lo >= 32 ? ~0u : ((1u << (nvq - lo)) - 1u)) : 0u;
                c += __popc(~acc[i] & vm);
            }
            counts[(uint64_t)p * n_blocks + blk] = c;
        } else {
            unsigned long long o = off[(uint64_t)p * n_blocks + blk];
#pragma unroll
            for (int i = 0; i < kRouteWB; ++i) {
                const uint64_t lo = 32ULL * i;
                const uint32_t vm = nvq > lo ? (nvq - lo >= 32 ? ~0u : ((1u << (nvq - lo)) - 1u)) : 0u;
                uint32_t r = ~acc[i] & vm;
                while (r) {
                    const int t = __ffs(r) - 1;
                    r &= r - 1;
                    if (o < cap) qidx[o] = qbase + (uint32_t)(qb + lo + (uint32_t)t);
                    ++o;
                }
            }
        }
    }
}

// ------------------------------------------------------------------ S3 ---
constexpr uint32_t kSmallRange = 4096;  // rows per work item of a partition routed to <= kSmallBatch queries

// Rows per work item of a partition with nq routed queries: a streaming (HBM-bound) partition is
// cut into short ranges, and a partition of at most three query chunks into quarter ranges, so that
// a large partition that few queries reach still yields many items and the persistent grid's last
// wave stays a small fraction of the scan (the item's query staging is cheap for few queries).
__device__ __forceinline__ uint32_t part_range_rows(unsigned long long nq, uint32_t range_rows) {
    if (nq <= (unsigned long long)kSmallBatch) return min(range_rows, kSmallRange);
    if (nq <= 3ULL * kChunk) return max((range_rows / 4) & ~255u, 256u);
    return range_rows;
}

// Per partition: routed query count -> (chunks of kChunk queries) x (ranges of
// range_rows rows) work items.
__global__ void k_items(const unsigned long long *__restrict__ word_off, uint64_t qw_total,
                        const uint32_t *__restrict__ part_row, const uint32_t *__restrict__ part_n, uint32_t n_parts,
                        unsigned long long *__restrict__ qoff, unsigned long long *__restrict__ item_cnt,
                        DevCounters *ctr, uint32_t range_rows) {
    uint32_t p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p > n_parts) return;
    const unsigned long long o = word_off[(uint64_t)p * qw_total];
    qoff[p] = o;
    if (p == n_parts) {
        item_cnt[p] = 0;
        ctr->routed = o;
        return;
    }
    const unsigned long long nq = word_off[(uint64_t)(p + 1) * qw_total] - o;
    const uint32_t rows = part_row[p + 1] - part_row[p];
    const unsigned long long nchunk = (nq + kChunk - 1) / kChunk;
    const uint32_t rr = part_range_rows(nq, range_rows);
    const unsigned long long nrange = (rows + rr - 1) / rr;
    item_cnt[p] = nchunk * nrange;
    if (nq) atomicAdd(&ctr->candidates, nq * (unsigned long long)part_n[p]);
}

// ------------------------------------------------------------- S4..S7 ---
// Two-level pre-filter (Alg. 4 generalised): level A tests the batch against
// the common mask of a 256-row block (8 tiles), level B tests the level-A
// survivors against the mask of each 32-row tile; only level-B survivors are
// checked against the tile's 32 sets (Alg. 3).
#ifndef TM_BLOCK_TILES
#define TM_BLOCK_TILES 8
#endif
constexpr int kBlockTiles = TM_BLOCK_TILES;  // tiles per level-A block (8: 256 rows)
constexpr int kSubB = 128;       // level-B survivors buffered per pass
constexpr int kQSub = 128;       // queries per unit

// Matches are staged per warp (kPend entries in shared memory) and emitted in batches: one
// global atomic per batch instead of one per matching warp step (the output counter is a single
// address every SM hits).
constexpr uint32_t kPend = 8;

// WORD1 survivor planes: word w (= 32-bit half w & 1 of block w >> 1) of level-B
// survivor k at sw[warp][w][k]; the plane stride (kSubW + 4 words = 400 B, 16 B mod 128)
// puts the six planes on disjoint bank quads, so the per-lane-plane LDS.128 of the
// pre-check is conflict-free.
#ifndef TM_SUBW
#define TM_SUBW 96
#endif
constexpr int kSubW = TM_SUBW;                         // level-B survivors per pass (WORD1)
constexpr int kSubWStride = kSubW + 4;

struct ScanSmem {
    uint64_t q0[kChunk], q1[kChunk], q2[kChunk];  // the item's query batch (SoA)
    uint16_t sa[kScanWarps][kChunk];               // per-warp level-A survivors (slots)
    union {
        uint4 sbuf[kScanWarps][kSubB];             // per-warp level-B survivors (see SurvivorLayout)
        uint32_t sw[kScanWarps][6][kSubWStride];   // WORD1: per-warp level-B survivors, word planes
    };
    uint16_t sbi[kScanWarps][kSubB];               // per-warp level-B survivors: slots
    uint64_t tmask[kScanWarps][3][kBlockTiles];    // per-warp: AND masks of the unit's tiles
    const uint32_t *qid;                           // batch slot -> query index in the call (global)
    unsigned long long item;
    unsigned int unit_ctr;
    unsigned long long cnt[3];                     // CTA totals: tile tests, pair checks, matched sets
    uint2 pend[kScanWarps][kPend];                 // per-warp matches (row, query) awaiting emission
};

// Shared memory of the streaming-only kernels (calls of <= kSmallBatch queries: every partition batch
// is small): the same members as ScanSmem, sized for the streaming path, so that residency is
// bounded by registers (8 CTAs/SM) instead of ScanSmem's 32 KB (7 CTAs/SM).
struct StreamSmem {
    uint64_t q0[kSmallBatch], q1[kSmallBatch], q2[kSmallBatch];
    uint16_t sa[kScanWarps][1];
    union {
        uint4 sbuf[kScanWarps][1];
        uint32_t sw[1][6][kSubWStride];   // warp 0's planes hold the batch (pre-check)
    };
    uint16_t sbi[kScanWarps][1];
    const uint32_t *qid;
    unsigned long long item;
    unsigned int unit_ctr;
    unsigned long long cnt[3];
    uint2 pend[kScanWarps][kPend];
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint4 lds128(uint32_t addr) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
    return v;
}

// acc |= B << j for each j in 0..3 with (a & ~v_j) == 0: one LOP3 with a predicate result and
// one predicated OR per survivor (no SEL / add chain)
// Two-word form: survivor j passes when (a & ~v_j) | (b & ~u_j) == 0.
__device__ __forceinline__ uint32_t pick_word(uint64_t s0, uint64_t s1, uint64_t s2, uint32_t w, bool valid) {
    const uint64_t lo = (w & 2u) ? s1 : s0;
    const uint64_t b = (w & 4u) ? s2 : lo;
    const uint32_t x = (w & 1u) ? (uint32_t)(b >> 32) : (uint32_t)b;
    return valid ? x : ~0u;
}

// WORD1: survivor k's six words into the per-warp word planes (stride kSubWStride), slot i
__device__ __forceinline__ void store_survivor(uint32_t *sw, uint16_t *sbi, uint32_t k, uint64_t a0, uint64_t a1,
                                               uint64_t a2, uint32_t i) {
    uint32_t *c = sw + k;
    c[0] = (uint32_t)a0;
    c[kSubWStride] = (uint32_t)(a0 >> 32);
    c[2 * kSubWStride] = (uint32_t)a1;
    c[3 * kSubWStride] = (uint32_t)(a1 >> 32);
    c[4 * kSubWStride] = (uint32_t)a2;
    c[5 * kSubWStride] = (uint32_t)(a2 >> 32);
    sbi[k] = (uint16_t)i;
}

// Four independent accumulators (one per survivor lane of the uint4) keep the predicated ORs
// off a single serial dependency chain; the caller ORs them together.
// IMAD = true: the predicated accumulate is an integer multiply-add (acc += one * bit; the bits of an
// accumulator are disjoint, so + is |), which runs on the FMA pipe instead of the ALU pipe: the
// pre-check then puts 2 of its 3 ops per pair on the ALU pipe (scripts/int_peak.cu measures both).
template <int B, bool IMAD = false>
__device__ __forceinline__ void precheck4x2(uint32_t &c0, uint32_t &c1, uint32_t &c2, uint32_t &c3, uint32_t a,
                                            uint4 v, uint32_t b, uint4 u, uint32_t one = 1u) {
    if constexpr (IMAD) {
        asm("{\n\t.reg .pred p0, p1, p2, p3;\n\t.reg .b32 t0, t1, t2, t3, s0, s1, s2, s3;\n\t"
            "not.b32 t0, %5;\n\tnot.b32 t1, %6;\n\tnot.b32 t2, %7;\n\tnot.b32 t3, %8;\n\t"
            "and.b32 t0, t0, %4;\n\tand.b32 t1, t1, %4;\n\tand.b32 t2, t2, %4;\n\tand.b32 t3, t3, %4;\n\t"
            "not.b32 s0, %10;\n\tnot.b32 s1, %11;\n\tnot.b32 s2, %12;\n\tnot.b32 s3, %13;\n\t"
            "and.b32 s0, s0, %9;\n\tand.b32 s1, s1, %9;\n\tand.b32 s2, s2, %9;\n\tand.b32 s3, s3, %9;\n\t"
            "or.b32 t0, t0, s0;\n\tor.b32 t1, t1, s1;\n\tor.b32 t2, t2, s2;\n\tor.b32 t3, t3, s3;\n\t"
            "setp.eq.u32 p0, t0, 0;\n\tsetp.eq.u32 p1, t1, 0;\n\tsetp.eq.u32 p2, t2, 0;\n\tsetp.eq.u32 p3, t3, 0;\n\t"
            "@p0 mad.lo.u32 %0, %18, %14, %0;\n\t@p1 mad.lo.u32 %1, %18, %15, %1;\n\t"
            "@p2 mad.lo.u32 %2, %18, %16, %2;\n\t@p3 mad.lo.u32 %3, %18, %17, %3;\n\t}"
            : "+r"(c0), "+r"(c1), "+r"(c2), "+r"(c3)
            : "r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"(b), "r"(u.x), "r"(u.y), "r"(u.z), "r"(u.w), "n"(B),
              "n"(B << 1), "n"(B << 2), "n"(B << 3), "r"(one));
        return;
    }
    asm("{\n\t.reg .pred p0, p1, p2, p3;\n\t.reg .b32 t0, t1, t2, t3, s0, s1, s2, s3;\n\t"
        "not.b32 t0, %5;\n\tnot.b32 t1, %6;\n\tnot.b32 t2, %7;\n\tnot.b32 t3, %8;\n\t"
        "and.b32 t0, t0, %4;\n\tand.b32 t1, t1, %4;\n\tand.b32 t2, t2, %4;\n\tand.b32 t3, t3, %4;\n\t"
        "not.b32 s0, %10;\n\tnot.b32 s1, %11;\n\tnot.b32 s2, %12;\n\tnot.b32 s3, %13;\n\t"
        "and.b32 s0, s0, %9;\n\tand.b32 s1, s1, %9;\n\tand.b32 s2, s2, %9;\n\tand.b32 s3, s3, %9;\n\t"
        "or.b32 t0, t0, s0;\n\tor.b32 t1, t1, s1;\n\tor.b32 t2, t2, s2;\n\tor.b32 t3, t3, s3;\n\t"
        "setp.eq.u32 p0, t0, 0;\n\tsetp.eq.u32 p1, t1, 0;\n\tsetp.eq.u32 p2, t2, 0;\n\tsetp.eq.u32 p3, t3, 0;\n\t"
        "@p0 or.b32 %0, %0, %14;\n\t@p1 or.b32 %1, %1, %15;\n\t@p2 or.b32 %2, %2, %16;\n\t@p3 or.b32 %3, %3, %17;\n\t}"
        : "+r"(c0), "+r"(c1), "+r"(c2), "+r"(c3)
        : "r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"(b), "r"(u.x), "r"(u.y), "r"(u.z), "r"(u.w), "n"(B),
          "n"(B << 1), "n"(B << 2), "n"(B << 3));
}

// 16-B streaming load of two consecutive rows of a plane (read-only path, no L1 allocation)
__device__ __forceinline__ ulonglong2 ldg_stream2(const uint64_t *ptr) {
    ulonglong2 v;
    asm volatile("ld.global.nc.L1::no_allocate.v2.u64 {%0, %1}, [%2];" : "=l"(v.x), "=l"(v.y) : "l"(ptr));
    return v;
}

__device__ __forceinline__ uint64_t shfl64(uint64_t v, int src) {
    return __shfl_sync(0xffffffffu, v, src);
}

__device__ __forceinline__ uint64_t keep_mask_before(uint64_t x) {
    // bits strictly before (more significant than) the leftmost one-bit of x; x != 0
    const int c = __clzll((long long)x);
    return c ? (~0ULL << (64 - c)) : 0ULL;
}

// Alg. 4 (reading R6): prefix = first with every position
// >= leftmost_nonzero_bit(first XOR last) cleared; whole first if equal.
__device__ __forceinline__ void tile_prefix(uint64_t f0, uint64_t f1, uint64_t f2, uint64_t l0, uint64_t l1,
                                            uint64_t l2, uint64_t &p0, uint64_t &p1, uint64_t &p2) {
    const uint64_t x0 = f0 ^ l0, x1 = f1 ^ l1, x2 = f2 ^ l2;
    uint64_t k0 = ~0ULL, k1 = ~0ULL, k2 = ~0ULL;
    if (x0) {
        k0 = keep_mask_before(x0);
        k1 = 0;
        k2 = 0;
    } else if (x1) {
        k1 = keep_mask_before(x1);
        k2 = 0;
    } else if (x2) {
        k2 = keep_mask_before(x2);
    }
    p0 = f0 & k0;
    p1 = f1 & k1;
    p2 = f2 & k2;
}

// Emit the (query, key) pairs of the lanes whose set matched: the key lookup and a
// warp-aggregated output reservation (replacing the per-pair atomic of PAPER.md:158).  bm = the
// warp's ballot of m (warp-uniform call); m lanes write their set's keys.
// Fused exchange (in-process multi-GPU database, tm_group.cu): the lanes' keys go straight to the
// query owner's receive region for this GPU (a peer pointer over NVLink) instead of the local output;
// one warp-aggregated reservation per owner present in the warp, on this GPU's counter of that
// owner (no remote atomics).  nk = the lane's key count, kb = its first key, qg = its query.
__device__ __forceinline__ uint32_t owner_of(uint32_t qg, const ScanParams &p) {
    uint32_t d = 0;
#pragma unroll
    for (int g = 1; g < kMaxOwners; ++g)
        if ((uint32_t)g < p.n_owners && qg >= p.xstart[g]) d = (uint32_t)g;
    return d;
}

__device__ __forceinline__ void emit_fused(uint32_t nk, uint32_t kb, uint32_t qg, const ScanParams &p, int lane) {
    const uint32_t d = nk ? owner_of(qg, p) : 0u;
    uint32_t todo = __ballot_sync(0xffffffffu, nk > 0);
    while (todo) {
        const int leader = __ffs(todo) - 1;
        const uint32_t dd = __shfl_sync(0xffffffffu, d, leader);
        const bool mine = nk > 0 && d == dd;
        todo &= ~__ballot_sync(0xffffffffu, mine);
        uint32_t v = mine ? nk : 0u, incl = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += t;
        }
        const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
        unsigned long long base = 0;
        if (lane == leader) base = atomicAdd(p.xcnt + dd, (unsigned long long)total);
        base = __shfl_sync(0xffffffffu, base, leader);
        if (mine) {
            unsigned long long o = base + (incl - v);
            uint64_t *dst = p.xout[dd];
            const uint64_t hi = (uint64_t)qg << 32;
            for (uint32_t j = 0; j < nk; ++j, ++o)
                if (o < p.xcap) dst[o] = hi | (uint64_t)__ldg(p.keys + kb + j);
        }
    }
}

template <bool FUSED>
__device__ __forceinline__ void emit_direct(bool m, uint32_t row, uint32_t qg, const ScanParams &p, int lane) {
    uint32_t kb = 0, nk = 0;
    if (m) {
        kb = __ldg(p.key_off + row);
        nk = __ldg(p.key_off + row + 1) - kb;
    }
    if constexpr (FUSED) {
        emit_fused(nk, kb, qg, p, lane);
        return;
    }
    uint32_t incl = nk;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    unsigned long long base = 0;
    if (lane == 31 && total) base = atomicAdd(&p.ctr->n_out, (unsigned long long)total);
    base = __shfl_sync(0xffffffffu, base, 31);
    unsigned long long o = base + (incl - nk);
    const uint64_t hi = (uint64_t)qg << 32;
    for (uint32_t j = 0; j < nk; ++j, ++o)
        if (o < p.cap) p.out[o] = hi | (uint64_t)__ldg(p.keys + kb + j);
}

// Emit the warp's staged matches (lanes 0..npend-1 take one each); warp-uniform call.
template <bool FUSED>
__device__ __forceinline__ void flush_pend(uint2 *pend, uint32_t &npend, const ScanParams &p, int lane) {
    if (!npend) return;
    __syncwarp();
    const bool m = (uint32_t)lane < npend;
    uint2 e = make_uint2(0u, 0u);
    if (m) e = pend[lane];
    uint32_t kb = 0, nk = 0;
    if (m) {
        kb = __ldg(p.key_off + e.x);
        nk = __ldg(p.key_off + e.x + 1) - kb;
    }
    if constexpr (FUSED) {
        emit_fused(nk, kb, e.y, p, lane);
        npend = 0;
        __syncwarp();
        return;
    }
    uint32_t incl = nk;
#pragma unroll
    for (int o = 1; o < (int)kPend; o <<= 1) {
        const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    const uint32_t total = __shfl_sync(0xffffffffu, incl, kPend - 1);
    unsigned long long base = 0;
    if (lane == (int)kPend - 1 && total) base = atomicAdd(&p.ctr->n_out, (unsigned long long)total);
    base = __shfl_sync(0xffffffffu, base, kPend - 1);
    unsigned long long o = base + (incl - nk);
    const uint64_t hi = (uint64_t)e.y << 32;
    for (uint32_t j = 0; j < nk; ++j, ++o)
        if (o < p.cap) p.out[o] = hi | (uint64_t)__ldg(p.keys + kb + j);
    npend = 0;
    __syncwarp();
}

// Stage the matches of one warp step (bm = ballot of m, nonzero, warp-uniform); a step with more
// matches than the stage holds is emitted directly.
template <bool FUSED>
__device__ __forceinline__ void emit_keys(bool m, uint32_t bm, uint32_t row, uint32_t qg, const ScanParams &p,
                                          int lane, uint2 *pend, uint32_t &npend) {
    const uint32_t c = __popc(bm);
    if (npend + c > kPend) flush_pend<FUSED>(pend, npend, p, lane);
    if (c > kPend) {
        emit_direct<FUSED>(m, row, qg, p, lane);
        return;
    }
    if (m) pend[npend + __popc(bm & ((1u << lane) - 1u))] = make_uint2(row, qg);
    npend += c;
}

// Block 2 of one survivor whose blocks 0-1 passed in some lane, then emit.
template <bool FUSED>
__device__ __forceinline__ void check_block2(bool hit01, uint32_t slot, uint64_t s2, uint32_t row,
                                             ScanSmem &sm, const ScanParams &p, int lane,
                                             uint32_t &matched, uint32_t &npend) {
    const bool m = hit01 && (s2 & ~sm.q2[slot]) == 0;
    const uint32_t b = __ballot_sync(0xffffffffu, m);
    if (b) {
        matched += __popc(b);
        emit_keys<FUSED>(m, b, row, __ldg(sm.qid + slot), p, lane, sm.pend[threadIdx.x >> 5], npend);
    }
}

// Warp AND over the first n lanes (others contribute all-ones).
__device__ __forceinline__ uint64_t warp_and(uint64_t v) {
#pragma unroll
    for (int o = 16; o; o >>= 1) v &= __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Persistent subset-scan kernel.  Work item = (partition p, query chunk c,
// row range r) from a global counter; the CTA stages the chunk's query
// signatures in shared memory, then its warps take units = (256-row block,
// query sub-range) from a shared counter.  Per unit: level A compacts the
// queries containing the block's common mask; per 32-row tile (one set per
// lane, in registers) level B compacts the level-A survivors containing the
// tile's mask, and each level-B survivor is checked block by block against
// the 32 sets: blocks 0-1 for all, block 2 when some lane passed (the subset
// check "amounts to a simple operation on each Bloom-filter block").
// Filters: 0 = Alg. 4 common prefix of first/last row; 1 = AND of the rows
// (precomputed per tile at build); 2 = none.
// Without WORD1 (variant 0): level-B survivors are 16-B entries (blocks 0, 1), tested four per
// iteration with one LDS.128 each, block 2 on a hit.
// WORD1: per-lane word pre-check.  Every row carries a build-time choice of two of its six
// 32-bit words (those with the most one-bits outside its tile's AND mask, k_word_select);
// each lane tests its set's two words against those words of 4 survivors per LDS.128 pair
// (s_w & ~q_w == 0 is necessary for s within q), collecting a 32-survivor pass mask in a
// register with no votes; only the (lane, survivor) pairs that pass (about 0.1% on the
// Twitter-like workload) get the full six-word check, in a divergent loop whose trip count
// is the largest per-lane pass count.
// MINB: resident CTAs per SM the register allocator must allow (__launch_bounds__); shared memory
// caps residency at 8 CTAs, which ptxas cannot see (the scan's shared memory is dynamic).
// STREAM: streaming path only (launched for calls of <= kSmallBatch queries), with StreamSmem.
// OPT: bit 0 = pre-check accumulate on the FMA pipe (precheck4x2<B, true>); bit 4 = lean tile
// set-up (the two pre-check words read from the build-time wwords plane, no per-lane selects).
__device__ unsigned long long g_scan_dbg[12];  // OPT & 512: pre-check pass statistics (diagnostic variant)

// BT: tiles per level-A block (<= kBlockTiles): 8 (256 rows) or 4 (128 rows; the default with small
// partitions)
template <bool WORD1 = false, int MINB = 8, bool STREAM = false, int OPT = 0, int BT = kBlockTiles>
__global__ void __launch_bounds__(kScanWarps * 32, MINB) k_scan(const ScanParams p) {
    static_assert(BT >= 1 && BT <= kBlockTiles, "level-A block of at most kBlockTiles tiles");
    constexpr bool kImad = (OPT & 1) != 0;
    constexpr bool kLean = WORD1 && !STREAM && (OPT & 16) != 0;
    constexpr bool kFused = (OPT & 64) != 0;  // emission into the owners' regions (in-process group)
    constexpr bool kDbg = WORD1 && !STREAM && (OPT & 512) != 0;    // pre-check pass statistics (g_scan_dbg)
    unsigned long long dbg[12];
    if constexpr (kDbg) {
#pragma unroll
        for (int i = 0; i < 12; ++i) dbg[i] = 0;
    }
    extern __shared__ __align__(16) unsigned char smem_raw[];
    using Smem = typename std::conditional<STREAM, StreamSmem, ScanSmem>::type;
    Smem &sm = *reinterpret_cast<Smem *>(smem_raw);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    // per-warp statistics, 32-bit (one item decides at most kChunk x range_rows pairs) and flushed to
    // the 64-bit global counters at every item boundary
    uint32_t st_tests = 0, st_checks = 0, st_matched = 0;
    uint32_t npend = 0;  // the warp's staged matches (sm.pend[warp])
    const unsigned long long n_items = p.item_off[p.n_parts];
    if (blockIdx.x == 0 && threadIdx.x == 0) p.ctr->n_items = n_items;
    if (p.ctr->routed > p.qcap) return;  // query lists truncated: the host grows qidx and re-runs
    if (threadIdx.x < 3) sm.cnt[threadIdx.x] = 0;  // ordered before any flush by the item loop's barrier
    uint16_t *sa = sm.sa[warp];
    uint4 *sbuf = sm.sbuf[warp];
    uint16_t *sbi = sm.sbi[warp];
    const uint32_t sb_addr = (uint32_t)__cvta_generic_to_shared(sbuf);

    for (;;) {
        if (lane == 0 && (st_tests | st_checks | st_matched)) {  // shared atomics: no global contention
            atomicAdd(&sm.cnt[0], (unsigned long long)st_tests);
            atomicAdd(&sm.cnt[1], (unsigned long long)st_checks);
            atomicAdd(&sm.cnt[2], (unsigned long long)st_matched);
        }
        st_tests = st_checks = st_matched = 0;
        if (threadIdx.x == 0) {
            sm.item = atomicAdd(&p.ctr->item_ctr, 1ULL);
            sm.unit_ctr = 0;
        }
        __syncthreads();
        const unsigned long long item = sm.item;
        if (item >= n_items) break;
        // partition: last p with item_off[p] <= item
        uint32_t lo = 0, hi = p.n_parts;  // invariant: item_off[lo] <= item < item_off[hi]
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (__ldg(p.item_off + mid) <= item) lo = mid; else hi = mid;
        }
        const uint32_t part = lo;
        const uint32_t prow = __ldg(p.part_row + part);
        const uint32_t rows = __ldg(p.part_row + part + 1) - prow;
        const uint32_t real_end = prow + __ldg(p.part_n + part);
        const unsigned long long pq0 = __ldg(p.qoff + part), pq1 = __ldg(p.qoff + part + 1);
        const uint32_t rr = part_range_rows(pq1 - pq0, p.range_rows);
        const uint32_t nrange = (rows + rr - 1) / rr;
        const unsigned long long local = item - __ldg(p.item_off + part);
        const uint32_t chunk = (uint32_t)(local / nrange), range = (uint32_t)(local % nrange);
        const unsigned long long qbeg = pq0 + (unsigned long long)chunk * kChunk;
        const uint32_t nq = (uint32_t)min((unsigned long long)kChunk, pq1 - qbeg);
        const uint32_t rlo = prow + range * rr;
        const uint32_t rhi = min(rlo + rr, prow + rows);

        if constexpr (STREAM) {
            if (nq > (uint32_t)kSmallBatch) __trap();  // the host launches STREAM kernels for Q <= kSmallBatch only
        }
        if (threadIdx.x == 0) sm.qid = p.qidx + qbeg;
        // stage the query batch (the batch of queries of partition p)
        for (uint32_t i = threadIdx.x; i < nq; i += blockDim.x) {
            const uint32_t q = __ldg(p.qidx + qbeg + i);
            sm.q0[i] = __ldg(p.q0 + q);
            sm.q1[i] = __ldg(p.q1 + q);
            sm.q2[i] = __ldg(p.q2 + q);
        }
        __syncthreads();

        if (nq <= (uint32_t)kSmallBatch) {
            // Small batch (a lightly loaded partition, a latency-bound call, the HBM sweep):
            // the pre-filter cannot pay off, so each warp streams 64-row units (two rows per
            // lane, all loads issued up front) and checks every row against every query on all
            // three blocks -- the HBM-bound regime of the scan.
            const uint32_t vend = min(real_end, rhi);
            // WORD1 with 3..8 queries: pre-check; one or two queries: the direct check below is cheaper
            const bool pre = WORD1 && nq > 4;
            // units: 64 rows (pre-check: two rows per lane) or 128 rows (direct: four rows per lane as
            // two 16-B loads per plane, 96 B in flight per lane)
            const uint32_t ush = pre ? 6u : 7u;
            const uint32_t nunit = (rhi - rlo + (1u << ush) - 1) >> ush;
            if (pre) {
                // the batch as six 32-bit word planes (warp 0's survivor planes; read-only here)
                if (threadIdx.x < 6 * kSmallBatch) {
                    const uint32_t w = threadIdx.x / kSmallBatch, j = threadIdx.x % kSmallBatch;
                    const uint64_t b = j < nq ? (w < 2 ? sm.q0[j] : w < 4 ? sm.q1[j] : sm.q2[j]) : 0ULL;
                    sm.sw[0][w][j] = (w & 1) ? (uint32_t)(b >> 32) : (uint32_t)b;
                }
                __syncthreads();
            }
            for (;;) {
                uint32_t u = 0;
                if (lane == 0) u = atomicAdd(&sm.unit_ctr, 1u);
                u = __shfl_sync(0xffffffffu, u, 0);
                if (u >= nunit) break;
                if (pre) {
                    // two-word pre-check of both rows against the batch (4 queries per LDS.128 pair),
                    // full check only on the (row, query) pairs that pass; rows (ra, ra + 1) per lane
                    // as one 16-B load per plane (a tile never straddles rhi)
                    const uint32_t ra = rlo + u * 64 + 2 * (uint32_t)lane, rb = ra + 1;
                    ulonglong2 v0 = make_ulonglong2(~0ULL, ~0ULL), v1 = v0, v2 = v0;
                    uint32_t wab = 0x1010u;
                    if (ra < rhi) {
                        v0 = ldg_stream2(p.w0 + ra);
                        v1 = ldg_stream2(p.w1 + ra);
                        v2 = ldg_stream2(p.w2 + ra);
                        wab = __ldg(reinterpret_cast<const unsigned short *>(p.wsel + ra));
                    }
                    const uint64_t a0 = v0.x, a1 = v1.x, a2 = v2.x, b0 = v0.y, b1 = v1.y, b2 = v2.y;
                    const bool va = ra < vend, vb = rb < vend;
                    const uint32_t wa = wab & 0xffu, wb = wab >> 8;
                    const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm.sw[0][0]);
                    constexpr uint32_t kPl = kSubWStride * 4;
                    const uint32_t xa = pick_word(a0, a1, a2, wa & 15u, va), ya = pick_word(a0, a1, a2, wa >> 4, va);
                    const uint32_t xb = pick_word(b0, b1, b2, wb & 15u, vb), yb = pick_word(b0, b1, b2, wb >> 4, vb);
                    const uint32_t pxa = base + (wa & 15u) * kPl, pya = base + (wa >> 4) * kPl;
                    const uint32_t pxb = base + (wb & 15u) * kPl, pyb = base + (wb >> 4) * kPl;
                    uint32_t c0 = 0, c1 = 0, c2 = 0, c3 = 0, d0 = 0, d1 = 0, d2 = 0, d3 = 0;
                    precheck4x2<1u>(c0, c1, c2, c3, xa, lds128(pxa), ya, lds128(pya));
                    precheck4x2<1u>(d0, d1, d2, d3, xb, lds128(pxb), yb, lds128(pyb));
                    if (nq > 4) {
                        precheck4x2<16u>(c0, c1, c2, c3, xa, lds128(pxa + 16), ya, lds128(pya + 16));
                        precheck4x2<16u>(d0, d1, d2, d3, xb, lds128(pxb + 16), yb, lds128(pyb + 16));
                    }
                    const uint32_t qmask = (1u << nq) - 1u;
                    uint32_t acc = va ? ((c0 | c1) | (c2 | c3)) & qmask : 0u;
                    acc |= vb ? (((d0 | d1) | (d2 | d3)) & qmask) << 16 : 0u;  // row b: bits 16..
                    while (__any_sync(0xffffffffu, acc != 0)) {
                        bool m = false;
                        uint32_t j = 0, row = ra;
                        if (acc) {
                            const uint32_t bit = (uint32_t)(__ffs(acc) - 1);
                            acc &= acc - 1;
                            const bool isb = bit >= 16;
                            j = bit & 15u;
                            row = isb ? rb : ra;
                            const uint64_t s0 = isb ? b0 : a0, s1 = isb ? b1 : a1, s2 = isb ? b2 : a2;
                            m = ((s0 & ~sm.q0[j]) | (s1 & ~sm.q1[j]) | (s2 & ~sm.q2[j])) == 0;
                        }
                        const uint32_t bm = __ballot_sync(0xffffffffu, m);
                        if (bm) {
                            st_matched += __popc(bm);
                            emit_keys<kFused>(m, bm, row, m ? __ldg(sm.qid + j) : 0u, p, lane, sm.pend[warp], npend);
                        }
                    }
                    const uint32_t u0 = rlo + u * 64;
                    st_checks += nq * (vend > u0 ? min(64u, vend - u0) : 0u);
                    continue;
                }
                // direct check: rows (r, r+1) and (r+64, r+65) per lane, r = base + 2 lane; a tile
                // is either wholly inside the range or wholly outside, so a pair never straddles rhi
                const uint32_t u0 = rlo + (u << 7);
                const uint32_t r0 = u0 + 2 * (uint32_t)lane, r1 = r0 + 64;
                ulonglong2 a0 = make_ulonglong2(~0ULL, ~0ULL), a1 = a0, a2 = a0, b0 = a0, b1 = a0, b2 = a0;
                if (r0 < rhi) {
                    a0 = ldg_stream2(p.w0 + r0);
                    a1 = ldg_stream2(p.w1 + r0);
                    a2 = ldg_stream2(p.w2 + r0);
                }
                if (r1 < rhi) {
                    b0 = ldg_stream2(p.w0 + r1);
                    b1 = ldg_stream2(p.w1 + r1);
                    b2 = ldg_stream2(p.w2 + r1);
                }
                const bool v0 = r0 < vend, v1 = r0 + 1 < vend, v2 = r1 < vend, v3 = r1 + 1 < vend;
                for (uint32_t j = 0; j < nq; ++j) {
                    const uint64_t q0 = sm.q0[j], q1 = sm.q1[j], q2 = sm.q2[j];
                    const bool h0 = v0 && ((a0.x & ~q0) | (a1.x & ~q1) | (a2.x & ~q2)) == 0;
                    const bool h1 = v1 && ((a0.y & ~q0) | (a1.y & ~q1) | (a2.y & ~q2)) == 0;
                    const bool h2 = v2 && ((b0.x & ~q0) | (b1.x & ~q1) | (b2.x & ~q2)) == 0;
                    const bool h3 = v3 && ((b0.y & ~q0) | (b1.y & ~q1) | (b2.y & ~q2)) == 0;
                    if (__any_sync(0xffffffffu, (h0 || h1) || (h2 || h3))) {
                        const uint32_t qg = __ldg(sm.qid + j);
                        const bool hh[4] = {h0, h1, h2, h3};
                        const uint32_t rr4[4] = {r0, r0 + 1, r1, r1 + 1};
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            const uint32_t bq = __ballot_sync(0xffffffffu, hh[e]);
                            if (bq) {
                                st_matched += __popc(bq);
                                emit_keys<kFused>(hh[e], bq, rr4[e], qg, p, lane, sm.pend[warp], npend);
                            }
                        }
                    }
                }
                st_checks += nq * (vend > u0 ? min(128u, vend - u0) : 0u);
            }
            __syncthreads();
            continue;
        }

        if constexpr (!STREAM) {
        const uint32_t ntile = (rhi - rlo) / kTile;
        const uint32_t nblock = (ntile + BT - 1) / BT;
        // unit = (256-row block, query sub-range), taken dynamically through unit_ctr;
        // few blocks: split the batch so every warp has work
        // (a small item -- few blocks -- is split over query sub-ranges until it has p.unit_target
        // units, so its warps finish together at the item barrier)
        const uint32_t nsplit = nblock >= p.unit_target
                                    ? 1u
                                    : min((p.unit_target + max(nblock, 1u) - 1) / max(nblock, 1u), (nq + 31) / 32);
        const uint32_t subsz = ((nq + nsplit - 1) / nsplit + 31) & ~31u;
        const uint32_t units = nblock * nsplit;
        for (;;) {
            uint32_t u = 0;
            if (lane == 0) u = atomicAdd(&sm.unit_ctr, 1u);
            u = __shfl_sync(0xffffffffu, u, 0);
            if (u >= units) break;
            const uint32_t blk = u / nsplit, sub = u % nsplit;
            const uint32_t qs = sub * subsz, qe = min(nq, qs + subsz);
            if (qs >= qe) continue;
            const uint32_t t_first = blk * BT, t_end = min(ntile, t_first + BT);
            const uint32_t brow0 = rlo + t_first * kTile;
            const uint32_t bend = min(rlo + t_end * kTile, real_end);  // real rows of the block
            // ---- level A: the block's common mask
            uint64_t f0 = 0, f1 = 0, f2 = 0;
            if (p.filter == 0) {
                tile_prefix(__ldg(p.w0 + brow0), __ldg(p.w1 + brow0), __ldg(p.w2 + brow0), __ldg(p.w0 + bend - 1),
                            __ldg(p.w1 + bend - 1), __ldg(p.w2 + bend - 1), f0, f1, f2);
            } else if (p.filter == 1) {
                const uint32_t t = brow0 / kTile + lane;
                const bool in = (uint32_t)lane < t_end - t_first;
                const uint64_t m0 = in ? __ldg(p.t0 + t) : ~0ULL, m1 = in ? __ldg(p.t1 + t) : ~0ULL,
                               m2 = in ? __ldg(p.t2 + t) : ~0ULL;
                if ((uint32_t)lane < (uint32_t)BT) {  // the block's tile masks, for level B
                    sm.tmask[warp][0][lane] = m0;
                    sm.tmask[warp][1][lane] = m1;
                    sm.tmask[warp][2][lane] = m2;
                }
                f0 = warp_and(m0);
                f1 = warp_and(m1);
                f2 = warp_and(m2);
            }
            uint32_t na = 0;
            if ((f0 != 0) + (f1 != 0) + (f2 != 0) <= 1) {
                // the block mask lives in one word (or none): test that word only (warp-uniform)
                const uint64_t *qw = f1 ? sm.q1 : (f2 ? sm.q2 : sm.q0);
                const uint64_t fm = f0 | f1 | f2;
                for (uint32_t qb = qs; qb < qe; qb += 32) {
                    const uint32_t i = qb + lane;
                    const bool ok = i < qe && (fm & ~qw[i]) == 0;
                    const uint32_t b = __ballot_sync(0xffffffffu, ok);
                    if (ok) sa[na + __popc(b & lt_mask)] = (uint16_t)i;
                    na += __popc(b);
                }
            } else if (f0 == 0 || f1 == 0 || f2 == 0) {
                // two nonzero words: test those two only
                const uint64_t *qa = f0 ? sm.q0 : sm.q1, *qb2 = f2 ? sm.q2 : sm.q1;
                const uint64_t fa = f0 ? f0 : f1, fb = f2 ? f2 : f1;
                for (uint32_t qb = qs; qb < qe; qb += 32) {
                    const uint32_t i = qb + lane;
                    const bool ok = i < qe && ((fa & ~qa[i]) | (fb & ~qb2[i])) == 0;
                    const uint32_t b = __ballot_sync(0xffffffffu, ok);
                    if (ok) sa[na + __popc(b & lt_mask)] = (uint16_t)i;
                    na += __popc(b);
                }
            } else {
                for (uint32_t qb = qs; qb < qe; qb += 32) {
                    const uint32_t i = qb + lane;
                    const bool ok = i < qe && ((f0 & ~sm.q0[i]) | (f1 & ~sm.q1[i]) | (f2 & ~sm.q2[i])) == 0;
                    const uint32_t b = __ballot_sync(0xffffffffu, ok);
                    if (ok) sa[na + __popc(b & lt_mask)] = (uint16_t)i;
                    na += __popc(b);
                }
            }
            st_tests += qe - qs;
            __syncwarp();
            if (na == 0) continue;
            // ---- per tile of the block
            for (uint32_t t = t_first; t < t_end; ++t) {
                const uint32_t row0 = rlo + t * kTile;
                const uint32_t row = row0 + lane;
                const uint32_t nvalid = min(32u, real_end - row0);
                const bool valid = (uint32_t)lane < nvalid;
                // rows are padded to whole tiles: every lane may load
                const uint64_t s0 = __ldg(p.w0 + row), s1 = __ldg(p.w1 + row), s2 = __ldg(p.w2 + row);
                uint64_t g0 = 0, g1 = 0, g2 = 0;
                if (p.filter == 0) {
                    tile_prefix(shfl64(s0, 0), shfl64(s1, 0), shfl64(s2, 0), shfl64(s0, nvalid - 1),
                                shfl64(s1, nvalid - 1), shfl64(s2, nvalid - 1), g0, g1, g2);
                } else if (p.filter == 1) {  // staged at level A (written before the __syncwarp there)
                    g0 = sm.tmask[warp][0][t - t_first];
                    g1 = sm.tmask[warp][1][t - t_first];
                    g2 = sm.tmask[warp][2][t - t_first];
                }
                // 32-bit halves of the lane's set (invalid lanes: all ones, never pass; the lean form
                // relies on the pre-check mask of invalid lanes being cleared instead)
                const uint32_t a0l = (kLean || valid) ? (uint32_t)s0 : ~0u, a0h = (kLean || valid) ? (uint32_t)(s0 >> 32) : ~0u;
                const uint32_t a1l = (kLean || valid) ? (uint32_t)s1 : ~0u, a1h = (kLean || valid) ? (uint32_t)(s1 >> 32) : ~0u;
                const uint32_t a2l = (kLean || valid) ? (uint32_t)s2 : ~0u, a2h = (kLean || valid) ? (uint32_t)(s2 >> 32) : ~0u;
                if constexpr (WORD1) {
                    uint32_t wsel, aw, aw2;
                    if constexpr (kLean) {
                        // the row's two pre-check words, precomputed at build (rows are padded to whole
                        // tiles, so every lane may load; invalid lanes' acc is cleared below)
                        wsel = (uint32_t)__ldg(p.wsel + row);
                        const uint2 ww = __ldg(p.wwords + row);
                        aw = ww.x;
                        aw2 = ww.y;
                    } else {
                        wsel = valid ? (uint32_t)__ldg(p.wsel + row) : 0x10u;
                        // branch-free word select: block wl >> 1, half wl & 1 (invalid lanes: all ones)
                        aw = pick_word(s0, s1, s2, wsel & 15u, valid);
                        aw2 = pick_word(s0, s1, s2, wsel >> 4, valid);
                    }
                    const uint32_t wl = wsel & 15u, wl2 = wsel >> 4;
                    st_tests += na;
                    const uint32_t *swp = sm.sw[warp][0];
                    const uint32_t sw_base = (uint32_t)__cvta_generic_to_shared(swp);
                    const uint32_t my_plane = sw_base + wl * (uint32_t)(kSubWStride * 4);
                    const uint32_t my_plane2 = sw_base + wl2 * (uint32_t)(kSubWStride * 4);
                    for (uint32_t j = 0; j < na;) {
                        // ---- level B: level-A survivors that contain the tile's mask -> word planes,
                        // 32 at a time until the buffer cannot take another 32 (full pre-check groups)
                        uint32_t nb = 0;
                        const uint32_t pe = na;
                        // two independent 32-survivor halves per step (ILP), then one more half
                        // when it still fits
                        uint32_t *swk = sm.sw[warp][0];
                        for (; j < na && nb <= (uint32_t)kSubW - 64; j += 64) {
                            const uint32_t ja = j + lane, jb = ja + 32;
                            // sa[0, pe) holds valid slots (< kChunk); lanes past pe read slot 0
                            const uint32_t ia = ja < pe ? (uint32_t)sa[ja] : 0u;
                            const uint32_t ib = jb < pe ? (uint32_t)sa[jb] : 0u;
                            const uint64_t a0 = sm.q0[ia], a1 = sm.q1[ia], a2 = sm.q2[ia];
                            const uint64_t b0 = sm.q0[ib], b1 = sm.q1[ib], b2 = sm.q2[ib];
                            const bool oka = ja < pe && ((g0 & ~a0) | (g1 & ~a1) | (g2 & ~a2)) == 0;
                            const bool okb = jb < pe && ((g0 & ~b0) | (g1 & ~b1) | (g2 & ~b2)) == 0;
                            const uint32_t ba = __ballot_sync(0xffffffffu, oka);
                            const uint32_t bb = __ballot_sync(0xffffffffu, okb);
                            if (oka) store_survivor(swk, sbi, nb + __popc(ba & lt_mask), a0, a1, a2, ia);
                            const uint32_t nba = nb + __popc(ba);
                            if (okb) store_survivor(swk, sbi, nba + __popc(bb & lt_mask), b0, b1, b2, ib);
                            nb = nba + __popc(bb);
                        }
                        if (j < na && nb <= (uint32_t)kSubW - 32) {
                            const uint32_t ja = j + lane;
                            const uint32_t ia = ja < pe ? (uint32_t)sa[ja] : 0u;
                            const uint64_t a0 = sm.q0[ia], a1 = sm.q1[ia], a2 = sm.q2[ia];
                            const bool oka = ja < pe && ((g0 & ~a0) | (g1 & ~a1) | (g2 & ~a2)) == 0;
                            const uint32_t ba = __ballot_sync(0xffffffffu, oka);
                            if (oka) store_survivor(swk, sbi, nb + __popc(ba & lt_mask), a0, a1, a2, ia);
                            nb += __popc(ba);
                            j += 32;
                        }
                        st_checks += nb * nvalid;
                        __syncwarp();
                        for (uint32_t k0 = 0; k0 < nb; k0 += 32) {
                            const uint32_t cnt = min(32u, nb - k0);
                            // ---- pre-check: the lane's word against 32 survivors, pass bits in acc
                            uint32_t c0 = 0, c1 = 0, c2 = 0, c3 = 0;
                            const uint32_t pa = my_plane + k0 * 4, pa2 = my_plane2 + k0 * 4;
#define TM_PRE(B, o) precheck4x2<B, kImad>(c0, c1, c2, c3, aw, lds128(pa + (o)), aw2, lds128(pa2 + (o)), p.one)
                            TM_PRE(1u << 0, 0);
                            TM_PRE(1u << 4, 16);
                            if (cnt > 8) {
                                TM_PRE(1u << 8, 32);
                                TM_PRE(1u << 12, 48);
                            }
                            if (cnt > 16) {
                                TM_PRE(1u << 16, 64);
                                TM_PRE(1u << 20, 80);
                            }
                            if (cnt > 24) {
                                TM_PRE(1u << 24, 96);
                                TM_PRE(1u << 28, 112);
                            }
#undef TM_PRE
                            uint32_t acc = (c0 | c1) | (c2 | c3);
                            if (cnt < 32) acc &= (1u << cnt) - 1u;
                            if (!valid) acc = 0;
                            if constexpr (kDbg) {
                                const uint32_t pc = __popc(acc);
                                const uint32_t mx = __reduce_max_sync(0xffffffffu, pc);
                                dbg[0] += __reduce_add_sync(0xffffffffu, pc);
                                dbg[1] += 1;
                                dbg[2] += mx;
                                dbg[3 + (mx == 0 ? 0 : mx == 1 ? 1 : mx == 2 ? 2 : mx <= 4 ? 3 : mx <= 8 ? 4 : mx <= 16 ? 5 : 6)] += 1;
                                dbg[10] += __reduce_add_sync(0xffffffffu, pc > 8 ? pc : 0u);
                                dbg[11] += __reduce_add_sync(0xffffffffu, pc ? 1u : 0u);
                            }
                            // ---- Alg. 3 on the pairs that passed: all six words, then emit
                            while (__any_sync(0xffffffffu, acc != 0)) {
                                bool m = false;
                                uint32_t e = 0;
                                if (acc) {
                                    e = k0 + (uint32_t)(__ffs(acc) - 1);
                                    acc &= acc - 1;
                                    const uint32_t *c = swp + e;
                                    m = ((a0l & ~c[0]) | (a0h & ~c[kSubWStride]) | (a1l & ~c[2 * kSubWStride]) |
                                         (a1h & ~c[3 * kSubWStride]) | (a2l & ~c[4 * kSubWStride]) |
                                         (a2h & ~c[5 * kSubWStride])) == 0;
                                }
                                const uint32_t bm = __ballot_sync(0xffffffffu, m);
                                if (bm) {
                                    st_matched += __popc(bm);
                                    emit_keys<kFused>(m, bm, row, m ? __ldg(sm.qid + sbi[e]) : 0u, p, lane, sm.pend[warp], npend);
                                }
                            }
                        }
                        __syncwarp();
                    }
                    continue;
                }
                for (uint32_t pb = 0; pb < na; pb += kSubB) {
                    const uint32_t pe = min(na, pb + kSubB);
                    // ---- level B: level-A survivors that contain the tile's mask
                    uint32_t nb = 0;
                    for (uint32_t j = pb; j < pe; j += 32) {
                        const uint32_t jj = j + lane;
                        bool ok = false;
                        uint64_t a0 = 0, a1 = 0, a2 = 0;
                        uint32_t i = 0;
                        if (jj < pe) {
                            i = sa[jj];
                            a0 = sm.q0[i];
                            a1 = sm.q1[i];
                            a2 = sm.q2[i];
                            ok = ((g0 & ~a0) | (g1 & ~a1) | (g2 & ~a2)) == 0;
                        }
                        const uint32_t b = __ballot_sync(0xffffffffu, ok);
                        if (ok) {
                            const uint32_t k = nb + __popc(b & lt_mask);
                            sbuf[k] = make_uint4((uint32_t)a0, (uint32_t)(a0 >> 32), (uint32_t)a1, (uint32_t)(a1 >> 32));
                            sbi[k] = (uint16_t)i;
                        }
                        nb += __popc(b);
                    }
                    st_tests += pe - pb;
                    st_checks += nb * nvalid;
                    // pad to a multiple of 4 with zeros (masked by k < nb below)
                    if ((uint32_t)lane < ((4 - (nb % 4)) % 4)) {
                        sbuf[nb + lane] = make_uint4(0, 0, 0, 0);
                        sbi[nb + lane] = 0;
                    }
                    __syncwarp();
                    // ---- Alg. 3: 4 survivors per iteration against the warp's 32 sets, blocks 0-1
                    // first (one LDS.128 each), block 2 only when some lane passed
                    for (uint32_t k = 0; k < nb; k += 4) {
                        bool h[4];
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            const uint4 v = lds128(sb_addr + (k + j) * 16);
                            h[j] = ((a0l & ~v.x) | (a0h & ~v.y) | (a1l & ~v.z) | (a1h & ~v.w)) == 0;
                        }
                        if (__any_sync(0xffffffffu, (h[0] | h[1]) | (h[2] | h[3]))) {
#pragma unroll
                            for (int j = 0; j < 4; ++j)
                                if (k + j < nb && __any_sync(0xffffffffu, h[j]))
                                    check_block2<kFused>(h[j], sbi[k + j], s2, row, sm, p, lane, st_matched, npend);
                        }
                    }
                    __syncwarp();
                }
            }
        }
        }  // !STREAM
        __syncthreads();
    }
    // the loop ends for all warps together (after the barrier that read the last item)
    flush_pend<kFused>(sm.pend[warp], npend, p, lane);
    if constexpr (kDbg) {
        if (lane == 0)
            for (int i = 0; i < 12; ++i) atomicAdd(&g_scan_dbg[i], dbg[i]);
    }
    if (lane == 0 && (st_tests | st_checks | st_matched)) {
        atomicAdd(&sm.cnt[0], (unsigned long long)st_tests);
        atomicAdd(&sm.cnt[1], (unsigned long long)st_checks);
        atomicAdd(&sm.cnt[2], (unsigned long long)st_matched);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (sm.cnt[0]) atomicAdd(&p.ctr->tile_tests, sm.cnt[0]);
        if (sm.cnt[1]) atomicAdd(&p.ctr->pair_checks, sm.cnt[1]);
        if (sm.cnt[2]) atomicAdd(&p.ctr->matched_sets, sm.cnt[2]);
    }
}

// ------------------------------------------------------------ dense scan ---
// Unfiltered subset scan (tables built with tile_filter = 2: the plain Alg. 3 scan, and the HBM
// roofline sweep of SURVEY 8(d)).  No pre-filter, so no survivor compaction: the item's query
// batch is staged once as six 32-bit word planes, every lane holds two consecutive rows, and the
// two-word pre-check of the filtered path (necessary condition, 3 ops per (row, query), four
// queries per LDS.128 pair) runs against the whole batch in groups of 32 queries; only passing
// (row, query) pairs get the full six-word check (Alg. 3) and are emitted.
// BULK = false: lanes load their rows straight from HBM (16-B non-allocating loads).
// BULK = true : each warp streams its 64-row units through a ring of kDenseStages shared-memory
//               stages filled by 1-D bulk copies (cp.async.bulk, completion on an mbarrier):
//               the next units are in flight while the current one is checked, with no
//               registers held for outstanding loads (north_star's "TMA staging of a
//               partition tile").
constexpr int kDenseStages = 3;
constexpr int kDenseRows = 64;                  // rows per unit (two per lane)
constexpr int kDpStride = kChunk + 4;           // word-plane stride: 16 B mod 128 -> planes on disjoint bank quads

struct DenseSmemBase {
    uint32_t dp[6][kDpStride];                  // the batch as word planes
    const uint32_t *qid;
    unsigned long long item;
    unsigned int unit_ctr;
    unsigned long long cnt[3];
    uint2 pend[kScanWarps][kPend];
};
struct DenseSmemBulk : DenseSmemBase {
    __align__(16) uint64_t stage[kScanWarps][kDenseStages][3 * kDenseRows];  // per warp: ring of row tiles
    __align__(16) uint8_t wstage[kScanWarps][kDenseStages][kDenseRows];      // their pre-check word bytes
    __align__(8) unsigned long long bar[kScanWarps][kDenseStages];           // one mbarrier per stage
};

__device__ __forceinline__ void mbar_init(unsigned long long *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(unsigned long long *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ bool mbar_try_wait(unsigned long long *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred P1;\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\tselp.u32 %0, 1, 0, P1;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

// 1-D bulk copy global -> shared (TMA engine), completing `bytes` on the mbarrier
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, unsigned long long *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

// OPT: bit 0 = FMA-pipe pre-check accumulate; bit 2 (direct loads only) = four rows per lane
// (128-row units, both row pairs' loads issued before the checks: twice the bytes in flight).
template <bool BULK, int OPT = 0>
__global__ void __launch_bounds__(kScanWarps * 32, BULK ? 6 : 7) k_dense(const ScanParams p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    using Smem = typename std::conditional<BULK, DenseSmemBulk, DenseSmemBase>::type;
    Smem &sm = *reinterpret_cast<Smem *>(smem_raw);
    constexpr bool kImad = (OPT & 1) != 0;
    constexpr bool kFused = (OPT & 64) != 0;  // emission into the owners' regions (in-process group)
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t st_checks = 0, st_matched = 0;
    uint32_t npend = 0;
    uint32_t par = 0;  // BULK: expected phase parity of each of the warp's stages (bit s)
    const unsigned long long n_items = p.item_off[p.n_parts];
    if (blockIdx.x == 0 && threadIdx.x == 0) p.ctr->n_items = n_items;
    if (p.ctr->routed > p.qcap) return;
    if (threadIdx.x < 3) sm.cnt[threadIdx.x] = 0;
    if constexpr (BULK) {
        if (lane == 0)
            for (int i = 0; i < kDenseStages; ++i) mbar_init(&sm.bar[warp][i], 1);
    }
    const uint32_t dp_base = smem_u32(sm.dp[0]);
    constexpr uint32_t kPl = kDpStride * 4;

    for (;;) {
        if (lane == 0 && (st_checks | st_matched)) {
            atomicAdd(&sm.cnt[1], (unsigned long long)st_checks);
            atomicAdd(&sm.cnt[2], (unsigned long long)st_matched);
        }
        st_checks = st_matched = 0;
        if (threadIdx.x == 0) {
            sm.item = atomicAdd(&p.ctr->item_ctr, 1ULL);
            sm.unit_ctr = 0;
        }
        __syncthreads();  // also orders the mbarrier inits before their first use
        const unsigned long long item = sm.item;
        if (item >= n_items) break;
        uint32_t lo = 0, hi = p.n_parts;
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (__ldg(p.item_off + mid) <= item) lo = mid; else hi = mid;
        }
        const uint32_t part = lo;
        const uint32_t prow = __ldg(p.part_row + part);
        const uint32_t rows = __ldg(p.part_row + part + 1) - prow;
        const uint32_t real_end = prow + __ldg(p.part_n + part);
        const unsigned long long pq0 = __ldg(p.qoff + part), pq1 = __ldg(p.qoff + part + 1);
        const uint32_t rr = part_range_rows(pq1 - pq0, p.range_rows);
        const uint32_t nrange = (rows + rr - 1) / rr;
        const unsigned long long local = item - __ldg(p.item_off + part);
        const uint32_t chunk = (uint32_t)(local / nrange), range = (uint32_t)(local % nrange);
        const unsigned long long qbeg = pq0 + (unsigned long long)chunk * kChunk;
        const uint32_t nq = (uint32_t)min((unsigned long long)kChunk, pq1 - qbeg);
        const uint32_t rlo = prow + range * rr;
        const uint32_t rhi = min(rlo + rr, prow + rows);
        const uint32_t vend = min(real_end, rhi);
        if (threadIdx.x == 0) sm.qid = p.qidx + qbeg;
        // the batch as six word planes
        for (uint32_t i = threadIdx.x; i < nq; i += blockDim.x) {
            const uint32_t q = __ldg(p.qidx + qbeg + i);
            const uint64_t a0 = __ldg(p.q0 + q), a1 = __ldg(p.q1 + q), a2 = __ldg(p.q2 + q);
            sm.dp[0][i] = (uint32_t)a0;
            sm.dp[1][i] = (uint32_t)(a0 >> 32);
            sm.dp[2][i] = (uint32_t)a1;
            sm.dp[3][i] = (uint32_t)(a1 >> 32);
            sm.dp[4][i] = (uint32_t)a2;
            sm.dp[5][i] = (uint32_t)(a2 >> 32);
        }
        __syncthreads();
        // rows per unit: 64 (two per lane), or 128 with kRows4 (four per lane, all loads issued first)
        constexpr bool kRows4 = !BULK && (OPT & 4) != 0;
        constexpr uint32_t kUnitRows = kRows4 ? 2 * kDenseRows : kDenseRows;
        const uint32_t nunit = (rhi - rlo + kUnitRows - 1) / kUnitRows;
        auto take = [&]() {
            uint32_t u = 0;
            if (lane == 0) u = atomicAdd(&sm.unit_ctr, 1u);
            return __shfl_sync(0xffffffffu, u, 0);
        };
        // BULK: fill stage si with unit u (lane 0): 3 planes + the word bytes, nr = 32 or 64 rows
        auto issue = [&](uint32_t si, uint32_t u) {
            if constexpr (BULK) {
                if (lane == 0) {
                    const uint32_t r0 = rlo + u * kDenseRows;
                    const uint32_t nr = min((uint32_t)kDenseRows, rhi - r0);
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // prior generic reads of the stage
                    mbar_expect_tx(&sm.bar[warp][si], nr * 25);
                    bulk_g2s(&sm.stage[warp][si][0], p.w0 + r0, nr * 8, &sm.bar[warp][si]);
                    bulk_g2s(&sm.stage[warp][si][kDenseRows], p.w1 + r0, nr * 8, &sm.bar[warp][si]);
                    bulk_g2s(&sm.stage[warp][si][2 * kDenseRows], p.w2 + r0, nr * 8, &sm.bar[warp][si]);
                    bulk_g2s(&sm.wstage[warp][si][0], p.wsel + r0, nr, &sm.bar[warp][si]);
                }
            }
        };
        // kLeanD (direct loads): the rows' pre-check words come from the build-time wwords plane
        constexpr bool kLeanD = !BULK && (OPT & 16) != 0;
        // direct loads of rows (r, r + 1) of a lane (all-ones past the range)
        auto load_pair = [&](uint32_t r, ulonglong2 &x0, ulonglong2 &x1, ulonglong2 &x2, uint32_t &xw, uint4 &ww) {
            x0 = x1 = x2 = make_ulonglong2(~0ULL, ~0ULL);
            xw = 0x1010u;
            ww = make_uint4(~0u, ~0u, ~0u, ~0u);
            if (r < rhi) {
                x0 = ldg_stream2(p.w0 + r);
                x1 = ldg_stream2(p.w1 + r);
                x2 = ldg_stream2(p.w2 + r);
                xw = __ldg(reinterpret_cast<const unsigned short *>(p.wsel + r));
                if constexpr (kLeanD) ww = __ldg(reinterpret_cast<const uint4 *>(p.wwords + r));
            }
        };
        // the two-word pre-check of rows (u0 + 2 lane, + 1) against the batch, full checks, emission
        auto check_pair = [&](const ulonglong2 v0, const ulonglong2 v1, const ulonglong2 v2, const uint32_t wab,
                              const uint32_t u0, const uint4 ww) {
                const uint32_t ra = u0 + 2 * (uint32_t)lane, rb = ra + 1;
                const uint64_t a0 = v0.x, a1 = v1.x, a2 = v2.x, b0 = v0.y, b1 = v1.y, b2 = v2.y;
                const bool va = ra < vend, vb = rb < vend;
                const uint32_t wa = wab & 0xffu, wb = wab >> 8;
                uint32_t xa, ya, xb, yb;
                if constexpr (kLeanD) {  // invalid rows: their pass masks are cleared below
                    xa = ww.x;
                    ya = ww.y;
                    xb = ww.z;
                    yb = ww.w;
                } else {
                    xa = pick_word(a0, a1, a2, wa & 15u, va);
                    ya = pick_word(a0, a1, a2, wa >> 4, va);
                    xb = pick_word(b0, b1, b2, wb & 15u, vb);
                    yb = pick_word(b0, b1, b2, wb >> 4, vb);
                }
                const uint32_t pxa = dp_base + (wa & 15u) * kPl, pya = dp_base + (wa >> 4) * kPl;
                const uint32_t pxb = dp_base + (wb & 15u) * kPl, pyb = dp_base + (wb >> 4) * kPl;
                for (uint32_t k0 = 0; k0 < nq; k0 += 32) {
                    uint32_t c0 = 0, c1 = 0, c2 = 0, c3 = 0, d0 = 0, d1 = 0, d2 = 0, d3 = 0;
                    const uint32_t o = k0 * 4;
    #define TM_DPRE(B, g)                                                                                        \
        precheck4x2<B, kImad>(c0, c1, c2, c3, xa, lds128(pxa + o + 16 * (g)), ya, lds128(pya + o + 16 * (g)), p.one); \
        precheck4x2<B, kImad>(d0, d1, d2, d3, xb, lds128(pxb + o + 16 * (g)), yb, lds128(pyb + o + 16 * (g)), p.one)
                    const uint32_t left = nq - k0;
                    TM_DPRE(1u << 0, 0);
                    if (left > 4) { TM_DPRE(1u << 4, 1); }
                    if (left > 8) { TM_DPRE(1u << 8, 2); }
                    if (left > 12) { TM_DPRE(1u << 12, 3); }
                    if (left > 16) { TM_DPRE(1u << 16, 4); }
                    if (left > 20) { TM_DPRE(1u << 20, 5); }
                    if (left > 24) { TM_DPRE(1u << 24, 6); }
                    if (left > 28) { TM_DPRE(1u << 28, 7); }
    #undef TM_DPRE
                    const uint32_t qmask = left >= 32 ? ~0u : ((1u << left) - 1u);
                    uint32_t acc_a = va ? ((c0 | c1) | (c2 | c3)) & qmask : 0u;
                    uint32_t acc_b = vb ? ((d0 | d1) | (d2 | d3)) & qmask : 0u;
                    // Alg. 3 on the pairs that passed: all six words, then emit (keys fused, S7)
                    while (__any_sync(0xffffffffu, (acc_a | acc_b) != 0)) {
                        bool m = false;
                        uint32_t j = 0, row = ra;
                        if (acc_a | acc_b) {
                            const bool isb = acc_a == 0;
                            uint32_t &acc = isb ? acc_b : acc_a;
                            j = k0 + (uint32_t)(__ffs(acc) - 1);
                            acc &= acc - 1;
                            row = isb ? rb : ra;
                            const uint64_t s0 = isb ? b0 : a0, s1 = isb ? b1 : a1, s2 = isb ? b2 : a2;
                            m = (((uint32_t)s0 & ~sm.dp[0][j]) | ((uint32_t)(s0 >> 32) & ~sm.dp[1][j]) |
                                 ((uint32_t)s1 & ~sm.dp[2][j]) | ((uint32_t)(s1 >> 32) & ~sm.dp[3][j]) |
                                 ((uint32_t)s2 & ~sm.dp[4][j]) | ((uint32_t)(s2 >> 32) & ~sm.dp[5][j])) == 0;
                        }
                        const uint32_t bm = __ballot_sync(0xffffffffu, m);
                        if (bm) {
                            st_matched += __popc(bm);
                            emit_keys<kFused>(m, bm, row, m ? __ldg(sm.qid + j) : 0u, p, lane, sm.pend[warp], npend);
                        }
                    }
                }
            st_checks += nq * (vend > u0 ? min((uint32_t)kDenseRows, vend - u0) : 0u);
        };
        // BULK: the warp's reserved units in issue order (stage of ring0 = si, ring1 = si + 1, ...);
        // rotated by value so no array is indexed dynamically (no local memory)
        static_assert(kDenseStages == 3, "the ring below is written for three stages");
        uint32_t ring0 = 0, ring1 = 0, ring2 = 0;
        if constexpr (BULK) {
            ring0 = take();
            if (ring0 < nunit) issue(0, ring0);
            ring1 = take();
            if (ring1 < nunit) issue(1, ring1);
            ring2 = take();
            if (ring2 < nunit) issue(2, ring2);
        }
        uint32_t si = 0;
        for (;;) {
            if constexpr (BULK) {
                const uint32_t u = ring0;
                if (u >= nunit) break;  // later reservations are larger: nothing is in flight
                while (!mbar_try_wait(&sm.bar[warp][si], (par >> si) & 1u)) {
                }
                par ^= 1u << si;
                const uint64_t *st = sm.stage[warp][si];
                ulonglong2 v0 = *reinterpret_cast<const ulonglong2 *>(st + 2 * lane);
                ulonglong2 v1 = *reinterpret_cast<const ulonglong2 *>(st + kDenseRows + 2 * lane);
                ulonglong2 v2 = *reinterpret_cast<const ulonglong2 *>(st + 2 * kDenseRows + 2 * lane);
                uint32_t wab = *reinterpret_cast<const unsigned short *>(&sm.wstage[warp][si][2 * lane]);
                if (rlo + u * kDenseRows + 2 * (uint32_t)lane >= rhi) {  // past a 32-row unit: stale stage bytes
                    v0 = v1 = v2 = make_ulonglong2(~0ULL, ~0ULL);
                    wab = 0x1010u;
                }
                __syncwarp();  // every lane has read the stage: refill it now
                const uint32_t nu = take();
                if (nu < nunit) issue(si, nu);
                ring0 = ring1;
                ring1 = ring2;
                ring2 = nu;
                si = si == kDenseStages - 1 ? 0 : si + 1;
                check_pair(v0, v1, v2, wab, rlo + u * kDenseRows, make_uint4(0u, 0u, 0u, 0u));
            } else if constexpr (kRows4) {
                const uint32_t u = take();
                if (u >= nunit) break;
                const uint32_t u0 = rlo + u * kUnitRows;
                ulonglong2 v0, v1, v2, y0, y1, y2;
                uint32_t wab, wcd;
                uint4 wwa, wwc;
                load_pair(u0 + 2 * (uint32_t)lane, v0, v1, v2, wab, wwa);  // 96 B per lane in flight
                load_pair(u0 + kDenseRows + 2 * (uint32_t)lane, y0, y1, y2, wcd, wwc);
                check_pair(v0, v1, v2, wab, u0, wwa);
                check_pair(y0, y1, y2, wcd, u0 + kDenseRows, wwc);
            } else {
                const uint32_t u = take();
                if (u >= nunit) break;
                ulonglong2 v0, v1, v2;
                uint32_t wab;
                uint4 ww;
                load_pair(rlo + u * kDenseRows + 2 * (uint32_t)lane, v0, v1, v2, wab, ww);
                check_pair(v0, v1, v2, wab, rlo + u * kDenseRows, ww);
            }
        }
        __syncthreads();
    }
    flush_pend<kFused>(sm.pend[warp], npend, p, lane);
    if (lane == 0 && (st_checks | st_matched)) {
        atomicAdd(&sm.cnt[1], (unsigned long long)st_checks);
        atomicAdd(&sm.cnt[2], (unsigned long long)st_matched);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (sm.cnt[1]) atomicAdd(&p.ctr->pair_checks, sm.cnt[1]);
        if (sm.cnt[2]) atomicAdd(&p.ctr->matched_sets, sm.cnt[2]);
    }
}

// ------------------------------------------------------------------ S8 ---
__global__ void k_split(const uint64_t *__restrict__ pairs, uint64_t n, uint32_t *__restrict__ q,
                        uint32_t *__restrict__ k) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t v = pairs[i];
    q[i] = (uint32_t)(v >> 32);
    k[i] = (uint32_t)v;
}

// q_off[i] = base + first index of query qlo + i in the sorted (q<<32 | key) pairs (lower bound),
// one thread per query of the range; q_off[nq] = base + n.
__global__ void k_query_offsets(const uint64_t *__restrict__ pairs, uint64_t n, uint64_t qlo, uint64_t nq,
                                uint64_t base, uint64_t *__restrict__ q_off) {
    const uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (j > nq) return;
    if (j == nq) {
        q_off[nq] = base + n;
        return;
    }
    const uint64_t key = (qlo + j) << 32;
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (__ldg(pairs + mid) < key) lo = mid + 1; else hi = mid;
    }
    q_off[j] = base + lo;
}

// ---------------------------------------------------------------- build ---
__global__ void k_gather_planes(const uint64_t *__restrict__ s0, const uint64_t *__restrict__ s1,
                                const uint64_t *__restrict__ s2, const uint32_t *__restrict__ idx, uint64_t n,
                                uint64_t *__restrict__ d0, uint64_t *__restrict__ d1, uint64_t *__restrict__ d2) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t j = idx[i];
    d0[i] = s0[j];
    d1[i] = s1[j];
    d2[i] = s2[j];
}

__global__ void k_gather_u64(const uint64_t *__restrict__ s, const uint32_t *__restrict__ idx, uint64_t n,
                             uint64_t *__restrict__ d) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) d[i] = s[idx[i]];
}

__global__ void k_iota(uint32_t *v, uint64_t n) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) v[i] = (uint32_t)i;
}

// Per row: which two of its six 32-bit words (w = 2 * block + half, half 1 = the high 32
// bits) have the most one-bits outside its tile's AND mask -- the words the WORD1 pre-check
// tests (low nibble: the best, high nibble: the second; ties: lowest w).  Any choice is
// lossless; this one makes the pre-check most selective.
__global__ void k_word_select(const uint64_t *__restrict__ w0, const uint64_t *__restrict__ w1,
                              const uint64_t *__restrict__ w2, const uint64_t *__restrict__ t0,
                              const uint64_t *__restrict__ t1, const uint64_t *__restrict__ t2, uint64_t rows,
                              uint8_t *__restrict__ wsel, uint2 *__restrict__ wwords) {
    uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (r >= rows) return;
    const uint64_t t = r / kTile;
    const uint64_t x[3] = {w0[r] & ~t0[t], w1[r] & ~t1[t], w2[r] & ~t2[t]};
    int best = 0, bc = -1, second = 1, sc = -1;
#pragma unroll
    for (int w = 0; w < 6; ++w) {
        const int c = __popc((uint32_t)(x[w >> 1] >> (32 * (w & 1))));
        if (c > bc) {
            second = best;
            sc = bc;
            bc = c;
            best = w;
        } else if (c > sc) {
            sc = c;
            second = w;
        }
    }
    wsel[r] = (uint8_t)(best | (second << 4));
    // the two words themselves (the lean scan reads them instead of selecting them per tile)
    const uint64_t v[3] = {w0[r], w1[r], w2[r]};
    wwords[r] = make_uint2((uint32_t)(v[best >> 1] >> (32 * (best & 1))), (uint32_t)(v[second >> 1] >> (32 * (second & 1))));
}

struct WidenAt {
    const uint32_t *v;
    uint64_t n;
    __device__ unsigned long long operator()(const uint64_t &i) const {
        return i < n ? (unsigned long long)v[i] : 0ULL;
    }
};

}  // namespace

// ------------------------------------------------------------ launchers ---
cudaError_t launch_hash_vocab(const uint8_t *bytes, const uint64_t *off, const uint64_t *hashes, uint64_t n_vocab,
                              uint64_t n_bytes, uint64_t *vsig, unsigned int *err, cudaStream_t s) {
    if (!n_vocab) return cudaSuccess;
    k_hash_vocab<<<grid_for(n_vocab, 256), 256, 0, s>>>(bytes, off, hashes, n_vocab, n_bytes, vsig, err);
    return cudaGetLastError();
}

cudaError_t launch_encode_sets(const uint64_t *vsig, const uint32_t *tag_idx, const uint64_t *set_off,
                               uint64_t n_sets, uint64_t n_tags, uint64_t n_vocab, uint64_t *w0, uint64_t *w1,
                               uint64_t *w2, unsigned int *err, cudaStream_t s) {
    if (!n_sets) return cudaSuccess;
    k_encode_sets<<<grid_for(n_sets, 256), 256, 0, s>>>(vsig, tag_idx, set_off, n_sets, n_tags, n_vocab, w0, w1, w2,
                                                         err);
    return cudaGetLastError();
}

uint64_t route_blocks(uint64_t n_q) { return (n_q + kRouteBlockQ - 1) / kRouteBlockQ; }

cudaError_t launch_route(int pass, const uint64_t *masks, uint32_t n_parts, const uint64_t *q0, const uint64_t *q1,
                         const uint64_t *q2, uint64_t n_q, uint32_t *counts, const unsigned long long *off,
                         uint32_t *qidx, unsigned long long cap, cudaStream_t s, uint32_t qbase) {
    const uint64_t nb = route_blocks(n_q);
    if (!nb || !n_parts) return cudaSuccess;
    const size_t smem = (size_t)kRouteWarps * 192 * kRouteWB * 4;  // 36 KB: within the default dynamic limit
    static_assert((size_t)kRouteWarps * 192 * kRouteWB * 4 <= 48 * 1024, "route Z needs the opt-in attribute");
    auto f = pass == 0 ? k_route<0> : k_route<1>;
    // enough warps to fill the GPU (~16 per SM) even for small batches: slice the partitions
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t groups = (n_parts + 31) / 32;
    const uint64_t want = (uint64_t)std::max(sms, 1) * 16;
    const uint32_t slices = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(groups, (want + nb - 1) / nb));
    f<<<grid_for(nb * slices, kRouteWarps), kRouteWarps * 32, smem, s>>>(masks, n_parts, q0, q1, q2, n_q, nb, counts,
                                                                         off, qidx, cap, qbase, slices);
    return cudaGetLastError();
}

cudaError_t launch_items(const unsigned long long *word_off, uint64_t qw, const uint32_t *part_row,
                         const uint32_t *part_n, uint32_t n_parts, unsigned long long *qoff,
                         unsigned long long *item_cnt, DevCounters *ctr, uint32_t range_rows, cudaStream_t s) {
    k_items<<<grid_for((uint64_t)n_parts + 1, 256), 256, 0, s>>>(word_off, qw, part_row, part_n, n_parts, qoff,
                                                                 item_cnt, ctr, range_rows);
    return cudaGetLastError();
}

namespace {
using ScanFn = void (*)(const ScanParams);
// FUSED: the same kernel with the fused-exchange emission (OPT bit 6), launched when
// ScanParams.n_owners > 1 (in-process partitioned groups); the local-output kernels stay untouched
template <int F>
ScanFn scan_fn_t(int variant) {
    // variants 1-4 of round 1 (8 survivors per iteration, all three blocks in the main loop, pair
    // unions) never won a tuning class and were removed in round 2; their numbers stay unused
    switch (variant) {
        case 0: return k_scan<false, 8, false, F>;  // no word pre-check: 4 survivors per iteration, blocks 0-1 first
        // 72 registers and 7 CTAs/SM, no spills: 2.00 ms at C2 vs 2.10 ms with 64 registers and
        // 8 CTAs (spills) and 2.05 ms with 76 registers and 6 CTAs (profiles/r1v29_minb.txt)
        case 5: return k_scan<true, 7, false, F>;
        case 6: return k_scan<false, 8, true, F>;   // streaming only, direct check
        case 7: return k_scan<true, 8, true, F>;    // streaming only, word pre-check
        case 8: return k_scan<true, 7, false, 1 | F>;  // 5 + pre-check accumulate on the FMA pipe
        case 9: return k_dense<false, 1 | F>;   // unfiltered dense scan, direct loads, FMA-pipe accumulate
        case 10: return k_dense<true, 1 | F>;   // unfiltered dense scan, bulk-copy (TMA) staged rows
        case 11: return k_dense<false, 0 | F>;
        case 12: return k_dense<true, 0 | F>;
        case 13: return k_dense<false, 5 | F>;  // 9 with four rows per lane
        case 14: return k_scan<true, 7, false, 17 | F>;  // 8 + lean tile set-up (the default)
        case 15: return k_dense<false, 21 | F>;  // 13 + the build-time pre-check words (no selects)
        case 16: return k_scan<true, 7, false, 17 | 512 | F>;  // 14 + pre-check pass statistics (diagnostic)
        case 17: return k_scan<true, 7, false, 17 | F, 4>;  // 14 with 128-row level-A blocks
        case 18: return k_scan<true, 7, false, 1 | F, 4>;   // 8 with 128-row level-A blocks
        default: return nullptr;
    }
}

ScanFn scan_fn(int variant, bool fused = false) { return fused ? scan_fn_t<64>(variant) : scan_fn_t<0>(variant); }
}  // namespace

size_t scan_smem(int variant) {
    if (variant == 9 || variant == 11 || variant == 13 || variant == 15) return sizeof(DenseSmemBase);

    if (variant == 10 || variant == 12) return sizeof(DenseSmemBulk);
    return (variant == 6 || variant == 7) ? sizeof(StreamSmem) : sizeof(ScanSmem);
}

int scan_variant_env() {
    // TM_SCAN_VARIANT forces a scan-kernel variant: 0 = no word pre-check;
    // 5 = per-lane two-word pre-check (WORD1); 8 = 5 + FMA-pipe accumulate; 14 = 8 + lean tile
    // set-up (default); 6 / 7 = streaming-only kernels (direct check / word pre-check; calls of
    // <= kSmallBatch queries, else mapped to 0 / 5 by the caller); 9-13, 15 = the dense
    // (unfiltered) scan (9 two rows per lane, 13 four, 10 / 12 bulk-copy staged, 11 / 12 without
    // the FMA accumulate, 15 = 13 with build-time pre-check words; 16 = 14 printing pre-check pass
    // statistics, a diagnostic; 17 / 18 = 14 / 8 with 128-row level-A blocks).  Unset or unknown (-1): the
    // handle tunes on its first calls.
    const char *e = getenv("TM_SCAN_VARIANT");
    if (!e) return -1;
    const int v = atoi(e);
    return (v >= 0 && v < kScanVariants && scan_fn(v)) ? v : -1;
}

uint32_t range_rows_env(uint64_t n_rows) {
    // measured (scripts/gpu_rangerows.sh): C2 (1M rows) 8192 ~ 4096 > 16384; C3 (100M rows)
    // 32768 is 3% faster than 8192 (fewer item barriers; still 450K items for 1184 CTAs)
    const uint32_t def = n_rows >= (1ULL << 24) ? 32768u : (uint32_t)kRangeRows;
    const char *e = getenv("TM_RANGE_ROWS");
    if (!e) return def;
    const long v = atol(e);
    // at most 2^20 rows: one item then decides < 2^32 pairs (the kernel's 32-bit per-item statistics)
    return (v >= 256 && v <= (1L << 20) && v % 256 == 0) ? (uint32_t)v : def;
}

uint32_t unit_target_env() {
    const char *e = getenv("TM_UNIT_TARGET");
    const long v = e ? atol(e) : 0;
    return (v >= 1 && v <= 64) ? (uint32_t)v : kUnitTarget;  // 8: +1% at C3 over 4 (profiles/r2j_ab_*)
}

int scan_grid(int device, int variant) {
    int sms = 0, per = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    ScanFn f = scan_fn(variant);
    if (!f) return 0;  // unused variant number
    cudaFuncSetAttribute(scan_fn(variant, true), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)scan_smem(variant));
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)scan_smem(variant));
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, f, kScanWarps * 32, scan_smem(variant));
    if (per < 1) per = 1;
    if (sms < 1) sms = 1;
    return sms * per;
}

void scan_debug_dump(int variant) {
    // variant 16 (diagnostic): print and reset the pre-check pass statistics of the last scan
    if (variant != 16) return;
    unsigned long long h[12] = {}, z[12] = {};
    if (cudaMemcpyFromSymbol(h, g_scan_dbg, sizeof h) != cudaSuccess) return;
    cudaMemcpyToSymbol(g_scan_dbg, z, sizeof z);
    fprintf(stderr, "scan_dbg passes %llu groups %llu iters(sum max) %llu hist[0,1,2,3-4,5-8,9-16,17-32] %llu %llu %llu %llu %llu %llu %llu heavy_passes %llu lanes_with_pass %llu\n",
            h[0], h[1], h[2], h[3], h[4], h[5], h[6], h[7], h[8], h[9], h[10], h[11]);
}

cudaError_t launch_scan(const ScanParams &p, int grid, cudaStream_t s, int variant) {
    scan_fn(variant, p.n_owners > 1)<<<grid, kScanWarps * 32, scan_smem(variant), s>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_word_select(const uint64_t *planes, const uint64_t *tand, uint64_t rows, uint8_t *wsel,
                               uint2 *wwords, cudaStream_t s) {
    if (!rows) return cudaSuccess;
    const uint64_t nt = rows / kTile;
    k_word_select<<<grid_for(rows, 256), 256, 0, s>>>(planes, planes + rows, planes + 2 * rows, tand, tand + nt,
                                                      tand + 2 * nt, rows, wsel, wwords);
    return cudaGetLastError();
}

cudaError_t launch_query_offsets(const uint64_t *pairs, uint64_t n, uint64_t qlo, uint64_t nq, uint64_t base,
                                 uint64_t *q_off, cudaStream_t s) {
    k_query_offsets<<<grid_for(nq + 1, 256), 256, 0, s>>>(pairs, n, qlo, nq, base, q_off);
    return cudaGetLastError();
}

cudaError_t launch_split(const uint64_t *pairs, uint64_t n, uint32_t *q, uint32_t *k, cudaStream_t s) {
    if (!n) return cudaSuccess;
    k_split<<<grid_for(n, 256), 256, 0, s>>>(pairs, n, q, k);
    return cudaGetLastError();
}

cudaError_t launch_gather_planes(const uint64_t *src0, const uint64_t *src1, const uint64_t *src2,
                                 const uint32_t *idx, uint64_t n, uint64_t *d0, uint64_t *d1, uint64_t *d2,
                                 cudaStream_t s) {
    if (!n) return cudaSuccess;
    k_gather_planes<<<grid_for(n, 256), 256, 0, s>>>(src0, src1, src2, idx, n, d0, d1, d2);
    return cudaGetLastError();
}

cudaError_t launch_gather_u64(const uint64_t *src, const uint32_t *idx, uint64_t n, uint64_t *dst,
                              cudaStream_t s) {
    if (!n) return cudaSuccess;
    k_gather_u64<<<grid_for(n, 256), 256, 0, s>>>(src, idx, n, dst);
    return cudaGetLastError();
}

cudaError_t launch_iota(uint32_t *v, uint64_t n, cudaStream_t s) {
    if (!n) return cudaSuccess;
    k_iota<<<grid_for(n, 256), 256, 0, s>>>(v, n);
    return cudaGetLastError();
}

// ----------------------------------------------------------------- CUB ---
cudaError_t cub_exclusive_scan_u32_u64(const uint32_t *in, unsigned long long *out, uint64_t n, void *tmp,
                                      size_t *tmp_bytes, cudaStream_t s) {
    // out[0..n] = exclusive prefix of in[0..n) widened to 64 bits; out[n] = total
    cub::CountingInputIterator<uint64_t> cnt(0);
    cub::TransformInputIterator<unsigned long long, WidenAt, cub::CountingInputIterator<uint64_t>> it(cnt,
                                                                                                     WidenAt{in, n});
    return cub::DeviceScan::ExclusiveSum(tmp, *tmp_bytes, it, out, (int64_t)(n + 1), s);
}

cudaError_t cub_exclusive_scan_u64(const unsigned long long *in, unsigned long long *out, uint64_t n, void *tmp,
                                   size_t *tmp_bytes, cudaStream_t s) {
    return cub::DeviceScan::ExclusiveSum(tmp, *tmp_bytes, in, out, (int64_t)n, s);
}

cudaError_t cub_sort_pairs_u64_u32(const uint64_t *kin, uint64_t *kout, const uint32_t *vin, uint32_t *vout,
                                   uint64_t n, void *tmp, size_t *tmp_bytes, cudaStream_t s) {
    return cub::DeviceRadixSort::SortPairs(tmp, *tmp_bytes, kin, kout, vin, vout, (int64_t)n, 0, 64, s);
}

cudaError_t cub_sort_keys_u64(uint64_t *k, uint64_t *kalt, uint64_t n, int end_bit, int *sel, void *tmp,
                              size_t *tmp_bytes, cudaStream_t s) {
    cub::DoubleBuffer<uint64_t> db(k, kalt);
    cudaError_t e = cub::DeviceRadixSort::SortKeys(tmp, *tmp_bytes, db, (int64_t)n, 0, end_bit, s);
    if (sel) *sel = db.selector;
    return e;
}

cudaError_t cub_unique_u64(const uint64_t *in, uint64_t *out, unsigned long long *n_out, uint64_t n, void *tmp,
                           size_t *tmp_bytes, cudaStream_t s) {
    return cub::DeviceSelect::Unique(tmp, *tmp_bytes, in, out, n_out, (int64_t)n, s);
}

}  // namespace tmb
