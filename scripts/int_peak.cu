// int_peak.cu -- INT/logic-pipe peak of this B200 ("64/clk is the CUDA-guide
// value ... must be measured on sm_100a by our microbenchmark").  The denominator of the scan
// kernel's ALU roofline (bench.py roofline.peak).
//
// Kernels (every thread runs 8 independent dependency chains so latency is hidden; a grid of
// 148 x 8 CTAs x 256 threads fills every SM):
//   lop3     : x_i = lop3(x_i, y, z)                      -- ALU pipe only (LOP3)
//   lop3_imad: x_i = lop3(...) ; w_i = w_i * a + b (IMAD)  -- ALU and FMA pipes in parallel
//   precheck : the scan's pre-check step per (row, survivor): LOP3 s = b & ~u; LOP3 with a
//              predicate r = (a & ~v) | s; @p OR acc, bit   -- 3 ALU ops
//   precheck_imad: the same with the predicated OR as an IMAD (acc += bit), FMA pipe
// ops/clk/SM = thread-ops / (SM cycles x SMs); cycles from clock64() inside the kernel.
// Output: one JSON line.  Usage: int_peak [iters]
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#define CK(x)                                                                       \
    do {                                                                            \
        cudaError_t e_ = (x);                                                       \
        if (e_ != cudaSuccess) {                                                    \
            fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
            exit(1);                                                                \
        }                                                                           \
    } while (0)

__device__ __forceinline__ uint32_t lop3_xor(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d;
    asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}

__device__ __forceinline__ uint32_t imad(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d;
    asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}

__global__ void k_lop3(uint32_t y, uint32_t z, int iters, uint32_t *out, long long *cyc) {
    uint32_t x[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x * 8 + i;
    const long long c0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 16; ++r)
#pragma unroll
            for (int i = 0; i < 8; ++i) x[i] = lop3_xor(x[i], y, z + r);
    }
    const long long c1 = clock64();
    uint32_t a = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) a ^= x[i];
    if (a == 0x12345678u) out[blockIdx.x] = a;
    if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
}

__global__ void k_lop3_imad(uint32_t y, uint32_t z, int iters, uint32_t *out, long long *cyc) {
    uint32_t x[4], w[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        x[i] = threadIdx.x * 8 + i;
        w[i] = threadIdx.x * 8 + 4 + i;
    }
    const long long c0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 16; ++r)
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                x[i] = lop3_xor(x[i], y, z + r);
                w[i] = imad(w[i], y, z + r);
            }
    }
    const long long c1 = clock64();
    uint32_t a = 0;
#pragma unroll
    for (int i = 0; i < 4; ++i) a ^= x[i] ^ w[i];
    if (a == 0x12345678u) out[blockIdx.x] = a;
    if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
}

// One pre-check step of 4 survivors (the scan's precheck4x2): 3 ALU ops per survivor.
template <bool IMAD>
__global__ void k_precheck(uint32_t y, uint32_t z, int iters, uint32_t *out, long long *cyc) {
    uint32_t a = threadIdx.x * 0x9e3779b9u, b = a ^ y;
    const uint32_t one = y & 1u;  // 1 at run time (y odd), opaque to ptxas: keeps the IMAD an IMAD
    uint32_t c[4] = {0, 0, 0, 0};
    uint32_t v[4], u[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        v[i] = y * (i + 1);
        u[i] = z * (i + 3);
    }
    const long long c0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 16; ++r) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                uint32_t s, t;
                asm volatile("lop3.b32 %0, %1, %2, 0, 0x30;" : "=r"(s) : "r"(b), "r"(u[i]));  // b & ~u
                if (IMAD) {
                    asm volatile(
                        "{\n\t.reg .pred p;\n\t"
                        "lop3.b32 %1, %2, %3, %4, 0xf2;\n\t"  // (a & ~v) | s
                        "setp.eq.u32 p, %1, 0;\n\t"
                        "@p mad.lo.u32 %0, %5, %6, %0;\n\t}"
                        : "+r"(c[i]), "=r"(t) : "r"(a), "r"(v[i]), "r"(s), "r"(1u << r), "r"(one));
                } else {
                    asm volatile(
                        "{\n\t.reg .pred p;\n\t"
                        "lop3.b32 %1, %2, %3, %4, 0xf2;\n\t"
                        "setp.eq.u32 p, %1, 0;\n\t"
                        "@p or.b32 %0, %0, %5;\n\t}"
                        : "+r"(c[i]), "=r"(t) : "r"(a), "r"(v[i]), "r"(s), "r"(1u << r));
                }
                v[i] += 0x3c6ef372u;  // vary the survivor words (not counted: IADD / IMAD)
            }
        }
    }
    const long long c1 = clock64();
    const uint32_t acc = c[0] ^ c[1] ^ c[2] ^ c[3];
    if (acc == 0x12345678u) out[blockIdx.x] = acc;
    if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
}

int main(int argc, char **argv) {
    const int iters = argc > 1 ? atoi(argv[1]) : 4096;
    int dev = 0, sms = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, dev));
    const int threads = 256, per_sm = 8, grid = sms * per_sm;
    uint32_t *out;
    long long *cyc;
    CK(cudaMalloc(&out, grid * 4));
    CK(cudaMalloc(&cyc, grid * 8));
    long long *hc = (long long *)malloc(grid * 8);
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    printf("{\"gpu\": \"%s\", \"sms\": %d, \"threads\": %d, \"ctas\": %d, \"iters\": %d", prop.name, sms, threads,
           grid, iters);
    struct K {
        const char *name;
        void (*f)(uint32_t, uint32_t, int, uint32_t *, long long *);
        double ops_per_iter;  // counted thread-ops per loop iteration
        const char *what;
    } ks[] = {
        {"lop3", k_lop3, 16 * 8, "LOP3 (ALU pipe)"},
        {"lop3_imad", k_lop3_imad, 16 * 8, "LOP3 + IMAD 1:1 (ALU + FMA pipes)"},
        {"precheck_alu", k_precheck<false>, 16 * 4 * 3, "pre-check step, 3 ALU ops per survivor"},
        {"precheck_imad", k_precheck<true>, 16 * 4 * 3, "pre-check step, predicated OR as IMAD"},
    };
    for (const K &k : ks) {
        double best = 0, best_clk = 0, best_mhz = 0;
        for (int rep = 0; rep < 5; ++rep) {
            CK(cudaEventRecord(e0));
            k.f<<<grid, threads>>>(0x5bd1e995u, 0x27d4eb2fu, iters, out, cyc);
            CK(cudaEventRecord(e1));
            CK(cudaEventSynchronize(e1));
            CK(cudaGetLastError());
            float ms = 0;
            CK(cudaEventElapsedTime(&ms, e0, e1));
            CK(cudaMemcpy(hc, cyc, grid * 8, cudaMemcpyDeviceToHost));
            long long cmax = 0;
            for (int i = 0; i < grid; ++i)
                if (hc[i] > cmax) cmax = hc[i];
            const double ops = (double)grid * threads * iters * k.ops_per_iter;
            const double tops = ops / (ms * 1e-3) / 1e12;
            // per_sm CTAs run concurrently on one SM; cmax = the longest CTA's SM cycles
            const double per_clk = ops / ((double)cmax * sms);
            if (tops > best) {
                best = tops;
                best_clk = per_clk;
                best_mhz = (double)cmax / (ms * 1e3);
            }
        }
        printf(", \"%s\": {\"tops\": %.3f, \"ops_per_clk_per_sm\": %.2f, \"sm_mhz_est\": %.0f, \"what\": \"%s\"}", k.name,
               best, best_clk, best_mhz, k.what);
    }
    printf("}\n");
    return 0;
}
