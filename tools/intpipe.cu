// intpipe.cu -- measured integer-pipe peaks on the B200 (the denominators for
// the "alu" roofline of the compute-bound configs).  Each kernel runs 8
// independent dependency chains per thread of one PTX op (asm volatile so
// nothing is folded), full occupancy, grid = 8 x SMs blocks of 256 threads.
// Prints one JSON object: per op, lanes (thread-ops) per clock per SM and
// ops/s for the whole GPU.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o intpipe tools/intpipe.cu && ./intpipe
#include <cstdio>
#include <cuda_runtime.h>

#define ITERS 4096

#define CHAIN8(OP)                                                                  \
    OP(a0) OP(a1) OP(a2) OP(a3) OP(a4) OP(a5) OP(a6) OP(a7)

__global__ void k_imad(unsigned *out, unsigned m, unsigned c) {
    unsigned a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
#define OP(x) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x) : "r"(m), "r"(c));
    for (int i = 0; i < ITERS; ++i) { CHAIN8(OP) }
#undef OP
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 ^ a1 ^ a2 ^ a3 ^ a4 ^ a5 ^ a6 ^ a7;
}
__global__ void k_imadhi(unsigned *out, unsigned m, unsigned c) {
    unsigned a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
#define OP(x) asm volatile("mad.hi.u32 %0, %0, %1, %2;" : "+r"(x) : "r"(m), "r"(c));
    for (int i = 0; i < ITERS; ++i) { CHAIN8(OP) }
#undef OP
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 ^ a1 ^ a2 ^ a3 ^ a4 ^ a5 ^ a6 ^ a7;
}
__global__ void k_iadd3(unsigned *out, unsigned m, unsigned c) {
    unsigned a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
#define OP(x) asm volatile("add.u32 %0, %0, %1;\n\tadd.u32 %0, %0, %2;" : "+r"(x) : "r"(m), "r"(c));
    for (int i = 0; i < ITERS; ++i) { CHAIN8(OP) }
#undef OP
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 ^ a1 ^ a2 ^ a3 ^ a4 ^ a5 ^ a6 ^ a7;
}
__global__ void k_imadwide(unsigned *out, unsigned m, unsigned c) {
    // acc_i = b_i * m + acc_i (64-bit accumulate of 32x32 products): the
    // pattern of a radix-2^31 product-scanning multiply
    unsigned long long a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6,
                       a7 = a0 + 7;
    unsigned b0 = c ^ threadIdx.x, b1 = b0 * 3, b2 = b0 * 5, b3 = b0 * 7, b4 = b0 * 9, b5 = b0 * 11, b6 = b0 * 13,
             b7 = b0 * 15;
#define OPW(x, b) asm volatile("mad.wide.u32 %0, %1, %2, %0;" : "+l"(x) : "r"(b), "r"(m));
    for (int i = 0; i < ITERS; ++i) {
        OPW(a0, b0) OPW(a1, b1) OPW(a2, b2) OPW(a3, b3) OPW(a4, b4) OPW(a5, b5) OPW(a6, b6) OPW(a7, b7)
        b0 += (unsigned)a0; b1 += (unsigned)a1; b2 += (unsigned)a2; b3 += (unsigned)a3;
        b4 += (unsigned)a4; b5 += (unsigned)a5; b6 += (unsigned)a6; b7 += (unsigned)a7;
    }
#undef OPW
    unsigned long long x = a0 ^ a1 ^ a2 ^ a3 ^ a4 ^ a5 ^ a6 ^ a7;
    out[blockIdx.x * blockDim.x + threadIdx.x] = (unsigned)x ^ (unsigned)(x >> 32);
}
// one limb product of an operand-scanning row as libup emits it:
// mad.lo.cc / madc.hi.cc pairs on a running 4-word window
__global__ void k_rowmac(unsigned *out, unsigned m, unsigned c) {
    unsigned r0 = threadIdx.x, r1 = r0 + 1, r2 = r0 + 2, r3 = r0 + 3, b0 = m, b1 = m ^ 7, b2 = m + 3, b3 = m * 5;
    unsigned a = c + threadIdx.x;
    for (int i = 0; i < ITERS / 2; ++i) {
        asm volatile(
            "mad.lo.cc.u32 %0, %4, %5, %0;\n\t"
            "madc.lo.cc.u32 %1, %4, %6, %1;\n\t"
            "madc.lo.cc.u32 %2, %4, %7, %2;\n\t"
            "madc.lo.cc.u32 %3, %4, %8, %3;\n\t"
            "mad.hi.cc.u32 %1, %4, %5, %1;\n\t"
            "madc.hi.cc.u32 %2, %4, %6, %2;\n\t"
            "madc.hi.cc.u32 %3, %4, %7, %3;\n\t"
            "madc.hi.u32 %0, %4, %8, %0;\n\t"
            : "+r"(r0), "+r"(r1), "+r"(r2), "+r"(r3)
            : "r"(a), "r"(b0), "r"(b1), "r"(b2), "r"(b3));
        a += r3;
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = r0 ^ r1 ^ r2 ^ r3;
}

// 32x32->64 products: one mul.wide per step vs a mul.lo + mul.hi pair
__global__ void k_mulwide(unsigned *out, unsigned m, unsigned c) {
    unsigned a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
#define OP(x) { unsigned long long r; asm volatile("mul.wide.u32 %0, %1, %2;" : "=l"(r) : "r"(x), "r"(m)); \
                x = (unsigned)r ^ (unsigned)(r >> 32); }
    for (int i = 0; i < ITERS; ++i) { CHAIN8(OP) }
#undef OP
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 ^ a1 ^ a2 ^ a3 ^ a4 ^ a5 ^ a6 ^ a7;
}
__global__ void k_mullohi(unsigned *out, unsigned m, unsigned c) {
    unsigned a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
#define OP(x) { unsigned lo, hi; asm volatile("mul.lo.u32 %0, %2, %3;\n\tmul.hi.u32 %1, %2, %3;" : "=r"(lo), "=r"(hi) : "r"(x), "r"(m)); \
                x = lo ^ hi; }
    for (int i = 0; i < ITERS; ++i) { CHAIN8(OP) }
#undef OP
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 ^ a1 ^ a2 ^ a3 ^ a4 ^ a5 ^ a6 ^ a7;
}

template <typename K>
double run(K kern, const char *name, double ops_per_thread, int sms, double &lanes_per_clk_sm, double &clk_ghz) {
    unsigned *out;
    int blocks = sms * 8, threads = 256;
    cudaMalloc(&out, sizeof(unsigned) * blocks * threads);
    kern<<<blocks, threads>>>(out, 0x9E3779B9u, 12345u);
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(e0);
        kern<<<blocks, threads>>>(out, 0x9E3779B9u, 12345u + rep);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    int khz = 0;
    cudaDeviceGetAttribute(&khz, cudaDevAttrClockRate, 0);
    clk_ghz = khz / 1e6;
    double ops = ops_per_thread * blocks * threads;
    double ops_s = ops / (best / 1e3);
    lanes_per_clk_sm = ops_s / (sms * clk_ghz * 1e9);
    cudaFree(out);
    return ops_s;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double l, g;
    printf("{\"sms\": %d", sms);
    double v;
    v = run(k_imad, "imad", 8.0 * ITERS, sms, l, g);
    printf(", \"imad\": {\"ops_per_s\": %.4e, \"lanes_per_clk_sm_at_max_clock\": %.2f}", v, l);
    v = run(k_imadhi, "imad_hi", 8.0 * ITERS, sms, l, g);
    printf(", \"imad_hi\": {\"ops_per_s\": %.4e, \"lanes_per_clk_sm_at_max_clock\": %.2f}", v, l);
    v = run(k_imadwide, "imad_wide", 8.0 * ITERS, sms, l, g);
    printf(", \"imad_wide\": {\"ops_per_s\": %.4e, \"lanes_per_clk_sm_at_max_clock\": %.2f}", v, l);
    v = run(k_iadd3, "iadd", 16.0 * ITERS, sms, l, g);
    printf(", \"iadd\": {\"ops_per_s\": %.4e, \"lanes_per_clk_sm_at_max_clock\": %.2f}", v, l);
    v = run(k_rowmac, "row_mac", 8.0 * (ITERS / 2), sms, l, g);
    printf(", \"mad_cc_chain\": {\"ops_per_s\": %.4e, \"lanes_per_clk_sm_at_max_clock\": %.2f, \"note\": \"PTX mad.lo/hi.cc ops (2 per limb product)\"}", v, l);
    v = run(k_mulwide, "mul_wide", 8.0 * ITERS, sms, l, g);
    printf(", \"mul_wide_products\": {\"ops_per_s\": %.4e, \"lanes_per_clk_sm_at_max_clock\": %.2f}", v, l);
    v = run(k_mullohi, "mul_lohi", 8.0 * ITERS, sms, l, g);
    printf(", \"mul_lo_hi_products\": {\"ops_per_s\": %.4e, \"lanes_per_clk_sm_at_max_clock\": %.2f}", v, l);
    printf(", \"clock_ghz_attr\": %.3f}\n", g);
    return 0;
}
