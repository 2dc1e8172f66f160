// tc_probe.cu -- standalone probe of the tcgen05 kind::i8 path used by
// csrc/contract_tc.cu: one CTA, A (128 x 32 u8) and B (N x 32 u8) written in
// the K-major no-swizzle core-matrix layout, one MMA, commit to an mbarrier
// (bounded wait), TMEM -> registers, compare with a host GEMM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/tc_probe tools/tc_probe.cu
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

typedef uint32_t u32;
typedef unsigned long long u64;

__device__ __forceinline__ u32 smem_u32(const void *p) { return (u32)__cvta_generic_to_shared(p); }

__device__ __forceinline__ u64 desc(u32 saddr, int lbo, int sbo) {
    return (u64)((saddr >> 4) & 0x3FFFu) | ((u64)(lbo >> 4) << 16) | ((u64)(sbo >> 4) << 32) | (1ull << 46);
}

// A: 128 rows, B: N rows, K = 32 bytes; layout per tile: [row/8][kchunk(2)][row%8][16]
__global__ void probe(const uint8_t *A, const uint8_t *B, int N, int lbo_mode, u32 *D, int *status) {
    __shared__ __align__(1024) uint8_t sa[128 * 32];
    __shared__ __align__(1024) uint8_t sb[256 * 32];
    __shared__ u32 s_taddr;
    __shared__ __align__(8) u64 mbar;
    const int tid = threadIdx.x;
    if (lbo_mode < 2) {
        // K-major: SBO = 256 (an 8-row group holds 2 K chunks of 128 B), LBO = 128
        for (int i = tid; i < 128 * 32; i += blockDim.x) {
            const int r = i / 32, k = i % 32;
            sa[(r >> 3) * 256 + (k >> 4) * 128 + (r & 7) * 16 + (k & 15)] = A[i];
        }
        for (int i = tid; i < N * 32; i += blockDim.x) {
            const int r = i / 32, k = i % 32;
            sb[(r >> 3) * 256 + (k >> 4) * 128 + (r & 7) * 16 + (k & 15)] = B[i];
        }
    } else {
        // MN-major: core matrix = 16 MN-contiguous bytes x 8 K rows (128 B);
        // MN chunks 128 B apart, 8-row K groups (M/16)*128 B apart
        for (int i = tid; i < 128 * 32; i += blockDim.x) {
            const int m = i / 32, k = i % 32;
            sa[(k >> 3) * (128 / 16) * 128 + (m >> 4) * 128 + (k & 7) * 16 + (m & 15)] = A[i];
        }
        for (int i = tid; i < N * 32; i += blockDim.x) {
            const int m = i / 32, k = i % 32;
            sb[(k >> 3) * (N / 16) * 128 + (m >> 4) * 128 + (k & 7) * 16 + (m & 15)] = B[i];
        }
    }
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" :: "r"(smem_u32(&s_taddr)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&mbar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const u32 taddr = s_taddr;
    if (tid == 0) {
        u32 idesc = (2u << 4) | ((u32)(N >> 3) << 17) | ((128u >> 4) << 24);
        u64 da, db;
        if (lbo_mode < 2) {
            const int lbo = lbo_mode ? 128 : 256, sbo = lbo_mode ? 256 : 128;   // mode 0: fields swapped
            da = desc(smem_u32(sa), lbo, sbo); db = desc(smem_u32(sb), lbo, sbo);
        } else {
            idesc |= (1u << 15) | (1u << 16);                                   // A, B MN-major
            // mode 2: LBO = K-group stride, SBO = MN-chunk stride; mode 3: swapped
            const int ka = (128 / 16) * 128, kb = (N / 16) * 128;
            if (lbo_mode == 2) { da = desc(smem_u32(sa), ka, 128); db = desc(smem_u32(sb), kb, 128); }
            else { da = desc(smem_u32(sa), 128, ka); db = desc(smem_u32(sb), 128, kb); }
        }
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                     :: "r"(taddr), "l"(da), "l"(db), "r"(idesc), "r"(0u));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(smem_u32(&mbar)));
    }
    u32 ok = 0;
    for (long it = 0; it < (1L << 24) && !ok; ++it)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                     : "=r"(ok) : "r"(smem_u32(&mbar)), "r"(0u) : "memory");
    if (!ok) { if (tid == 0) *status = 2; }
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (ok && tid < 128) {
        const int warp = tid >> 5;
        for (int c0 = 0; c0 < N; c0 += 4) {
            u32 v0, v1, v2, v3;
            asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(v0), "=r"(v1), "=r"(v2), "=r"(v3) : "r"(taddr + ((u32)(32 * warp) << 16) + (u32)c0));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            D[tid * N + c0] = v0; D[tid * N + c0 + 1] = v1; D[tid * N + c0 + 2] = v2; D[tid * N + c0 + 3] = v3;
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" :: "r"(taddr));
    if (tid == 0 && ok) *status = 1;
}

int main() {
    for (int N : {96, 256, 16}) {
        for (int lbo_mode : {1, 2, 3}) {
            std::vector<uint8_t> A(128 * 32), B(N * 32);
            srand(N + lbo_mode);
            for (auto &x : A) x = rand() & 255;
            for (auto &x : B) x = rand() & 255;
            uint8_t *dA, *dB; u32 *dD; int *dS;
            cudaMalloc(&dA, A.size()); cudaMalloc(&dB, B.size());
            cudaMalloc(&dD, 128 * N * 4); cudaMalloc(&dS, 4);
            cudaMemcpy(dA, A.data(), A.size(), cudaMemcpyHostToDevice);
            cudaMemcpy(dB, B.data(), B.size(), cudaMemcpyHostToDevice);
            cudaMemset(dD, 0, 128 * N * 4); cudaMemset(dS, 0, 4);
            probe<<<1, 128>>>(dA, dB, N, lbo_mode, dD, dS);
            cudaError_t e = cudaDeviceSynchronize();
            std::vector<u32> D(128 * N);
            int st = 0;
            cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
            cudaMemcpy(&st, dS, 4, cudaMemcpyDeviceToHost);
            long bad = 0, first = -1;
            for (int m = 0; m < 128; ++m)
                for (int n = 0; n < N; ++n) {
                    u32 ref = 0;
                    for (int k = 0; k < 32; ++k) ref += (u32)A[m * 32 + k] * B[n * 32 + k];
                    if (ref != D[m * N + n]) { if (first < 0) first = m * N + n; ++bad; }
                }
            printf("N=%d mode=%d err=%s status=%d mismatches=%ld first=%ld", N, lbo_mode,
                   cudaGetErrorString(e), st, bad, first);
            if (first >= 0) {
                const int m = first / N, n = first % N;
                u32 ref = 0;
                for (int k = 0; k < 32; ++k) ref += (u32)A[m * 32 + k] * B[n * 32 + k];
                printf(" (m=%d n=%d got=%u want=%u)", m, n, D[first], ref);
            }
            printf("\n");
            fflush(stdout);
            if (e != cudaSuccess) return 1;
        }
    }
    return 0;
}
