// coresid_probe.cu -- can a light integer kernel share the SMs with the
// limb-quad tensor-core contraction (k_contract_tq, ~204 KB of shared memory
// and 6 warps per SM)?  Times the contraction alone, a spin kernel alone
// (3 x 256-thread blocks per SM, 64 registers, no memory traffic) and both on
// two streams; if they co-reside the pair takes ~max, not the sum.  Also
// prints the spin kernel's start time relative to the contraction's end.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/coresid tools/coresid_probe.cu \
//        -Lpaper_conf_icde_lixylz24_b200 -l:libup.so -Xlinker -rpath=$PWD/paper_conf_icde_lixylz24_b200
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

extern "C" cudaError_t upk_launch_contract_tq(const uint32_t *A, long long lda, int La, const uint32_t *B, long long ldb,
                                              int Lb, long long n, int sign, unsigned long long *ws, uint32_t *ticket,
                                              uint32_t *result, int LA, int num_sms, cudaStream_t st);

__global__ void __launch_bounds__(256, 4) spin(long long iters, unsigned *out, unsigned long long *t0) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        *t0 = t;
    }
    unsigned a = threadIdx.x, b = blockIdx.x;
    for (long long i = 0; i < iters; ++i) { a = a * 1664525u + b; b ^= a >> 7; }
    if (a == 0x12345678u) out[0] = b;
}

__global__ void stamp(unsigned long long *t) { asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(*t)); }

int main() {
    const long long n = 12500000;
    const int L = 21, G = 6;
    const long long ld = (n + 3) & ~3ll;
    uint32_t *A, *B, *res, *ticket;
    unsigned long long *ws, *tt;
    unsigned *o;
    cudaMalloc(&A, (size_t)G * ld * 16);
    cudaMalloc(&B, (size_t)G * ld * 16);
    cudaMemset(A, 1, (size_t)G * ld * 16);
    cudaMemset(B, 2, (size_t)G * ld * 16);
    cudaMalloc(&ws, 8 * 4096); cudaMemset(ws, 0, 8 * 4096);
    cudaMalloc(&ticket, 64); cudaMemset(ticket, 0, 64);
    cudaMalloc(&res, 4 * 64);
    cudaMalloc(&o, 64);
    cudaMalloc(&tt, 64);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaFuncSetAttribute(spin, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaStream_t s1, s2;
    cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto tc = [&](cudaStream_t s) { upk_launch_contract_tq(A, ld, L, B, ld, L, n, 1, ws, ticket, res, 43, sms, s); };
    const long long iters = 20000;
    auto sp = [&](cudaStream_t s) { spin<<<3 * sms, 256, 0, s>>>(iters, o, tt); };
    float ms;
    for (int w = 0; w < 3; ++w) { tc(s1); sp(s2); }
    cudaDeviceSynchronize();
    cudaEventRecord(e0, s1); for (int r = 0; r < 10; ++r) tc(s1); cudaEventRecord(e1, s1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1); printf("tc alone     %.4f ms\n", ms / 10);
    cudaEventRecord(e0, s2); for (int r = 0; r < 10; ++r) sp(s2); cudaEventRecord(e1, s2); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1); printf("spin alone   %.4f ms\n", ms / 10);
    for (int order = 0; order < 2; ++order) {
        cudaDeviceSynchronize();
        cudaEventRecord(e0, s1);
        cudaStreamWaitEvent(s2, e0, 0);
        for (int r = 0; r < 10; ++r) {
            if (order == 0) { tc(s1); sp(s2); } else { sp(s2); tc(s1); }
            cudaEvent_t j; cudaEventCreateWithFlags(&j, cudaEventDisableTiming);
            cudaEventRecord(j, s2); cudaStreamWaitEvent(s1, j, 0);
            cudaEventRecord(j, s1); cudaStreamWaitEvent(s2, j, 0);
            cudaEventDestroy(j);
        }
        cudaEventRecord(e1, s1); cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1); printf("both (%s first) %.4f ms\n", order ? "spin" : "tc", ms / 10);
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
