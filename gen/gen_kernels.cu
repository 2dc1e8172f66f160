// gen_kernels.cu -- device twin of gen/synth.py's counter-based generator
// (INPUT GENERATION ONLY: holds none of the method's arithmetic).  Built into
// gen/libupgen.so; bit-identical to synth.uniform_range() by construction
// (same SplitMix64 finaliser, same counter layout, same rejection order).
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}

__device__ __forceinline__ uint32_t word(uint64_t key, uint64_t row, uint32_t att, uint32_t j) {
    const uint64_t ctr = (row << 32) | (uint64_t)((att << 10) | j);
    return (uint32_t)(mix64(key ^ mix64(ctr)) & 0xffffffffull);
}

constexpr int kMaxW = 128;

__global__ void __launch_bounds__(256) k_uniform(uint64_t key, long long row0, long long n, int W, uint32_t topmask,
                                                 const uint32_t *__restrict__ lo, const uint32_t *__restrict__ hi,
                                                 int is_signed, uint32_t *__restrict__ mag, uint8_t *__restrict__ neg,
                                                 unsigned int *fail) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const uint64_t row = (uint64_t)(row0 + i);
        bool done = false;
        for (uint32_t att = 0; att < 4096 && !done; ++att) {
            // compare candidate with lo and hi, most significant word first
            int cl = 0, ch = 0;   // sign of (cand - lo), (cand - hi) once decided
            for (int j = W - 1; j >= 0; --j) {
                uint32_t w = word(key, row, att, (uint32_t)j);
                if (j == W - 1) w &= topmask;
                if (cl == 0 && w != lo[j]) cl = w > lo[j] ? 1 : -1;
                if (ch == 0 && w != hi[j]) ch = w > hi[j] ? 1 : -1;
            }
            if (cl >= 0 && ch <= 0) {
                for (int j = 0; j < W; ++j) {
                    uint32_t w = word(key, row, att, (uint32_t)j);
                    if (j == W - 1) w &= topmask;
                    mag[i * W + j] = w;
                }
                neg[i] = is_signed ? (uint8_t)(word(key, row, att, (uint32_t)W) & 1u) : (uint8_t)0;
                done = true;
            }
        }
        if (!done) atomicAdd(fail, 1u);
    }
}

}  // namespace

extern "C" int upgen_uniform(uint64_t key, long long row0, long long n, int W, uint32_t topmask, const uint32_t *d_lo,
                             const uint32_t *d_hi, int is_signed, uint32_t *d_mag, uint8_t *d_neg,
                             unsigned int *d_fail, void *stream) {
    if (W < 1 || W > kMaxW || n < 0) return 1;
    if (n == 0) return 0;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    long long want = (n + 255) / 256, cap = (long long)sms * 16;
    int grid = (int)(want < cap ? want : cap);
    k_uniform<<<grid, 256, 0, (cudaStream_t)stream>>>(key, row0, n, W, topmask, d_lo, d_hi, is_signed, d_mag, d_neg,
                                                       d_fail);
    return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
