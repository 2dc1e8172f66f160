// kernels.cu -- static (nvcc, sm_100a) kernels of libup: column codec (row a3
// ingestion / row a12 read-back) and the exact multi-rank combine (row a13).
#include <cuda_runtime.h>
#include <stdint.h>

#include "up_dev.cuh"

using up::u32;
using up::u64;

namespace {

// sign-magnitude rows (n x W words, neg bytes) -> L two's-complement planes.
// One thread per row; planes written coalesced.  |mag| >= 10^p sets F_RANGE
// (bound = 10^p in L limbs, a DECIMAL(p,s) holds |m| < 10^p, Eq. 1).
__global__ void __launch_bounds__(256) k_from_bin(const u32 *__restrict__ mag, int W, const uint8_t *__restrict__ neg,
                                                  long long n, const u32 *__restrict__ bound, int L,
                                                  u32 *__restrict__ out, long long ld, u32 *flags) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    u32 fl = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const u32 *m = mag + i * W;
        // range check, most significant limb first
        int cmp = 0;   // -1: m < bound, +1: m >= bound decided
        for (int j = (W > L ? W : L) - 1; j >= 0 && cmp == 0; --j) {
            const u32 a = j < W ? m[j] : 0u, b = j < L ? bound[j] : 0u;
            if (a != b) cmp = a < b ? -1 : 1;
        }
        if (cmp >= 0) fl |= up::F_RANGE;
        const u32 ng = (neg && neg[i]) ? 1u : 0u;
        const u32 mask = 0u - ng;
        u64 carry = ng;
        for (int j = 0; j < L; ++j) {
            const u64 t = (u64)((j < W ? m[j] : 0u) ^ mask) + carry;
            out[(long long)j * ld + i] = (u32)t;
            carry = t >> 32;
        }
    }
    if (fl) atomicOr(flags, fl);
}

// L two's-complement planes -> sign-magnitude rows (n x L words, neg bytes)
__global__ void __launch_bounds__(256) k_to_bin(const u32 *__restrict__ planes, int L, long long ld, long long n,
                                                u32 *__restrict__ mag, uint8_t *__restrict__ neg) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const u32 ng = planes[(long long)(L - 1) * ld + i] >> 31;
        const u32 mask = 0u - ng;
        u64 carry = ng;
        for (int j = 0; j < L; ++j) {
            const u64 t = (u64)(planes[(long long)j * ld + i] ^ mask) + carry;
            mag[i * L + j] = (u32)t;
            carry = t >> 32;
        }
        neg[i] = (uint8_t)ng;
    }
}

// limb planes -> limb quads (up.h UP_LAYOUT_QUADS): quad g of row i =
// limbs 4g..4g+3 as one uint4 at q[g*ldq + i]; limb L = the sign flag (1 for a
// negative row), the limbs above it 0.  One thread per (row, quad): 16-byte
// stores coalesced across the warp.
__global__ void __launch_bounds__(256) k_planes_to_quads(const u32 *__restrict__ planes, int L, long long ld,
                                                         long long n, uint4 *__restrict__ q, long long ldq) {
    const int G = (L + 1 + 3) / 4;
    const long long total = n * G, stride = (long long)gridDim.x * blockDim.x;
    for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
        const long long i = t % n;
        const int g = (int)(t / n);
        u32 w[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const int j = 4 * g + k;
            w[k] = j < L ? planes[(long long)j * ld + i] : j == L ? planes[(long long)(L - 1) * ld + i] >> 31 : 0u;
        }
        q[(long long)g * ldq + i] = make_uint4(w[0], w[1], w[2], w[3]);
    }
}

// limb quads -> limb planes (the flag and padding limbs are dropped)
__global__ void __launch_bounds__(256) k_quads_to_planes(const uint4 *__restrict__ q, long long ldq, int L, long long n,
                                                         u32 *__restrict__ planes, long long ld) {
    const int G = (L + 3) / 4;   // quads holding value limbs
    const long long total = n * G, stride = (long long)gridDim.x * blockDim.x;
    for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
        const long long i = t % n;
        const int g = (int)(t / n);
        const uint4 v = q[(long long)g * ldq + i];
        const u32 w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int k = 0; k < 4; ++k)
            if (4 * g + k < L) planes[(long long)(4 * g + k) * ld + i] = w[k];
    }
}

// out = sum of nranks la-limb two's-complement partials, mod 2^(32 la), in
// rank order (exact; order only matters for readability -- integer sums
// commute).  One block: limb-parallel 64-bit column sums, then one carry pass.
__global__ void __launch_bounds__(1024) k_combine(const u32 *__restrict__ parts, int nranks, int la,
                                                  u32 *__restrict__ out) {
    extern __shared__ u64 col[];
    for (int j = threadIdx.x; j < la; j += blockDim.x) {
        u64 t = 0;
        for (int r = 0; r < nranks; ++r) t += parts[(long long)r * la + j];
        col[j] = t;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        u64 carry = 0;
        for (int j = 0; j < la; ++j) {
            const u64 t = (col[j] & 0xffffffffull) + carry;
            out[j] = (u32)t;
            carry = (t >> 32) + (col[j] >> 32);
        }
    }
}

// Split-SUM combine: out = sum of the partials, partial `scaled` multiplied by
// the unsigned constant scale[0..nsc) first (two's complement mod 2^(32 la):
// exact).  Column j: 64-bit sums of the low and high halves of its products,
// then one carry pass.
__global__ void __launch_bounds__(1024) k_combine_scaled(const u32 *__restrict__ parts, int nparts, int la, int scaled,
                                                         const u32 *__restrict__ scale, int nsc, u32 *__restrict__ out) {
    extern __shared__ u64 col[];
    u64 *hi = col + la;
    const u32 *sp = parts + (long long)scaled * la;
    for (int j = threadIdx.x; j < la; j += blockDim.x) {
        u64 lo = 0, h = 0;
        for (int r = 0; r < nparts; ++r)
            if (r != scaled) lo += parts[(long long)r * la + j];
        for (int m = 0; m < nsc && m <= j; ++m) {
            const u64 pr = (u64)sp[j - m] * scale[m];
            lo += (u32)pr;
            h += pr >> 32;
        }
        col[j] = lo;
        hi[j] = h;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        u64 carry = 0;
        for (int j = 0; j < la; ++j) {
            // value at limb j: lo[j] + hi[j] 2^32 (+ carry from below)
            const u64 t = (col[j] & 0xffffffffull) + carry;
            out[j] = (u32)t;
            carry = (t >> 32) + (col[j] >> 32) + hi[j];
        }
    }
}

// Compact byte-aligned rows (the paper's cDecimal, P:L843-873 / Fig. 4):
// Lb bytes per row, little-endian magnitude, the sign in the top bit of the
// last byte.  A block stages its 256 contiguous records with 32-bit loads
// (256*Lb is a multiple of 4), then each thread assembles its row's limbs.
__global__ void __launch_bounds__(256) k_from_compact(const uint8_t *__restrict__ bytes, int Lb, long long n,
                                                      const u32 *__restrict__ bound, int L, u32 *__restrict__ out,
                                                      long long ld, u32 *flags) {
    extern __shared__ u32 stage[];
    const uint8_t *sb = reinterpret_cast<const uint8_t *>(stage);
    u32 fl = 0;
    for (long long base = (long long)blockIdx.x * 256; base < n; base += (long long)gridDim.x * 256) {
        const long long rows = n - base < 256 ? n - base : 256;
        const long long nbytes = rows * Lb;
        const uint8_t *src = bytes + base * Lb;
        __syncthreads();
        if ((reinterpret_cast<uintptr_t>(src) & 3) == 0) {
            const u32 *src4 = reinterpret_cast<const u32 *>(src);
            for (long long w = threadIdx.x; w < nbytes / 4; w += blockDim.x) stage[w] = __ldcs(src4 + w);
            for (long long b = (nbytes / 4) * 4 + threadIdx.x; b < nbytes; b += blockDim.x)
                reinterpret_cast<uint8_t *>(stage)[b] = src[b];
        } else {
            for (long long b = threadIdx.x; b < nbytes; b += blockDim.x) reinterpret_cast<uint8_t *>(stage)[b] = src[b];
        }
        __syncthreads();
        if (threadIdx.x < rows) {
            const uint8_t *rb = sb + threadIdx.x * Lb;
            const u32 ng = rb[Lb - 1] >> 7;
            const u32 mask = 0u - ng;
            // range: |m| < 10^p, compared limb-wise from the top
            int cmp = 0;
            for (int j = L - 1; j >= 0 && cmp == 0; --j) {
                u32 m = 0;
                for (int b = 0; b < 4; ++b) {
                    const int k = 4 * j + b;
                    u32 v = k < Lb ? rb[k] : 0u;
                    if (k == Lb - 1) v &= 0x7Fu;
                    m |= v << (8 * b);
                }
                if (m != bound[j]) cmp = m < bound[j] ? -1 : 1;
            }
            if (cmp >= 0) fl |= up::F_RANGE;
            u64 carry = ng;
            const long long i = base + threadIdx.x;
            for (int j = 0; out && j < L; ++j) {   // out == nullptr: range check only (compact-resident column)
                u32 m = 0;
                for (int b = 0; b < 4; ++b) {
                    const int k = 4 * j + b;
                    u32 v = k < Lb ? rb[k] : 0u;
                    if (k == Lb - 1) v &= 0x7Fu;
                    m |= v << (8 * b);
                }
                const u64 t = (u64)(m ^ mask) + carry;
                out[(long long)j * ld + i] = (u32)t;
                carry = t >> 32;
            }
        }
    }
    if (fl) atomicOr(flags, fl);
}

// L two's-complement planes -> compact rows (Lb bytes, sign in the top bit)
__global__ void __launch_bounds__(256) k_to_compact(const u32 *__restrict__ planes, int L, long long ld, long long n,
                                                    uint8_t *__restrict__ bytes, int Lb) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const u32 ng = planes[(long long)(L - 1) * ld + i] >> 31;
        const u32 mask = 0u - ng;
        u64 carry = ng;
        uint8_t *rb = bytes + i * Lb;
        for (int j = 0; j < L; ++j) {
            const u64 t = (u64)(planes[(long long)j * ld + i] ^ mask) + carry;
            carry = t >> 32;
            const u32 m = (u32)t;
            for (int b = 0; b < 4; ++b) {
                const int k = 4 * j + b;
                if (k < Lb) rb[k] = (uint8_t)(m >> (8 * b));
            }
        }
        rb[Lb - 1] = (uint8_t)((rb[Lb - 1] & 0x7Fu) | (ng << 7));
    }
}

// Multi-rank combine of grouped aggregates (NEXT-4; aggregate typing
// P:L1069-1080).  parts: nranks x part_words u32, each rank's output of
// up_group_aggregate run with AVG replaced by SUM (its partial state); counts:
// nranks x G row counts.  One thread per (aggregate, group):
//   SUM  -- exact two's-complement sum over ranks;
//   MIN / MAX -- signed multi-limb min / max over the ranks whose group is non-empty;
//   AVG  -- trunc(|SUM| 10^4 / COUNT) sign(SUM) of the combined SUM and COUNT
//           (reading Q4 truncation; COUNT 0 -> 0).
struct AggDesc {
    int kind, Lp, Lr, pad;
    long long poff, roff;
};
__global__ void __launch_bounds__(128) k_group_combine(const u32 *__restrict__ parts, int nranks, long long part_words,
                                                       const unsigned long long *__restrict__ counts, int G, int n_aggs,
                                                       const AggDesc *__restrict__ d, u32 *__restrict__ out,
                                                       unsigned long long *__restrict__ counts_out) {
    const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (t < G && counts_out) {
        unsigned long long c = 0;
        for (int r = 0; r < nranks; ++r) c += counts[(long long)r * G + t];
        counts_out[t] = c;
    }
    if (t >= (long long)G * n_aggs) return;
    const int a = (int)(t / G), g = (int)(t % G);
    const AggDesc ad = d[a];
    u32 *o = out + ad.roff + (long long)g * ad.Lr;
    unsigned long long cnt = 0;
    for (int r = 0; r < nranks; ++r) cnt += counts[(long long)r * G + g];
    if (ad.kind == 1 || ad.kind == 2) {   // MIN / MAX over non-empty ranks
        int best = -1;
        for (int r = 0; r < nranks; ++r) {
            if (counts[(long long)r * G + g] == 0) continue;
            if (best < 0) { best = r; continue; }
            const u32 *x = parts + (long long)r * part_words + ad.poff + (long long)g * ad.Lp;
            const u32 *y = parts + (long long)best * part_words + ad.poff + (long long)g * ad.Lp;
            int cmp = 0;   // signed compare x vs y
            if ((int)x[ad.Lp - 1] != (int)y[ad.Lp - 1]) cmp = (int)x[ad.Lp - 1] < (int)y[ad.Lp - 1] ? -1 : 1;
            for (int j = ad.Lp - 2; j >= 0 && cmp == 0; --j)
                if (x[j] != y[j]) cmp = x[j] < y[j] ? -1 : 1;
            if ((ad.kind == 1 && cmp < 0) || (ad.kind == 2 && cmp > 0)) best = r;
        }
        for (int j = 0; j < ad.Lr; ++j)
            o[j] = best < 0 ? 0u : parts[(long long)best * part_words + ad.poff + (long long)g * ad.Lp + (j < ad.Lp ? j : ad.Lp - 1)];
        return;
    }
    // SUM over ranks (Lp limbs, two's complement), kept in up to 80 limbs
    constexpr int MAXL = 80;
    u32 acc[MAXL];
    const int L = ad.Lp < MAXL ? ad.Lp : MAXL;
    for (int j = 0; j < L; ++j) acc[j] = 0u;
    for (int r = 0; r < nranks; ++r) {
        const u32 *x = parts + (long long)r * part_words + ad.poff + (long long)g * ad.Lp;
        u64 c = 0;
        for (int j = 0; j < L; ++j) {
            const u64 v = (u64)acc[j] + x[j] + c;
            acc[j] = (u32)v;
            c = v >> 32;
        }
    }
    if (ad.kind == 0) {
        for (int j = 0; j < ad.Lr; ++j) o[j] = j < L ? acc[j] : ((acc[L - 1] >> 31) ? 0xFFFFFFFFu : 0u);
        return;
    }
    // AVG: |S| 10^4 / COUNT, truncated, with the sign of S
    const u32 ng = acc[L - 1] >> 31;
    u32 mag[MAXL + 1];
    {
        u64 c = ng;
        for (int j = 0; j < L; ++j) {
            const u64 v = (u64)(acc[j] ^ (0u - ng)) + c;
            mag[j] = (u32)v;
            c = v >> 32;
        }
        u64 m = 0;   // x 10^4
        for (int j = 0; j < L; ++j) {
            const u64 v = (u64)mag[j] * 10000u + m;
            mag[j] = (u32)v;
            m = v >> 32;
        }
        mag[L] = (u32)m;
    }
    if (cnt == 0) {
        for (int j = 0; j < ad.Lr; ++j) o[j] = 0u;
        return;
    }
    unsigned __int128 rem = 0;
    for (int j = L; j >= 0; --j) {
        const unsigned __int128 cur = (rem << 32) | mag[j];
        mag[j] = (u32)(cur / cnt);
        rem = cur % cnt;
    }
    u64 c = ng;
    for (int j = 0; j < ad.Lr; ++j) {
        const u64 v = (u64)((j <= L ? mag[j] : 0u) ^ (0u - ng)) + c;
        o[j] = (u32)v;
        c = v >> 32;
    }
}

int grid_for(long long n, int threads) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    long long want = (n + threads - 1) / threads;
    long long cap = (long long)sms * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

}  // namespace

extern "C" {

cudaError_t upk_launch_from_bin(const uint32_t *mag, int W, const uint8_t *neg, long long n, const uint32_t *bound,
                                int L, uint32_t *out, long long ld, uint32_t *flags, cudaStream_t st) {
    k_from_bin<<<grid_for(n, 256), 256, 0, st>>>(mag, W, neg, n, bound, L, out, ld, flags);
    return cudaGetLastError();
}

cudaError_t upk_launch_to_bin(const uint32_t *planes, int L, long long ld, long long n, uint32_t *mag, uint8_t *neg,
                              cudaStream_t st) {
    k_to_bin<<<grid_for(n, 256), 256, 0, st>>>(planes, L, ld, n, mag, neg);
    return cudaGetLastError();
}

cudaError_t upk_launch_from_compact(const uint8_t *bytes, int Lb, long long n, const uint32_t *bound, int L,
                                   uint32_t *out, long long ld, uint32_t *flags, cudaStream_t st) {
    const size_t smem = (size_t)256 * Lb + 16;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(k_from_compact, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    long long want = (n + 255) / 256, cap = (long long)sms * 8;
    k_from_compact<<<(int)(want < 1 ? 1 : (want < cap ? want : cap)), 256, smem, st>>>(bytes, Lb, n, bound, L, out, ld,
                                                                                  flags);
    return cudaGetLastError();
}

cudaError_t upk_launch_to_compact(const uint32_t *planes, int L, long long ld, long long n, uint8_t *bytes, int Lb,
                                 cudaStream_t st) {
    k_to_compact<<<grid_for(n, 256), 256, 0, st>>>(planes, L, ld, n, bytes, Lb);
    return cudaGetLastError();
}

cudaError_t upk_launch_planes_to_quads(const uint32_t *planes, int L, long long ld, long long n, uint32_t *quads,
                                      long long ldq, cudaStream_t st) {
    k_planes_to_quads<<<grid_for(n * ((L + 4) / 4), 256), 256, 0, st>>>(planes, L, ld, n, (uint4 *)quads, ldq);
    return cudaGetLastError();
}

cudaError_t upk_launch_quads_to_planes(const uint32_t *quads, long long ldq, int L, long long n, uint32_t *planes,
                                      long long ld, cudaStream_t st) {
    k_quads_to_planes<<<grid_for(n * ((L + 3) / 4), 256), 256, 0, st>>>((const uint4 *)quads, ldq, L, n, planes, ld);
    return cudaGetLastError();
}

cudaError_t upk_launch_group_combine(const uint32_t *parts, int nranks, long long part_words,
                                     const unsigned long long *counts, int G, int n_aggs, const void *d_descs,
                                     uint32_t *out, unsigned long long *counts_out, cudaStream_t st) {
    const long long nt = (long long)G * n_aggs > G ? (long long)G * n_aggs : G;
    k_group_combine<<<(int)((nt + 127) / 128), 128, 0, st>>>(parts, nranks, part_words, counts, G, n_aggs,
                                                             (const AggDesc *)d_descs, out, counts_out);
    return cudaGetLastError();
}

cudaError_t upk_launch_combine(const uint32_t *partials, int nranks, int la, uint32_t *out, cudaStream_t st) {
    const size_t smem = sizeof(u64) * (size_t)la;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(k_combine, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    k_combine<<<1, 1024, smem, st>>>(partials, nranks, la, out);
    return cudaGetLastError();
}

cudaError_t upk_launch_combine_scaled(const uint32_t *partials, int nparts, int la, uint32_t *out, int scaled,
                                      const uint32_t *scale, int nsc, cudaStream_t st) {
    const size_t smem = 2 * sizeof(u64) * (size_t)la;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(k_combine_scaled, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
    }
    k_combine_scaled<<<1, 1024, smem, st>>>(partials, nparts, la, scaled, scale, nsc, out);
    return cudaGetLastError();
}

}  // extern "C"
