// groupby.cu -- GROUP BY on DECIMAL key columns:
// the paper sorts with DECIMAL comparison operators to group (P:L730-734,
// Sec. II-C).  Here the comparison is folded into a stable LSD radix sort over
// the keys' two's-complement limb planes (least significant key column and
// limb first; the top limb of each key has its sign bit flipped so unsigned
// order equals signed order), after which equal keys are adjacent: one pass
// marks the first row of every run by comparing all key limbs with the
// previous sorted row, a prefix sum numbers the runs, and a scatter writes the
// dense id back to each row.  The radix sort and the scans are written here
// (no CUB): per 8-bit digit a tile histogram, an exclusive scan of the
// digit-major counts, and a stable scatter whose in-tile ranks come from
// warp match masks (__match_any_sync) and per-warp digit counts.
#include <cuda_runtime.h>

#include <mutex>
#include <string>

#include "../../include/up.h"

up_status up_internal_fail(up_status st, const std::string &msg);
void up_internal_add_launches(up_ctx *c, long long k);
up_status up_internal_scratch(up_ctx *c, size_t bytes, void **out);
std::mutex &up_internal_mutex(up_ctx *c);

namespace {

constexpr int kMaxKeyPlanes = 64;

struct KeyPlanes {
    const uint32_t *p[kMaxKeyPlanes];
    int np;
};

__global__ void k_gb_iota(uint32_t *perm, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        perm[i] = (uint32_t)i;
}

// key[i] = plane[perm[i]] (sign bit flipped for the top limb of a key column)
__global__ void k_gb_gather(const uint32_t *__restrict__ plane, const uint32_t *__restrict__ perm,
                            uint32_t *__restrict__ key, long long n, uint32_t flip) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        key[i] = plane[perm[i]] ^ flip;
}

// most significant pass: excluded rows (negative id) sort last
__global__ void k_gb_gather_excl(const int32_t *__restrict__ ids, const uint32_t *__restrict__ perm,
                                 uint32_t *__restrict__ key, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        key[i] = ids[perm[i]] < 0 ? 1u : 0u;
}

// head[i] = 1 iff sorted row i is included and its key differs from row i-1's
// (all key limbs compared: DECIMAL equality of every key column)
__global__ void k_gb_heads(const KeyPlanes kp, const int32_t *__restrict__ ids, const uint32_t *__restrict__ perm,
                           uint32_t *__restrict__ head, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const uint32_t r = perm[i];
        uint32_t h = 0;
        if (ids[r] >= 0) {
            if (i == 0) {
                h = 1;
            } else {
                const uint32_t q = perm[i - 1];   // included too: excluded rows are sorted last
                for (int j = 0; j < kp.np; ++j) h |= kp.p[j][r] != kp.p[j][q];
            }
        }
        head[i] = h;
    }
}

__global__ void k_gb_scatter(const uint32_t *__restrict__ perm, const uint32_t *__restrict__ head,
                             const uint32_t *__restrict__ gid, int32_t *__restrict__ ids, long long *__restrict__ first,
                             long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const uint32_t r = perm[i];
        if (ids[r] < 0) continue;
        const uint32_t g = gid[i] - 1u;
        ids[r] = (int32_t)g;
        if (first && head[i]) first[g] = (long long)r;   // stable sort from row order: smallest row of the group
    }
}

// ------------------------------------------------------------------ radix sort
constexpr int RS_THREADS = 256, RS_ROUNDS = 16, RS_TILE = RS_THREADS * RS_ROUNDS, RADIX = 256;
constexpr int SCAN_CHUNK = 4096;

// cnt[d * nt + t] = rows of tile t whose digit (key >> shift) & 255 is d
__global__ void __launch_bounds__(RS_THREADS) k_rs_hist(const uint32_t *__restrict__ key, long long n, int shift,
                                                         uint32_t *__restrict__ cnt, long long nt) {
    __shared__ uint32_t h[RADIX];
    for (long long t = blockIdx.x; t < nt; t += gridDim.x) {
        h[threadIdx.x] = 0u;
        __syncthreads();
        const long long b0 = t * RS_TILE;
        for (int r = 0; r < RS_ROUNDS; ++r) {
            const long long i = b0 + (long long)r * RS_THREADS + threadIdx.x;
            if (i < n) atomicAdd(&h[(key[i] >> shift) & 255u], 1u);
        }
        __syncthreads();
        cnt[(long long)threadIdx.x * nt + t] = h[threadIdx.x];
        __syncthreads();
    }
}

// stable scatter of one 8-bit digit: rows keep their input order within a
// digit (tile offsets from the scanned counts, ranks inside a tile by rounds
// of 256 rows: warp peers by __match_any_sync, lower warps by per-warp counts)
__global__ void __launch_bounds__(RS_THREADS) k_rs_scatter(const uint32_t *__restrict__ kin, const uint32_t *__restrict__ vin,
                                                            uint32_t *__restrict__ kout, uint32_t *__restrict__ vout,
                                                            long long n, int shift, const uint32_t *__restrict__ off,
                                                            long long nt) {
    __shared__ uint32_t run[RADIX];
    __shared__ uint32_t wc[RS_THREADS / 32][RADIX];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const uint32_t lt = (1u << lane) - 1u;
    for (long long t = blockIdx.x; t < nt; t += gridDim.x) {
        run[tid] = off[(long long)tid * nt + t];
        const long long b0 = t * RS_TILE;
        for (int r = 0; r < RS_ROUNDS; ++r) {
            for (int w = 0; w < RS_THREADS / 32; ++w) wc[w][tid] = 0u;
            __syncthreads();
            const long long i = b0 + (long long)r * RS_THREADS + tid;
            const bool valid = i < n;
            const uint32_t k = valid ? kin[i] : 0u;
            const uint32_t d = valid ? (k >> shift) & 255u : 256u;
            const uint32_t peers = __match_any_sync(0xFFFFFFFFu, d);
            if (valid && (peers & lt) == 0u) wc[warp][d] = __popc(peers);
            __syncthreads();
            if (valid) {
                uint32_t pos = run[d] + __popc(peers & lt);
                for (int w = 0; w < warp; ++w) pos += wc[w][d];
                kout[pos] = k;
                vout[pos] = vin[i];
            }
            __syncthreads();
            uint32_t add = 0u;
            for (int w = 0; w < RS_THREADS / 32; ++w) add += wc[w][tid];
            run[tid] += add;
            __syncthreads();
        }
    }
}

// scans of u32 arrays (exclusive or inclusive), three phases: chunk sums,
// one block scanning the chunk sums, each chunk scanned with its offset
__global__ void __launch_bounds__(256) k_scan_sums(const uint32_t *__restrict__ in, long long m,
                                                    uint32_t *__restrict__ part) {
    __shared__ uint32_t red[256];
    const long long c = blockIdx.x, b0 = c * SCAN_CHUNK;
    uint32_t s = 0;
    for (int i = threadIdx.x; i < SCAN_CHUNK; i += 256)
        if (b0 + i < m) s += in[b0 + i];
    red[threadIdx.x] = s;
    __syncthreads();
    for (int w = 128; w > 0; w >>= 1) {
        if (threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
        __syncthreads();
    }
    if (threadIdx.x == 0) part[c] = red[0];
}
__global__ void __launch_bounds__(1024) k_scan_parts(uint32_t *part, long long np) {
    __shared__ uint32_t tot[1024];
    const long long per = (np + 1023) / 1024, lo = threadIdx.x * per;
    uint32_t s = 0;
    for (long long i = lo; i < lo + per && i < np; ++i) s += part[i];
    tot[threadIdx.x] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t acc = 0;
        for (int i = 0; i < 1024; ++i) { const uint32_t v = tot[i]; tot[i] = acc; acc += v; }
    }
    __syncthreads();
    uint32_t acc = tot[threadIdx.x];
    for (long long i = lo; i < lo + per && i < np; ++i) { const uint32_t v = part[i]; part[i] = acc; acc += v; }
}
// (in and out may be the same array: no __restrict__ -- each element is read before it is written)
__global__ void __launch_bounds__(256) k_scan_apply(const uint32_t *in, uint32_t *out, long long m,
                                                     const uint32_t *__restrict__ part, int inclusive) {
    __shared__ uint32_t seg[256];
    const long long c = blockIdx.x, b0 = c * SCAN_CHUNK;
    constexpr int PER = SCAN_CHUNK / 256;   // consecutive elements per thread
    const long long lo = b0 + (long long)threadIdx.x * PER;
    uint32_t s = 0;
    for (int i = 0; i < PER; ++i)
        if (lo + i < m) s += in[lo + i];
    seg[threadIdx.x] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t acc = part[c];
        for (int i = 0; i < 256; ++i) { const uint32_t v = seg[i]; seg[i] = acc; acc += v; }
    }
    __syncthreads();
    uint32_t acc = seg[threadIdx.x];
    for (int i = 0; i < PER; ++i) {
        if (lo + i >= m) break;
        const uint32_t v = in[lo + i];
        if (inclusive) { acc += v; out[lo + i] = acc; } else { out[lo + i] = acc; acc += v; }
    }
}

cudaError_t scan_u32(const uint32_t *in, uint32_t *out, long long m, uint32_t *part, bool inclusive, cudaStream_t st,
                     long long &launches) {
    const long long nc = (m + SCAN_CHUNK - 1) / SCAN_CHUNK;
    k_scan_sums<<<(unsigned)nc, 256, 0, st>>>(in, m, part);
    k_scan_parts<<<1, 1024, 0, st>>>(part, nc);
    k_scan_apply<<<(unsigned)nc, 256, 0, st>>>(in, out, m, part, inclusive ? 1 : 0);
    launches += 3;
    return cudaGetLastError();
}

// one stable LSD pass over `bits` key bits (<= 32, 8 per digit pass): (k, v) -> sorted, ping-pong buffers
cudaError_t radix_sort_pairs(uint32_t *&k, uint32_t *&v, uint32_t *&k2, uint32_t *&v2, long long n, int bits,
                             uint32_t *cnt, uint32_t *part, cudaStream_t st, long long &launches) {
    const long long nt = (n + RS_TILE - 1) / RS_TILE;
    const int grid = (int)(nt < 148 * 8 ? nt : 148 * 8);
    for (int shift = 0; shift < bits; shift += 8) {
        k_rs_hist<<<grid, RS_THREADS, 0, st>>>(k, n, shift, cnt, nt);
        ++launches;
        cudaError_t e = scan_u32(cnt, cnt, (long long)RADIX * nt, part, false, st, launches);
        if (e != cudaSuccess) return e;
        k_rs_scatter<<<grid, RS_THREADS, 0, st>>>(k, v, k2, v2, n, shift, cnt, nt);
        ++launches;
        uint32_t *tk = k, *tv = v;
        k = k2; v = v2; k2 = tk; v2 = tv;
    }
    return cudaGetLastError();
}

int grid_for(long long n) {
    long long b = (n + 255) / 256;
    return (int)(b < 148 * 16 ? (b < 1 ? 1 : b) : 148 * 16);
}

}  // namespace

extern "C" up_status up_group_ids(up_ctx *c, const up_column *keys, int nkeys, int32_t *d_ids, int64_t *n_groups,
                                  int64_t *d_first, void *stream) {
    if (!c || !keys || nkeys < 1 || !n_groups || (!d_ids && keys[0].n > 0)) return up_internal_fail(UP_E_INVAL, "group_ids: need ctx, keys, d_ids, n_groups");
    const long long n = keys[0].n;
    KeyPlanes kp;
    kp.np = 0;
    for (int k = 0; k < nkeys; ++k) {
        const up_column &col = keys[k];
        if (col.n != n) return up_internal_fail(UP_E_INVAL, "group_ids: key columns differ in length");
        if (col.layout != UP_LAYOUT_PLANES) return up_internal_fail(UP_E_UNSUPPORTED, "group_ids: key columns must be limb planes");
        if (col.p < 1 || col.limbs != up_limbs(col.p) || (n > 0 && !col.data) || col.ld < n)
            return up_internal_fail(UP_E_INVAL, "group_ids: bad key column descriptor");
        for (int j = 0; j < col.limbs; ++j) {
            if (kp.np == kMaxKeyPlanes) return up_internal_fail(UP_E_UNSUPPORTED, "group_ids: more than 64 key limbs");
            kp.p[kp.np++] = col.data + (long long)j * col.ld;
        }
    }
    if (n >= (1ll << 32)) return up_internal_fail(UP_E_UNSUPPORTED, "group_ids: more than 2^32-1 rows");
    *n_groups = 0;
    if (n == 0) return UP_OK;
    cudaStream_t st = (cudaStream_t)stream;
    // the ctx scratch may be reallocated by up_internal_scratch: hold the ctx lock for the whole call
    std::lock_guard<std::mutex> lock(up_internal_mutex(c));
#define GB_TRY(x)                                                                                     \
    do {                                                                                              \
        const cudaError_t e_ = (x);                                                                   \
        if (e_ != cudaSuccess) return up_internal_fail(UP_E_CUDA, std::string("group_ids: " #x ": ") + \
                                                       cudaGetErrorString(e_));                       \
    } while (0)
    // scratch (the ctx's persistent buffer): keys x2, perm x2, head, gid, digit counts, scan partials
    const long long nt = (n + RS_TILE - 1) / RS_TILE;
    const size_t words = ((6 * (size_t)n + 63) / 64) * 64;
    const size_t cwords = (size_t)RADIX * (size_t)nt + 64;
    const size_t pwords = (size_t)((RADIX * nt > n ? RADIX * nt : n) + SCAN_CHUNK - 1) / SCAN_CHUNK + 64;
    void *base = nullptr;
    if (up_status e = up_internal_scratch(c, (words + cwords + pwords) * sizeof(uint32_t), &base)) return e;
    uint32_t *k0 = (uint32_t *)base;
    uint32_t *k1 = k0 + n, *p0 = k0 + 2 * n, *p1 = k0 + 3 * n, *head = k0 + 4 * n, *gid = k0 + 5 * n;
    uint32_t *cnt = k0 + words, *part = cnt + cwords;
    uint32_t *kc = k0, *kn = k1, *pc = p0, *pn = p1;
    const int grid = grid_for(n);
    long long launches = 0;
    k_gb_iota<<<grid, 256, 0, st>>>(pc, n);
    ++launches;
    // LSD: last key column first, least significant limb first
    for (int k = nkeys - 1; k >= 0; --k) {
        const up_column &col = keys[k];
        for (int j = 0; j < col.limbs; ++j) {
            const uint32_t flip = j == col.limbs - 1 ? 0x80000000u : 0u;
            k_gb_gather<<<grid, 256, 0, st>>>(col.data + (long long)j * col.ld, pc, kc, n, flip);
            ++launches;
            GB_TRY(radix_sort_pairs(kc, pc, kn, pn, n, 32, cnt, part, st, launches));
        }
    }
    k_gb_gather_excl<<<grid, 256, 0, st>>>(d_ids, pc, kc, n);
    ++launches;
    GB_TRY(radix_sort_pairs(kc, pc, kn, pn, n, 8, cnt, part, st, launches));
    k_gb_heads<<<grid, 256, 0, st>>>(kp, d_ids, pc, head, n);
    ++launches;
    GB_TRY(scan_u32(head, gid, n, part, true, st, launches));
    uint32_t total = 0;
    GB_TRY(cudaMemcpyAsync(&total, gid + (n - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    k_gb_scatter<<<grid, 256, 0, st>>>(pc, head, gid, d_ids, reinterpret_cast<long long *>(d_first), n);
    ++launches;
    up_internal_add_launches(c, launches);
    GB_TRY(cudaGetLastError());
    GB_TRY(cudaStreamSynchronize(st));
#undef GB_TRY
    *n_groups = (int64_t)total;
    return UP_OK;
}
