// groupby.cu -- GROUP BY on DECIMAL key columns:
// the paper sorts with DECIMAL comparison operators to group (P:L730-734,
// Sec. II-C).  Here the comparison is folded into a stable LSD radix sort over
// the keys' two's-complement limb planes (least significant key column and
// limb first; the top limb of each key has its sign bit flipped so unsigned
// order equals signed order), after which equal keys are adjacent: one pass
// marks the first row of every run by comparing all key limbs with the
// previous sorted row, a prefix sum numbers the runs, and a scatter writes the
// dense id back to each row.  The radix-sort and scan primitives are CUB's
// (library code, like cuBLAS for a GEMM); the key handling is ours.
#include <cuda_runtime.h>

#include <cub/cub.cuh>
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
    // scratch (the ctx's persistent buffer): keys x2, perm x2, head, gid, then CUB's temp storage
    uint32_t *k0 = nullptr;
    size_t tsort = 0, tscan = 0;
    {
        cub::DoubleBuffer<uint32_t> kq(nullptr, nullptr), pq(nullptr, nullptr);
        GB_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tsort, kq, pq, n, 0, 32, st));
        GB_TRY(cub::DeviceScan::InclusiveSum(nullptr, tscan, (uint32_t *)nullptr, (uint32_t *)nullptr, n, st));
    }
    const size_t tbytes = tsort > tscan ? tsort : tscan;
    const size_t words = ((6 * (size_t)n + 63) / 64) * 64;
    void *base = nullptr;
    if (up_status e = up_internal_scratch(c, words * sizeof(uint32_t) + tbytes, &base)) return e;
    k0 = (uint32_t *)base;
    void *temp = (void *)(k0 + words);
    uint32_t *k1 = k0 + n, *p0 = k0 + 2 * n, *p1 = k0 + 3 * n, *head = k0 + 4 * n, *gid = k0 + 5 * n;
    cub::DoubleBuffer<uint32_t> kb(k0, k1), pb(p0, p1);
    const int grid = grid_for(n);
    long long launches = 0;
    k_gb_iota<<<grid, 256, 0, st>>>(pb.Current(), n);
    ++launches;
    // LSD: last key column first, least significant limb first
    for (int k = nkeys - 1; k >= 0; --k) {
        const up_column &col = keys[k];
        for (int j = 0; j < col.limbs; ++j) {
            const uint32_t flip = j == col.limbs - 1 ? 0x80000000u : 0u;
            k_gb_gather<<<grid, 256, 0, st>>>(col.data + (long long)j * col.ld, pb.Current(), kb.Current(), n, flip);
            ++launches;
            size_t tb = tbytes;
            GB_TRY(cub::DeviceRadixSort::SortPairs(temp, tb, kb, pb, n, 0, 32, st));
        }
    }
    k_gb_gather_excl<<<grid, 256, 0, st>>>(d_ids, pb.Current(), kb.Current(), n);
    ++launches;
    {
        size_t tb = tbytes;
        GB_TRY(cub::DeviceRadixSort::SortPairs(temp, tb, kb, pb, n, 0, 1, st));
    }
    k_gb_heads<<<grid, 256, 0, st>>>(kp, d_ids, pb.Current(), head, n);
    ++launches;
    {
        size_t tb = tbytes;
        GB_TRY(cub::DeviceScan::InclusiveSum(temp, tb, head, gid, n, st));
    }
    uint32_t total = 0;
    GB_TRY(cudaMemcpyAsync(&total, gid + (n - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    k_gb_scatter<<<grid, 256, 0, st>>>(pb.Current(), head, gid, d_ids, reinterpret_cast<long long *>(d_first), n);
    ++launches;
    up_internal_add_launches(c, launches);
    GB_TRY(cudaGetLastError());
    GB_TRY(cudaStreamSynchronize(st));
#undef GB_TRY
    *n_groups = (int64_t)total;
    return UP_OK;
}
