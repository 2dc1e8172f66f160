// up_wide.cuh -- warp-per-row arithmetic on wide numbers staged in shared
// memory (rows a3/a6/a7/a10/a11 for DECIMAL columns of ~40+ limbs, e.g.
// cfg3 at DECIMAL(1000,100) = 104 limbs).  Embedded into NVRTC kernels next to
// up_dev.cuh.
//
// A warp owns one row at a time (the paper's TPI = 32 threads per instance,
// P:L1312-1418).  Operands live in the warp's shared-memory slice; lanes own
// contiguous chunks for carry-propagating passes (ballot carry-lookahead, see
// Grp<32>) and own balanced sets of product COLUMNS for multiplication, so a
// product is accumulated as exact 96-bit column sums with no per-row carry
// normalisation at all when only the SUM is needed.
#pragma once

namespace up {
namespace wide {

// two's complement (L limbs in smem) -> magnitude in place; returns the sign (0/1)
template <int L>
__device__ __forceinline__ u32 to_mag(u32 *x) {
    constexpr int CH = (L + 31) / 32;
    const Grp<32> g;
    const u32 sign = x[L - 1] >> 31;
    if (!sign) return 0u;
    u32 c[CH];
#pragma unroll
    for (int i = 0; i < CH; ++i) {
        const int j = g.gl * CH + i;
        c[i] = j < L ? x[j] : 0xFFFFFFFFu;
    }
    g_cond_neg<32, CH>(g, c, 1u);
#pragma unroll
    for (int i = 0; i < CH; ++i) {
        const int j = g.gl * CH + i;
        if (j < L) x[j] = c[i];
    }
    __syncwarp();
    return 1u;
}

// Column sums of the product of magnitudes a (LA limbs) x b (LB limbs), added
// as exact 64-bit slots into acc[k] (+ carries into acc[k+1]): value added =
// a*b = sum_k colsum_k 2^(32k), colsum_k = sum_{i+j=k} a_i b_j (< 2^71).
// Columns are dealt to lanes in pairs whose term counts add up to a constant,
// so every lane runs the same trip count.
template <int LA, int LB>
__device__ __forceinline__ void colsum_product(const u32 *a, const u32 *b, u64 *acc) {
    constexpr int NK = LA + LB - 1;                  // columns 0 .. NK-1
    constexpr int NPAIR = (NK + 1) / 2;
    const int lane = threadIdx.x & 31;
    for (int pr = lane; pr < NPAIR; pr += 32) {
        // pair column k with NK-1-k (when equal, a single column)
#pragma unroll
        for (int half = 0; half < 2; ++half) {
            const int k = half == 0 ? pr : NK - 1 - pr;
            if (half == 1 && k == pr) break;
            const int ilo = k - (LB - 1) > 0 ? k - (LB - 1) : 0;
            const int ihi = k < LA - 1 ? k : LA - 1;
            u64 lo = 0;
            u32 hi = 0;
            int i = ilo;
            for (; i + 3 <= ihi; i += 4) {
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const u64 p = (u64)a[i + u] * b[k - i - u];
                    lo += p;
                    hi += lo < p ? 1u : 0u;
                }
            }
            for (; i <= ihi; ++i) {
                const u64 p = (u64)a[i] * b[k - i];
                lo += p;
                hi += lo < p ? 1u : 0u;
            }
            // value lo + hi*2^64 at column k: slots k (low 32), k+1 (next 32), k+2 (hi)
            const u32 l0 = (u32)lo;
            const u64 l1 = (lo >> 32) | 0ull;
            if (l0) atomicAdd(&acc[k], (u64)l0);
            if (l1) atomicAdd(&acc[k + 1], l1);
            if (hi) atomicAdd(&acc[k + 2], (u64)hi);
        }
    }
}

// u (NU limbs) = a (LA limbs) * c (LC limbs, constant), magnitudes, written to
// smem (NU >= LA + LC - 1 .. LA + LC; the top limb receives the last carry).
// Lanes own chunks of CH output limbs: exact column sums, local carry, then
// a shuffled 64-bit carry and a ballot-resolved 1-bit carry between lanes.
template <int LA, int LC, int NU>
__device__ __forceinline__ void mul_const(const u32 *a, const u32 (&c)[LC], u32 *u) {
    constexpr int CH = (NU + 31) / 32 < 2 ? 2 : (NU + 31) / 32;   // >= 2: the 64-bit carry spans two limbs
    const Grp<32> g;
    u32 limb[CH];
    u64 carry = 0;   // local running carry (< 2^40)
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const int k = g.gl * CH + t;
        u64 lo = carry;
        u32 hi = 0;
        if (k < NU) {
#pragma unroll
            for (int q = 0; q < LC; ++q) {
                const int i = k - q;
                if (i >= 0 && i < LA) {
                    const u64 p = (u64)a[i] * c[q];
                    lo += p;
                    hi += lo < p ? 1u : 0u;
                }
            }
        }
        limb[t] = (u32)lo;
        carry = (lo >> 32) | ((u64)hi << 32);
    }
    // carry out of this chunk goes to the next lane's lowest limbs
    const u32 c0 = g.up1((u32)carry), c1 = g.up1((u32)(carry >> 32));
    limb[0] = add_cc(limb[0], c0);
    limb[1] = addc_cc(limb[1], c1);
#pragma unroll
    for (int t = 2; t < CH; ++t) limb[t] = addc_cc(limb[t], 0u);
    const u32 cy = addc(0u, 0u);
    chunk_inc(limb, g.carry_in(cy != 0u, chunk_all_ones(limb), 0u));
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const int k = g.gl * CH + t;
        if (k < NU) u[k] = limb[t];
    }
    __syncwarp();
}

// 1-bit borrow/carry passes over a window w[0..N) in smem, lanes owning CH limbs
template <int N>
__device__ __forceinline__ u32 sub_lo_hi(u32 *w, const u32 *v, int nv, u32 qhat) {
    // w -= qhat * v (v has nv limbs, w has nv+1 limbs = N); returns the final borrow (1 = negative)
    constexpr int CH = (N + 31) / 32;
    const Grp<32> g;
    u32 x[CH], lo[CH], hi[CH];
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const int i = g.gl * CH + t;
        x[t] = i < N ? w[i] : 0u;
        const u32 vi = i < nv ? v[i] : 0u;
        const u64 p = (u64)qhat * vi;
        lo[t] = (u32)p;
        hi[t] = (u32)(p >> 32);
    }
    // hi parts land one limb up
    u32 hs[CH];
    const u32 hin = g.up1(hi[CH - 1]);
#pragma unroll
    for (int t = 0; t < CH; ++t) hs[t] = t == 0 ? hin : hi[t - 1];
    // pass 1: x -= lo
    x[0] = sub_cc(x[0], lo[0]);
#pragma unroll
    for (int t = 1; t < CH; ++t) x[t] = subc_cc(x[t], lo[t]);
    u32 b1 = 0u - subc(0u, 0u);
    {
        u32 z = 0;
#pragma unroll
        for (int t = 0; t < CH; ++t) z |= x[t];
        const u32 bin = g.carry_in(b1 != 0u, z == 0u, 0u);
        x[0] = sub_cc(x[0], bin);
#pragma unroll
        for (int t = 1; t < CH; ++t) x[t] = subc_cc(x[t], 0u);
        (void)subc(0u, 0u);
    }
    const u32 top1 = (u32)__shfl_sync(0xFFFFFFFFu, (int)b1, 31);   // not used for the sign (see below)
    (void)top1;
    // pass 2: x -= hs
    x[0] = sub_cc(x[0], hs[0]);
#pragma unroll
    for (int t = 1; t < CH; ++t) x[t] = subc_cc(x[t], hs[t]);
    u32 b2 = 0u - subc(0u, 0u);
    {
        u32 z = 0;
#pragma unroll
        for (int t = 0; t < CH; ++t) z |= x[t];
        const u32 bin = g.carry_in(b2 != 0u, z == 0u, 0u);
        x[0] = sub_cc(x[0], bin);
#pragma unroll
        for (int t = 1; t < CH; ++t) x[t] = subc_cc(x[t], 0u);
        (void)subc(0u, 0u);
    }
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const int i = g.gl * CH + t;
        if (i < N) w[i] = x[t];
    }
    __syncwarp();
    // the window is negative iff its top limb (index nv) has the sign bit set:
    // 0 <= w - qhat*v + v*... holds within (-v, v*2^32) so the top limb decides
    return w[nv] >> 31;
}

template <int N>
__device__ __forceinline__ void add_back(u32 *w, const u32 *v, int nv) {
    constexpr int CH = (N + 31) / 32;
    const Grp<32> g;
    u32 x[CH], y[CH];
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const int i = g.gl * CH + t;
        x[t] = i < N ? w[i] : 0u;
        y[t] = i < nv ? v[i] : 0u;
    }
    x[0] = add_cc(x[0], y[0]);
#pragma unroll
    for (int t = 1; t < CH; ++t) x[t] = addc_cc(x[t], y[t]);
    const u32 c = addc(0u, 0u);
    chunk_inc(x, g.carry_in(c != 0u, chunk_all_ones(x), 0u));
#pragma unroll
    for (int t = 0; t < CH; ++t) {
        const int i = g.gl * CH + t;
        if (i < N) w[i] = x[t];
    }
    __syncwarp();
}

// Knuth D on magnitudes staged in smem, warp-cooperative:
// q[0..NQ) = floor(u / v) (u: NU limbs, v: NV limbs), flags F_DIVZERO /
// F_OVERFLOW (q >= 2^(32 NQ)).  scratch: NU + NV + 1 (un) + NV (vn) words.
template <int NU, int NV, int NQ>
__device__ __forceinline__ u32 divq(const u32 *u, const u32 *v, u32 *q, u32 *scratch) {
    constexpr int NN = NU + NV + 1;
    constexpr int NQE = NQ < NU ? NQ : NU;
    const int lane = threadIdx.x & 31;
    u32 *un = scratch, *vn = scratch + NN;
    // top nonzero limb of v
    int top = -1;
    for (int i = lane; i < NV; i += 32) if (v[i]) top = i;
    top = (int)__reduce_max_sync(0xFFFFFFFFu, (unsigned)(top + 1)) - 1;
    for (int i = lane; i < NQ; i += 32) q[i] = 0u;
    if (top < 0) { __syncwarp(); return F_DIVZERO; }
    const int z = NV - 1 - top;
    const u32 sh = __clz(v[top]);
    // vn = v << (32 z + sh), un = u << (32 z + sh)
    for (int i = lane; i < NV; i += 32) {
        const int s = i - z;
        const u32 hi = s >= 0 ? v[s] : 0u, lo = s - 1 >= 0 ? v[s - 1] : 0u;
        vn[i] = __funnelshift_l(lo, hi, sh);
    }
    for (int i = lane; i < NN; i += 32) {
        const int s = i - z;
        const u32 hi = (s >= 0 && s < NU) ? u[s] : 0u, lo = (s - 1 >= 0 && s - 1 < NU) ? u[s - 1] : 0u;
        un[i] = __funnelshift_l(lo, hi, sh);
    }
    __syncwarp();
    // overflow: q >= 2^(32 NQE) iff un[NQE ..] >= vn (as an NN-NQE limb number)
    if (NQE < NU) {
        int hi_nz = 0;
        for (int i = NQE + NV + lane; i < NN; i += 32) hi_nz |= un[i] != 0u;
        // compare un[NQE .. NQE+NV) with vn from the top: first differing limb
        int diff = -1;
        for (int i = lane; i < NV; i += 32) if (un[NQE + i] != vn[i]) diff = i;
        diff = (int)__reduce_max_sync(0xFFFFFFFFu, (unsigned)(diff + 1)) - 1;
        const bool ge = __any_sync(0xFFFFFFFFu, hi_nz) || diff < 0 || un[NQE + (diff < 0 ? 0 : diff)] > vn[diff < 0 ? 0 : diff];
        if (ge) { __syncwarp(); return F_OVERFLOW; }
    }
    const u32 vt = vn[NV - 1], vs = NV >= 2 ? vn[NV - 2] : 0u;
    for (int j = NQE - 1; j >= 0; --j) {
        u32 *w = un + j;   // window w[0..NV]
        const u32 w2 = w[NV], w1 = w[NV - 1], w0 = NV >= 2 ? w[NV - 2] : 0u;
        u32 qhat;
        u64 rhat;
        if (w2 >= vt) {
            qhat = 0xFFFFFFFFu;
            rhat = (u64)w1 + vt;
        } else {
            u32 rr;
            qhat = div_2by1(w2, w1, vt, rr);
            rhat = rr;
        }
        if (NV >= 2)
            while (rhat < 0x100000000ull && (u64)qhat * vs > ((rhat << 32) | w0)) { --qhat; rhat += vt; }
        __syncwarp();
        const u32 neg = sub_lo_hi<NV + 1>(w, vn, NV, qhat);
        if (neg) {
            --qhat;
            add_back<NV + 1>(w, vn, NV);
        }
        if (lane == 0) q[j] = qhat;
    }
    __syncwarp();
    return 0u;
}


// Balanced column sums for LA == LB == L: work item k < L-1 covers column k
// (k+1 terms) then column k+L (L-1-k terms); item L-1 covers column L-1
// (L terms): every item is exactly L terms, and at step t the a-index is t
// for every lane (a broadcast read).  acc gets colsum_k as 3 x 32-bit slots.
template <int L>
__device__ __forceinline__ void colsum_product_sq(const u32 *a, const u32 *b, u64 *acc) {
    const int lane = threadIdx.x & 31;
    for (int k = lane; k < L; k += 32) {
        u64 lo = 0;
        u32 hi = 0;
        int col = k;
#pragma unroll 4
        for (int t = 0; t < L; ++t) {
            if (t == k + 1) {   // switch from column k to column k+L (never for k = L-1)
                if ((u32)lo) atomicAdd(&acc[col], (u64)(u32)lo);
                if (lo >> 32) atomicAdd(&acc[col + 1], lo >> 32);
                if (hi) atomicAdd(&acc[col + 2], (u64)hi);
                lo = 0;
                hi = 0;
                col = k + L;
            }
            const int bi = t <= k ? k - t : k + L - t;
            const u64 p = (u64)a[t] * b[bi];
            lo += p;
            hi += lo < p ? 1u : 0u;
        }
        if ((u32)lo) atomicAdd(&acc[col], (u64)(u32)lo);
        if (lo >> 32) atomicAdd(&acc[col + 1], lo >> 32);
        if (hi) atomicAdd(&acc[col + 2], (u64)hi);
    }
}

// |q| < bound (NQ limbs each, in smem / constant) -- warp-cooperative compare
template <int NQ>
__device__ __forceinline__ bool lt_bound(const u32 *q, const u32 (&bound)[NQ]) {
    const int lane = threadIdx.x & 31;
    int diff = -1;
#pragma unroll
    for (int i = 0; i < NQ; ++i)
        if ((i & 31) == lane && q[i] != bound[i]) diff = i;
    diff = (int)__reduce_max_sync(0xFFFFFFFFu, (unsigned)(diff + 1)) - 1;
    if (diff < 0) return false;   // equal
    u32 qd = 0, bd = 0;
#pragma unroll
    for (int i = 0; i < NQ; ++i)
        if (i == diff) { qd = q[i]; bd = bound[i]; }
    return qd < bd;
}

// Last-block tail of the wide SUM: term t's slots in ws (pos at off_t, neg at
// off_t + ns_t) are normalised to LA limbs, scaled by the alignment constant
// 10^k_t (kc_t limbs) and added with sign sg_t.  One thread; LA <= 512.
__device__ __noinline__ void wide_final(const u64 *ws_pos, const u64 *ws_neg, int ns, const u32 *kc, int nkc,
                                        int sg, int LA, u32 *acc /* LA limbs, local */) {
    u32 x[512];
    u64 cp = 0, cn = 0;
    u32 borrow = 0;
    for (int j = 0; j < LA; ++j) {
        u64 tp = cp, tn = cn;
        if (j < ns) { tp += (u32)ws_pos[j]; tn += (u32)ws_neg[j]; }
        if (j >= 1 && j - 1 < ns) { tp += ws_pos[j - 1] >> 32; tn += ws_neg[j - 1] >> 32; }
        cp = tp >> 32;
        cn = tn >> 32;
        const u64 d = (u64)(u32)tp - (u32)tn - borrow;
        x[j] = (u32)d;
        borrow = (u32)(d >> 63);
    }
    // y = x * 10^k mod 2^(32 LA), then acc += sg * y
    u32 y[512];
    for (int j = 0; j < LA; ++j) y[j] = 0u;
    for (int i = 0; i < LA; ++i) {
        u64 c = 0;
        const u32 xi = x[i];
        for (int q = 0; q < nkc && i + q < LA; ++q) {
            const u64 t = (u64)xi * kc[q] + y[i + q] + c;
            y[i + q] = (u32)t;
            c = t >> 32;
        }
        if (i + nkc < LA) {
            for (int j = i + nkc; j < LA && c; ++j) {
                const u64 t = (u64)y[j] + c;
                y[j] = (u32)t;
                c = t >> 32;
            }
        }
    }
    u64 c = sg < 0 ? 1 : 0;
    for (int j = 0; j < LA; ++j) {
        const u32 yy = sg < 0 ? ~y[j] : y[j];
        const u64 t = (u64)acc[j] + yy + c;
        acc[j] = (u32)t;
        c = t >> 32;
    }
}
}  // namespace wide
}  // namespace up
