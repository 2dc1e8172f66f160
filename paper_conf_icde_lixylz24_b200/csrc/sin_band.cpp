// sin_band.cpp -- sin_P(x) (row a9, SURVEY §8c-Q13 from Query 5 P:L2197-2249)
// as a skewed band of terms: the B200 design of the fixed-point Taylor sine.
//
// Per row, x = m 10^-s (DECIMAL(p,s), |m| < 10^9, 2s < 32), X2 = m^2 and
//   t_1 = |m| 10^(P-s),  t_(k+1) = floor(t_k X2 / (10^(2s) (2k)(2k+1))),
//   S = sum_k (-1)^(k-1) t_k,  result sign(m) S at scale P.
// With 10^(2s) (2k)(2k+1) = 2^(2s) D_k (D_k = 5^(2s) (2k)(2k+1) < 2^64) the
// kernel keeps Y_k = t_k 2^(o_k) (o_1 = 0) and per term computes
//   Q = floor(Y_k X2 / D_k)          (one Horner long division, MS -> LS)
//   o' = o_k + 2s;  Y_(k+1) = (Q with its low o' bits cleared) / B^[o' >= 32]
// (floor(floor(a/b)/c) = floor(a/(bc)) makes t_(k+1) = floor(Q / 2^o')).
//
// Why Horner: the dividend Y_k X2 is fed as NON-normalised product digits
// A_i = lo(y_i X2) + mid(y_(i-1) X2) + hi(y_(i-2) X2) (< 3B, B = 2^32) -- no
// carry ever travels upward -- so digit i of Q depends only on digits >= i
// of Y_k (through the running remainder R) and on nothing below.  The
// quotient digit is a Moller-Granlund 3-by-2 step against the normalised
// D~ = D_k 2^sh; V = Y X2 2^sh is streamed as
//   V_i = lo32(A_(i-sd) << sb) + (A_(i-sd-1) >> (32 - sb))   (sh = 32 sd + sb),
// whose carry c (<= 2) belongs to the position above, already consumed:
// R := R + c (Horner).  R + c >= D~ (probability ~2^-63 per digit) means a
// quotient digit >= B: +1 into the digit emitted one step earlier.
//
// The skew: term k+1 can consume digit i of Y_(k+1) as soon as term k has
// emitted it, so G consecutive terms of one row run CONCURRENTLY on G lanes,
// term b of the band DELTA digits behind term b-1 (a systolic wavefront over
// a shared-memory digit array): every lane has independent work every step,
// which the single-chain kernels lacked (ncu: 'wait' stalls on the serial
// remainder chain, profiles/r02_s1/ncu_sin1000.json).  The running sum is a
// carry-save array of signed 64-bit slots S 2^c = sum_k (-1)^(k-1) Y_k 2^(c-o_k),
// c = max o_k; each term adds its input digit when it loads it.
// tools/sin_model.py is the word-level Python model of these recurrences.
#include <cmath>
#include <cstdint>
#include <sstream>
#include <string>
#include <vector>

#include "codegen.h"
#include "hbig.h"

namespace uph {

namespace {

// bank-conflict-minimising padded row stride (words) for lanes (r, b) that
// touch word (base - DELTA b) of row r; elt = 1 (u32) or 2 (u64 words)
int pick_stride(int R, int G, int DELTA, int elt, int RPL) {
    int best = R, bestc = 1 << 30;
    for (int rs = R; rs < R + 64; ++rs) {
        int cnt[32] = {0};
        for (int b = 0; b < G; ++b)              // one access instruction: row slots g RPL + q, q fixed
            for (int g = 0; g < 32 / G; ++g) {
                const long long idx = (long long)(1000 - DELTA * b) * rs + g * RPL;
                for (int e = 0; e < elt; ++e) cnt[(idx * elt + e) & 31]++;
            }
        int mx = 0;
        for (int i = 0; i < 32; ++i) mx = std::max(mx, cnt[i]);
        if (mx < bestc) { bestc = mx; best = rs; }
    }
    return best;
}

std::string hex_arr(const std::vector<uint32_t> &w) {
    std::ostringstream o;
    o << "{";
    for (size_t i = 0; i < w.size(); ++i) o << (i ? "," : "") << "0x" << std::hex << w[i] << std::dec << "u";
    o << "}";
    return o.str();
}

// The kernel body (constants come as #defines in front of it).
const char *kBandBody = R"KERNEL(
// Shared memory of the (one-warp) block: S slots [WS][RSS] (u64), then the Y
// digit slots [WY][RSY] (u32); row slot rr of the warp is column rr.
extern __shared__ __align__(16) u64 Ssm[];
#define YSM (reinterpret_cast<u32 *>(Ssm + WS * RSS))
// explicit shared-window addresses (bytes) in the hot loop: one LDS/STS per
// access, no per-access address materialisation; predicated, branch-free
__device__ __forceinline__ u32 lds32p(bool p, u32 a) {
    u32 v = 0u;
    asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.shared.u32 %0, [%1]; }" : "+r"(v) : "r"(a), "r"((u32)p));
    return v;
}
__device__ __forceinline__ void sts32p(bool p, u32 a, u32 v) {
    asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q st.shared.u32 [%0], %1; }" :: "r"(a), "r"(v), "r"((u32)p) : "memory");
}
__device__ __forceinline__ u64 lds64p(bool p, u32 a) {
    u64 v = 0ull;
    asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.shared.u64 %0, [%1]; }" : "+l"(v) : "r"(a), "r"((u32)p));
    return v;
}
__device__ __forceinline__ void sts64p(bool p, u32 a, u64 v) {
    asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q st.shared.u64 [%0], %1; }" :: "r"(a), "l"(v), "r"((u32)p) : "memory");
}

// signed carry-save slots of row rr (value sum_l S_l 2^(32 l), S_l signed
// 64-bit) -> S_l in [0, 2^32) for l < WS-1, the top slot signed
__device__ __forceinline__ void s_normalize(int rr) {
    long long carry = 0;
    for (int l = 0; l < WS - 1; ++l) {
        const long long t = (long long)Ssm[l * RSS + rr] + carry;
        Ssm[l * RSS + rr] = (u64)(u32)t;
        carry = t >> 32;
    }
    Ssm[(WS - 1) * RSS + rr] = (u64)((long long)Ssm[(WS - 1) * RSS + rr] + carry);
}
// digit jo (< WS-1) of the normalised value >> CSC (exact: value = S 2^CSC);
// digit WS-2 takes the low CSC bits of the signed top slot
__device__ __forceinline__ u32 s_digit(int rr, int jo) {
#if CSC == 0
    return (u32)Ssm[jo * RSS + rr];
#else
    return (u32)((Ssm[jo * RSS + rr] >> CSC) | (Ssm[(jo + 1) * RSS + rr] << (32 - CSC)));
#endif
}
__device__ __forceinline__ long long s_top(int rr) { return (long long)Ssm[(WS - 1) * RSS + rr] >> CSC; }

// lanes: g = lane / G owns the RPL row slots rr = g RPL + q of this warp
// (R = RPL 32 / G rows), b = lane % G is the term index in the band; the RPL
// rows of a lane run the same term (same D_k, o_k, drop, mask) as independent
// remainder chains interleaved in one instruction stream
extern "C" __global__ void __launch_bounds__(32) upk(const up_kparams P) {
    u32 *const Ysm = YSM;
    const int lane = threadIdx.x;
    const int gl = lane / G, b = lane % G;
    const int rr0 = gl * RPL;
    const unsigned FULL = 0xFFFFFFFFu;
    u32 fl = 0;
#pragma unroll
    for (int q = 0; q < RPL; ++q)
        for (int l = b; l < WS; l += G) Ssm[l * RSS + rr0 + q] = 0ull;
    __syncwarp();   // lane b == 0 of the row group reads (negates) these slots below
    int since_norm = 0;
    u32 acc_neg[RPL];     // SUM: the row slot's accumulator currently holds -(sum)
#pragma unroll
    for (int q = 0; q < RPL; ++q) acc_neg[q] = 0u;
    const long long n = P.n;
    const long long groups = (n + R - 1) / R;
    for (long long grp = blockIdx.x; grp < groups; grp += gridDim.x) {
        u32 ng[RPL], x0[RPL], x1[RPL];
        bool valid[RPL];
        long long row[RPL];
        int top = -1;
#pragma unroll
        for (int q = 0; q < RPL; ++q) {
            const int rr = rr0 + q;
            row[q] = grp * R + rr;
            valid[q] = row[q] < n;
            const u32 xv = valid[q] ? __ldcs(P.col[0] + row[q]) : 0u;
            ng[q] = xv >> 31;
            const u32 mx = ng[q] ? 0u - xv : xv;
            const u64 X2 = (u64)mx * mx;
            x0[q] = (u32)X2;
            x1[q] = (u32)(X2 >> 32);
            // ---- Y_1 = |m| 10^(P-s) (slot l = digit l), lane b == 0 of the row group
            if (b == 0) {
                u64 c = 0;
                for (int l = 0; l < W; ++l) {
                    const u64 t = mulw(POW10PS[l], mx) + c;
                    const u32 v = (u32)t;
                    Ysm[l * RSY + rr] = v;
                    c = t >> 32;
                    if (v && l > top) top = l;
                }
                for (int l = W; l < WY; ++l) Ysm[l * RSY + rr] = 0u;
#if SUM
                // sum of sign(m) S over rows: the slot accumulates with the sign of the
                // current row; negate it in place when the sign changes
                if (ng[q] != acc_neg[q]) {
                    for (int l = 0; l < WS; ++l) Ssm[l * RSS + rr] = 0ull - Ssm[l * RSS + rr];
                    acc_neg[q] = ng[q];
                }
#else
                for (int l = 0; l < WS; ++l) Ssm[l * RSS + rr] = 0ull;
#endif
            }
        }
        top = __shfl_sync(FULL, top, gl * G);
        __syncwarp();
        int J0 = (int)__reduce_max_sync(FULL, (unsigned)(top + 1)) - 1 + 3 + SDMAX;   // top + 3 + sd
        bool live = __any_sync(FULL, top >= 0);
        u32 kbase = 1;
        while (live) {
            const u32 k = kbase + (u32)b;
            const uint4 e = DTAB[k <= KT ? k - 1 : KT - 1];
            if (k > KT) fl |= F_INVAL;        // never reached for |x| < 10^(p-s) (host bound)
            const u32 d0 = e.x, d1 = e.y, v = e.z;
            const int sd = (int)(e.w >> 5);
            const u32 sb = e.w & 31u;
            const u64 Dn = ((u64)d1 << 32) | d0;
            const u32 o = (TWO_S * (k - 1u)) & 31u;
            const u32 o2 = o + TWO_S;
            const int drop = (int)(o2 >> 5);
            const u32 onew = o2 & 31u;
            const u32 mask = onew ? ~((1u << onew) - 1u) : 0xFFFFFFFFu;
            const u32 esh = CSC - o;                      // S addend = Y_k digit << esh
            const bool negt = (k & 1u) == 0u;             // (-1)^(k-1)
            const int jb = J0 + DELTA * b, jtop = J0 + b;
            const int steps = DELTA * (G - 1) + J0 + 1;
            const int jld = 3 + sd;
#if NEGSH0
            // negative terms have esh = 0: add ~y (= 2^32 - 1 - y) per loaded slot, then
            // subtract 2^(32 n) - 1 once (n = slots this term loads): S[n] -= 1, S[0] += 1
            const u32 xm = negt ? 0xFFFFFFFFu : 0u;
            if (negt) {
                const int nl = jtop - 2 - sd;
                if (nl > 0) {
#pragma unroll
                    for (int q = 0; q < RPL; ++q) {
                        atomicAdd(&Ssm[nl * RSS + rr0 + q], ~0ull);
                        atomicAdd(&Ssm[rr0 + q], 1ull);
                    }
                }
            }
            __syncwarp();
#else
            const u64 smsk = negt ? ~0ull : 0ull;
#endif
            const u32 nd1 = 0u - d1;
            u32 r1[RPL], r0[RPL], qprev[RPL], p0a[RPL], p0b[RPL], p1a[RPL], Alo[RPL], ynext[RPL];
            // running shared-window byte addresses of row rr0's load / store slots (row q: + 4q / 8q)
            const u32 ybase = (u32)__cvta_generic_to_shared(Ysm), sbase = (u32)__cvta_generic_to_shared(Ssm);
            u32 yl = ybase + 4u * (u32)((jb - 3 - sd) * RSY + rr0);
            u32 yw = ybase + 4u * (u32)((jb - drop) * RSY + rr0);
            u32 sl = sbase + 8u * (u32)((jb - 3 - sd) * RSS + rr0);
            // software pipeline: the digit step tau + 1 consumes was written at step <= tau - 1
            // (DELTA >= 6 + sd), so it is loaded one step ahead, off the remainder chain
            const bool ld0 = (unsigned)jb <= (unsigned)jtop && jb >= jld;
#pragma unroll
            for (int q = 0; q < RPL; ++q) {
                r1[q] = r0[q] = qprev[q] = p0a[q] = p0b[q] = p1a[q] = Alo[q] = 0u;
                ynext[q] = lds32p(ld0, yl + 4u * q);
            }
            // unrolled by 2: the digit-history rotation (p0b <- p0a <- p0, Alo) becomes
            // register renaming instead of moves (SASS: 84 -> 76 instructions per step)
#pragma unroll 2
            for (int tau = 0; tau < steps; ++tau) {
                const int j = jb - tau;
                const bool act = (unsigned)j <= (unsigned)jtop;
                const bool ld = act && j >= jld;
                const bool ldn = (unsigned)(j - 1) <= (unsigned)jtop && j - 1 >= jld;
                const bool st = act && j >= drop;
                const u32 qm = j == drop ? mask : 0xFFFFFFFFu;
#pragma unroll
                for (int q = 0; q < RPL; ++q) {
                    const u32 y = ynext[q];
                    ynext[q] = lds32p(ldn, yl - 4u * RSY + 4u * q);
                    {   // running sum: S 2^c += (-1)^(k-1) Y_k 2^(c - o_k)   (y = 0: no-op)
#if NEGSH0
                        const u64 a = ((u64)y << esh) ^ xm;
#else
                        const u64 a = (((u64)y << esh) ^ smsk) - smsk;
#endif
                        const u32 sq = sl + 8u * q;
#if SPLIT
                        const u64 s0 = lds64p(ld, sq), s1 = lds64p(ld, sq + 8u * RSS);
                        const long long sa = (long long)a;
                        sts64p(ld, sq, s0 + (u64)(u32)(u64)sa);
                        sts64p(ld, sq + 8u * RSS, s1 + (u64)(sa >> 32));
#else
                        sts64p(ld, sq, lds64p(ld, sq) + a);
#endif
                    }
                    // product digit stream: y X2 = p0 + p1 B + p2 B^2
                    const u64 pa = mulw(y, x0[q]);
                    const u64 pb = mulw(y, x1[q]);
                    u32 p1, p2;
                    asm("add.cc.u32 %0, %2, %3; addc.u32 %1, %4, 0;" : "=r"(p1), "=r"(p2)
                        : "r"((u32)pb), "r"((u32)(pa >> 32)), "r"((u32)(pb >> 32)));
                    const u32 p0 = (u32)pa;
                    // A at the new position = p0(2 ago) + p1(1 ago) + p2(now)  (< 3B)
                    const u64 A = (u64)p0b[q] + p1a[q] + p2;
                    // V digit: lo32(Aprev << sb) + (A >> (32 - sb)); its carry goes into R
                    const u64 vs = (u64)(Alo[q] << sb) + (A >> (32u - sb));
                    const u32 u0 = (u32)vs;
                    u64 T = (((u64)r1[q] << 32) | r0[q]) + (vs >> 32);
                    if (__builtin_expect(T >= Dn, 0)) {   // quotient digit >= B (p ~ 2^-63): +1 into the digit emitted last step
                        T -= Dn;
                        if (act && j + 1 <= jtop) {
                            const u32 pv = qprev[q] + 1u;
                            if (pv == 0u) fl |= F_INVAL;   // second-order ripple (p ~ 2^-95): flagged, never silent
                            sts32p(j + 1 >= drop, yw + 4u * RSY + 4u * q, j + 1 == drop ? (pv & mask) : pv);
                        }
                    }
                    // Moller-Granlund 3-by-2 step (T:u0) / Dn, T < Dn
                    u32 qd;
                    {
                        const u32 u2 = (u32)(T >> 32), u1 = (u32)T;
                        const u64 qq = mulw(v, u2) + T;
                        u32 q1 = (u32)(qq >> 32);
                        const u32 q0 = (u32)qq;
                        const u32 rh = u1 + q1 * nd1;
                        u64 rm = ((((u64)rh) << 32) | u0) - mulw(d0, q1) - Dn;
                        q1 += 1u;
                        if ((u32)(rm >> 32) >= q0) { q1 -= 1u; rm += Dn; }
                        if (__builtin_expect(rm >= Dn, 0)) { q1 += 1u; rm -= Dn; }
                        r1[q] = (u32)(rm >> 32);
                        r0[q] = (u32)rm;
                        qd = q1;
                    }
                    sts32p(st, yw + 4u * q, qd & qm);
                    qprev[q] = qd;
                    p0b[q] = p0a[q]; p0a[q] = p0; p1a[q] = p1;
                    Alo[q] = (u32)A;
                }
                yl -= 4u * RSY; yw -= 4u * RSY; sl -= 8u * RSS;
                __syncwarp();
            }
            kbase += G;
            // the band's last term (k = kbase - 1) wrote Y_kbase into slots [0, J0 + G - 1 - drop]:
            // find each row's top digit, then clear the slots the next band's first term
            // may read above it (they can hold digits of earlier, longer terms)
            int tp = -1;
            if (b == 0) {
                const u32 ol = (TWO_S * (kbase - 2u)) & 31u;
                const int t0 = min(J0 + G - 1 - (int)((ol + TWO_S) >> 5), WY - 1);
#pragma unroll
                for (int q = 0; q < RPL; ++q) {
                    int t = t0;
                    while (t >= 0 && Ysm[t * RSY + rr0 + q] == 0u) --t;
                    for (int l = t + 1; l <= t + SDMAX + 3 && l < WY; ++l) Ysm[l * RSY + rr0 + q] = 0u;
                    tp = max(tp, t);
                }
            }
            tp = __shfl_sync(FULL, tp, gl * G);
            live = __any_sync(FULL, tp >= 0);
            J0 = (int)__reduce_max_sync(FULL, (unsigned)(tp + 1)) - 1 + 3 + SDMAX;
            if (kbase > KT + G) { fl |= F_INVAL; break; }
            __syncwarp();
        }
        // ---- row end
#if SUM
        if (++since_norm >= NR) {
            since_norm = 0;
            if (b == 0)
#pragma unroll
                for (int q = 0; q < RPL; ++q) s_normalize(rr0 + q);
        }
#else
        if (b == 0) {
#pragma unroll
            for (int q = 0; q < RPL; ++q) {
                const int rr = rr0 + q;
                s_normalize(rr);
                // out = sign(m) (S 2^c >> c), two's complement, LO limbs
                const u32 msk = 0u - ng[q];
                u32 cy = ng[q];
                for (int jo = 0; jo < LO; ++jo) {
                    const u64 t = (u64)(s_digit(rr, jo) ^ msk) + cy;
                    cy = (u32)(t >> 32);
                    if (valid[q]) P.out[(long long)jo * P.ld_out + row[q]] = (u32)t;
                }
            }
        }
#endif
        __syncwarp();
    }
    if (fl) atomicOr(P.flags, fl);
#if SUM
    // commit this lane's row slots' S (signed, x 2^c) into the pos / neg workspace
    if (b == 0) {
#pragma unroll
        for (int q = 0; q < RPL; ++q) {
            const int rr = rr0 + q;
            if (acc_neg[q])
                for (int l = 0; l < WS; ++l) Ssm[l * RSS + rr] = 0ull - Ssm[l * RSS + rr];
            s_normalize(rr);
            for (int jo = 0; jo < WS - 1; ++jo) {
                const u32 dgt = s_digit(rr, jo);
                if (dgt) atomicAdd(&P.ws[jo], (u64)dgt);
            }
            const long long tv = s_top(rr);
            if (tv > 0) atomicAdd(&P.ws[WS - 1], (u64)tv);
            if (tv < 0) atomicAdd(&P.ws[WS + WS - 1], (u64)(-tv));
        }
    }
    __threadfence();
    __syncwarp();
    u32 last = 0;
    if (lane == 0) last = atomicAdd(P.ticket, 1u) == gridDim.x - 1 ? 1u : 0u;
    last = __shfl_sync(FULL, last, 0);
    if (!last) return;
    __threadfence();
    if (lane == 0) {
        *P.ticket = 0u;
        u64 cp = 0, cn = 0;
        u32 borrow = 0;
        u64 pprev = 0, nprev = 0;
        for (int jo = 0; jo < LA; ++jo) {
            const u64 pj = jo < WS ? atomicExch(&P.ws[jo], 0ull) : 0ull;
            const u64 nj = jo < WS ? atomicExch(&P.ws[WS + jo], 0ull) : 0ull;
            const u64 tpos = cp + (u32)pj + (pprev >> 32), tneg = cn + (u32)nj + (nprev >> 32);
            pprev = pj; nprev = nj;
            cp = tpos >> 32; cn = tneg >> 32;
            const u64 d = (u64)(u32)tpos - (u32)tneg - borrow;
            P.result[jo] = (u32)d;
            borrow = (u32)(d >> 63);
        }
        for (int jo = LA; jo < WS; ++jo) { P.ws[jo] = 0ull; P.ws[WS + jo] = 0ull; }
    }
#endif
}
)KERNEL";

}  // namespace

std::string gen_sin_kernel_band(int P, int p, int s, int Lout, int LA, bool sum, int G_req, SinBandInfo &info,
                                std::string &err, int rpl_req) {
    if (p > 9 || s > p || s > P || p - s > 1 || 2 * s >= 32) { err = "band sine: unsupported type"; return ""; }
    const int W = limbs_for_precision(P + 23) + 2;
    // number of terms: t_(k+1) <= t_k x^2 / ((2k)(2k+1)), |x| < 10^(p-s)
    int kmax = 1;
    {
        const double lx2 = 2.0 * (p - s) * std::log(10.0);
        double lt = (P + p - s + 1) * std::log(10.0);
        while (lt > -1.0 && kmax < 200000) { lt += lx2 - std::log((double)(2 * kmax) * (2 * kmax + 1)); ++kmax; }
        kmax += 2;
    }
    int G = G_req;
    // lanes per row (measured, profiles/r02_s2-s3): P = 5000 (W = 520) G = 16, P = 20000 G = 32
    if (G <= 0) G = W <= 160 ? 4 : W <= 700 ? 16 : 32;
    if (G != 1 && G != 2 && G != 4 && G != 8 && G != 16 && G != 32) { err = "band sine: G must divide 32"; return ""; }
    // rows per lane: independent remainder chains per instruction stream; measured
    // (profiles/r02_s5) RPL = 2 / 4 halve the resident warps (shared memory per
    // row) for no ILP gain: P = 5000 9.3e5 (RPL 1) vs 6.5e5 (2) vs 3.5e5 (4) rows/s
    const int RPL = rpl_req > 0 ? rpl_req : 1;
    if (RPL != 1 && RPL != 2 && RPL != 4) { err = "band sine: rows per lane must be 1, 2 or 4"; return ""; }
    const int R = RPL * 32 / G;
    const int KT = kmax + G + 2;
    // D_k table (normalised), sh split into (sd, sb)
    std::vector<uint32_t> tab;
    int sdmax = 0;
    unsigned __int128 c5 = 1;
    for (int i = 0; i < 2 * s; ++i) c5 *= 5u;
    for (int k = 1; k <= KT; ++k) {
        const unsigned __int128 D = c5 * (unsigned __int128)((uint64_t)(2 * k) * (uint64_t)(2 * k + 1));
        if (D >> 64) { err = "band sine: D_k >= 2^64"; return ""; }
        const uint64_t d = (uint64_t)D;
        const int sh = __builtin_clzll(d);
        const uint64_t dn = d << sh;
        const unsigned __int128 all = ~(unsigned __int128)0 >> 32;   // 2^96 - 1
        const uint64_t v = (uint64_t)(all / dn) - (1ull << 32);
        tab.insert(tab.end(), {(uint32_t)dn, (uint32_t)(dn >> 32), (uint32_t)v, (uint32_t)sh});
        sdmax = std::max(sdmax, sh >> 5);
    }
    const int DELTA = 6 + sdmax;   // load one step ahead + the one-step carry fix-up window
    const int WY = W + G + 8 + sdmax;
    const int WS = WY + 2;
    // S scale c = max o_k, single-slot adds when sum_rows(addends) stays < 2^62
    int csc = 0;
    for (int k = 1; k <= 64; ++k) csc = std::max(csc, (2 * s * (k - 1)) & 31);
    const double per_row = std::log2((double)kmax + G) + 32 + csc;
    const bool split = per_row > 60.0;
    int NR = 1;
    if (!split) NR = (int)std::max(1.0, std::floor(std::pow(2.0, 61.0 - per_row)));
    else NR = (int)std::max(1.0, std::floor(std::pow(2.0, 61.0 - (std::log2((double)kmax + G) + 33))));
    const int RSY = pick_stride(R, G, DELTA, 1, RPL), RSS = pick_stride(R, G, DELTA, 2, RPL);
    // negative (even-k) terms have o_k = c for every even k (s = 8: o = 16; s = 0: o = 0)
    bool negsh0 = true;
    for (int kk = 2; kk <= 64; kk += 2) negsh0 = negsh0 && (((2 * s * (kk - 1)) & 31) == csc);
    info.G = G;
    info.rows_per_block = R;
    info.smem = WS * RSS * 8 + WY * RSY * 4;
    info.ws_slots = 2 * WS;
    info.delta = DELTA;
    info.W = W;
    if (info.smem > 227 * 1024) { err = "band sine: row state exceeds shared memory"; return ""; }
    if (sum && 2 * WS > 65536) { err = "band sine: SUM workspace"; return ""; }

    std::ostringstream k;
    k << "// generated by libup: sin_taylor (skewed band) P=" << P << " x DECIMAL(" << p << "," << s << ") W=" << W
      << " G=" << G << " DELTA=" << DELTA << " KT=" << KT << (sum ? " SUM" : " eval") << "\n";
    k << "#include \"up_dev.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n";
    k << "#define W " << W << "\n#define WY " << WY << "\n#define WS " << WS << "\n#define G " << G << "\n#define R "
      << R << "\n#define RPL " << RPL << "\n#define DELTA " << DELTA << "\n#define SDMAX " << sdmax << "\n#define KT " << KT << "\n#define TWO_S "
      << 2 * s << "u\n#define CSC " << csc << "\n#define SPLIT " << (split ? 1 : 0) << "\n#define NR " << NR
      << "\n#define NEGSH0 " << (negsh0 ? 1 : 0) << "\n#define RSY " << RSY << "\n#define RSS " << RSS << "\n#define SUM " << (sum ? 1 : 0) << "\n#define LO "
      << Lout << "\n#define LA " << LA << "\n";
    k << "__device__ const u32 POW10PS[W] = " << hex_arr(HBig::pow10(P - s).twos(W, false)) << ";\n";
    k << "__device__ const uint4 DTAB[KT] = {";
    for (int i = 0; i < KT; ++i)
        k << (i ? "," : "") << "{" << tab[4 * i] << "u," << tab[4 * i + 1] << "u," << tab[4 * i + 2] << "u,"
          << tab[4 * i + 3] << "u}";
    k << "};\n";
    k << kBandBody;
    return k.str();
}

}  // namespace uph
