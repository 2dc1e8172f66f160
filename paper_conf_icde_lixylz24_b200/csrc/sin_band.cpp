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
// Why Horner: the dividend Y_k X2 is fed as NON-normalised product chunks
// (64-bit chunks c_m of two Y digits: c_m X2 = L_m + H_m 2^64,
// A_m = L_m + H_(m-1), 65 bits) -- no carry ever travels upward -- so chunk m
// of Q depends only on chunks >= m of Y_k (through the running remainder R)
// and on nothing below.  The quotient chunk is a Moller-Granlund 2-by-1 step
// on 64-bit words against the normalised D~ = D_k 2^sh (one word); V = Y X2
// 2^sh is streamed as V_m = lo64(A_m << sh) + (A_(m-1) >> (64 - sh)), whose
// carry (<= 1) belongs to the position above, already consumed: R := R + c
// (Horner).  R + c >= D~ (probability ~2^-63 per chunk) means a quotient
// chunk >= 2^64: +1 into the chunk emitted one step earlier.  (Round 2 first
// ran this on 32-bit digits with 3-by-2 steps; the chunk version halves the
// dependent steps: P = 2000 +27 %, P = 20000 +20 %, profiles/r02_s15-s16.)
// The skew: term k+1 can consume digit i of Y_(k+1) as soon as term k has
// emitted it, so G consecutive terms of one row run CONCURRENTLY on G lanes,
// term b of the band DELTA chunks behind term b-1 (a systolic wavefront over
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

std::string hex_arr(const std::vector<uint32_t> &w) {
    std::ostringstream o;
    o << "{";
    for (size_t i = 0; i < w.size(); ++i) o << (i ? "," : "") << "0x" << std::hex << w[i] << std::dec << "u";
    o << "}";
    return o.str();
}


// The 64-bit-chunk band (default): the same recurrences with the division
// run on digit PAIRS -- c_m = y_2m + y_(2m+1) B, c_m X2 = L_m + H_m 2^64,
// A_m = L_m + H_(m-1) (65 bits, no carry travels upward),
// V_m = lo64(A_m << sh) + (A_(m-1) >> (64 - sh)) (sh = clz64 D_k, carry <= 1
// into R: Horner), one Moller-Granlund 2-by-1 step on 64-bit words per chunk
// against D~ = D_k 2^sh.  Half the steps of the 32-bit band for the same
// digits; the offsets o_k, drops and masks stay per 32-bit digit (quotient
// digit i goes to Y digit i - drop).  tools/sin_model.py::term_divide64 is
// the word-level model.  One row per lane group.
const char *kBand64Body = R"KERNEL(
extern __shared__ __align__(16) u64 Ssm[];
#define YSM (reinterpret_cast<u32 *>(Ssm + WS * RSS))
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
__device__ __forceinline__ void s_normalize(int rr) {
    long long carry = 0;
    for (int l = 0; l < WS - 1; ++l) {
        const long long t = (long long)Ssm[l * RSS + rr] + carry;
        Ssm[l * RSS + rr] = (u64)(u32)t;
        carry = t >> 32;
    }
    Ssm[(WS - 1) * RSS + rr] = (u64)((long long)Ssm[(WS - 1) * RSS + rr] + carry);
}
__device__ __forceinline__ u32 s_digit(int rr, int jo) {
#if CSC == 0
    return (u32)Ssm[jo * RSS + rr];
#else
    return (u32)((Ssm[jo * RSS + rr] >> CSC) | (Ssm[(jo + 1) * RSS + rr] << (32 - CSC)));
#endif
}
__device__ __forceinline__ long long s_top(int rr) { return (long long)Ssm[(WS - 1) * RSS + rr] >> CSC; }
// S 2^c += (-1)^(k-1) y 2^(c - o_k) at the slot of address sa (y = 0: no-op)
__device__ __forceinline__ void s_add(bool p, u32 sa, u32 y, u32 esh, u32 xm, u64 smsk) {
#if NEGSH0
    const u64 a = ((u64)y << esh) ^ xm;
#else
    const u64 a = (((u64)y << esh) ^ smsk) - smsk;
#endif
#if SPLIT
    const u64 s0 = lds64p(p, sa), s1 = lds64p(p, sa + 8u * RSS);
    const long long sv = (long long)a;
    sts64p(p, sa, s0 + (u64)(u32)(u64)sv);
    sts64p(p, sa + 8u * RSS, s1 + (u64)(sv >> 32));
#else
    sts64p(p, sa, lds64p(p, sa) + a);
#endif
}

// lanes: g = lane / G owns row slot rr = g (R = 32 / G rows per warp),
// b = lane % G is the term index in the band
extern "C" __global__ void __launch_bounds__(32) upk(const up_kparams P) {
    u32 *const Ysm = YSM;
    const int lane = threadIdx.x;
    const int gl = lane / G, b = lane % G;
    const int rr = gl;
    const unsigned FULL = 0xFFFFFFFFu;
    u32 fl = 0;
    for (int l = b; l < WS; l += G) Ssm[l * RSS + rr] = 0ull;
    __syncwarp();   // lane b == 0 of the row group reads (negates) these slots below
    int since_norm = 0;
    u32 acc_neg = 0u;   // SUM: the row slot's accumulator currently holds -(sum)
    const long long n = P.n;
    const long long groups = (n + R - 1) / R;
    const u32 ybase = (u32)__cvta_generic_to_shared(Ysm), sbase = (u32)__cvta_generic_to_shared(Ssm);
    for (long long grp = blockIdx.x; grp < groups; grp += gridDim.x) {
        const long long row = grp * R + rr;
        const bool valid = row < n;
        const u32 xv = valid ? __ldcs(P.col[0] + row) : 0u;
        const u32 ng = xv >> 31;
        const u32 mx = ng ? 0u - xv : xv;
        const u64 X2 = (u64)mx * mx;
        int top = -1;
        // ---- Y_1 = |m| 10^(P-s) (slot l = digit l), lane b == 0 of the row group
        if (b == 0) {
            u64 c = 0;
            for (int l = 0; l < W; ++l) {
                const u64 t = mulw(POW10PS[l], mx) + c;
                const u32 v = (u32)t;
                Ysm[l * RSY + rr] = v;
                c = t >> 32;
                if (v) top = l;
            }
            for (int l = W; l < WY; ++l) Ysm[l * RSY + rr] = 0u;
#if SUM
            if (ng != acc_neg) {
                for (int l = 0; l < WS; ++l) Ssm[l * RSS + rr] = 0ull - Ssm[l * RSS + rr];
                acc_neg = ng;
            }
#else
            for (int l = 0; l < WS; ++l) Ssm[l * RSS + rr] = 0ull;
#endif
        }
        __syncwarp();
        // chunk units: the first term's V is nonzero up to chunk (top >> 1) + 2
        int mtop = (int)__reduce_max_sync(FULL, (unsigned)(top + 1)) - 1;
        bool live = mtop >= 0;
        int J0 = (mtop >> 1) + 2;
        u32 kbase = 1;
        while (live) {
            const u32 k = kbase + (u32)b;
            const u32 ki = k <= KT ? k - 1 : KT - 1;
            if (k > KT) fl |= F_INVAL;        // never reached for |x| < 10^(p-s) (host bound)
            const uint4 e = DTAB[ki];
            const u32 sh = SHT[ki];
            const u64 Dn = ((u64)e.y << 32) | e.x;
            const u64 V64 = ((u64)e.w << 32) | e.z;
            const u32 o = (TWO_S * (k - 1u)) & 31u;
            const u32 o2 = o + TWO_S;
            const int drop = (int)(o2 >> 5);
            const u32 onew = o2 & 31u;
            const u32 mask = onew ? ~((1u << onew) - 1u) : 0xFFFFFFFFu;
            const u32 esh = CSC - o;                      // S addend = Y_k digit << esh
            const bool negt = (k & 1u) == 0u;             // (-1)^(k-1)
            const int jb = J0 + DELTA * b, jtop = J0 + b; // chunk positions: start, top
            const int steps = DELTA * (G - 1) + J0 + 1;
#if NEGSH0
            const u32 xm = negt ? 0xFFFFFFFFu : 0u;
            const u64 smsk = 0ull;
            if (negt) {   // ~y per loaded digit: subtract 2^(32 nl) - 1 once (nl digits: chunks 0 .. jtop - 2)
                const int nl = 2 * (jtop - 1);
                if (nl > 0) { atomicAdd(&Ssm[nl * RSS + rr], ~0ull); atomicAdd(&Ssm[rr], 1ull); }
            }
            __syncwarp();
#else
            const u32 xm = 0u;
            const u64 smsk = negt ? ~0ull : 0ull;
#endif
            // step at chunk position j: load chunk j - 2 (digits 2j-4, 2j-3), add its
            // digits into S, form A_(j-1) and V_j, emit quotient chunk j (Y digits
            // 2j - drop, 2j + 1 - drop); the next chunk is loaded one step ahead
            u32 yl = ybase + 4u * (u32)((2 * (jb - 2)) * RSY + rr);
            u32 sl = sbase + 8u * (u32)((2 * (jb - 2)) * RSS + rr);
            u32 yw = ybase + 4u * (u32)((2 * jb - drop) * RSY + rr);
            const bool ld0 = (unsigned)jb <= (unsigned)jtop && jb >= 2;
            u32 ya = lds32p(ld0, yl), yb = lds32p(ld0, yl + 4u * RSY);
            u64 Rm = 0ull, qprev = 0ull, Lprev = 0ull, Aplo = 0ull;
#pragma unroll 2
            for (int tau = 0; tau < steps; ++tau) {
                const int j = jb - tau;
                const bool act = (unsigned)j <= (unsigned)jtop;
                const bool ld = act && j >= 2;
                const bool ldn = (unsigned)(j - 1) <= (unsigned)jtop && j >= 3;
                const u32 y0 = ya, y1 = yb;
                ya = lds32p(ldn, yl - 8u * RSY);
                yb = lds32p(ldn, yl - 4u * RSY);
                s_add(ld, sl, y0, esh, xm, smsk);
                s_add(ld, sl + 8u * RSS, y1, esh, xm, smsk);
                // c_(j-2) X2 = L + H 2^64
                const u64 cw = ((u64)y1 << 32) | y0;
                const unsigned __int128 pr = (unsigned __int128)cw * X2;
                const u64 L = (u64)pr, H = (u64)(pr >> 64);
                // A_(j-1) = L_(j-1) + H_(j-2) (65 bits); V_j = lo64(A_j << sh) + (A_(j-1) >> (64 - sh))
                u64 Alo, Vj;
                u32 Ahi, cV;
                asm("add.cc.u64 %0, %2, %3; addc.u32 %1, 0, 0;" : "=l"(Alo), "=r"(Ahi) : "l"(Lprev), "l"(H));
                // A_(j-1) >> (64 - sh), branch-free for sh = 0 .. 63 (sh differs per lane)
                const u64 spill = ((Alo >> 1) >> (63u - sh)) | ((u64)Ahi << sh);
                asm("add.cc.u64 %0, %2, %3; addc.u32 %1, 0, 0;" : "=l"(Vj), "=r"(cV) : "l"(Aplo << sh), "l"(spill));
                u64 T = Rm + cV;     // the carry belongs to position j + 1 (Horner)
                if (__builtin_expect(T >= Dn, 0)) {   // quotient chunk >= 2^64 (p ~ 2^-63): +1 into chunk j + 1
                    T -= Dn;
                    if (act && j + 1 <= jtop) {
                        const u64 pv = qprev + 1ull;
                        if (pv == 0ull) fl |= F_INVAL;   // second-order ripple (p ~ 2^-127): flagged, never silent
                        sts32p(true, yw + 8u * RSY, (u32)pv);
                        sts32p(true, yw + 12u * RSY, (u32)(pv >> 32));
                    }
                }
                u64 Rn;
                const u64 q = mg_step64(T, Vj, Dn, V64, Rn);
                Rm = Rn;
                // quotient digits 2j, 2j+1 -> Y digits 2j - drop, 2j + 1 - drop (digit drop masked)
                sts32p(act && 2 * j >= drop, yw, (u32)q & (2 * j == drop ? mask : 0xFFFFFFFFu));
                sts32p(act, yw + 4u * RSY, (u32)(q >> 32) & (2 * j + 1 == drop ? mask : 0xFFFFFFFFu));
                qprev = q;
                Lprev = L; Aplo = Alo;
                yl -= 8u * RSY; yw -= 8u * RSY; sl -= 16u * RSS;
                __syncwarp();
            }
            kbase += G;
            // the band's last term (k = kbase - 1) wrote Y_kbase digits [0, 2 (J0 + G - 1) + 1 - drop]:
            // find each row's top digit and zero the digit(s) above it the next first term reads
            int tp = -1;
            if (b == 0) {
                const u32 ol = (TWO_S * (kbase - 2u)) & 31u;
                const int t0 = min(2 * (J0 + G - 1) + 1 - (int)((ol + TWO_S) >> 5), WY - 1);
                int t = t0;
                while (t >= 0 && Ysm[t * RSY + rr] == 0u) --t;
                for (int l = t + 1; l <= t + 2 && l < WY; ++l) Ysm[l * RSY + rr] = 0u;
                tp = t;
            }
            __syncwarp();
            mtop = (int)__reduce_max_sync(FULL, (unsigned)(tp + 1)) - 1;
            live = mtop >= 0;
            J0 = (mtop >> 1) + 2;
            if (kbase > KT + G) { fl |= F_INVAL; break; }
        }
        // ---- row end
#if SUM
        if (++since_norm >= NR) {
            since_norm = 0;
            if (b == 0) s_normalize(rr);
        }
#else
        if (b == 0) {
            s_normalize(rr);
            const u32 msk = 0u - ng;
            u32 cy = ng;
            for (int jo = 0; jo < LO; ++jo) {
                const u64 t = (u64)(s_digit(rr, jo) ^ msk) + cy;
                cy = (u32)(t >> 32);
                if (valid) P.out[(long long)jo * P.ld_out + row] = (u32)t;
            }
        }
#endif
        __syncwarp();
    }
    if (fl) atomicOr(P.flags, fl);
#if SUM
    if (b == 0) {
        if (acc_neg)
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
                                std::string &err) {
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
    // lanes per row (measured with packed row slots, profiles/r02_s40): P = 2000 (W = 213)
    // G = 4 5.87e6 rows/s (G = 8: 5.19e6), P = 3000 G = 4 2.78e6 (G = 8: 2.50e6), P = 5000
    // G = 8 1.23e6 (G = 4: 0.89e6, G = 16: 1.12e6), P = 10000 G = 16 3.41e5 (G = 32:
    // 3.10e5), P = 20000 G = 32 9.53e4 (G = 16: 7.36e4).  Fewer lanes: less pipeline
    // fill (DELTA (G - 1) steps per band); more: more rows resident (shared memory)
    if (G <= 0) G = W <= 350 ? 4 : W <= 700 ? 8 : W <= 1500 ? 16 : 32;
    if (G != 1 && G != 2 && G != 4 && G != 8 && G != 16 && G != 32) { err = "band sine: G must divide 32"; return ""; }
    // one row per lane group (two rows per lane were measured slower, profiles/r02_s5)
    const int R = 32 / G;
    const int KT = kmax + G + 2;
    // D_k table: normalised D~ = D_k 2^sh (one 64-bit word), its 2-by-1 reciprocal, sh
    std::vector<uint32_t> tab, sht;
    unsigned __int128 c5 = 1;
    for (int i = 0; i < 2 * s; ++i) c5 *= 5u;
    for (int k = 1; k <= KT; ++k) {
        const unsigned __int128 D = c5 * (unsigned __int128)((uint64_t)(2 * k) * (uint64_t)(2 * k + 1));
        if (D >> 64) { err = "band sine: D_k >= 2^64"; return ""; }
        const uint64_t d = (uint64_t)D;
        const int sh = __builtin_clzll(d);
        const uint64_t dn = d << sh;
        const uint64_t v64 = (uint64_t)(~(unsigned __int128)0 / dn);   // floor((2^128-1)/dn) - 2^64 (mod 2^64)
        tab.insert(tab.end(), {(uint32_t)dn, (uint32_t)(dn >> 32), (uint32_t)v64, (uint32_t)(v64 >> 32)});
        sht.push_back((uint32_t)sh);
    }
    // chunk steps: lane b - 1 finalises chunk m (incl. its carry fix-up) at its step for
    // m - 3, lane b loads it (one ahead) at its step for m + 1: DELTA >= 5
    const int DELTA = 5;
    // Y digits written up to 2 (J0 + G - 1) + 1 <= W + 2G + 2; S slots up to W + 2G
    const int WY = W + 2 * G + 8;
    const int WS = WY + 2;
    // S scale c = max o_k, single-slot adds when sum_rows(addends) stays < 2^62
    int csc = 0;
    for (int k = 1; k <= 64; ++k) csc = std::max(csc, (2 * s * (k - 1)) & 31);
    const double per_row = std::log2((double)kmax + G) + 32 + csc;
    const bool split = per_row > 60.0;
    int NR = 1;
    if (!split) NR = (int)std::max(1.0, std::floor(std::pow(2.0, 61.0 - per_row)));
    else NR = (int)std::max(1.0, std::floor(std::pow(2.0, 61.0 - (std::log2((double)kmax + G) + 33))));
    // lanes of one step touch digits 2 DELTA apart (lane b) in rows g
    // row slots packed (stride R): padding the strides against the 2-way bank
    // conflicts of lanes b and b + 4 cost more resident rows than it saved
    // (P = 5000: 0.99e6 -> 1.23e6 rows/s without it, P = 2000 +1 %, r02_s39)
    const int RSY = R, RSS = R;
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
    k << "// generated by libup: sin_taylor (skewed band, 64-bit chunks) P=" << P << " x DECIMAL(" << p << "," << s << ") W=" << W
      << " G=" << G << " DELTA=" << DELTA << " KT=" << KT << (sum ? " SUM" : " eval") << "\n";
    k << "#include \"up_dev.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n";
    k << "#define W " << W << "\n#define WY " << WY << "\n#define WS " << WS << "\n#define G " << G << "\n#define R "
      << R << "\n#define DELTA " << DELTA << "\n#define KT " << KT << "\n#define TWO_S "
      << 2 * s << "u\n#define CSC " << csc << "\n#define SPLIT " << (split ? 1 : 0) << "\n#define NR " << NR
      << "\n#define NEGSH0 " << (negsh0 ? 1 : 0) << "\n#define RSY " << RSY << "\n#define RSS " << RSS << "\n#define SUM " << (sum ? 1 : 0) << "\n#define LO "
      << Lout << "\n#define LA " << LA << "\n";
    k << "__device__ const u32 POW10PS[W] = " << hex_arr(HBig::pow10(P - s).twos(W, false)) << ";\n";
    k << "__device__ const uint4 DTAB[KT] = {";
    for (int i = 0; i < KT; ++i)
        k << (i ? "," : "") << "{" << tab[4 * i] << "u," << tab[4 * i + 1] << "u," << tab[4 * i + 2] << "u,"
          << tab[4 * i + 3] << "u}";
    k << "};\n";
    k << "__device__ const unsigned char SHT[KT] = {";
    for (int i = 0; i < KT; ++i) k << (i ? "," : "") << sht[i];
    k << "};\n";
    k << kBand64Body;
    return k.str();
}

}  // namespace uph
