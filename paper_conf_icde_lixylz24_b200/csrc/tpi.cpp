// tpi.cpp -- per-operator kernels with TPI threads per instance (SURVEY
// NEXT-3; the paper's multi-threading arithmetic, §III-E1,
// measured in Fig. 13): c = a op b for op in + - * /, one row
// per group of G lanes (G = TPI in {1, 2, 4, 8, 16, 32}).
//
//  * Loads: limb-plane columns -- lane gl reads the contiguous limbs
//    [gl ML, (gl + 1) ML) of its row and turns them into a magnitude with a
//    group carry-lookahead negation; compact columns (the paper's cDecimal
//    rows) -- lane gl reads bytes [4 gl lt, 4 (gl + 1) lt) of the row, lt =
//    ceil(Lb / (4 TPI)) words: Listing 3's coalesced group load.
//    Magnitudes land in shared memory, one slice per row.
//  * * and the alignment products 10^k of + / -: lane gl forms the result
//    columns [gl MR, (gl + 1) MR) of the schoolbook product, each
//    a 128-bit sum of 32 x 32 -> 64 products, normalises them and hands its
//    carry to the next lane until no carry is left (warp vote);
//  * + / -: two's complement by group negation, then one group add/sub with a
//    ballot carry-lookahead (Grp::carry_in, up_dev.cuh);
//  * /: per thread (TPI = 1), Q = trunc(|A| 10^(s2+4) / |B|) (P:L1049-1058,
//    reading Q4) by Knuth's long division (divmod_mag, the fused kernels' path)
//    or by Newton-Raphson: the reciprocal of the divisor's top
//    limbs d^-1_(i+1) = d^-1_i (2 - d d^-1_i) in fixed point (NQ + 2 limbs of
//    precision) from a 64-bit seed, the quotient estimate (dividend top) x d^-1, then an exact
//    remainder correction.  Both exact; NR costs more multiplies for the short
//    typed quotients of DECIMAL division (measured).
// Values and flags equal up_eval_expr("c1 op c2") on the same columns.
#include <cstdint>
#include <sstream>
#include <string>
#include <vector>

#include "codegen.h"
#include "expr.h"
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

const char *kTpiBody = R"KERNEL(
// 128-bit column sums of the schoolbook product x * y (x: LX limbs, y: LY
// limbs, shared or constant memory) for columns [gl MR, (gl + 1) MR), then
// the group's carries: r = (x * y) mod 2^(32 G MR), lane chunks
template <int LX, int LY>
__device__ __forceinline__ void grp_mul_cols(const Grp<G> &g, const u32 *x, const u32 *y, u32 (&r)[MR]) {
    unsigned __int128 carry = 0;
#pragma unroll
    for (int c = 0; c < MR; ++c) {
        const int t = g.gl * MR + c;
        unsigned __int128 acc = carry;
        const int i0 = t - (LY - 1) > 0 ? t - (LY - 1) : 0;
        const int i1 = t < LX - 1 ? t : LX - 1;
        for (int i = i0; i <= i1; ++i) acc += (unsigned __int128)((u64)x[i] * y[t - i]);
        r[c] = (u32)acc;
        carry = acc >> 32;
    }
#if G > 1
    unsigned __int128 pend = carry;          // to be added at the next lane's lowest limb
    for (int it = 0; it < G; ++it) {
        const u32 w0 = g.up1((u32)pend), w1 = g.up1((u32)(pend >> 32)), w2 = g.up1((u32)(pend >> 64)),
                  w3 = g.up1((u32)(pend >> 96));
        unsigned __int128 cin = ((unsigned __int128)w3 << 96) | ((unsigned __int128)w2 << 64) |
                                ((unsigned __int128)w1 << 32) | w0;
        if (!__any_sync(0xFFFFFFFFu, cin != 0)) break;
#pragma unroll
        for (int c = 0; c < MR; ++c) {
            const unsigned __int128 s = (unsigned __int128)r[c] + cin;
            r[c] = (u32)s;
            cin = s >> 32;
        }
        pend = cin;
    }
#endif
}

// row magnitude (L limbs) into shared memory dst[0..L), returns the sign
template <int L, int LBYTES>
__device__ __forceinline__ u32 load_mag(const Grp<G> &g, const u32 *col, long long ld, long long row, bool valid, u32 *dst) {
#if G == 1
    constexpr int ML = L;
#else
    constexpr int ML = (L + G - 1) / G;
#endif
    if constexpr (LBYTES == 0) {     // limb planes, two's complement
        u32 ch[ML];
#pragma unroll
        for (int i = 0; i < ML; ++i) {
            const int j = g.gl * ML + i;
            ch[i] = (valid && j < L) ? __ldcs(col + (long long)j * ld + row) : 0u;
        }
        // sign = top bit of limb L-1 (lane (L-1) / ML)
        u32 topw = 0u;
#pragma unroll
        for (int i = 0; i < ML; ++i) if (g.gl * ML + i == L - 1) topw = ch[i];
        const u32 ng = g.bcast(topw, (L - 1) / ML) >> 31;
#pragma unroll
        for (int i = 0; i < ML; ++i) if (g.gl * ML + i >= L) ch[i] = 0u - ng;   // sign extension
        g_cond_neg(g, ch, ng);
#pragma unroll
        for (int i = 0; i < ML; ++i) { const int j = g.gl * ML + i; if (j < L) dst[j] = ch[i]; }
        return ng;
    } else {                          // compact rows (Listing 3): lane gl reads lt words of the row
        constexpr int LT = (LBYTES + 4 * G - 1) / (4 * G);
        const unsigned char *rb = reinterpret_cast<const unsigned char *>(col) + row * LBYTES;
        unsigned char *db = reinterpret_cast<unsigned char *>(dst);
#pragma unroll
        for (int i = 0; i < 4 * LT; ++i) {
            const int k = g.gl * 4 * LT + i;
            if (k < 4 * L) db[k] = (valid && k < LBYTES) ? rb[k] : (unsigned char)0;
        }
        __syncwarp();
        const u32 ng = (db[LBYTES - 1] >> 7) & 1u;
        __syncwarp();
        if (g.gl == (LBYTES - 1) / (4 * LT)) db[LBYTES - 1] &= 0x7Fu;
        return ng;
    }
}

extern "C" __global__ void __launch_bounds__(256) upk(const up_kparams P) {
    constexpr int RB = 256 / G;                       // rows per block iteration
    extern __shared__ u32 tsm[];                      // RB magnitude slices of a, then of b
    const Grp<G> g;
    const int rloc = threadIdx.x / G;
    u32 *const sar = tsm + rloc * (LA_ + 1), *const sbr = tsm + RB * (LA_ + 1) + rloc * (LB_ + 1);
    u32 fl = 0;
    const long long n = P.n;
    for (long long r0 = (long long)blockIdx.x * RB; r0 < n; r0 += (long long)gridDim.x * RB) {
        const long long row = r0 + rloc;
        const bool valid = row < n;
        const u32 nga = load_mag<LA_, CA>(g, P.col[0], P.ld[0], row, valid, sar);
        const u32 ngb = load_mag<LB_, CB>(g, P.col[1], P.ld[1], row, valid, sbr);
        __syncwarp();
#if OP == 0 || OP == 1                                 // + / -
        u32 ra[MR], rb2[MR];
        grp_mul_cols<LA_, KA>(g, sar, CONSTA, ra);
        grp_mul_cols<LB_, KB>(g, sbr, CONSTB, rb2);
        g_cond_neg(g, ra, nga);
        g_cond_neg(g, rb2, ngb);
        g_addsub(g, ra, rb2, OP == 1 ? 1u : 0u);
        const u32 *res = ra;
#elif OP == 2                                          // *
        u32 ra[MR];
        grp_mul_cols<LA_, LB_>(g, sar, sbr, ra);
        g_cond_neg(g, ra, nga ^ ngb);
        const u32 *res = ra;
#else                                                  // / (G == 1)
        u32 a[LA_], b[LB_], u[NU], q[NQ];
#pragma unroll
        for (int i = 0; i < LA_; ++i) a[i] = sar[i];
#pragma unroll
        for (int i = 0; i < LB_; ++i) b[i] = sbr[i];
        u32 cu[KU];
#pragma unroll
        for (int i = 0; i < KU; ++i) cu[i] = CONSTU[i];
        mul_mag<LA_, KU, NU>(u, a, cu);
        u32 f;
#if NRDIV
        f = nr_divmod<NU, LB_, NQ>(q, u, b);
#else
        u32 rem[LB_];
        f = divmod_mag<NU, LB_, NQ, false>(q, rem, u, b);
#endif
        // typed quotient bound |Q| < 10^p (reading Q5)
        u32 bq[NQ];
#pragma unroll
        for (int i = 0; i < NQ; ++i) bq[i] = QBOUND[i];
        if (!f && !lt(q, bq)) f = F_OVERFLOW;
        if (valid) fl |= f;
        const u32 m = 0u - (nga ^ ngb);
        u64 cy = nga ^ ngb;
#pragma unroll
        for (int i = 0; i < NQ; ++i) { const u64 t = (u64)(q[i] ^ m) + cy; q[i] = (u32)t; cy = t >> 32; }
        const u32 *res = q;
#endif
        if (valid) {
#pragma unroll
            for (int c = 0; c < MR; ++c) {
                const int t = g.gl * MR + c;
                if (t < LO) __stcs(P.out + (long long)t * P.ld_out + row, res[c]);
            }
        }
        __syncwarp();
    }
    if (fl) atomicOr(P.flags, fl);
}
)KERNEL";

// Newton-Raphson division, per thread, exact:
//   normalise v (top bit of limb NV-1 set) and u by the same shift;
//   X = floor(B^K / vt) for the divisor's top T = min(NV, NQ + 2) limbs,
//     K = T + NQ + 2 (X carries NQ + 2 limbs of the quotient's precision),
//     seeded from the top 64 bits (X0 = floor((2^128 - 1) / d64) B^(K-T-2)),
//     X <- X + X (B^K - vt X) / B^K (d^-1 (2 - d d^-1)) until converged, then
//     fixed exactly against the remainder B^K - vt X;
//   q = (top limbs of u) X / B^K, then corrected with the exact remainder
//     u - q v (tools-level model: no correction step was ever needed).
const char *kNrDiv = R"KERNEL(
template <int N> __device__ __forceinline__ bool neg_top(const u32 (&a)[N]) { return (a[N - 1] >> 31) != 0u; }
template <int N> __device__ __forceinline__ void add_to(u32 (&a)[N], const u32 *b, int nb) {
    u64 c = 0;
#pragma unroll
    for (int i = 0; i < N; ++i) { const u64 t = (u64)a[i] + (i < nb ? b[i] : 0u) + c; a[i] = (u32)t; c = t >> 32; }
}
template <int N> __device__ __forceinline__ void sub_from(u32 (&a)[N], const u32 *b, int nb) {
    u64 br = 0;
#pragma unroll
    for (int i = 0; i < N; ++i) {
        const u64 t = (u64)a[i] - (u64)(i < nb ? b[i] : 0u) - br;
        a[i] = (u32)t;
        br = (t >> 63) & 1u;
    }
}
template <int N> __device__ __forceinline__ void inc_n(u32 (&a)[N]) {
    u64 c = 1;
#pragma unroll
    for (int i = 0; i < N; ++i) { const u64 t = (u64)a[i] + c; a[i] = (u32)t; c = t >> 32; }
}
template <int N> __device__ __forceinline__ void dec_n(u32 (&a)[N]) {
    u64 b = 1;
#pragma unroll
    for (int i = 0; i < N; ++i) { const u64 t = (u64)a[i] - b; a[i] = (u32)t; b = (t >> 63) & 1u; }
}

template <int XU, int XV, int XQ>
__device__ __noinline__ u32 nr_divmod(u32 (&q)[XQ], const u32 (&u)[XU], const u32 (&v)[XV]) {
    zero(q);
    if (is_zero(v)) return F_DIVZERO;
    // --- normalise (as divmod_mag): shift v and u left by S = 32 z + sh bits
    int top = 0;
#pragma unroll
    for (int i = 0; i < XV; ++i) top = v[i] ? i : top;
    const int z = XV - 1 - top;
    u32 vn[XV];
    copy(vn, v);
    constexpr int XN = XU + XV;
    u32 un[XN];
    zext<XU, XN>(un, u);
    if (z) {
        shl_limbs_dyn<XV, XV>(vn, z);
        shl_limbs_dyn<XN, XV>(un, z);
    }
    const u32 sh = __clz(vn[XV - 1]);
    shl_bits(vn, sh);
    shl_bits(un, sh);
    // --- overflow: q >= 2^(32 XQ) iff (un >> 32 XQ) >= vn
    constexpr int XQE = XQ < XU ? XQ : XU;
    {
        u32 R[XV];
#pragma unroll
        for (int i = 0; i < XV; ++i) R[i] = (XQE + i < XN) ? un[(XQE + i < XN) ? XQE + i : 0] : 0u;
        u32 hi = 0;
#pragma unroll
        for (int i = XQE + XV; i < XN; ++i) hi |= un[i];
        if (hi != 0u || !lt(R, vn)) return F_OVERFLOW;
    }
    if constexpr (XV == 1) {   // one-limb divisor: X = floor(B^2 / d) fits 33 bits; short division is the same cost
        u32 rr[1];
        return divmod_mag<XN, 1, XQ, false>(q, rr, un, vn);
    } else {
        constexpr int T = XQ + 2 < XV ? XQ + 2 : XV;      // divisor limbs the reciprocal uses
        constexpr int K = T + XQ + 2;                     // X = floor(B^K / vt) in (B^(XQ+2), 2 B^(XQ+2)]
        constexpr int TX = XQ + 3;
        constexpr int NE = K + 2;                         // B^K - vt X, two's complement
        u32 vt[T];
#pragma unroll
        for (int i = 0; i < T; ++i) vt[i] = vn[XV - T + i];
        // --- seed: X0 = floor((2^128 - 1) / d64) B^(K-T-2), d64 = top 64 bits of vt
        u32 X[TX];
        zero(X);
        {
            const u64 d64 = ((u64)vt[T - 1] << 32) | vt[T - 2];
            const unsigned __int128 x0 = (~(unsigned __int128)0) / d64;     // in (2^64, 2^65]
            X[K - T - 2] = (u32)x0;
            X[K - T - 1] = (u32)(x0 >> 32);
            X[K - T] = (u32)(x0 >> 64);
        }
        // --- Newton-Raphson: E = B^K - vt X, X += X E / B^K (each step doubles the correct bits)
        constexpr int ITER = (32 * TX <= 128) ? 2 : (32 * TX <= 256) ? 3 : (32 * TX <= 512) ? 4 : (32 * TX <= 1024) ? 5
                           : (32 * TX <= 2048) ? 6 : 7;
#pragma unroll 1
        for (int it = 0; it < ITER; ++it) {
            u32 p[NE];
            mul_mag<T, TX, NE>(p, vt, X);
            u32 e[NE];
            zero(e);
            e[K] = 1u;                                    // B^K
            sub_from(e, p, NE);
            const bool eneg = neg_top(e);
            if (eneg) { for (int i = 0; i < NE; ++i) e[i] = ~e[i]; inc_n(e); }
            u32 pe[TX + NE];
            mul_mag<TX, NE, TX + NE>(pe, X, e);
            u32 dx[TX + 2];
#pragma unroll
            for (int i = 0; i < TX + 2; ++i) dx[i] = pe[K + i];
            u32 Xw[TX + 2];
            zext<TX, TX + 2>(Xw, X);
            if (eneg) sub_from(Xw, dx, TX + 2); else add_to(Xw, dx, TX + 2);
#pragma unroll
            for (int i = 0; i < TX; ++i) X[i] = Xw[i];
        }
        // --- exact fix: 0 <= B^K - vt X < vt
#pragma unroll 1
        for (int it = 0; it < 8; ++it) {
            u32 p[NE];
            mul_mag<T, TX, NE>(p, vt, X);
            u32 e[NE];
            zero(e);
            e[K] = 1u;
            sub_from(e, p, NE);
            if (neg_top(e)) { dec_n(X); continue; }
            u32 vte[NE];
            zext<T, NE>(vte, vt);
            if (!lt(e, vte)) { inc_n(X); continue; }
            break;
        }
        // --- quotient estimate: (un >> 32 (XV - T)) X >> 32 K
        constexpr int XUT = XQE + T + 1;                  // dividend top limbs (q < B^XQE)
        u32 ut[XUT];
#pragma unroll
        for (int i = 0; i < XUT; ++i) ut[i] = (XV - T + i < XN) ? un[(XV - T + i < XN) ? XV - T + i : 0] : 0u;
        u32 pq[XUT + TX];
        mul_mag<XUT, TX, XUT + TX>(pq, ut, X);
        u32 qh[XQE + 1];
#pragma unroll
        for (int i = 0; i < XQE + 1; ++i) qh[i] = (K + i < XUT + TX) ? pq[(K + i < XUT + TX) ? K + i : 0] : 0u;
        // --- exact correction with the full remainder r = un - qh vn (XN + 1 limbs, signed)
        u32 r[XN + 1];
        zext<XN, XN + 1>(r, un);
        {
            u32 pv[XQE + 1 + XV];
            mul_mag<XQE + 1, XV, XQE + 1 + XV>(pv, qh, vn);
            sub_from(r, pv, XQE + 1 + XV);
        }
        u32 vw[XN + 1];
        zext<XV, XN + 1>(vw, vn);
        int steps = 0;
        while (neg_top(r) && steps < 8) { add_to(r, vw, XN + 1); dec_n(qh); ++steps; }
        while (!lt(r, vw) && steps < 8) { sub_from(r, vw, XN + 1); inc_n(qh); ++steps; }
        if (steps >= 8) return F_INVAL;                  // never: the estimate is within a few units
#pragma unroll
        for (int i = 0; i < XQ; ++i) q[i] = i <= XQE ? qh[i <= XQE ? i : 0] : 0u;
        return 0u;
    }
}
)KERNEL";

}  // namespace

std::string gen_tpi_kernel(int op, const ColType &ta, const ColType &tb, const Node *root, int G, bool nr_div,
                           TpiInfo &info, std::string &err) {
    if (G != 1 && G != 2 && G != 4 && G != 8 && G != 16 && G != 32) { err = "tpi must be 1, 2, 4, 8, 16 or 32"; return ""; }
    if (op == 3 && G != 1) { err = "division runs one row per thread (tpi = 1)"; return ""; }
    const int LO = root->L;
    const int MR = (LO + G - 1) / G;
    std::ostringstream k;
    k << "// generated by libup: tpi operator kernel op=" << "+-*/"[op] << " TPI=" << G << " a (" << ta.p << "," << ta.s
      << ") b (" << tb.p << "," << tb.s << ") -> (" << root->p << "," << root->s << ")" << (nr_div ? " NR" : "") << "\n";
    k << "#include \"up_dev.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n";
    k << "#define G " << G << "\n#define OP " << op << "\n#define LA_ " << ta.limbs << "\n#define LB_ " << tb.limbs
      << "\n#define LO " << LO << "\n#define MR " << MR << "\n#define CA " << ta.Lb << "\n#define CB " << tb.Lb
      << "\n#define NRDIV " << (nr_div ? 1 : 0) << "\n";
    if (op <= 1) {
        const int s = root->s;
        const std::vector<uint32_t> ca = HBig::pow10(s - ta.s).w, cb = HBig::pow10(s - tb.s).w;
        k << "#define KA " << ca.size() << "\n#define KB " << cb.size() << "\n";
        k << "__device__ const u32 CONSTA[" << ca.size() << "] = " << hex_arr(ca) << ";\n";
        k << "__device__ const u32 CONSTB[" << cb.size() << "] = " << hex_arr(cb) << ";\n";
    }
    if (op == 3) {
        const std::vector<uint32_t> cu = HBig::pow10(tb.s + 4).w;
        const int NU = ta.limbs + (int)cu.size();
        k << "#define KU " << cu.size() << "\n#define NU " << NU << "\n#define NQ " << LO << "\n";
        k << "__device__ const u32 CONSTU[" << cu.size() << "] = " << hex_arr(cu) << ";\n";
        k << "__device__ const u32 QBOUND[" << LO << "] = " << hex_arr(HBig::pow10(root->p).twos(LO, false)) << ";\n";
        k << kNrDiv;
    }
    k << kTpiBody;
    info.rows_per_block = 256 / G;
    info.dyn_smem = (256 / G) * (ta.limbs + tb.limbs + 2) * 4;
    if (info.dyn_smem > 200 * 1024) { err = "tpi: operands too wide for the block's shared memory"; return ""; }
    return k.str();
}

}  // namespace uph
