// contract_tc.cu -- SUM over rows of c_a * c_b (a top-level column product of
// SELECT SUM(expr), SURVEY §8a rows a6 + a11) on the 5th-generation tensor
// cores, exact.
//
// The SUM of a product of two DECIMAL columns is a dense contraction over the
// row index: with byte digits a_x (x < 4La) of the two's-complement limb
// planes of c_a, and the sign digit a_{4La} = s_a (weight -2^(32 La)),
//     SUM_i a_i b_i = SUM_{x,y} sgn(x,y) 2^(8(x+y)) D[x][y],
//     D[x][y] = SUM_i a_x(i) b_y(i)                    (u8 x u8 -> s32),
// sgn = -1 when exactly one of x, y is a sign digit (schoolbook product of
// P:L576-607 with the row sum of P:L1069-1080 moved inside it, which SUM's
// linearity allows).  D is one integer GEMM (M = digits of c_a, N = digits
// of c_b, K = rows) issued as tcgen05.mma kind::i8 with the accumulator in
// TMEM.  A control warp's lane 0 brings each stage's limb-plane boxes (c_a's
// limbs of the M tile, c_b's of the N group, KC rows) into shared memory with
// 2-D TMA copies completing on mbarriers; 16 transform warps rewrite them in
// the canonical MN-major no-swizzle core-matrix layout -- a WORD transpose:
// the 16 digit bytes of one row in a 16-digit chunk are the little-endian
// words of 4 consecutive limbs -- and the control lane issues the MMAs and
// commits them to an mbarrier.  Every <= 32768 rows (255^2 * 32768 < 2^31) the accumulator is
// drained: each thread reads its TMEM lane (one digit x) and adds D[x][y]
// into per-CTA anti-diagonal sums (u64, shared memory).  At the end the
// CTAs add their sums into 32-bit-aligned u64 slots (positive and negative
// parts) with global atomics and the last CTA normalises them into LA
// two's-complement limbs: exact for any row count < 2^32.
//
// Roles: M tile (128 digits of c_a) x N group (<= 512 digits of c_b, the
// TMEM width), so one CTA's accumulator fits TMEM; CTAs of the same row block
// run the roles of the same rows (c_b re-reads hit L2).
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>

namespace {

typedef uint32_t u32;
typedef unsigned long long u64;

constexpr int THREADS = 512;            // transform warps (16); + 1 control warp
constexpr int NRAW_MAX = 4;              // raw (TMA-filled) stages in flight, at most
constexpr int MAX_SLOTS = 1024;
constexpr int MAX_ROLE_LIMBS = 256;
constexpr int ABOX_MAX = 32;             // c_a limbs per M tile (128 digits)

struct TcArgs {
    const u32 *A, *B;
    long long lda, ldb, n;
    int La, Lb;
    int n_mtiles, n_groups, n_roles, n_rblocks;
    u64 *ws;          // 2 * nsl slots: positive, negative (zero on entry, re-zeroed)
    u32 *ticket;
    u32 *result;      // LA limbs
    int LA, nsl, sign;
    int abox, bbox;   // c_a limbs per M-tile box (<= 32), c_b limbs per N-group box (<= 129)
    int nst;          // raw stages (2..NRAW_MAX), as many as shared memory holds
};

__device__ __forceinline__ u32 smem_u32(const void *p) { return (u32)__cvta_generic_to_shared(p); }

// MN-major, no swizzle: a core matrix is 16 digit bytes (MN) x 8 rows (K),
// 128 B; SBO = 128 B (next 16-digit chunk), LBO = next 8-row group
// (chunks x 128 B).  Verified against a host GEMM by tools/tc_probe.cu.
__device__ __forceinline__ u64 umma_desc_mn(u32 saddr, u32 lbo) {
    return (u64)((saddr >> 4) & 0x3FFFu) | ((u64)((lbo >> 4) & 0x3FFFu) << 16) | ((u64)(128 >> 4) << 32) | (1ull << 46);
}

// bounded wait: a lost completion traps (launch error) instead of hanging.
// try_wait with a suspend-time hint parks the warp instead of spinning.
__device__ __forceinline__ void mbar_wait(u32 mb, u32 parity) {
    u32 ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
                 "selp.u32 %0, 1, 0, p;\n\t}\n" : "=r"(ok) : "r"(mb), "r"(parity), "r"(1000000u) : "memory");
    if (ok) return;
    for (long long spins = 0;; ++spins) {
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}\n" : "=r"(ok) : "r"(mb), "r"(parity), "r"(1000000u) : "memory");
        if (ok) return;
        if (spins == (1ll << 24)) {
            printf("contract_tc: mbarrier wait timed out (block %d thread %d parity %u)\n", blockIdx.x, threadIdx.x, parity);
            __trap();
        }
    }
}

// per-CTA digit sums -> 32-bit-aligned u64 slots of the global workspace (a
// value v at byte position d is v * 2^(8(d%4)) at slot d/4: three 32-bit
// pieces); positive and negative parts apart
__device__ __forceinline__ void commit_digit_sums(const u64 *dpos, const u64 *dneg, int ND, int dbase, u64 *ws, int nsl) {
    u64 *wpos = ws, *wneg = ws + nsl;
    for (int i = threadIdx.x; i < 2 * ND; i += blockDim.x) {
        const bool ng = i >= ND;
        const int dd = ng ? i - ND : i;
        const u64 v = (ng ? dneg : dpos)[dd];
        if (!v) continue;
        const int d = dbase + dd, sl = d >> 2, r = 8 * (d & 3);
        const u32 p0 = (u32)(v << r);
        const u32 p1 = r ? (u32)(v >> (32 - r)) : (u32)(v >> 32);
        const u32 p2 = r ? (u32)(v >> (64 - r)) : 0u;
        u64 *dst = ng ? wneg : wpos;
        if (p0 && sl < nsl) atomicAdd(&dst[sl], (u64)p0);
        if (p1 && sl + 1 < nsl) atomicAdd(&dst[sl + 1], (u64)p1);
        if (p2 && sl + 2 < nsl) atomicAdd(&dst[sl + 2], (u64)p2);
    }
    __threadfence();
    __syncthreads();
}

// the last CTA (ticket) takes the slots (re-zeroing them) and normalises
// positive - negative into LA two's-complement limbs (negated for sign < 0)
__device__ void finish_last_cta(u64 *ws, int nsl, u32 *ticket, u32 *result, int LA, int sign, unsigned char *smem,
                                u32 *s_last) {
    if (threadIdx.x == 0) *s_last = (atomicAdd(ticket, 1u) == gridDim.x - 1) ? 1u : 0u;
    __syncthreads();
    if (!*s_last) return;
    __threadfence();
    u64 *wpos = ws, *wneg = ws + nsl;
    u64 *sp = reinterpret_cast<u64 *>(smem), *sn = sp + nsl;    // reuse shared memory (nsl <= MAX_SLOTS)
    for (int i = threadIdx.x; i < nsl; i += blockDim.x) { sp[i] = atomicExch(&wpos[i], 0ull); sn[i] = atomicExch(&wneg[i], 0ull); }
    __syncthreads();
    if (threadIdx.x == 0) {
        *ticket = 0u;
        u64 cp = 0, cn = 0;
        u32 borrow = 0, cneg = sign < 0 ? 1u : 0u;
        for (int j = 0; j < LA; ++j) {
            u64 tp = cp, tn = cn;
            if (j < nsl) { tp += (u32)sp[j]; tn += (u32)sn[j]; }
            if (j >= 1 && j - 1 < nsl) { tp += sp[j - 1] >> 32; tn += sn[j - 1] >> 32; }
            cp = tp >> 32; cn = tn >> 32;
            const u64 d = (u64)(u32)tp - (u32)tn - borrow;
            borrow = (u32)(d >> 63);
            if (sign < 0) {
                const u64 g = (u64)(~(u32)d) + cneg;
                cneg = (u32)(g >> 32);
                result[j] = (u32)g;
            } else {
                result[j] = (u32)d;
            }
        }
    }
}

// A role's operand tile: digits [dbase, dbase + extent) of one column; its raw
// stage holds the limbs lo .. lo + nl - 1 (+ the top limb when only the sign
// digit falls into the tile)
struct Opnd {
    int dbase, L, lo, nl, raw_off;   // raw_off: first raw slot (limbs)
    bool extra_top;                  // raw slot nl holds limb L - 1
    int ndig;                        // digits to write: [0, ndig) local
};

template <int KC>
__global__ void __launch_bounds__(THREADS + 32, 1) k_contract_tc(const TcArgs P, const __grid_constant__ CUtensorMap tA,
                                                                  const __grid_constant__ CUtensorMap tB) {
    constexpr int DRAIN_CHUNKS = 32768 / KC; // s32 accumulators drained every 32768 rows
    extern __shared__ __align__(1024) unsigned char smem[];
    __shared__ u32 s_taddr;
    __shared__ __align__(8) u64 s_full[NRAW_MAX], s_empty[NRAW_MAX], s_cfull[2], s_mdone[2], s_drained;
    __shared__ u32 s_last;

    // warps 0..THREADS/32-1 transform raw limb rows into the MMA layout (warps
    // 0-3 also drain TMEM lanes 0-127); the last warp issues the TMA copies and the MMAs
    const int NRAW = P.nst;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int role = blockIdx.x % P.n_roles, rblock = blockIdx.x / P.n_roles;
    const int mt = role % P.n_mtiles, grp = role / P.n_mtiles;
    const int MA = 4 * P.La + 1, MB = 4 * P.Lb + 1;
    const int x0 = 128 * mt, y0 = 512 * grp;               // first digits of this role
    const int ny = min(512, MB - y0);
    const int W = (ny + 15) & ~15;                         // MMA N extent (<= 512)
    const int N0 = W > 256 ? 256 : W, N1 = W - N0;         // two N tiles at most
    const u32 tcols = W <= 32 ? 32 : W <= 64 ? 64 : W <= 128 ? 128 : W <= 256 ? 256 : 512;

    // raw stage = TMA boxes [ABOX limbs | P.bbox limbs] x KC rows (rows >= n and
    // limbs >= L arrive zero-filled); a box starts one limb early when only the
    // sign digit of its column falls into the tile (it needs the top limb)
    Opnd oa, ob;
    oa.dbase = x0; oa.L = P.La; oa.lo = x0 / 4; oa.nl = max(0, min(P.La, (x0 + 128) / 4) - oa.lo);
    oa.extra_top = (4 * P.La >= x0 && 4 * P.La < x0 + 128) && oa.nl == 0;
    oa.ndig = min(128, MA - x0);
    oa.raw_off = 0;
    ob.dbase = y0; ob.L = P.Lb; ob.lo = y0 / 4; ob.nl = max(0, min(P.Lb, (y0 + W) / 4) - ob.lo);
    ob.extra_top = (4 * P.Lb >= y0 && 4 * P.Lb < y0 + W) && ob.nl == 0;
    ob.ndig = ny;
    ob.raw_off = P.abox;
    const int box_a = oa.extra_top ? P.La - 1 : oa.lo, box_b = ob.extra_top ? P.Lb - 1 : ob.lo;
    const int nraw_limbs = P.abox + P.bbox;

    // shared: [NRAW raw stages: limb x KC words][2 canonical stages: A 128 x KC | B W x KC][digit sums]
    const int raw_bytes = nraw_limbs * KC * 4;
    const int a_bytes = 128 * KC, b_bytes = W * KC, st_bytes = a_bytes + b_bytes;
    const u32 LBO_A = (128 / 16) * 128, LBO_B = (u32)(W / 16) * 128;   // bytes per 8-row group of a tile
    unsigned char *raw0 = smem;
    unsigned char *canon0 = smem + NRAW * raw_bytes;
    const int ND = 128 + W;
    u64 *dpos = reinterpret_cast<u64 *>(canon0 + 2 * st_bytes);
    u64 *dneg = dpos + ND;

    for (int i = tid; i < (2 * st_bytes) / 16; i += blockDim.x) reinterpret_cast<uint4 *>(canon0)[i] = make_uint4(0, 0, 0, 0);
    for (int i = tid; i < 2 * ND; i += blockDim.x) dpos[i] = 0ull;
    __syncwarp();
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(&s_taddr)), "r"(tcols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        for (int i = 0; i < NRAW; ++i) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&s_full[i])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(&s_empty[i])), "r"(THREADS / 32));
        }
        for (int i = 0; i < 2; ++i) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(&s_cfull[i])), "r"(THREADS / 32));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&s_mdone[i])));
        }
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 4;" :: "r"(smem_u32(&s_drained)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const u32 taddr = s_taddr;

    const long long n = P.n;
    const long long nchunks = (n + KC - 1) / KC;
    // a contiguous range of chunks per row block: consecutive stages read
    // consecutive segments of every limb plane
    const long long c_begin = nchunks * rblock / P.n_rblocks, c_end = nchunks * (rblock + 1) / P.n_rblocks;
    const long long my_chunks = c_end - c_begin;
    auto is_drain = [&](int t) { return ((t + 1) % DRAIN_CHUNKS) == 0 || t == (int)my_chunks - 1; };

    if (warp == THREADS / 32) {
        // ---------------- control warp: bulk copies + MMA issue
        auto issue = [&](int t, int rs) {   // the role's limb rows of local chunk t -> raw stage rs = t % NRAW (2 TMA boxes)
            if (lane != 0) return;
            const int row0 = (int)((c_begin + t) * KC);
            const u32 mb = smem_u32(&s_full[rs]);
            const u32 tx = (u32)(nraw_limbs * KC * 4);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(mb), "r"(tx) : "memory");
            const u32 dst = smem_u32(raw0 + rs * raw_bytes);
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                         :: "r"(dst), "l"(&tA), "r"(row0), "r"(box_a), "r"(mb) : "memory");
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                         :: "r"(dst + (u32)(P.abox * KC * 4)), "l"(&tB), "r"(row0), "r"(box_b), "r"(mb) : "memory");
        };
        for (int t = 0; t < NRAW && t < (int)my_chunks; ++t) issue(t, t);
        // s32 accumulate, u8 x u8, A and B MN-major (bits 15, 16)
        const u32 idesc0 = (2u << 4) | (1u << 15) | (1u << 16) | ((u32)(N0 >> 3) << 17) | ((128u >> 4) << 24);
        const u32 idesc1 = (2u << 4) | (1u << 15) | (1u << 16) | ((u32)(N1 >> 3) << 17) | ((128u >> 4) << 24);
        int drains = 0, rs = 0;
        u32 rph = 0;                                       // raw stage rs, its use parity
        for (int t = 0; t < (int)my_chunks; ++t) {
            const int cs = t & 1;
            if (lane == 0) {
                mbar_wait(smem_u32(&s_cfull[cs]), (u32)((t >> 1) & 1));           // canonical stage written
                const bool fresh = (t == 0) || is_drain(t - 1);
                if (t > 0 && is_drain(t - 1)) mbar_wait(smem_u32(&s_drained), (u32)(drains++ & 1));   // TMEM read out
                asm volatile("tcgen05.fence::after_thread_sync;");
                const u32 a_addr = smem_u32(canon0 + cs * st_bytes), b_addr = a_addr + (u32)a_bytes;
#pragma unroll
                for (int kk = 0; kk < KC / 32; ++kk) {
                    const u32 acc = (!fresh || kk > 0) ? 1u : 0u;
                    const u64 da = umma_desc_mn(a_addr + kk * 4 * LBO_A, LBO_A);
                    const u64 db0 = umma_desc_mn(b_addr + kk * 4 * LBO_B, LBO_B);
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                 "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                                 :: "r"(taddr), "l"(da), "l"(db0), "r"(idesc0), "r"(acc));
                    if (N1 > 0) {
                        const u64 db1 = umma_desc_mn(b_addr + (N0 / 16) * 128 + kk * 4 * LBO_B, LBO_B);
                        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                     "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                                     :: "r"(taddr + (u32)N0), "l"(da), "l"(db1), "r"(idesc1), "r"(acc));
                    }
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                             :: "r"(smem_u32(&s_mdone[cs])));
                if (t + NRAW < (int)my_chunks) mbar_wait(smem_u32(&s_empty[rs]), rph);   // raw stage read
            }
            __syncwarp();
            if (t + NRAW < (int)my_chunks) issue(t + NRAW, rs);
            if (++rs == NRAW) { rs = 0; rph ^= 1u; }
        }
    } else {
        // ---------------- transform warps: word transpose into the MN-major layout.
        // Task = (16-digit chunk c of a tile, row r): the chunk's bytes in row r
        // are the little-endian words of limbs 4c..4c+3 -> 4 LDS.32 (consecutive
        // rows across lanes) and one STS.128 (lanes 16 B apart: conflict-free).
        // The word at the sign digit's position is the row's sign bit; words of
        // limbs beyond the column stay zero.  Task list fixed for the whole run.
        constexpr int MAXT = KC == 256 ? 16 : 10;                       // (8 + 32) chunks x 128 rows / 512 threads
        const int ca_used = min(8, (oa.ndig + 15) / 16), cb_used = (ob.ndig + 15) / 16;
        const int tasks = (ca_used + cb_used) * KC;
        u32 t_src[MAXT], t_dst[MAXT], t_mode[MAXT];   // raw word offset of the first word; canonical byte offset; word kinds
        int nt = 0;
#pragma unroll
        for (int k = 0; k < MAXT; ++k) {
            t_src[k] = 0; t_dst[k] = 0; t_mode[k] = 0;
            const int task = tid + THREADS * k;
            if (task >= tasks) continue;
            nt = k + 1;
            const int cidx = task / KC, r = task % KC;
            const bool isA = cidx < ca_used;
            const Opnd &o = isA ? oa : ob;
            const int c = isA ? cidx : cidx - ca_used;
            const int blo = isA ? box_a : box_b;
            const int nbox = isA ? P.abox : P.bbox;
            // word q of the chunk = limb (dbase/4 + 4c + q); kinds: 0 normal, 1 sign, 2 zero
            u32 mode = 0;
            int first_slot = -1;
            for (int q = 0; q < 4; ++q) {
                const int lj = o.dbase / 4 + 4 * c + q;        // global limb index of this word
                u32 kind;
                if (lj < o.L) kind = 0;
                else if (lj == o.L) kind = 1;
                else kind = 2;
                if (kind == 0 && first_slot < 0) first_slot = lj - blo;
                mode |= kind << (2 * q);
            }
            // sign word reads the top limb's slot
            const int sign_slot = o.L - 1 - blo;
            if (first_slot < 0) first_slot = sign_slot;          // chunk holding only the sign digit
            (void)nbox;
            t_src[k] = (u32)((o.raw_off + first_slot) * KC + r) | ((u32)(sign_slot - first_slot + 8) << 24);
            t_dst[k] = (u32)((isA ? 0 : a_bytes) + (r >> 3) * (int)(isA ? LBO_A : LBO_B) + c * 128 + (r & 7) * 16);
            t_mode[k] = mode;
        }
        int rs = 0;
        u32 rph = 0;
        for (int t = 0; t < (int)my_chunks; ++t, rs = (rs + 1 == NRAW) ? 0 : rs + 1, rph ^= (rs == 0) ? 1u : 0u) {
            const int cs = t & 1;
            mbar_wait(smem_u32(&s_full[rs]), rph);                                  // raw rows landed
            if (t >= 2) mbar_wait(smem_u32(&s_mdone[cs]), (u32)(((t - 2) >> 1) & 1));  // canonical stage free
            const u32 *raw = reinterpret_cast<const u32 *>(raw0 + rs * raw_bytes);
            unsigned char *canon = canon0 + cs * st_bytes;
#pragma unroll
            for (int k = 0; k < MAXT; ++k) {
                if (k >= nt) break;
                const u32 src = t_src[k] & 0xFFFFFFu, mode = t_mode[k];
                uint4 out;
                if (mode == 0) {                                // the common case: 4 limbs of the column
                    out.x = raw[src]; out.y = raw[src + KC]; out.z = raw[src + 2 * KC]; out.w = raw[src + 3 * KC];
                } else {
                    const int sdel = (int)(t_src[k] >> 24) - 8;
                    const u32 sgn = raw[(int)src + sdel * KC] >> 31;
                    u32 wq[4];
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const u32 kind = (mode >> (2 * q)) & 3u;
                        wq[q] = kind == 0 ? raw[src + q * KC] : kind == 1 ? sgn : 0u;
                    }
                    out = make_uint4(wq[0], wq[1], wq[2], wq[3]);
                }
                *reinterpret_cast<uint4 *>(canon + t_dst[k]) = out;
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0) {
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(&s_empty[rs])) : "memory");
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(&s_cfull[cs])) : "memory");
            }
            if (warp < 4 && is_drain(t)) {
                // accumulator drain: MMAs of chunk t done -> D[x][y] into the digit sums
                mbar_wait(smem_u32(&s_mdone[cs]), (u32)((t >> 1) & 1));
                asm volatile("tcgen05.fence::after_thread_sync;");
                const int x = x0 + 32 * warp + lane;       // this thread's digit of c_a (TMEM lane)
                const bool xs = (x == 4 * P.La), xv = x < MA;
                for (int c0 = 0; c0 < W; c0 += 32) {
                    u32 v[32];
                    const u32 ta = taddr + ((u32)(32 * warp) << 16) + (u32)c0;
                    asm volatile(
                        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
                          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
                          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
                        : "r"(ta));
                    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                    if (xv) {
#pragma unroll
                        for (int k = 0; k < 32; ++k) {
                            const int y = y0 + c0 + k;
                            if (y < MB && v[k]) {
                                const bool neg = xs != (y == 4 * P.Lb);
                                atomicAdd(&(neg ? dneg : dpos)[x - x0 + y - y0], (u64)v[k]);
                            }
                        }
                    }
                }
                asm volatile("tcgen05.fence::before_thread_sync;");
                __syncwarp();
                if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(&s_drained)) : "memory");
            }
        }
    }
    __syncthreads();

    commit_digit_sums(dpos, dneg, ND, x0 + y0, P.ws, P.nsl);
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(taddr), "r"(tcols));
    finish_last_cta(P.ws, P.nsl, P.ticket, P.result, P.LA, P.sign, smem, &s_last);
}

// ---------------------------------------------------------------------------
// Limb-quad columns (UP_LAYOUT_QUADS, up.h): quad g of row i is the 16 bytes
// of limbs 4g..4g+3 at ((uint4 *)data)[g*ld + i], limb L holds the sign flag
// (1 = negative) and the padding limbs are zero.  A quad plane is one
// contiguous run of 16-byte rows, so a 2-D TMA box {2 KC u64 = KC rows, nq
// quads} (rows >= n and quads >= G zero-filled) lands in shared memory as
// [quad][row][16 B]: 8 consecutive rows of one quad are exactly one MN-major
// core matrix (16 digit bytes x 8 rows, 128 B), so the MMAs read the
// TMA-landed stage directly -- no transform warps.  (A 3-D box with a 16-byte
// inner dimension was measured at 3.6 TB/s: the copy engine's per-row cost;
// the 2 KB inner rows of this one are not limited by it.)  Descriptors: K-direction core-matrix stride (LBO) 128 B,
// MN-direction stride (SBO) KC * 16 B (the next quad), the layout
// tools/tc_probe.cu mode 2 verified with other strides.
//
// Warps: 0-3 drain TMEM (lane = digit of c_a), 4 = TMA producer, 5 = MMA
// issuer.  Accumulators are double-buffered in TMEM when two fit, so the MMA
// warp never waits for a drain of the previous window.

constexpr int TQ_THREADS = 192;
constexpr int TQ_MAXST = 8;

struct TqArgs {
    long long n;
    int La, Lb, Ga, Gb;           // limbs, quads (incl. the sign-flag limb)
    int n_mtiles, n_groups, n_roles, n_rblocks;
    int nqb;                      // B box quads (<= 32)
    int nst;                      // stages
    u64 *ws;
    u32 *ticket;
    u32 *result;
    int LA, nsl, sign;
};

__device__ __forceinline__ u64 umma_desc(u32 saddr, u32 lbo, u32 sbo) {
    return (u64)((saddr >> 4) & 0x3FFFu) | ((u64)((lbo >> 4) & 0x3FFFu) << 16) | ((u64)((sbo >> 4) & 0x3FFFu) << 32) |
           (1ull << 46);
}

template <int KC>
__global__ void __launch_bounds__(TQ_THREADS, 1) k_contract_tq(const TqArgs P, const __grid_constant__ CUtensorMap tA,
                                                               const __grid_constant__ CUtensorMap tB) {
    constexpr int DRAIN_CHUNKS = 32768 / KC;
    extern __shared__ __align__(1024) unsigned char smem[];
    __shared__ u32 s_taddr;
    __shared__ __align__(8) u64 s_full[TQ_MAXST], s_empty[TQ_MAXST], s_mdone[2], s_drained[2];
    __shared__ u32 s_last;

    const int NST = P.nst;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int role = blockIdx.x % P.n_roles, rblock = blockIdx.x / P.n_roles;
    const int mt = role % P.n_mtiles, grp = role / P.n_mtiles;
    const int MA = 4 * P.La + 1, MB = 4 * P.Lb + 1;        // digits incl. the sign digit
    const int x0 = 128 * mt, y0 = 512 * grp;
    const int nqw = min(32, P.Gb - 32 * grp);              // quads of c_b in this group
    const int W = 16 * nqw;                                // MMA N extent
    const int N0 = W > 256 ? 256 : W, N1 = W - N0;
    const u32 tcols = W <= 32 ? 32 : W <= 64 ? 64 : W <= 128 ? 128 : W <= 256 ? 256 : 512;
    const int nbuf = tcols <= 256 ? 2 : 1;                 // TMEM accumulators

    const int a_bytes = 8 * KC * 16, st_bytes = a_bytes + P.nqb * KC * 16;
    const int ND = 128 + W;
    u64 *dpos = reinterpret_cast<u64 *>(smem + NST * st_bytes);
    u64 *dneg = dpos + ND;
    for (int i = tid; i < 2 * ND; i += blockDim.x) dpos[i] = 0ull;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(&s_taddr)), "r"(tcols * nbuf));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        for (int i = 0; i < NST; ++i) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&s_full[i])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&s_empty[i])));
        }
        for (int i = 0; i < 2; ++i) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&s_mdone[i])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 4;" :: "r"(smem_u32(&s_drained[i])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const u32 taddr = s_taddr;

    const long long nchunks = (P.n + KC - 1) / KC;
    const long long c_begin = nchunks * rblock / P.n_rblocks, c_end = nchunks * (rblock + 1) / P.n_rblocks;
    const int my_chunks = (int)(c_end - c_begin);
    // accumulation window w covers local chunks [w * DRAIN_CHUNKS, ...); it
    // ends at a drain
    auto is_drain = [&](int t) { return ((t + 1) % DRAIN_CHUNKS) == 0 || t == my_chunks - 1; };

    if (warp == 4) {
        // ---------------- TMA producer
        if (lane == 0) {
            const u32 tx = (u32)st_bytes;
            for (int t = 0; t < my_chunks; ++t) {
                const int s = t % NST;
                if (t >= NST) mbar_wait(smem_u32(&s_empty[s]), (u32)(((t / NST) - 1) & 1));
                const int row0 = (int)((c_begin + t) * KC);
                const u32 mb = smem_u32(&s_full[s]);
                const u32 dst = smem_u32(smem + s * st_bytes);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(mb), "r"(tx) : "memory");
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                             :: "r"(dst), "l"(&tA), "r"(2 * row0), "r"(8 * mt), "r"(mb) : "memory");
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                             :: "r"(dst + (u32)a_bytes), "l"(&tB), "r"(2 * row0), "r"(32 * grp), "r"(mb) : "memory");
            }
        }
    } else if (warp == 5) {
        // ---------------- MMA issuer: s32 += u8 x u8, A and B MN-major
        if (lane == 0) {
            const u32 idesc0 = (2u << 4) | (1u << 15) | (1u << 16) | ((u32)(N0 >> 3) << 17) | ((128u >> 4) << 24);
            const u32 idesc1 = (2u << 4) | (1u << 15) | (1u << 16) | ((u32)(N1 >> 3) << 17) | ((128u >> 4) << 24);
            const u32 SBO = (u32)KC * 16u;
            int win = 0;                                    // accumulation window
            bool fresh = true;
            for (int t = 0; t < my_chunks; ++t) {
                const int s = t % NST;
                const int buf = win % nbuf;
                if (fresh && win >= nbuf) mbar_wait(smem_u32(&s_drained[buf]), (u32)(((win - nbuf) / nbuf) & 1));
                mbar_wait(smem_u32(&s_full[s]), (u32)((t / NST) & 1));
                asm volatile("tcgen05.fence::after_thread_sync;");
                const u32 a_addr = smem_u32(smem + s * st_bytes), b_addr = a_addr + (u32)a_bytes;
                const u32 tacc = taddr + (u32)buf * tcols;
#pragma unroll
                for (int kk = 0; kk < KC / 32; ++kk) {
                    const u32 acc = (!fresh || kk > 0) ? 1u : 0u;
                    const u64 da = umma_desc(a_addr + kk * 512, 128, SBO);
                    const u64 db0 = umma_desc(b_addr + kk * 512, 128, SBO);
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                 "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                                 :: "r"(tacc), "l"(da), "l"(db0), "r"(idesc0), "r"(acc));
                    if (N1 > 0) {
                        const u64 db1 = umma_desc(b_addr + 16 * SBO + kk * 512, 128, SBO);
                        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                     "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
                                     :: "r"(tacc + (u32)N0), "l"(da), "l"(db1), "r"(idesc1), "r"(acc));
                    }
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                             :: "r"(smem_u32(&s_empty[s])));
                fresh = false;
                if (is_drain(t)) {
                    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                                 :: "r"(smem_u32(&s_mdone[buf])));
                    ++win;
                    fresh = true;
                }
            }
        }
    } else {
        // ---------------- drain warps 0-3: TMEM lane 32 * warp + lane = digit x of c_a
        const int x = x0 + 32 * warp + lane;
        const bool xs = (x == 4 * P.La), xv = x < MA;
        const int nwin = my_chunks > 0 ? (my_chunks + DRAIN_CHUNKS - 1) / DRAIN_CHUNKS : 0;
        for (int win = 0; win < nwin; ++win) {
            const int buf = win % nbuf;
            mbar_wait(smem_u32(&s_mdone[buf]), (u32)((win / nbuf) & 1));
            asm volatile("tcgen05.fence::after_thread_sync;");
            for (int c0 = 0; c0 < W; c0 += 32) {
                u32 v[32];
                const u32 ta = taddr + (u32)buf * tcols + ((u32)(32 * warp) << 16) + (u32)c0;
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                    "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                    : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                      "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
                      "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
                      "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
                    : "r"(ta));
                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                if (xv) {
#pragma unroll
                    for (int k = 0; k < 32; ++k) {
                        const int y = y0 + c0 + k;
                        if (c0 + k < W && y < MB && v[k]) {
                            const bool neg = xs != (y == 4 * P.Lb);
                            atomicAdd(&(neg ? dneg : dpos)[x - x0 + y - y0], (u64)v[k]);
                        }
                    }
                }
            }
            asm volatile("tcgen05.fence::before_thread_sync;");
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(&s_drained[buf])) : "memory");
        }
    }
    __syncthreads();

    commit_digit_sums(dpos, dneg, ND, x0 + y0, P.ws, P.nsl);
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(taddr), "r"(tcols * nbuf));
    finish_last_cta(P.ws, P.nsl, P.ticket, P.result, P.LA, P.sign, smem, &s_last);
}

typedef CUresult (*EncodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// 2-D map of a column's limb planes: dim 0 = rows (n, contiguous), dim 1 = limbs (stride ld words)
cudaError_t make_tmap(CUtensorMap *m, const u32 *data, long long n, int L, long long ld, int box_rows, int box_limbs) {
    static EncodeTiled enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult q;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &q);
        if (e != cudaSuccess) return e;
        if (q != cudaDriverEntryPointSuccess || !enc) return cudaErrorSymbolNotFound;
    }
    const cuuint64_t dims[2] = {(cuuint64_t)(n > 0 ? n : 1), (cuuint64_t)L};
    const cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
    const cuuint32_t box[2] = {(cuuint32_t)box_rows, (cuuint32_t)box_limbs};
    const cuuint32_t es[2] = {1, 1};
    const CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, (void *)data, dims, strides, box, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

// 2-D map of a limb-quad column: dim 0 = a quad plane as u64 (2 per row,
// contiguous), dim 1 = quads (ld * 16 B apart); box {2 KC, nq}
cudaError_t make_tmap_quads(CUtensorMap *m, const u32 *data, long long n, int G, long long ld, int box_rows, int box_q) {
    static EncodeTiled enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult q;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &q);
        if (e != cudaSuccess) return e;
        if (q != cudaDriverEntryPointSuccess || !enc) return cudaErrorSymbolNotFound;
    }
    const cuuint64_t dims[2] = {(cuuint64_t)(n > 0 ? 2 * n : 2), (cuuint64_t)G};
    const cuuint64_t strides[1] = {(cuuint64_t)ld * 16};
    const cuuint32_t box[2] = {(cuuint32_t)(2 * box_rows), (cuuint32_t)box_q};
    const cuuint32_t es[2] = {1, 1};
    const CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, (void *)data, dims, strides, box, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

template <int KC>
cudaError_t launch_tq(TqArgs P, const u32 *A, long long lda, const u32 *B, long long ldb, int num_sms, cudaStream_t st) {
    CUtensorMap tA, tB;
    cudaError_t e = make_tmap_quads(&tA, A, P.n, P.Ga, lda, KC, 8);
    if (e != cudaSuccess) return e;
    e = make_tmap_quads(&tB, B, P.n, P.Gb, ldb, KC, P.nqb);
    if (e != cudaSuccess) return e;
    const size_t st_bytes = (size_t)(8 + P.nqb) * KC * 16;
    const int Wmax = 16 * P.nqb;
    const size_t sums = sizeof(u64) * (size_t)(2 * (128 + Wmax));
    P.nst = TQ_MAXST;
    while (P.nst > 2 && (size_t)P.nst * st_bytes + sums > 225 * 1024) --P.nst;
    size_t smem = (size_t)P.nst * st_bytes + sums;
    if (smem > 225 * 1024) return cudaErrorInvalidValue;
    if (smem < sizeof(u64) * 2 * (size_t)P.nsl) smem = sizeof(u64) * 2 * (size_t)P.nsl;
    e = cudaFuncSetAttribute(k_contract_tq<KC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const long long nchunks = (P.n + KC - 1) / KC;
    long long rb = (long long)num_sms / P.n_roles;
    if (rb < 1) rb = 1;
    if (rb > nchunks) rb = nchunks > 0 ? nchunks : 1;
    if (const char *f = getenv("UP_TC_RBLOCKS")) rb = atoll(f) > 0 ? atoll(f) : rb;   // tests: force mid-run drains
    P.n_rblocks = (int)rb;
    k_contract_tq<KC><<<(unsigned)(rb * P.n_roles), TQ_THREADS, smem, st>>>(P, tA, tB);
    return cudaGetLastError();
}

template <int KC>
cudaError_t launch_kc(TcArgs P, int W, int nraw_limbs, int num_sms, cudaStream_t st) {
    CUtensorMap tA, tB;
    cudaError_t e0 = make_tmap(&tA, P.A, P.n, P.La, P.lda, KC, P.abox);
    if (e0 != cudaSuccess) return e0;
    e0 = make_tmap(&tB, P.B, P.n, P.Lb, P.ldb, KC, P.bbox);
    if (e0 != cudaSuccess) return e0;
    const size_t sums = sizeof(u64) * (size_t)(2 * (128 + W));
    const size_t fixed = 2 * (size_t)(128 + W) * KC + sums;
    P.nst = NRAW_MAX;
    while (P.nst > 2 && (size_t)P.nst * nraw_limbs * KC * 4 + fixed > 225 * 1024) --P.nst;
    size_t smem = (size_t)P.nst * nraw_limbs * KC * 4 + fixed;
    if (smem > 225 * 1024) return cudaErrorInvalidValue;
    if (smem < sizeof(u64) * 2 * (size_t)P.nsl) smem = sizeof(u64) * 2 * (size_t)P.nsl;
    cudaError_t e = cudaFuncSetAttribute(k_contract_tc<KC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const int tcols = W <= 32 ? 32 : W <= 64 ? 64 : W <= 128 ? 128 : W <= 256 ? 256 : 512;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_contract_tc<KC>, THREADS + 32, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
    if (per_sm > 512 / tcols) per_sm = 512 / tcols;      // TMEM columns per SM
    if (per_sm > 2) per_sm = 2;
    const long long nchunks = (P.n + KC - 1) / KC;
    long long rb = ((long long)num_sms * per_sm) / P.n_roles;
    if (rb < 1) rb = 1;
    if (rb > nchunks) rb = nchunks > 0 ? nchunks : 1;
    if (const char *f = getenv("UP_TC_RBLOCKS")) rb = atoll(f) > 0 ? atoll(f) : rb;   // tests: force mid-run drains
    P.n_rblocks = (int)rb;
    k_contract_tc<KC><<<(unsigned)(rb * P.n_roles), THREADS + 32, smem, st>>>(P, tA, tB);
    return cudaGetLastError();
}

}  // namespace

extern "C" {

// Slots of the global workspace the kernel needs (2 * nsl), for the caller's check.
int upk_contract_tc_slots(int La, int Lb) { return 2 * (La + Lb + 3); }

// SUM_rows(sign * c_a * c_b) into `result` (LA limbs, two's complement).
// ws: >= upk_contract_tc_slots u64, zero on entry (left zero); ticket zero.
cudaError_t upk_launch_contract_tc(const uint32_t *A, long long lda, int La, const uint32_t *B, long long ldb, int Lb,
                                   long long n, int sign, unsigned long long *ws, uint32_t *ticket, uint32_t *result,
                                   int LA, int num_sms, cudaStream_t st) {
    TcArgs P;
    P.A = A; P.B = B; P.lda = lda; P.ldb = ldb; P.n = n; P.La = La; P.Lb = Lb;
    const int MA = 4 * La + 1, MB = 4 * Lb + 1;
    P.n_mtiles = (MA + 127) / 128;
    P.n_groups = (MB + 511) / 512;
    P.n_roles = P.n_mtiles * P.n_groups;
    P.ws = ws; P.ticket = ticket; P.result = result; P.LA = LA; P.nsl = La + Lb + 3; P.sign = sign;
    if (P.nsl > MAX_SLOTS) return cudaErrorInvalidValue;
    const int W = ((MB < 512 ? MB : 512) + 15) & ~15;
    P.bbox = (W / 4 < Lb ? W / 4 : Lb) + 1;               // group limbs (+1: a sign-only tile starts one limb early)
    if (P.bbox > 128 + 1) P.bbox = 129;
    P.abox = La < ABOX_MAX ? La : ABOX_MAX;
    const int nraw = P.abox + P.bbox;
    if (nraw > MAX_ROLE_LIMBS) return cudaErrorInvalidValue;
    // stage depth (measured on B200, profiles/r01_kc/): 256 rows when 2 raw + 2
    // canonical stages fit (cfg3 p = 200: 1.098e10 -> 1.128e10 rows/s), else
    // 128 rows with >= 3 raw stages, else 64
    const size_t need256 = (size_t)2 * nraw * 256 * 4 + 2 * (size_t)(128 + W) * 256;
    const size_t need128 = (size_t)3 * nraw * 128 * 4 + 2 * (size_t)(128 + W) * 128;   // >= 3 raw stages at 128 rows
    const int max_tasks = (8 + W / 16) * 128;             // transform tasks per 128-row stage (<= 512 x MAXT)
    if (need256 + 16 * 1024 <= 220 * 1024 && max_tasks * 2 <= 512 * 16) return launch_kc<256>(P, W, nraw, num_sms, st);
    if (need128 + 16 * 1024 <= 220 * 1024 && max_tasks <= 5120) return launch_kc<128>(P, W, nraw, num_sms, st);
    return launch_kc<64>(P, W, nraw, num_sms, st);
}

// The same SUM over limb-quad columns (UP_LAYOUT_QUADS): A, B are the quad
// arrays (uint4 per row and quad, lda/ldb rows per quad plane); the columns
// hold La / Lb limbs plus the sign-flag limb (Ga / Gb = ceil((L + 1) / 4) quads).
cudaError_t upk_launch_contract_tq(const uint32_t *A, long long lda, int La, const uint32_t *B, long long ldb, int Lb,
                                   long long n, int sign, unsigned long long *ws, uint32_t *ticket, uint32_t *result,
                                   int LA, int num_sms, cudaStream_t st) {
    if (n >= (1ll << 30)) return cudaErrorInvalidValue;   // TMA coordinate 2 * row must fit int32
    TqArgs P;
    P.n = n; P.La = La; P.Lb = Lb;
    P.Ga = (La + 1 + 3) / 4; P.Gb = (Lb + 1 + 3) / 4;
    P.n_mtiles = (P.Ga + 7) / 8;
    P.n_groups = (P.Gb + 31) / 32;
    P.n_roles = P.n_mtiles * P.n_groups;
    P.nqb = P.Gb < 32 ? P.Gb : 32;
    P.ws = ws; P.ticket = ticket; P.result = result; P.LA = LA; P.nsl = La + Lb + 3; P.sign = sign;
    if (P.nsl > MAX_SLOTS) return cudaErrorInvalidValue;
    // stage rows: 128 (the TMA box's 256-element limit at 2 u64 per row) when
    // 3 stages fit, else 64
    const size_t row_bytes = (size_t)(8 + P.nqb) * 16, sums = sizeof(u64) * 2 * (128 + 16 * (size_t)P.nqb);
    if (3 * 128 * row_bytes + sums <= 225 * 1024) return launch_tq<128>(P, A, lda, B, ldb, num_sms, st);
    return launch_tq<64>(P, A, lda, B, ldb, num_sms, st);
}

}  // extern "C"
