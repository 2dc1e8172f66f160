// codegen.cpp -- kernel specialisation (row a2): emits one fused CUDA kernel
// per (typed expression, column types, variant) for NVRTC.
//
// P:L779-841 §III-B: DECIMAL sizes p, s, Lw are baked in as compile-time
// constants of the generated code; expand -> evaluate -> write in
// one kernel; §III-D2: constants (literals, 10^k alignment
// factors, 10^p overflow bounds) are converted once here, not per tuple.
// B200 layout: limb planes, one or four rows per thread with
// 128-bit loads, intermediates in registers, SUM fused into the same kernel.
#include "codegen.h"

#include <cstdlib>
#include <functional>
#include <map>
#include <sstream>

namespace uph {

std::string mul_variant_define() { return ""; }

std::string launch_bounds(int threads, int min_blocks) {
    std::string s = "__launch_bounds__(" + std::to_string(threads);
    if (min_blocks > 0) s += ", " + std::to_string(min_blocks);
    return s + ")";
}

namespace {

std::string limbs_init(const std::vector<uint32_t> &w) {
    std::ostringstream o;
    o << "{";
    for (size_t i = 0; i < w.size(); ++i) o << (i ? "," : "") << "0x" << std::hex << w[i] << std::dec << "u";
    o << "}";
    return o.str();
}

int mag_limbs_of_pow10(int k) {   // limbs of the magnitude 10^k - 1 (at least 1)
    int bl = HBig::pow10(k).bitlen();   // bitlen(10^k - 1) <= bitlen(10^k)
    return std::max(1, (bl + 31) / 32);
}

// Window of the top-limb division decision (div_top_decide in up_dev.cuh):
// T divisor limbs, T = max(limbs(C), limbs(q)) + 1 (UP_DIVTOP_T2: + 2), so an
// undecided row has probability ~(q0 + C)/v_h, below 2^-30 for a divisor whose
// top limb is not tiny (cfg3: ~2^-33); undecided rows run the full division,
// so the window only trades speed.  Used when the divisor is wider than the
// window and the dividend reaches into it.  Returns T, or 0.
int div_top_window(const Node *n) {
    if (n->op != Op::Div) return 0;
    const int La = n->l->L, Lb = n->r->L;
    const int NC = (int)HBig::pow10(n->r->s + 4).w.size();
    const int T = std::max(NC, n->L) + 1;
    const int E = Lb - T;
    return (E > 0 && La > E) ? T : 0;
}

// columns read only as operands of top-limb divisions are not loaded whole:
// those divisions read the limbs they need from global memory
void div_only_uses(const Node *n, std::vector<int> &uses, std::vector<int> &div_uses) {
    if (!n) return;
    if (n->op == Op::Col) { uses[(size_t)n->col]++; return; }
    if (div_top_window(n)) {
        for (const Node *ch : {n->l.get(), n->r.get()}) {
            if (ch->op == Op::Col) { uses[(size_t)ch->col]++; div_uses[(size_t)ch->col]++; }
            else div_only_uses(ch, uses, div_uses);
        }
        return;
    }
    div_only_uses(n->l.get(), uses, div_uses);
    div_only_uses(n->r.get(), uses, div_uses);
}

struct Emitter {
    std::ostringstream o;
    std::ostringstream pre;   // out-of-line helpers, emitted before eval_row
    int tmp = 0;
    std::vector<bool> lazy;   // column c is read from global memory by the divisions that use it
    std::vector<bool> quad;   // column c is stored as limb quads (limb j at g + (j>>2)*l + (j&3))
    std::string fresh(const char *pfx) { return std::string(pfx) + std::to_string(tmp++); }
    bool is_lazy(const Node *n) const { return n->op == Op::Col && (size_t)n->col < lazy.size() && lazy[(size_t)n->col]; }
    // limb j (static) of operand n: register array x, or a global load for a lazy column
    std::string limb(const Node *n, const std::string &x, int j) const {
        if (is_lazy(n)) return "__ldg(g" + std::to_string(n->col) + " + " + lazy_off(n->col, j) + ")";
        return x + "[" + std::to_string(j) + "]";
    }
    // limb j of the decision window: for a lazy limb-quad column the window's
    // quads are loaded once with 16-byte loads (and shared by the two operands
    // when they are the same column)
    std::map<std::pair<int, int>, std::string> wq;   // (column, quad) -> uint4 of this division's window
    std::string top_limb(const Node *n, const std::string &x, int j) {
        if (!is_lazy(n)) return limb(n, x, j);
        if (!quad[(size_t)n->col]) {   // plane limb, requested before the decision's branches
            const std::pair<int, int> key(n->col, 1000000 + j);
            auto it = wq.find(key);
            if (it == wq.end()) {
                std::string v = fresh("w");
                o << "    const u32 " << v << " = ld_issue1(g" << n->col << " + " << lazy_off(n->col, j) << ");\n";
                it = wq.emplace(key, v).first;
            }
            return it->second;
        }
        const auto key = std::make_pair(n->col, j >> 2);
        auto it = wq.find(key);
        if (it == wq.end()) {
            std::string v = fresh("q");
            o << "    const uint4 " << v << " = ld_issue4(g" << n->col << " + (long long)" << (j >> 2) << " * l" << n->col << ");\n";
            it = wq.emplace(key, v).first;
        }
        static const char *f[4] = {".x", ".y", ".z", ".w"};
        return it->second + f[j & 3];
    }
    // the whole operand as a register array (loads a lazy column)
    std::string whole(const Node *n, const std::string &x) {
        if (!is_lazy(n)) return x;
        std::string t = fresh("t");
        o << "    u32 " << t << "[" << n->L << "];\n#pragma unroll\n    for (int j = 0; j < " << n->L << "; ++j) " << t
          << "[j] = __ldg(g" << n->col << " + " << lazy_off(n->col, -1) << ");\n";
        return t;
    }
    // word offset of limb j (-1: the loop variable j) of a lazy column from its row pointer
    std::string lazy_off(int col, int j) const {
        const std::string J = j < 0 ? "j" : std::to_string(j), l = "l" + std::to_string(col);
        if ((size_t)col < quad.size() && quad[(size_t)col])
            return j < 0 ? "(long long)(j >> 2) * " + l + " + (j & 3)"
                         : "(long long)" + std::to_string(j >> 2) + " * " + l + " + " + std::to_string(j & 3);
        return "(long long)" + J + " * " + l;
    }

    // constant array of exactly `n` limbs holding v (truncated / zero padded)
    std::string konst(const HBig &v, int n) {
        std::string k = fresh("k");
        std::vector<uint32_t> w((size_t)n, 0);
        for (int i = 0; i < n; ++i) w[(size_t)i] = v.limb((size_t)i);
        o << "    const u32 " << k << "[" << n << "] = " << limbs_init(w) << ";\n";
        return k;
    }

    // x (child with Lx limbs) scaled by 10^k into L limbs, signed
    std::string aligned(const std::string &x, int Lx, int k, int L) {
        std::string t = fresh("t");
        if (k == 0) {
            o << "    u32 " << t << "[" << L << "]; sext<" << Lx << "," << L << ">(" << t << ", " << x << ");\n";
            return t;
        }
        HBig c = HBig::pow10(k);
        int Lc = (int)c.w.size();
        int Lcd = std::min(Lc, L);
        long cost_direct = (long)L * Lcd;
        long cost_abs = (long)Lx * Lc + 3L * L + Lx;
        if (cost_direct <= cost_abs) {
            std::string kc = konst(c, Lcd);
            o << "    u32 " << t << "[" << L << "]; mul_signed_direct<" << Lx << "," << Lcd << "," << L << ">(" << t << ", " << x << ", " << kc << ");\n";
        } else {
            std::string kc = konst(c, Lc);
            o << "    u32 " << t << "[" << L << "]; mul_signed_abs<" << Lx << "," << Lc << "," << L << ">(" << t << ", " << x << ", " << kc << ", 0u);\n";
        }
        return t;
    }

    std::string emit(const Node *n) {
        switch (n->op) {
        case Op::Col: return "x" + std::to_string(n->col);
        case Op::Lit: {
            std::string t = fresh("t");
            o << "    const u32 " << t << "[" << n->L << "] = " << limbs_init(n->lit.twos(n->L, false)) << ";\n";
            return t;
        }
        case Op::Cast: {   // exact upward re-typing (optimiser output)
            std::string a = emit(n->l.get());
            return aligned(a, n->l->L, n->s - n->l->s, n->L);
        }
        case Op::Neg: {
            std::string a = emit(n->l.get());
            std::string t = fresh("t");
            o << "    u32 " << t << "[" << n->L << "]; sext<" << n->l->L << "," << n->L << ">(" << t << ", " << a << "); cond_neg(" << t << ", 1u);\n";
            return t;
        }
        default: break;
        }
        const Node *L_ = n->l.get(), *R_ = n->r.get();
        std::string a = emit(L_), b = emit(R_);
        const int L = n->L;
        std::string t = fresh("t");
        switch (n->op) {
        case Op::Add: case Op::Sub: {
            // align the smaller scale upward, x10^(s_hi - s_lo), then one carry chain
            std::string A = aligned(a, L_->L, n->s - L_->s, L);
            std::string B = aligned(b, R_->L, n->s - R_->s, L);
            o << "    u32 " << t << "[" << L << "]; " << (n->op == Op::Add ? "add" : "sub") << "<" << L << ">(" << t << ", " << A << ", " << B << ");\n";
            return t;
        }
        case Op::Mul: {
            const int La = L_->L, Lb = R_->L;
            long cost_direct = (long)L * (L + 1) / 2;
            long cost_abs = (long)La * Lb + 4L * L + 2L * (La + Lb);
            if (cost_direct <= cost_abs) {
                std::string ax = fresh("t"), bx = fresh("t");
                o << "    u32 " << ax << "[" << L << "]; sext<" << La << "," << L << ">(" << ax << ", " << a << ");\n";
                o << "    u32 " << bx << "[" << L << "]; sext<" << Lb << "," << L << ">(" << bx << ", " << b << ");\n";
                o << "    u32 " << t << "[" << L << "]; mul_mag<" << L << "," << L << "," << L << ">(" << t << ", " << ax << ", " << bx << ");\n";
            } else {
                std::string ub = fresh("t"), nb = fresh("n");
                o << "    u32 " << ub << "[" << Lb << "], " << nb << "; abs_copy(" << ub << ", " << b << ", " << nb << ");\n";
                o << "    u32 " << t << "[" << L << "]; mul_signed_abs<" << La << "," << Lb << "," << L << ">(" << t << ", " << a << ", " << ub << ", " << nb << ");\n";
            }
            return t;
        }
        case Op::Div: {
            // Q = sign * trunc(|A| * 10^(s2+4) / |B|)  (reading Q4)
            const int La = L_->L, Lb = R_->L;
            const int k = R_->s + 4;
            const int NU = mag_limbs_of_pow10(L_->p + k);
            HBig c = HBig::pow10(k);
            std::string ua = fresh("t"), na = fresh("n"), ub = fresh("t"), nb = fresh("n"), uu = fresh("t"), rr = fresh("t");
            std::string kc = konst(c, (int)c.w.size());
            const int T = div_top_window(n);
            if (T) {
                // top-limb decision (div_top_decide), the full Knuth division only for undecided rows
                const int E = Lb - T, NAH = La - E;
                std::string ah = fresh("t"), vh = fresh("t");
                // the window's limbs (quad columns: their 16-byte loads are emitted here)
                wq.clear();
                std::vector<std::string> av, bv;
                for (int j = 0; j < NAH; ++j) av.push_back(top_limb(L_, a, E + j));
                for (int j = 0; j < T; ++j) bv.push_back(top_limb(R_, b, E + j));
                const std::string atop = top_limb(L_, a, La - 1), btop = top_limb(R_, b, Lb - 1);
                // signs in {0,1} (cond_neg's contract); complement masks 0 - sign
                o << "    u32 " << t << "[" << L << "], " << na << " = " << atop << " >> 31, " << nb << " = " << btop << " >> 31;\n";
                o << "    u32 " << ah << "[" << NAH << "], " << vh << "[" << T << "];\n";
                for (int j = 0; j < NAH; ++j) o << "    " << ah << "[" << j << "] = " << av[(size_t)j] << " ^ (0u - " << na << ");\n";
                for (int j = 0; j < T; ++j) o << "    " << vh << "[" << j << "] = " << bv[(size_t)j] << " ^ (0u - " << nb << ");\n";
                o << "    if (!div_top_decide<" << NAH << "," << T << "," << c.w.size() << "," << L << ">(" << t << ", " << ah << ", " << vh << ", " << kc << ")) {\n";
                if (is_lazy(L_) && is_lazy(R_)) {
                    // both operands are columns: the (rare) full division runs out
                    // of line, so its wide arrays do not share the row loop's registers
                    const std::string fn = fresh("divfb"), rt = fn + "_r";
                    const int la = L_->col, lb = R_->col;
                    auto ld = [&](int col, const char *g, const char *l) {
                        const bool qd = quad[(size_t)col];
                        return std::string("__ldg(") + g + " + " + (qd ? std::string("(long long)(j >> 2) * ") + l + " + (j & 3)" : std::string("(long long)j * ") + l) + ")";
                    };
                    pre << "struct " << rt << " { u32 w[" << L << "]; u32 fl; };\n";
                    pre << "__device__ __noinline__ " << rt << " " << fn << "(const u32 *__restrict__ ga, long long la, const u32 *__restrict__ gb, long long lb) {\n";
                    pre << "    const u32 kc[" << c.w.size() << "] = " << limbs_init(std::vector<uint32_t>(c.w.begin(), c.w.end())) << ";\n";
                    pre << "    u32 fa[" << La << "], fb[" << Lb << "];\n";
                    pre << "#pragma unroll\n    for (int j = 0; j < " << La << "; ++j) fa[j] = " << ld(la, "ga", "la") << ";\n";
                    pre << "#pragma unroll\n    for (int j = 0; j < " << Lb << "; ++j) fb[j] = " << ld(lb, "gb", "lb") << ";\n";
                    pre << "    u32 ua[" << La << "], ub[" << Lb << "], na, nb; abs_copy(ua, fa, na); abs_copy(ub, fb, nb);\n";
                    pre << "    u32 uu[" << NU << "]; mul_mag<" << La << "," << c.w.size() << "," << NU << ">(uu, ua, kc);\n";
                    pre << "    u32 rr[" << Lb << "]; " << rt << " r;\n";
                    pre << "    r.fl = divmod_mag<" << NU << "," << Lb << "," << L << ",false>(r.w, rr, uu, ub);\n";
                    pre << "    return r;\n}\n\n";
                    o << "    { const " << rt << " r = " << fn << "(g" << la << ", l" << la << ", g" << lb << ", l" << lb << "); fl |= r.fl;\n";
                    o << "#pragma unroll\n      for (int j = 0; j < " << L << "; ++j) " << t << "[j] = r.w[j]; }\n";
                    o << "    }\n";
                    std::string kb = konst(HBig::pow10(n->p), L);
                    o << "    if (!lt(" << t << ", " << kb << ")) fl |= F_OVERFLOW;\n";
                    o << "    cond_neg(" << t << ", " << na << " ^ " << nb << ");\n";
                    return t;
                }
                const std::string fa = whole(L_, a), fb = whole(R_, b);
                o << "    u32 " << ua << "[" << La << "], " << ub << "[" << Lb << "], " << na << "x, " << nb << "x; abs_copy(" << ua << ", " << fa << ", " << na << "x); abs_copy(" << ub << ", " << fb << ", " << nb << "x);\n";
                o << "    u32 " << uu << "[" << NU << "]; mul_mag<" << La << "," << c.w.size() << "," << NU << ">(" << uu << ", " << ua << ", " << kc << ");\n";
                o << "    u32 " << rr << "[" << Lb << "];\n";
                o << "    fl |= divmod_mag<" << NU << "," << Lb << "," << L << ",false>(" << t << ", " << rr << ", " << uu << ", " << ub << ");\n";
                o << "    }\n";
            } else {
            o << "    u32 " << ua << "[" << La << "], " << na << "; abs_copy(" << ua << ", " << a << ", " << na << ");\n";
            o << "    u32 " << ub << "[" << Lb << "], " << nb << "; abs_copy(" << ub << ", " << b << ", " << nb << ");\n";
            o << "    u32 " << uu << "[" << NU << "]; mul_mag<" << La << "," << c.w.size() << "," << NU << ">(" << uu << ", " << ua << ", " << kc << ");\n";
            o << "    u32 " << t << "[" << L << "], " << rr << "[" << Lb << "];\n";
            o << "    fl |= divmod_mag<" << NU << "," << Lb << "," << L << ",false>(" << t << ", " << rr << ", " << uu << ", " << ub << ");\n";
            }
            // declared-type check |Q| < 10^p (reading Q5: the paper's bound can fail)
            std::string kb = konst(HBig::pow10(n->p), L);
            o << "    if (!lt(" << t << ", " << kb << ")) fl |= F_OVERFLOW;\n";
            o << "    cond_neg(" << t << ", " << na << " ^ " << nb << ");\n";
            return t;
        }
        case Op::Mod: {
            // r = sign(A) * (|A| mod |B|)  (reading Q7)
            const int La = L_->L, Lb = R_->L;
            std::string ua = fresh("t"), na = fresh("n"), ub = fresh("t"), nb = fresh("n"), q = fresh("t"), rr = fresh("t");
            o << "    u32 " << ua << "[" << La << "], " << na << "; abs_copy(" << ua << ", " << a << ", " << na << ");\n";
            o << "    u32 " << ub << "[" << Lb << "], " << nb << "; abs_copy(" << ub << ", " << b << ", " << nb << ");\n";
            o << "    u32 " << q << "[" << La << "], " << rr << "[" << Lb << "];\n";
            o << "    fl |= divmod_mag<" << La << "," << Lb << "," << La << ",true>(" << q << ", " << rr << ", " << ua << ", " << ub << ");\n";
            o << "    u32 " << t << "[" << L << "]; zext<" << Lb << "," << L << ">(" << t << ", " << rr << "); cond_neg(" << t << ", " << na << ");\n";
            return t;
        }
        default: break;
        }
        return "";
    }
};

}  // namespace

std::string gen_expr_kernel(const Node *root, const std::vector<ColType> &cols, const GenOpts &opt, GenInfo &info) {
    std::vector<bool> used(cols.size(), false);
    used_columns(root, used);
    const int LOUT = root->L;
    const bool narrow = max_limbs(root) <= 8 && !uses_divmod(root);
    const int R = narrow ? 4 : 1;
    info.rows_per_thread = R;
    bool any_compact = false;
    for (size_t c = 0; c < cols.size(); ++c) any_compact = any_compact || (used[c] && cols[c].Lb > 0);

    Emitter E;
    {
        std::vector<int> uses(cols.size(), 0), div_uses(cols.size(), 0);
        div_only_uses(root, uses, div_uses);
        E.lazy.assign(cols.size(), false);
        E.quad.assign(cols.size(), false);
        for (size_t c = 0; c < cols.size(); ++c) {
            E.lazy[c] = used[c] && cols[c].Lb == 0 && uses[c] > 0 && uses[c] == div_uses[c];
            E.quad[c] = cols[c].Q;
        }
    }
    std::string res = E.emit(root);

    std::ostringstream k;
    k << "// generated by libup codegen: " << canonical(root) << "  type (" << root->p << "," << root->s << ") L=" << LOUT << "\n";
    k << mul_variant_define() << "#include \"up_dev.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n\n";
    // per-row evaluation with everything in registers
    k << E.pre.str();
    k << "__device__ __forceinline__ void eval_row(";
    bool first = true;
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c]) continue;
        if (E.lazy[c]) k << (first ? "" : ", ") << "const u32 *__restrict__ g" << c << ", long long l" << c;
        else k << (first ? "" : ", ") << "const u32 (&x" << c << ")[" << cols[c].limbs << "]";
        first = false;
    }
    k << (first ? "" : ", ") << "u32 (&res)[" << LOUT << "], u32 &fl) {\n";
    k << E.o.str();
    k << "    sext<" << LOUT << "," << LOUT << ">(res, " << res << ");\n}\n\n";

    const bool cs = LOUT <= 8;
    const int LA = opt.sum ? opt.LA : LOUT;
    // chain accumulator: LOUT + 1 limbs per thread (< 2^31 rows per thread),
    // its sign as a negative count at slot KC -- not LA limbs (LA can be 20x LOUT)
    const int KC = std::min(LA, LOUT + 1);
    const int NS = cs ? LOUT : KC;
    // registers held across the row: node widths, minus columns only the
    // top-limb divisions read (loaded per division, not kept)
    std::function<int(const Node *)> live = [&](const Node *x) -> int {
        if (!x) return 0;
        if (E.is_lazy(x)) return 0;
        return std::max(x->L, std::max(live(x->l.get()), live(x->r.get())));
    };
    // occupancy: a kernel whose wide columns are all read lazily by top-limb
    // divisions keeps a narrow state per row -> 4 blocks/SM (64 registers; the
    // rare full-division fallback spills).  Measured on cfg3's rest kernel:
    // 2 -> 4 blocks/SM 1.227 -> 1.145 ms per step (profiles/r01_minblocks/).
    bool any_lazy = false;
    for (size_t c = 0; c < cols.size(); ++c) any_lazy = any_lazy || E.lazy[c];
    const int min_blocks = (R == 1 && any_lazy && live(root) <= 16) ? 4 : (R == 1 && live(root) <= 64) ? 2 : 0;
    k << "extern \"C\" __global__ void " << launch_bounds(256, min_blocks) << " upk(const up_kparams P) {\n";
    k << "    constexpr int R = " << R << ";\n";
    k << "    u32 fl = 0;\n";
    if (opt.sum) k << "    griddep_launch_dependents();\n";
    if (opt.sum) {
        if (cs) k << "    AccCS<" << LOUT << "> acc; acc.init();\n";
        else k << "    AccChain<" << LOUT << "," << KC << "> acc; acc.init();\n";
    }
    k << "    const long long n = P.n;\n";
    if (any_compact) {
        // Compact columns (NEXT-2, the paper's cDecimal rows read in place,
        // P:L843-873, Listing 1's expand step P:L942-948): tiles of 256 R rows;
        // each compact column's tile bytes (256 R Lb, a multiple of 16) are
        // brought into shared memory by ONE 1-D TMA bulk copy (cp.async.bulk)
        // completing on an mbarrier, double-buffered: the copy of the block's
        // next tile is in flight while its threads expand and evaluate the
        // current one.  The last tile copies rows * Lb rounded up to 16 bytes
        // (compact allocations are padded, up.h).
        int tile_bytes = 0;
        k << "    extern __shared__ __align__(128) unsigned char cdyn[];\n";
        for (size_t c = 0; c < cols.size(); ++c) {
            if (!used[c] || cols[c].Lb == 0) continue;
            const int words = ((256 * R * cols[c].Lb) / 4 + 4 + 31) / 32 * 32;   // + pad for the expand's look-ahead
            k << "    u32 *const cs" << c << "_0 = reinterpret_cast<u32 *>(cdyn) + " << tile_bytes / 4
              << ", *const cs" << c << "_1 = reinterpret_cast<u32 *>(cdyn) + " << tile_bytes / 4 + words << ";\n";
            tile_bytes += 2 * 4 * words;
        }
        info.dyn_smem = tile_bytes;
        k << "    __shared__ __align__(8) u64 cmb[2];\n";
        k << "    constexpr long long TILE = 256 * R;\n";
        k << "    const long long ntiles = (n + TILE - 1) / TILE;\n";
        k << "    if (threadIdx.x == 0) { mbar_init(&cmb[0], 1); mbar_init(&cmb[1], 1); mbar_fence_init(); }\n";
        k << "    __syncthreads();\n";
        // issue(tile, stage): one thread, all compact columns of the tile
        k << "    auto issue = [&](long long tile, int st) {\n";
        k << "        const long long t0 = tile * TILE; const long long rows = n - t0 < TILE ? n - t0 : TILE;\n";
        k << "        u32 total = 0;\n";
        for (size_t c = 0; c < cols.size(); ++c) {
            if (!used[c] || cols[c].Lb == 0) continue;
            k << "        const u32 nb" << c << " = (u32)((rows * " << cols[c].Lb << " + 15) / 16 * 16); total += nb" << c << ";\n";
        }
        k << "        mbar_expect_tx(&cmb[st], total);\n";
        for (size_t c = 0; c < cols.size(); ++c) {
            if (!used[c] || cols[c].Lb == 0) continue;
            k << "        bulk_g2s(st ? cs" << c << "_1 : cs" << c << "_0, reinterpret_cast<const unsigned char *>(P.col[" << c << "]) + t0 * "
              << cols[c].Lb << ", nb" << c << ", &cmb[st]);\n";
        }
        k << "    };\n";
        k << "    if (threadIdx.x == 0 && (long long)blockIdx.x < ntiles) issue(blockIdx.x, 0);\n";
        k << "    int it = 0;\n";
        k << "    for (long long tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++it) {\n";
        k << "        const int st = it & 1;\n";
        k << "        if (threadIdx.x == 0 && tile + gridDim.x < ntiles) { fence_proxy_async_smem(); issue(tile + gridDim.x, st ^ 1); }\n";
        k << "        mbar_wait_parity(&cmb[st], (u32)(it >> 1) & 1u);\n";
        k << "        const long long base = tile * TILE + (long long)threadIdx.x * R;\n";
        k << "        const bool live = base < n;\n";
    } else {
        k << "    const long long stride = (long long)gridDim.x * blockDim.x * R;\n";
        k << "    for (long long base = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * R; base < n; base += stride) {\n";
        k << "        const bool live = true;\n";
    }
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c] || cols[c].Lb == 0) continue;
        // thread's rows: tile bytes [tid R Lb, (tid + 1) R Lb); row r's limbs by
        // funnel shifts, the sign = top bit of its last byte, then two's complement
        const int Lc = cols[c].limbs, Lb = cols[c].Lb;
        const int NW = (R * Lb + 3) / 4 + 1;
        k << "        u32 x" << c << "[R][" << Lc << "];\n";
        k << "        { const int b0 = (int)threadIdx.x * " << R * Lb << ";\n";
        k << "          const u32 *w = (st ? cs" << c << "_1 : cs" << c << "_0) + (b0 >> 2); const u32 sh0 = (u32)(b0 & 3) * 8u;\n";
        k << "          u32 wv[" << NW + 1 << "];\n";
        k << "#pragma unroll\n          for (int i = 0; i < " << NW + 1 << "; ++i) wv[i] = w[i];\n";
        k << "          u32 al[" << NW << "];   // the thread's bytes, word-aligned\n";
        k << "#pragma unroll\n          for (int i = 0; i < " << NW << "; ++i) al[i] = __funnelshift_r(wv[i], wv[i + 1], sh0);\n";
        for (int r = 0; r < R; ++r) {
            const int rb = r * Lb;                      // row byte offset in al[]
            const int sbit = 8 * (rb + Lb - 1) + 7;    // sign bit (absolute bit in al[])
            k << "          { const u32 ng = (al[" << sbit / 32 << "] >> " << sbit % 32 << ") & 1u; const u32 m = 0u - ng; u64 cy = ng;\n";
            for (int j = 0; j < Lc; ++j) {
                const int bit0 = 8 * rb + 32 * j;       // limb j's first bit in al[]
                const int mag_bits = 8 * Lb - 1 - 32 * j;   // magnitude bits left in this row from limb j
                std::string v;
                if (mag_bits <= 0) v = "0u";
                else {
                    v = (bit0 % 32) ? "__funnelshift_r(al[" + std::to_string(bit0 / 32) + "], al[" + std::to_string(bit0 / 32 + 1) +
                                          "], " + std::to_string(bit0 % 32) + "u)"
                                    : "al[" + std::to_string(bit0 / 32) + "]";
                    if (mag_bits < 32) v = "(" + v + " & " + std::to_string((1u << mag_bits) - 1u) + "u)";
                }
                k << "            { const u64 t = (u64)(" << v << " ^ m) + cy; x" << c << "[" << r << "][" << j
                  << "] = (u32)t; cy = t >> 32; }\n";
            }
            k << "          }\n";
        }
        k << "        }\n";
    }
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c] || E.lazy[c] || cols[c].Lb > 0) continue;
        const int Lc = cols[c].limbs;
        k << "        u32 x" << c << "[R][" << Lc << "] = {};\n";
        if (cols[c].Q) {   // limb quads: one 16-byte load per quad and row
            k << "        if (live) { const uint4 *q = reinterpret_cast<const uint4 *>(P.col[" << c << "]) + base; const long long ld = P.ld[" << c << "];\n";
            k << "#pragma unroll\n          for (int r = 0; r < R; ++r) ld_quads<" << Lc << "," << (R == 1 ? "true" : "false") << ">(x" << c << "[r], q + r, ld); }\n";
            continue;
        }
        k << "        if (live) { const u32 *p = P.col[" << c << "] + base; const long long ld = P.ld[" << c << "];\n";
        if (R == 4) {
            k << "#pragma unroll\n          for (int j = 0; j < " << Lc << "; ++j) { const uint4 v = __ldcs(reinterpret_cast<const uint4 *>(p + j * ld));"
                 " x" << c << "[0][j] = v.x; x" << c << "[1][j] = v.y; x" << c << "[2][j] = v.z; x" << c << "[3][j] = v.w; } }\n";
        } else {
            k << "#pragma unroll\n          for (int j = 0; j < " << Lc << "; ++j) x" << c << "[0][j] = __ldcs(p + j * ld); }\n";
        }
    }
    const bool store = !opt.sum && !opt.cmp;
    if (store) k << "        u32 res[R][" << LOUT << "];\n";
    k << "#pragma unroll\n        for (int r = 0; r < (live ? R : 0); ++r) {\n";
    k << "            u32 fr = 0; u32 v[" << LOUT << "];\n";
    k << "            eval_row(";
    first = true;
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c]) continue;
        if (E.lazy[c] && cols[c].Q) k << (first ? "" : ", ") << "P.col[" << c << "] + 4 * (base + r), 4 * P.ld[" << c << "]";
        else if (E.lazy[c]) k << (first ? "" : ", ") << "P.col[" << c << "] + base + r, P.ld[" << c << "]";
        else k << (first ? "" : ", ") << "x" << c << "[r]";
        first = false;
    }
    k << (first ? "" : ", ") << "v, fr);\n";
    if (opt.cmp) {
        // WHERE: exact sign of lhs - rhs (P:L730-734 comparison operators)
        static const char *pred[] = {"", "ng", "ng || z", "!ng && !z", "!ng", "z", "!z"};
        k << "            if (base + r < n) { fl |= fr; const bool ng = (v[" << LOUT - 1 << "] >> 31) != 0u; const bool z = is_zero(v);\n";
        k << "              if (!(" << pred[opt.cmp] << ")) reinterpret_cast<int *>(P.out)[base + r] = -1; }\n";
    } else {
        k << "            if (base + r < n) { fl |= fr;" << (opt.sum ? " acc.add(v);" : "") << " }\n";
    }
    if (store) k << "#pragma unroll\n            for (int j = 0; j < " << LOUT << "; ++j) res[r][j] = v[j];\n";
    k << "        }\n";
    if (store) {
        if (R == 4)
            k << "        if (live)\n#pragma unroll\n        for (int j = 0; j < " << LOUT << "; ++j) __stcs(reinterpret_cast<uint4 *>(P.out + j * P.ld_out + base), make_uint4(res[0][j], res[1][j], res[2][j], res[3][j]));\n";
        else
            k << "        if (live)\n#pragma unroll\n        for (int j = 0; j < " << LOUT << "; ++j) __stcs(P.out + j * P.ld_out + base, res[0][j]);\n";
    }
    if (any_compact) k << "        __syncthreads();\n";
    k << "    }\n";
    k << "    if (fl) atomicOr(P.flags, fl);\n";
    if (opt.sum) {
        // the SUM workspace / ticket / result of the previous launch on this
        // stream are re-used: wait for it (no-op without a PDL launch)
        k << "    griddep_wait();\n";
        info.pdl = true;
        k << "    __shared__ u64 sm[(256 / 32) * " << (NS + 1) << "];\n";
        k << "    u64 vals[" << (NS + 1) << "];\n";
        if (cs) {
            k << "#pragma unroll\n    for (int j = 0; j < " << NS << "; ++j) vals[j] = acc.s[j];\n";
            k << "    vals[" << NS << "] = acc.neg;\n";
            k << "    block_commit<" << NS << "," << LA << "," << LOUT << ">(vals, P.ws, P.ticket, P.result, sm);\n";
        } else {
            k << "#pragma unroll\n    for (int j = 0; j < " << NS << "; ++j) vals[j] = acc.a[j];\n";
            k << "    vals[" << NS << "] = " << (KC < LA ? "(u64)(acc.a[" + std::to_string(KC - 1) + "] >> 31)" : std::string("0ull")) << ";\n";
            k << "    block_commit<" << NS << "," << LA << "," << NS << ">(vals, P.ws, P.ticket, P.result, sm);\n";
        }
        info.ws_slots = NS + 1;
    }
    k << "}\n";
    return k.str();
}


// ---------------------------------------------------------------------------
// Grouped aggregation (NEXT-4; the paper's moderngpu multi-pass
// SUM/MAX/MIN/AVG of P:L1480-1537 becomes ONE pass): every distinct
// expression is evaluated once per row (shared column loads) and folded into
// its group's record:
//   private mode (records fit shared memory per thread): each thread owns a
//     record per group in shared memory ([slot][thread] layout, conflict-free)
//     -- one 64-bit add per limb per row, no atomics, no warp collectives;
//     4 rows per thread with 128-bit loads when every operand is narrow;
//   warp mode (wide records): a warp's rows of one group are combined with
//     redux.sync and merged into a per-block record (smem atomics; MIN/MAX
//     under a per-record lock).
// Record: SUM = carry-save slots + negative count; MIN/MAX = best value (MIN
// as MAX of the bitwise complement); COUNT.  Blocks commit SUM slots with
// 64-bit atomics and MIN/MAX records to scratch; the last block (ticket)
// normalises, reduces MIN/MAX over blocks and finalises
// AVG = trunc(SUM * 10^4 / COUNT) (division rule with the divisor
// DECIMAL(ceil(log10 N)+1, 0): s2 = 0, so 10^(s2+4)).
std::string gen_group_agg_kernel(const std::vector<AggItem> &aggs, const std::vector<ColType> &cols, int G,
                                 GenInfo &info, int &mm_words) {
    // distinct expressions
    std::vector<const Node *> exprs;
    std::vector<std::string> names;
    std::vector<int> expr_of(aggs.size());
    for (size_t a = 0; a < aggs.size(); ++a) {
        std::string cn = canonical(aggs[a].root) + "@" + std::to_string(aggs[a].root->p) + "," + std::to_string(aggs[a].root->s);
        size_t e = 0;
        while (e < names.size() && names[e] != cn) ++e;
        if (e == names.size()) { names.push_back(cn); exprs.push_back(aggs[a].root); }
        expr_of[a] = (int)e;
    }
    const int NE = (int)exprs.size();
    // slot layout per group: [0] count, then per summed expression L+1 slots
    std::vector<int> sum_off(NE, -1);
    int SLOTS = 1;
    for (size_t a = 0; a < aggs.size(); ++a) {
        const int e = expr_of[a];
        if ((aggs[a].kind == AGG_SUM || aggs[a].kind == AGG_AVG) && sum_off[e] < 0) {
            sum_off[e] = SLOTS;
            SLOTS += exprs[e]->L + 1;
        }
    }
    // MIN/MAX records per group: one best value per MIN/MAX aggregate
    std::vector<int> mm_off(aggs.size(), -1), mm_idx(aggs.size(), -1);
    int MMW = 0, NMM = 0;
    for (size_t a = 0; a < aggs.size(); ++a)
        if (aggs[a].kind == AGG_MIN || aggs[a].kind == AGG_MAX) {
            mm_off[a] = MMW;
            mm_idx[a] = NMM++;
            MMW += exprs[expr_of[a]]->L;
        }
    mm_words = MMW;
    std::vector<bool> used(cols.size(), false);
    for (const Node *e : exprs) used_columns(e, used);
    int maxL = 0;
    bool divmod = false;
    for (const Node *e : exprs) { maxL = std::max(maxL, max_limbs(e)); divmod = divmod || uses_divmod(e); }

    // private records: T threads x G x (SLOTS u64 + MMW u32) within ~110 KB (2 blocks / SM)
    const size_t per_thread = (size_t)G * ((size_t)SLOTS * 8 + (size_t)MMW * 4);
    // block size maximising resident threads per SM under the 228 KB of shared
    // memory (1 KB reserved per block); measured on B200: more resident warps
    // beat larger blocks (Q1 shape: T = 32 0.80 ms vs T = 128 0.89 ms)
    int T = 0, best_threads = 0;
    for (int t : {256, 128, 64, 32}) {
        const size_t blk = per_thread * (size_t)t + 1024;
        const int nb = std::min<int>({32, 2048 / t, (int)((228u * 1024u) / blk)});
        if (nb >= 1 && per_thread * (size_t)t <= 220 * 1024 && nb * t >= best_threads) { best_threads = nb * t; T = t; }
    }
    const bool priv = T > 0;
    const int R = priv && maxL <= 8 && !divmod ? 4 : 1;
    if (!priv) T = 256;

    std::ostringstream k;
    k << "// generated by libup codegen: grouped aggregation, G=" << G << (priv ? " (private records)" : " (warp records)") << "\n";
    static const char *const kNames[] = {"SUM", "MIN", "MAX", "AVG"};
    for (size_t a = 0; a < aggs.size(); ++a)
        k << "//   agg " << a << ": " << kNames[aggs[a].kind] << "(" << names[(size_t)expr_of[a]] << ")\n";
    k << mul_variant_define() << "#include \"up_dev.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n\n";
    for (int e = 0; e < NE; ++e) {
        Emitter E;
        std::string res = E.emit(exprs[e]);
        k << "__device__ __forceinline__ void eval_" << e << "(";
        bool first = true;
        for (size_t c = 0; c < cols.size(); ++c) {
            if (!used[c]) continue;
            k << (first ? "" : ", ") << "const u32 (&x" << c << ")[" << cols[c].limbs << "]";
            first = false;
        }
        k << (first ? "" : ", ") << "u32 (&res)[" << exprs[e]->L << "], u32 &fl) {\n" << E.o.str();
        k << "    sext<" << exprs[e]->L << "," << exprs[e]->L << ">(res, " << res << ");\n}\n\n";
    }
    auto eval_one = [&](int e, const char *ind, const char *row) {
        k << ind << "u32 v" << e << "[" << exprs[e]->L << "]; eval_" << e << "(";
        bool first = true;
        for (size_t c = 0; c < cols.size(); ++c) {
            if (!used[c]) continue;
            k << (first ? "" : ", ") << "x" << c << row;
            first = false;
        }
        k << (first ? "" : ", ") << "v" << e << ", fr);\n";
    };
    k << "constexpr int G = " << G << ", SLOTS = " << SLOTS << ", MMW = " << std::max(MMW, 1) << ", NMM = " << std::max(NMM, 1)
      << ", T = " << T << ", R = " << R << ";\n";
    k << "extern \"C\" __global__ void " << launch_bounds(T) << " upk(const up_kparams P) {\n";
    k << "    extern __shared__ __align__(16) u64 gsm[];\n";
    k << "    const int tid = threadIdx.x;\n";
    k << "    u32 fl = 0;\n";
    k << "    const long long n = P.n;\n";
    if (priv) {
        // ---------------- private mode: [slot][thread] records
        k << "    u32 *gmm = reinterpret_cast<u32 *>(gsm + (long long)G * SLOTS * T);\n";
        k << "    for (int q = 0; q < G * SLOTS; ++q) gsm[q * T + tid] = 0ull;\n";
        if (NMM) {
            k << "    for (int g = 0; g < G; ++g) {\n";
            for (size_t a = 0; a < aggs.size(); ++a) {
                if (mm_off[a] < 0) continue;
                const int L = exprs[expr_of[a]]->L;
                k << "        for (int j = 0; j < " << L << "; ++j) gmm[(g * MMW + " << mm_off[a] << " + j) * T + tid] = j == " << L - 1 << " ? 0x80000000u : 0u;\n";
            }
            k << "    }\n";
        }
        k << "    const long long stride = (long long)gridDim.x * T * R;\n";
        k << "    for (long long base = ((long long)blockIdx.x * T + tid) * R; base < n; base += stride) {\n";
        k << "        int gi[R];\n";
        if (R == 4) {
            k << "        if (!P.group) { gi[0] = gi[1] = gi[2] = gi[3] = 0; }\n";
            k << "        else if (base + 3 < n) { const int4 q = __ldcs(reinterpret_cast<const int4 *>(P.group + base)); gi[0] = q.x; gi[1] = q.y; gi[2] = q.z; gi[3] = q.w; }\n";
            k << "        else { for (int r = 0; r < 4; ++r) gi[r] = base + r < n ? P.group[base + r] : -1; }\n";
        } else {
            k << "        gi[0] = P.group ? __ldcs(P.group + base) : 0;\n";
        }
        for (size_t c = 0; c < cols.size(); ++c) {
            if (!used[c]) continue;
            const int Lc = cols[c].limbs;
            k << "        u32 x" << c << "[R][" << Lc << "];\n";
            k << "        { const u32 *p = P.col[" << c << "] + base; const long long ld = P.ld[" << c << "];\n";
            if (R == 4)
                k << "#pragma unroll\n          for (int j = 0; j < " << Lc << "; ++j) { const uint4 v = __ldcs(reinterpret_cast<const uint4 *>(p + j * ld));"
                     " x" << c << "[0][j] = v.x; x" << c << "[1][j] = v.y; x" << c << "[2][j] = v.z; x" << c << "[3][j] = v.w; } }\n";
            else
                k << "#pragma unroll\n          for (int j = 0; j < " << Lc << "; ++j) x" << c << "[0][j] = __ldcs(p + j * ld); }\n";
        }
        k << "#pragma unroll\n        for (int r = 0; r < R; ++r) {\n";
        k << "            int g = base + r < n ? gi[r] : -1;\n";
        k << "            if (g >= G) { fl |= F_INVAL; g = -1; }\n";
        k << "            u32 fr = 0;\n";
        k << "            u64 *rec = gsm + (long long)(g < 0 ? 0 : g) * SLOTS * T + tid;\n";
        k << "            if (g >= 0) rec[0] += 1ull;\n";
        for (int e = 0; e < NE; ++e) {
            eval_one(e, "            ", "[r]");
            k << "            if (g >= 0) {\n";
            if (sum_off[e] >= 0) {
                const int L = exprs[e]->L;
                k << "#pragma unroll\n                for (int j = 0; j < " << L << "; ++j) rec[(" << sum_off[e] << " + j) * T] += v" << e << "[j];\n";
                k << "                rec[" << sum_off[e] + L << " * T] += v" << e << "[" << L - 1 << "] >> 31;\n";
            }
            for (size_t a = 0; a < aggs.size(); ++a) {
                if (mm_off[a] < 0 || expr_of[a] != e) continue;
                const int L = exprs[e]->L;
                const char *inv = aggs[a].kind == AGG_MAX ? "" : "~";
                k << "                { u32 *b = gmm + (g * MMW + " << mm_off[a] << ") * T + tid; u32 w[" << L << "], cur[" << L << "];\n";
                k << "#pragma unroll\n                  for (int j = 0; j < " << L << "; ++j) { w[j] = " << inv << "v" << e << "[j]; cur[j] = b[j * T]; }\n";
                k << "                  if (gt_signed<" << L << ">(w, cur)) {\n#pragma unroll\n                    for (int j = 0; j < " << L << "; ++j) b[j * T] = w[j]; } }\n";
            }
            k << "            }\n";
        }
        k << "            if (g >= 0) fl |= fr;\n";
        k << "        }\n    }\n";
        k << "    if (fl) atomicOr(P.flags, fl);\n";
        k << "    __syncthreads();\n";
        // block totals: slot q summed over the T records (rotated start: conflict-free)
        k << "    for (int q = tid; q < G * SLOTS; q += T) {\n";
        k << "        u64 t = 0;\n";
        k << "        for (int i = 0; i < T; ++i) t += gsm[q * T + ((i + tid) & (T - 1))];\n";
        k << "        if (t) atomicAdd(&P.ws[q], t);\n    }\n";
        if (NMM) {
            k << "    for (int q = tid; q < G * NMM; q += T) {\n";
            k << "        const int g = q / NMM, m = q - g * NMM;\n";
            k << "        switch (m) {\n";
            for (size_t a = 0; a < aggs.size(); ++a) {
                if (mm_off[a] < 0) continue;
                const int L = exprs[expr_of[a]]->L;
                k << "        case " << mm_idx[a] << ": {\n";
                k << "            const u32 *b = gmm + (g * MMW + " << mm_off[a] << ") * T;\n";
                k << "            u32 best[" << L << "], w[" << L << "];\n";
                k << "            for (int j = 0; j < " << L << "; ++j) best[j] = b[j * T];\n";
                k << "            for (int i = 1; i < T; ++i) {\n";
                k << "                for (int j = 0; j < " << L << "; ++j) w[j] = b[j * T + i];\n";
                k << "                if (gt_signed<" << L << ">(w, best)) for (int j = 0; j < " << L << "; ++j) best[j] = w[j];\n";
                k << "            }\n";
                k << "            u32 *o = P.scratch + (long long)blockIdx.x * G * MMW + g * MMW + " << mm_off[a] << ";\n";
                k << "            for (int j = 0; j < " << L << "; ++j) o[j] = best[j];\n";
                k << "            break; }\n";
            }
            k << "        }\n    }\n";
        }
        k << "    __syncthreads();\n";
    } else {
        // ---------------- warp mode: per-block records, warp-combined updates
        k << "    u32 *gmm = reinterpret_cast<u32 *>(gsm + G * SLOTS);\n";
        k << "    u32 *glk = gmm + G * MMW;\n";
        k << "    for (int i = tid; i < G * SLOTS; i += blockDim.x) gsm[i] = 0ull;\n";
        k << "    for (int i = tid; i < G * NMM; i += blockDim.x) glk[i] = 0u;\n";
        if (NMM) {
            k << "    for (int g = tid; g < G; g += blockDim.x) {\n";
            for (size_t a = 0; a < aggs.size(); ++a) {
                if (mm_off[a] < 0) continue;
                const int L = exprs[expr_of[a]]->L;
                k << "        for (int j = 0; j < " << L << "; ++j) gmm[g * MMW + " << mm_off[a] << " + j] = j == " << L - 1 << " ? 0x80000000u : 0u;\n";
            }
            k << "    }\n";
        }
        k << "    __syncthreads();\n";
        k << "    const int lane = tid & 31;\n";
        k << "    const long long stride = (long long)gridDim.x * blockDim.x;\n";
        k << "    for (long long wb = (long long)blockIdx.x * blockDim.x + (tid & ~31); wb < n; wb += stride) {\n";
        k << "        const long long i = wb + lane;\n";
        k << "        const long long ii = i < n ? i : n - 1;\n";
        k << "        int g = i < n ? (P.group ? __ldcs(P.group + ii) : 0) : -1;\n";
        k << "        if (g >= G) { fl |= F_INVAL; g = -1; }\n";
        for (size_t c = 0; c < cols.size(); ++c) {
            if (!used[c]) continue;
            k << "        u32 x" << c << "[" << cols[c].limbs << "];\n";
            k << "#pragma unroll\n        for (int j = 0; j < " << cols[c].limbs << "; ++j) x" << c << "[j] = __ldcs(P.col[" << c << "] + j * P.ld[" << c << "] + ii);\n";
        }
        k << "        u32 fr = 0;\n";
        k << "        const bool act = g >= 0;\n";
        // pass -1: COUNT; pass e: expression e (evaluated just before its pass: one value live at a time)
        for (int e = -1; e < NE; ++e) {
            if (e >= 0) eval_one(e, "        ", "");
            k << "        for (u32 pend = __ballot_sync(0xffffffffu, act); pend; ) {\n";
            k << "            const int ldr = __ffs(pend) - 1;\n";
            k << "            const int gl = __shfl_sync(0xffffffffu, g, ldr);\n";
            k << "            const bool mine = act && g == gl;\n";
            k << "            const u32 peers = __ballot_sync(0xffffffffu, mine);\n";
            k << "            pend &= ~peers;\n";
            k << "            if (mine) {\n";
            k << "                u64 *gs = gsm + gl * SLOTS;\n";
            k << "                const bool lead = lane == ldr;\n";
            if (e < 0) k << "                if (lead) atomicAdd(&gs[0], (u64)__popc(peers));\n";
            else {
                if (sum_off[e] >= 0) k << "                grp_sum_update<" << exprs[e]->L << ">(v" << e << ", peers, lead, gs + " << sum_off[e] << ");\n";
                for (size_t a = 0; a < aggs.size(); ++a) {
                    if (mm_off[a] < 0 || expr_of[a] != e) continue;
                    const int L = exprs[e]->L;
                    k << "                { u32 w[" << L << "];\n#pragma unroll\n                  for (int j = 0; j < " << L << "; ++j) w[j] = "
                      << (aggs[a].kind == AGG_MAX ? "" : "~") << "v" << e << "[j];\n";
                    k << "                  grp_max_update<" << L << ">(w, peers, lane, gmm + gl * MMW + " << mm_off[a] << ", glk + gl * NMM + " << mm_idx[a] << "); }\n";
                }
            }
            k << "            }\n        }\n";
        }
        k << "        if (act) fl |= fr;\n";
        k << "    }\n";
        k << "    if (fl) atomicOr(P.flags, fl);\n";
        k << "    __syncthreads();\n";
        k << "    for (int i = tid; i < G * SLOTS; i += blockDim.x) { const u64 t = gsm[i]; if (t) atomicAdd(&P.ws[i], t); }\n";
        if (NMM) k << "    for (int i = tid; i < G * MMW; i += blockDim.x) P.scratch[(long long)blockIdx.x * G * MMW + i] = gmm[i];\n";
    }
    // ---------------- common tail: last block normalises and finalises
    k << "    __threadfence();\n    __syncthreads();\n";
    k << "    __shared__ u32 s_last;\n";
    k << "    if (tid == 0) s_last = (atomicAdd(P.ticket, 1u) == gridDim.x - 1) ? 1u : 0u;\n";
    k << "    __syncthreads();\n    if (!s_last) return;\n    __threadfence();\n";
    k << "    for (int i = tid; i < G * SLOTS; i += blockDim.x) gsm[i] = atomicExch(&P.ws[i], 0ull);\n";
    k << "    __syncthreads();\n";
    k << "    if (tid == 0) *P.ticket = 0u;\n";
    k << "    for (int g = tid; g < G; g += blockDim.x) P.counts[g] = gsm[g * SLOTS];\n";
    k << "    for (int t = tid; t < " << aggs.size() << " * G; t += blockDim.x) {\n";
    k << "        const int a = t / G, g = t - a * G;\n";
    k << "        const u64 *gs = gsm + g * SLOTS;\n";
    k << "        const u64 cnt = gs[0];\n";
    k << "        switch (a) {\n";
    for (size_t a = 0; a < aggs.size(); ++a) {
        const int e = expr_of[a], L = exprs[e]->L, LA = aggs[a].LA, Lr = aggs[a].Lr;
        k << "        case " << a << ": {\n";
        k << "            u32 *o = P.result + " << aggs[a].off << "ll + (long long)g * " << Lr << ";\n";
        if (aggs[a].kind == AGG_SUM) {
            k << "            u32 r[" << LA << "]; slots_to_limbs<" << L << "," << LA << ">(r, gs + " << sum_off[e] << ");\n";
            k << "            for (int j = 0; j < " << Lr << "; ++j) o[j] = r[j];\n";
        } else if (aggs[a].kind == AGG_AVG) {
            // Q = sign * trunc(|SUM| * 10^4 / COUNT)  (P:L1076-1080 with the P:L1049-1058 quotient)
            k << "            u32 sm_[" << LA << "]; slots_to_limbs<" << L << "," << LA << ">(sm_, gs + " << sum_off[e] << ");\n";
            k << "            u32 ng; u32 ab[" << LA << "]; abs_copy(ab, sm_, ng);\n";
            k << "            u32 u[" << LA + 1 << "]; mul_1<" << LA << ">(u, ab, 10000u);\n";
            k << "            const u32 dv[2] = {(u32)cnt, (u32)(cnt >> 32)};\n";
            k << "            u32 q[" << Lr << "], rr[2];\n";
            k << "            if (cnt) { divmod_mag<" << LA + 1 << ",2," << Lr << ",false>(q, rr, u, dv); cond_neg(q, ng); } else zero(q);\n";
            k << "            for (int j = 0; j < " << Lr << "; ++j) o[j] = q[j];\n";
        } else {
            k << "            u32 b[" << L << "];\n";
            k << "            for (int j = 0; j < " << L << "; ++j) b[j] = j == " << L - 1 << " ? 0x80000000u : 0u;\n";
            k << "            for (unsigned blk = 0; blk < gridDim.x; ++blk) {\n";
            k << "                const u32 *c = P.scratch + (long long)blk * G * MMW + g * MMW + " << mm_off[a] << ";\n";
            k << "                u32 w[" << L << "];\n";
            k << "                for (int j = 0; j < " << L << "; ++j) w[j] = c[j];\n";
            k << "                if (gt_signed<" << L << ">(w, b)) for (int j = 0; j < " << L << "; ++j) b[j] = w[j];\n";
            k << "            }\n";
            k << "            for (int j = 0; j < " << L << "; ++j) o[j] = cnt ? " << (aggs[a].kind == AGG_MAX ? "b[j]" : "~b[j]") << " : 0u;\n";
        }
        k << "            break; }\n";
    }
    k << "        }\n    }\n}\n";
    info.rows_per_thread = R;
    info.threads = T;
    info.ws_slots = G * SLOTS;
    if (priv)
        info.dyn_smem = (int)((per_thread * (size_t)T + 15) & ~(size_t)15);
    else
        info.dyn_smem = (int)(((size_t)G * SLOTS * 8 + (size_t)G * std::max(MMW, 1) * 4 + (size_t)G * std::max(NMM, 1) * 4 + 15) & ~(size_t)15);
    // the last block re-reads G * SLOTS slots into gsm: the smem must hold them
    info.dyn_smem = std::max(info.dyn_smem, (int)(((size_t)G * SLOTS * 8 + 15) & ~(size_t)15));
    return k.str();
}


// ---------------------------------------------------------------------------
// Wide SUM regime (rows a10/a11 at ~40+ limbs, cfg3 DECIMAL(500..1000,...)):
// SELECT SUM(sum_t +-term_t) = sum_t +-10^(s_out - s_t) SUM(term_t) exactly
// (alignment is an exact x10^k and SUM is linear), so each term is summed on
// its own and the constant alignment is applied once at the end.  Terms:
// c_i, c_i*c_j, c_i/c_j.  One warp per row; a product is summed as exact
// column sums (no per-row carry normalisation); a quotient runs a
// warp-cooperative Knuth D on shared-memory operands.
namespace {

struct WTerm {
    int kind;   // 0 col, 1 mul, 2 div
    int sign;   // +1 / -1
    const Node *n;
    int ca = -1, cb = -1;
};

bool flatten(const Node *n, int sign, std::vector<WTerm> &out) {
    switch (n->op) {
    case Op::Add: return flatten(n->l.get(), sign, out) && flatten(n->r.get(), sign, out);
    case Op::Sub: return flatten(n->l.get(), sign, out) && flatten(n->r.get(), -sign, out);
    case Op::Neg: return flatten(n->l.get(), -sign, out);
    case Op::Col: out.push_back({0, sign, n, n->col, -1}); return true;
    case Op::Mul:
        if (n->l->op == Op::Col && n->r->op == Op::Col) { out.push_back({1, sign, n, n->l->col, n->r->col}); return true; }
        return false;
    case Op::Div:
        if (n->l->op == Op::Col && n->r->op == Op::Col) { out.push_back({2, sign, n, n->l->col, n->r->col}); return true; }
        return false;
    default: return false;
    }
}

}  // namespace

std::string gen_wide_sum_kernel(const Node *root, const std::vector<ColType> &cols, int LA, GenInfo &info) {
    std::vector<WTerm> terms;
    if (!flatten(root, 1, terms) || terms.empty() || terms.size() > 8) return "";
    std::vector<bool> used(cols.size(), false);
    used_columns(root, used);
    constexpr int NW = 8;
    std::ostringstream k;
    k << "// generated by libup codegen (wide SUM regime): " << canonical(root) << "  type (" << root->p << "," << root->s
      << ") LA=" << LA << "\n";
    k << mul_variant_define() << "#include \"up_dev.cuh\"\n#include \"up_wide.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n\n";
    // smem plan (in u32 words; u64 slot arrays first for alignment)
    int slot_words = 0;
    std::vector<int> slot_off(terms.size()), slot_n(terms.size());
    for (size_t t = 0; t < terms.size(); ++t) {
        const WTerm &w = terms[t];
        int ns = 0;
        if (w.kind == 0) ns = cols[(size_t)w.ca].limbs + 1;
        if (w.kind == 1) ns = cols[(size_t)w.ca].limbs + cols[(size_t)w.cb].limbs + 2;
        if (w.kind == 2) ns = w.n->L + 1;
        slot_off[t] = slot_words;
        slot_n[t] = ns;
        slot_words += 2 * ns;   // pos and neg u64 arrays (counted in u64 units here)
    }
    if (slot_words * 2 > 16000) return "";
    // per-warp scratch: staged columns + magnitude copies + division scratch
    int stage = 0;
    std::vector<int> stage_off(cols.size(), -1);
    for (size_t c = 0; c < cols.size(); ++c)
        if (used[c]) { stage_off[c] = stage; stage += cols[c].limbs; }
    int scratch = stage;   // scratch follows the staged columns in the warp's slice
    int magA = 0, magB = 0, divU = 0, divS = 0, divQ = 0, maxA = 0, maxB = 0;
    for (auto &w : terms) {
        if (w.kind == 0) continue;
        maxA = std::max(maxA, cols[(size_t)w.ca].limbs);
        maxB = std::max(maxB, cols[(size_t)w.cb].limbs);
    }
    magA = scratch; scratch += maxA;
    magB = scratch; scratch += maxB;
    int maxNU = 0, maxNS = 0, maxNQ = 0;
    for (auto &w : terms) {
        if (w.kind != 2) continue;
        const Node *A = w.n->l.get(), *B = w.n->r.get();
        const int NU = mag_limbs_of_pow10(A->p + B->s + 4);
        const int NV = B->L;
        maxNU = std::max(maxNU, NU);
        maxNS = std::max(maxNS, NU + NV + 1 + NV);
        maxNQ = std::max(maxNQ, w.n->L);
    }
    divU = scratch; scratch += maxNU;
    divS = scratch; scratch += maxNS;
    divQ = scratch; scratch += maxNQ;
    const int per_warp = scratch;
    const int smem_bytes = slot_words * 8 + NW * per_warp * 4;
    if (smem_bytes > 200 * 1024) return "";
    info.rows_per_thread = 1;
    info.ws_slots = slot_words;
    info.dyn_smem = smem_bytes;
    info.threads = NW * 32;
    info.rows_per_block = NW;

    k << "extern \"C\" __global__ void __launch_bounds__(" << NW * 32 << ") upk(const up_kparams P) {\n";
    k << "    constexpr int NW = " << NW << ", PER_WARP = " << per_warp << ", SLOTS = " << slot_words << ";\n";
    k << "    extern __shared__ u64 smem64[];\n";
    k << "    u64 *slots = smem64;\n";
    k << "    u32 *wbase = reinterpret_cast<u32 *>(smem64 + SLOTS);\n";
    k << "    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;\n";
    k << "    u32 *my = wbase + warp * PER_WARP;\n";
    k << "    for (int i = tid; i < SLOTS; i += blockDim.x) slots[i] = 0ull;\n";
    k << "    u32 fl = 0;\n";
    k << "    const long long n = P.n;\n";
    k << "    for (long long r0 = (long long)blockIdx.x * NW; r0 < n; r0 += (long long)gridDim.x * NW) {\n";
    k << "        __syncthreads();\n";
    // cooperative, sector-coalesced staging: 8 consecutive threads read 8 rows of one plane
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c]) continue;
        const int Lc = cols[c].limbs;
        k << "        for (int idx = tid; idx < " << Lc << " * NW; idx += blockDim.x) { const int j = idx / NW, w = idx % NW;\n"
             "            const long long row = r0 + w;\n"
             "            wbase[w * PER_WARP + " << stage_off[c] << " + j] = row < n ? __ldcs(P.col[" << c << "] + (long long)j * P.ld[" << c << "] + row) : 0u; }\n";
    }
    k << "        __syncthreads();\n";
    k << "        if (r0 + warp < n) {\n";
    for (size_t t = 0; t < terms.size(); ++t) {
        const WTerm &w = terms[t];
        const std::string pos = "(slots + " + std::to_string(slot_off[t]) + ")";
        const std::string neg = "(slots + " + std::to_string(slot_off[t] + slot_n[t]) + ")";
        k << "            { // term " << t << ": " << (w.sign > 0 ? "+" : "-") << canonical(w.n) << "\n";
        if (w.kind == 0) {
            const int Lc = cols[(size_t)w.ca].limbs;
            k << "              const u32 *x = my + " << stage_off[(size_t)w.ca] << ";\n";
            k << "              for (int j = lane; j < " << Lc << "; j += 32) if (x[j]) atomicAdd(&" << pos << "[j], (u64)x[j]);\n";
            k << "              if (lane == 0 && (x[" << Lc - 1 << "] >> 31)) atomicAdd(&" << neg << "[" << Lc << "], 1ull);\n";
        } else {
            const int La = cols[(size_t)w.ca].limbs, Lb = cols[(size_t)w.cb].limbs;
            k << "              u32 *A = my + " << magA << ", *B = my + " << magB << ";\n";
            k << "              for (int j = lane; j < " << La << "; j += 32) A[j] = my[" << stage_off[(size_t)w.ca] << " + j];\n";
            k << "              for (int j = lane; j < " << Lb << "; j += 32) B[j] = my[" << stage_off[(size_t)w.cb] << " + j];\n";
            k << "              __syncwarp();\n";
            k << "              const u32 sa = wide::to_mag<" << La << ">(A), sb = wide::to_mag<" << Lb << ">(B);\n";
            if (w.kind == 1) {
                k << "              u64 *acc = (sa ^ sb) ? " << neg << " : " << pos << ";\n";
                if (La == Lb) k << "              wide::colsum_product_sq<" << La << ">(A, B, acc);\n";
                else k << "              wide::colsum_product<" << La << "," << Lb << ">(A, B, acc);\n";
            } else {
                const Node *An = w.n->l.get(), *Bn = w.n->r.get();
                const int kk = Bn->s + 4;
                const int NU = mag_limbs_of_pow10(An->p + kk);
                HBig c = HBig::pow10(kk);
                const int LC = (int)c.w.size();
                const int NQ = w.n->L;
                std::vector<uint32_t> cw(c.w.begin(), c.w.end());
                k << "              const u32 KC[" << LC << "] = " << limbs_init(cw) << ";\n";
                k << "              u32 *U = my + " << divU << ", *Q = my + " << divQ << ";\n";
                k << "              wide::mul_const<" << La << "," << LC << "," << NU << ">(A, KC, U);\n";
                k << "              u32 f = wide::divq<" << NU << "," << Lb << "," << NQ << ">(U, B, Q, my + " << divS << ");\n";
                std::vector<uint32_t> bw = HBig::pow10(w.n->p).twos(NQ, false);
                k << "              const u32 BOUND[" << NQ << "] = " << limbs_init(bw) << ";\n";
                k << "              if (!f && !wide::lt_bound<" << NQ << ">(Q, BOUND)) f = F_OVERFLOW;\n";
                k << "              fl |= f;\n";
                k << "              if (!f) { u64 *acc = (sa ^ sb) ? " << neg << " : " << pos << ";\n"
                     "                for (int j = lane; j < " << NQ << "; j += 32) if (Q[j]) atomicAdd(&acc[j], (u64)Q[j]); }\n";
            }
        }
        k << "              __syncwarp();\n            }\n";
    }
    k << "        }\n";
    k << "    }\n";
    k << "    if (fl) atomicOr(P.flags, fl);\n";
    // commit all slots; last block combines
    k << "    __syncthreads();\n";
    k << "    for (int i = tid; i < SLOTS; i += blockDim.x) if (slots[i]) atomicAdd(&P.ws[i], slots[i]);\n";
    k << "    __threadfence();\n    __syncthreads();\n";
    k << "    __shared__ u32 s_last;\n";
    k << "    if (tid == 0) s_last = (atomicAdd(P.ticket, 1u) == gridDim.x - 1) ? 1u : 0u;\n";
    k << "    __syncthreads();\n    if (!s_last) return;\n    __threadfence();\n";
    k << "    for (int i = tid; i < SLOTS; i += blockDim.x) slots[i] = atomicExch(&P.ws[i], 0ull);\n";
    k << "    __syncthreads();\n";
    k << "    if (tid == 0) {\n";
    k << "        *P.ticket = 0u;\n";
    k << "        u32 acc[" << LA << "];\n        for (int j = 0; j < " << LA << "; ++j) acc[j] = 0u;\n";
    for (size_t t = 0; t < terms.size(); ++t) {
        const WTerm &w = terms[t];
        const int kt = root->s - w.n->s;
        HBig c = HBig::pow10(kt);
        std::vector<uint32_t> cw(c.w.begin(), c.w.end());
        k << "        { const u32 KT[" << cw.size() << "] = " << limbs_init(cw) << ";\n";
        k << "          wide::wide_final(slots + " << slot_off[t] << ", slots + " << slot_off[t] + slot_n[t] << ", "
          << slot_n[t] << ", KT, " << cw.size() << ", " << w.sign << ", " << LA << ", acc); }\n";
    }
    k << "        for (int j = 0; j < " << LA << "; ++j) P.result[j] = acc[j];\n";
    k << "    }\n";
    k << "}\n";
    return k.str();
}

// ---------------------------------------------------------------------------
// Row contraction for SUM of a column product (cfg3's c1*c2): over all rows,
// sum a*b = sum_k 2^(32k) sum_{i+j=k} (sum_rows A_i B_j)  -  sign corrections,
// with A, B the raw two's-complement limbs read as unsigned (a = A - s_a 2^(32 La)):
//   sum ab = sum AB - 2^(32 La) sum s_a B - 2^(32 Lb) sum s_b A + 2^(32(La+Lb)) sum s_a s_b.
// Each warp owns K consecutive product columns and keeps exact 96-bit
// carry-save column sums across all its rows (one row per lane): per a-limb
// one load of A_i and one of the sliding B window, K IMAD.WIDE products, no
// per-row carry propagation and no per-row sign handling.  The last block
// normalises pos - neg into LA limbs (negated for a '-' term) at P.result.
std::string gen_contract_kernel(int La, int Lb, int LA, int sign, int col_a, int col_b, GenInfo &info) {
    const int NK = La + Lb + 1;                 // columns 0 .. La+Lb (the last for s_a s_b)
    const int K = (NK + 7) / 8 <= 16 ? 8 : 16;  // keep a block <= 16 warps (registers per thread)
    const int CR = (NK + K - 1) / K;            // column ranges = warps per block
    const int NSL = NK + 3;                     // slot columns (carries of the top column)
    if (CR > 32) return "";
    info.threads = CR * 32;
    info.rows_per_block = 32;
    info.ws_slots = 2 * NSL;
    info.dyn_smem = 0;
    std::ostringstream k;
    k << "// generated by libup: row contraction SUM(c" << col_a + 1 << "*c" << col_b + 1 << ") La=" << La << " Lb=" << Lb
      << " K=" << K << " ranges=" << CR << "\n";
    k << mul_variant_define() << "#include \"up_dev.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n\n";
    k << "extern \"C\" __global__ void __launch_bounds__(" << CR * 32 << ") upk(const up_kparams P) {\n";
    k << "    constexpr int LA_ = " << La << ", LB_ = " << Lb << ", K = " << K << ", NSL = " << NSL << ";\n";
    k << "    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;\n";
    k << "    const int k0 = warp * K;\n";
    k << "    const u32 *A = P.col[" << col_a << "], *B = P.col[" << col_b << "];\n";
    k << "    const long long lda = P.ld[" << col_a << "], ldb = P.ld[" << col_b << "];\n";
    // 96-bit carry-save column sums a0:a1:a2 (add.cc chains on the IMAD.WIDE product)
    // split accumulators: low and high 32-bit halves of every product summed in
    // separate u64s (2^32 additions each before overflow): no carry flags live
    // across products, so ptxas never spills condition codes
    k << "    u64 alo[K], ahi[K], cor[K]; u64 ss = 0;\n";
    k << "#pragma unroll\n    for (int m = 0; m < K; ++m) { alo[m] = 0ull; ahi[m] = 0ull; cor[m] = 0ull; }\n";
    k << "    const int ilo = k0 - (LB_ - 1) > 0 ? k0 - (LB_ - 1) : 0;\n";
    k << "    const int ihi = k0 + K - 1 < LA_ - 1 ? k0 + K - 1 : LA_ - 1;\n";
    k << "    const int ib0 = ilo - ilo % K;\n";
    k << "    const long long n = P.n;\n";
    k << "    for (long long r0 = (long long)blockIdx.x * 32; r0 < n; r0 += (long long)gridDim.x * 32) {\n";
    k << "        const long long row = r0 + lane;\n";
    k << "        if (row < n) {\n";
    // circular window: slot (j mod K) holds B_j; at step i column m reads slot (k0+m-i) mod K
    k << "            u32 c[K];\n";
    k << "#pragma unroll\n            for (int m = 0; m < K; ++m) { const int j = k0 + m - ib0; c[m] = (j >= 0 && j < LB_) ? __ldg(B + (long long)j * ldb + row) : 0u; }\n";
    k << "            for (int ib = ib0; ib <= ihi; ib += K) {\n";
    k << "#pragma unroll\n              for (int u = 0; u < K; ++u) {\n";
    k << "                const int i = ib + u;\n";
    k << "                const u32 ai = (i >= ilo && i <= ihi) ? __ldg(A + (long long)i * lda + row) : 0u;\n";
    k << "#pragma unroll\n                for (int m = 0; m < K; ++m) {\n";
    k << "                    u64 p; asm(\"mul.wide.u32 %0, %1, %2;\" : \"=l\"(p) : \"r\"(ai), \"r\"(c[(m - u + K) % K]));\n";
    k << "                    alo[m] += (u32)p; ahi[m] += (u32)(p >> 32);\n";
    k << "                }\n";
    k << "                { const int j = k0 - i - 1; c[K - 1 - u] = (j >= 0 && j < LB_) ? __ldg(B + (long long)j * ldb + row) : 0u; }\n";
    k << "              }\n";
    k << "            }\n";
    // sign corrections
    k << "            const u32 sa = __ldg(A + (long long)(LA_ - 1) * lda + row) >> 31;\n";
    k << "            const u32 sb = __ldg(B + (long long)(LB_ - 1) * ldb + row) >> 31;\n";
    k << "            if (sa) {\n#pragma unroll\n              for (int m = 0; m < K; ++m) { const int j = k0 + m - LA_; if (j >= 0 && j < LB_) cor[m] += __ldg(B + (long long)j * ldb + row); } }\n";
    k << "            if (sb) {\n#pragma unroll\n              for (int m = 0; m < K; ++m) { const int j = k0 + m - LB_; if (j >= 0 && j < LA_) cor[m] += __ldg(A + (long long)j * lda + row); } }\n";
    k << "            ss += sa & sb;\n";
    k << "        }\n";
    k << "    }\n";
    // warp reduce (value a0 + a1 2^32 + a2 2^64 per column, exact in u64 slots below)
    // column value = alo + ahi 2^32 = lo + hi 2^64 (exact)
    k << "    u64 lo[K], hi[K];\n";
    k << "#pragma unroll\n    for (int m = 0; m < K; ++m) { const u64 t = alo[m] + (ahi[m] << 32); hi[m] = (ahi[m] >> 32) + (t < alo[m] ? 1ull : 0ull); lo[m] = t; }\n";
    k << "#pragma unroll\n    for (int m = 0; m < K; ++m) {\n";
    k << "#pragma unroll\n        for (int o = 16; o > 0; o >>= 1) {\n";
    k << "            const u64 l2 = __shfl_down_sync(0xFFFFFFFFu, lo[m], o); const u64 h2 = __shfl_down_sync(0xFFFFFFFFu, hi[m], o);\n";
    k << "            const u64 s = lo[m] + l2; hi[m] += h2 + (s < l2 ? 1ull : 0ull); lo[m] = s;\n";
    k << "            cor[m] += __shfl_down_sync(0xFFFFFFFFu, cor[m], o);\n";
    k << "        }\n    }\n";
    k << "#pragma unroll\n    for (int o = 16; o > 0; o >>= 1) ss += __shfl_down_sync(0xFFFFFFFFu, ss, o);\n";
    k << "    u64 *pos = P.ws, *neg = P.ws + NSL;\n";
    k << "    if (lane == 0) {\n";
    k << "#pragma unroll\n        for (int m = 0; m < K; ++m) {\n";
    k << "            const int col = k0 + m;\n";
    k << "            if (col + 2 < NSL) {\n";
    k << "                if ((u32)lo[m]) atomicAdd(&pos[col], (u64)(u32)lo[m]);\n";
    k << "                if (lo[m] >> 32) atomicAdd(&pos[col + 1], lo[m] >> 32);\n";
    k << "                if (hi[m]) atomicAdd(&pos[col + 2], hi[m]);\n";
    k << "                if ((u32)cor[m]) atomicAdd(&neg[col], (u64)(u32)cor[m]);\n";
    k << "                if (cor[m] >> 32) atomicAdd(&neg[col + 1], cor[m] >> 32);\n";
    k << "            }\n        }\n";
    k << "        if (warp == 0 && ss) atomicAdd(&pos[LA_ + LB_], ss);\n";
    k << "    }\n";
    // last block: normalise pos - neg (sign) into LA limbs
    k << "    __threadfence();\n    __syncthreads();\n";
    k << "    __shared__ u32 s_last;\n";
    k << "    if (threadIdx.x == 0) s_last = (atomicAdd(P.ticket, 1u) == gridDim.x - 1) ? 1u : 0u;\n";
    k << "    __syncthreads();\n    if (!s_last) return;\n    __threadfence();\n";
    k << "    __shared__ u64 sp[NSL], sn[NSL];\n";
    k << "    for (int i = threadIdx.x; i < NSL; i += blockDim.x) { sp[i] = atomicExch(&pos[i], 0ull); sn[i] = atomicExch(&neg[i], 0ull); }\n";
    k << "    __syncthreads();\n";
    k << "    if (threadIdx.x == 0) {\n";
    k << "        *P.ticket = 0u;\n";
    k << "        u64 cp = 0, cn = 0; u32 borrow = 0, cneg = " << (sign < 0 ? 1 : 0) << "u;\n";
    k << "        for (int j = 0; j < " << LA << "; ++j) {\n";
    k << "            u64 tp = cp, tn = cn;\n";
    k << "            if (j < NSL) { tp += (u32)sp[j]; tn += (u32)sn[j]; }\n";
    k << "            if (j >= 1 && j - 1 < NSL) { tp += sp[j - 1] >> 32; tn += sn[j - 1] >> 32; }\n";
    k << "            cp = tp >> 32; cn = tn >> 32;\n";
    k << "            const u64 d = (u64)(u32)tp - (u32)tn - borrow;\n";
    k << "            borrow = (u32)(d >> 63);\n";
    if (sign < 0) {
        k << "            const u64 ng = (u64)(~(u32)d) + cneg; cneg = (u32)(ng >> 32);\n";
        k << "            P.result[j] = (u32)ng;\n";
    } else {
        k << "            P.result[j] = (u32)d;\n";
    }
    k << "        }\n    }\n";
    k << "}\n";
    return k.str();
}


namespace {
void flatten_any(const Node *n, int sign, std::vector<std::pair<int, const Node *>> &out) {
    switch (n->op) {
    case Op::Add: flatten_any(n->l.get(), sign, out); flatten_any(n->r.get(), sign, out); return;
    case Op::Sub: flatten_any(n->l.get(), sign, out); flatten_any(n->r.get(), -sign, out); return;
    case Op::Neg: flatten_any(n->l.get(), -sign, out); return;
    default: out.push_back({sign, n}); return;
    }
}
std::unique_ptr<Node> clone_node(const Node *n) {
    auto c = std::make_unique<Node>();
    c->op = n->op; c->col = n->col; c->lit = n->lit; c->p = n->p; c->s = n->s; c->L = n->L;
    if (n->l) c->l = clone_node(n->l.get());
    if (n->r) c->r = clone_node(n->r.get());
    return c;
}
}  // namespace

// SUM(root) = sum of SUM(+-ci*cj) over the top-level column-product terms at
// the output scale (row contraction kernels) + 10^rest_scale * SUM(rest), the
// rest summed at its own scale (fused per-thread kernel).  Exact: SUM is linear and every
// term is an exact part of the row value.  Products below another scale, or
// too small to be compute-bound, stay in the rest.
bool split_sum_terms(const Node *root, const std::vector<ColType> &cols, int min_products,
                     std::vector<SplitTerm> &prods, std::unique_ptr<Node> &rest, int &rest_scale) {
    const Node *body = root->op == Op::Cast ? root->l.get() : root;
    const int s_out = root->s;
    std::vector<std::pair<int, const Node *>> terms;
    flatten_any(body, 1, terms);
    std::vector<std::pair<int, const Node *>> others;
    for (auto &t : terms) {
        const Node *n = t.second;
        if (n->op == Op::Mul && n->l->op == Op::Col && n->r->op == Op::Col && n->s == s_out &&
            cols[(size_t)n->l->col].limbs * cols[(size_t)n->r->col].limbs >= min_products)
            prods.push_back({t.first, n->l->col, n->r->col});
        else
            others.push_back(t);
    }
    if (prods.empty()) return false;
    rest.reset();
    if (!others.empty()) {
        std::unique_ptr<Node> acc;
        bool acc_neg = false;
        for (auto &t : others) {
            auto c = clone_node(t.second);
            const bool ng = t.first < 0;
            if (!acc) { acc = std::move(c); acc_neg = ng; continue; }
            auto m = std::make_unique<Node>();
            if (acc_neg && !ng) { m->op = Op::Sub; m->l = std::move(c); m->r = std::move(acc); acc_neg = false; }
            else { m->op = acc_neg == ng ? Op::Add : Op::Sub; m->l = std::move(acc); m->r = std::move(c); }
            acc = std::move(m);
        }
        if (acc_neg) { auto m = std::make_unique<Node>(); m->op = Op::Neg; m->l = std::move(acc); acc = std::move(m); }
        std::string err;
        type_tree(acc.get(), cols, err);
        if (!err.empty() || acc->s > s_out) return false;
        // the rest is summed at its own scale; its partial is multiplied by
        // 10^rest_scale in the combine (SUM is linear: no per-row alignment)
        rest_scale = s_out - acc->s;
        rest = std::move(acc);
    }
    return true;
}
}  // namespace uph
