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

#include <sstream>

namespace uph {

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

struct Emitter {
    std::ostringstream o;
    int tmp = 0;
    std::string fresh(const char *pfx) { return std::string(pfx) + std::to_string(tmp++); }

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
            o << "    u32 " << ua << "[" << La << "], " << na << "; abs_copy(" << ua << ", " << a << ", " << na << ");\n";
            o << "    u32 " << ub << "[" << Lb << "], " << nb << "; abs_copy(" << ub << ", " << b << ", " << nb << ");\n";
            std::string kc = konst(c, (int)c.w.size());
            o << "    u32 " << uu << "[" << NU << "]; mul_mag<" << La << "," << c.w.size() << "," << NU << ">(" << uu << ", " << ua << ", " << kc << ");\n";
            o << "    u32 " << t << "[" << L << "], " << rr << "[" << Lb << "];\n";
            o << "    fl |= divmod_mag<" << NU << "," << Lb << "," << L << ",false>(" << t << ", " << rr << ", " << uu << ", " << ub << ");\n";
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

    Emitter E;
    std::string res = E.emit(root);

    std::ostringstream k;
    k << "// generated by libup codegen: " << canonical(root) << "  type (" << root->p << "," << root->s << ") L=" << LOUT << "\n";
    k << "#include \"up_dev.cuh\"\n#include \"up_kparams.h\"\nusing namespace up;\n\n";
    // per-row evaluation with everything in registers
    k << "__device__ __forceinline__ void eval_row(";
    bool first = true;
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c]) continue;
        k << (first ? "" : ", ") << "const u32 (&x" << c << ")[" << cols[c].limbs << "]";
        first = false;
    }
    k << (first ? "" : ", ") << "u32 (&res)[" << LOUT << "], u32 &fl) {\n";
    k << E.o.str();
    k << "    sext<" << LOUT << "," << LOUT << ">(res, " << res << ");\n}\n\n";

    const bool cs = LOUT <= 8;
    const int LA = opt.sum ? opt.LA : LOUT;
    const int NS = cs ? LOUT : LA;
    k << "extern \"C\" __global__ void __launch_bounds__(256) upk(const up_kparams P) {\n";
    k << "    constexpr int R = " << R << ";\n";
    k << "    u32 fl = 0;\n";
    if (opt.sum) {
        if (cs) k << "    AccCS<" << LOUT << "> acc; acc.init();\n";
        else k << "    AccChain<" << LOUT << "," << LA << "> acc; acc.init();\n";
    }
    k << "    const long long n = P.n;\n";
    k << "    const long long stride = (long long)gridDim.x * blockDim.x * R;\n";
    k << "    for (long long base = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * R; base < n; base += stride) {\n";
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c]) continue;
        const int Lc = cols[c].limbs;
        k << "        u32 x" << c << "[R][" << Lc << "];\n";
        k << "        { const u32 *p = P.col[" << c << "] + base; const long long ld = P.ld[" << c << "];\n";
        if (R == 4) {
            k << "#pragma unroll\n          for (int j = 0; j < " << Lc << "; ++j) { const uint4 v = __ldcs(reinterpret_cast<const uint4 *>(p + j * ld));"
                 " x" << c << "[0][j] = v.x; x" << c << "[1][j] = v.y; x" << c << "[2][j] = v.z; x" << c << "[3][j] = v.w; } }\n";
        } else {
            k << "#pragma unroll\n          for (int j = 0; j < " << Lc << "; ++j) x" << c << "[0][j] = __ldcs(p + j * ld); }\n";
        }
    }
    if (!opt.sum) k << "        u32 res[R][" << LOUT << "];\n";
    k << "#pragma unroll\n        for (int r = 0; r < R; ++r) {\n";
    k << "            u32 fr = 0; u32 v[" << LOUT << "];\n";
    k << "            eval_row(";
    first = true;
    for (size_t c = 0; c < cols.size(); ++c) {
        if (!used[c]) continue;
        k << (first ? "" : ", ") << "x" << c << "[r]";
        first = false;
    }
    k << (first ? "" : ", ") << "v, fr);\n";
    k << "            if (base + r < n) { fl |= fr;" << (opt.sum ? " acc.add(v);" : "") << " }\n";
    if (!opt.sum) k << "#pragma unroll\n            for (int j = 0; j < " << LOUT << "; ++j) res[r][j] = v[j];\n";
    k << "        }\n";
    if (!opt.sum) {
        if (R == 4)
            k << "#pragma unroll\n        for (int j = 0; j < " << LOUT << "; ++j) __stcs(reinterpret_cast<uint4 *>(P.out + j * P.ld_out + base), make_uint4(res[0][j], res[1][j], res[2][j], res[3][j]));\n";
        else
            k << "#pragma unroll\n        for (int j = 0; j < " << LOUT << "; ++j) __stcs(P.out + j * P.ld_out + base, res[0][j]);\n";
    }
    k << "    }\n";
    k << "    if (fl) atomicOr(P.flags, fl);\n";
    if (opt.sum) {
        k << "    __shared__ u64 sm[(256 / 32) * " << (NS + 1) << "];\n";
        k << "    u64 vals[" << (NS + 1) << "];\n";
        if (cs) {
            k << "#pragma unroll\n    for (int j = 0; j < " << NS << "; ++j) vals[j] = acc.s[j];\n";
            k << "    vals[" << NS << "] = acc.neg;\n";
            k << "    block_commit<" << NS << "," << LA << "," << LOUT << ">(vals, P.ws, P.ticket, P.result, sm);\n";
        } else {
            k << "#pragma unroll\n    for (int j = 0; j < " << NS << "; ++j) vals[j] = acc.a[j];\n";
            k << "    vals[" << NS << "] = 0ull;\n";
            k << "    block_commit<" << NS << "," << LA << "," << LA << ">(vals, P.ws, P.ticket, P.result, sm);\n";
        }
        info.ws_slots = NS + 1;
    }
    k << "}\n";
    return k.str();
}

}  // namespace uph
