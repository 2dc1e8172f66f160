// expr.cpp -- parser + typing for DECIMAL expressions (rows a1/a2).
#include "expr.h"

#include <cctype>

namespace uph {

namespace {

struct Parser {
    const std::string &s;
    size_t i = 0;
    int ncols;
    std::string err;

    Parser(const std::string &src, int nc) : s(src), ncols(nc) {}
    void ws() { while (i < s.size() && (s[i] == ' ' || s[i] == '\t' || s[i] == '\n')) ++i; }
    bool fail(const std::string &m) { if (err.empty()) err = m + " at offset " + std::to_string(i); return false; }

    std::unique_ptr<Node> mk(Op op, std::unique_ptr<Node> l, std::unique_ptr<Node> r) {
        auto n = std::make_unique<Node>();
        n->op = op; n->l = std::move(l); n->r = std::move(r);
        return n;
    }
    std::unique_ptr<Node> primary() {
        ws();
        if (i >= s.size()) { fail("unexpected end"); return nullptr; }
        char c = s[i];
        if (c == '(') {
            ++i;
            auto e = sum();
            if (!e) return nullptr;
            ws();
            if (i >= s.size() || s[i] != ')') { fail("expected ')'"); return nullptr; }
            ++i;
            return e;
        }
        if (c == 'c' || c == 'C') {
            ++i;
            size_t st = i;
            long k = 0;
            while (i < s.size() && isdigit((unsigned char)s[i])) { k = k * 10 + (s[i] - '0'); ++i; if (k > 1000000) break; }
            if (i == st || k < 1 || k > ncols) { fail("bad column reference"); return nullptr; }
            auto n = std::make_unique<Node>();
            n->op = Op::Col; n->col = (int)k - 1;
            return n;
        }
        if (isdigit((unsigned char)c) || c == '.') {
            std::string ip, fp;
            while (i < s.size() && isdigit((unsigned char)s[i])) ip += s[i++];
            if (i < s.size() && s[i] == '.') { ++i; while (i < s.size() && isdigit((unsigned char)s[i])) fp += s[i++]; }
            if (ip.empty() && fp.empty()) { fail("bad literal"); return nullptr; }
            auto n = std::make_unique<Node>();
            n->op = Op::Lit;
            HBig::from_dec(ip + fp, n->lit);
            n->s = (int)fp.size();
            int nd = n->lit.dec_digits();
            n->p = std::max(std::max(nd, n->s), 1);
            return n;
        }
        fail(std::string("unexpected '") + c + "'");
        return nullptr;
    }
    std::unique_ptr<Node> unary() {
        ws();
        if (i < s.size() && s[i] == '-') { ++i; auto a = unary(); if (!a) return nullptr; return mk(Op::Neg, std::move(a), nullptr); }
        if (i < s.size() && s[i] == '+') { ++i; return unary(); }
        return primary();
    }
    std::unique_ptr<Node> product() {
        auto a = unary();
        if (!a) return nullptr;
        for (;;) {
            ws();
            if (i >= s.size()) return a;
            Op op;
            if (s[i] == '*') op = Op::Mul; else if (s[i] == '/') op = Op::Div; else if (s[i] == '%') op = Op::Mod; else return a;
            ++i;
            auto b = unary();
            if (!b) return nullptr;
            a = mk(op, std::move(a), std::move(b));
        }
    }
    std::unique_ptr<Node> sum() {
        auto a = product();
        if (!a) return nullptr;
        for (;;) {
            ws();
            if (i >= s.size()) return a;
            Op op;
            if (s[i] == '+') op = Op::Add; else if (s[i] == '-') op = Op::Sub; else return a;
            ++i;
            auto b = product();
            if (!b) return nullptr;
            a = mk(op, std::move(a), std::move(b));
        }
    }
};

}  // namespace

std::unique_ptr<Node> parse_expr(const std::string &src, int ncols, std::string &err) {
    Parser P(src, ncols);
    auto t = P.sum();
    P.ws();
    if (t && P.i != src.size()) { P.fail("trailing input"); t.reset(); }
    if (!t) err = P.err.empty() ? "parse error" : P.err;
    return t;
}

int type_tree(Node *n, const std::vector<ColType> &cols, std::string &err) {
    switch (n->op) {
    case Op::Col: {
        const ColType &c = cols[(size_t)n->col];
        n->p = c.p; n->s = c.s;
        break;
    }
    case Op::Lit: break;
    case Op::Cast: {   // keeps the target (p,s) set by the optimiser
        if (int e = type_tree(n->l.get(), cols, err)) return e;
        if (n->s < n->l->s) { err = "internal: downward cast"; return 1; }
        break;
    }
    case Op::Neg: {
        if (int e = type_tree(n->l.get(), cols, err)) return e;
        n->p = n->l->p; n->s = n->l->s;
        break;
    }
    default: {
        if (int e = type_tree(n->l.get(), cols, err)) return e;
        if (int e = type_tree(n->r.get(), cols, err)) return e;
        const int p1 = n->l->p, s1 = n->l->s, p2 = n->r->p, s2 = n->r->s;
        switch (n->op) {
        case Op::Add: case Op::Sub:
            if (s1 >= s2) { n->p = std::max(p1, p2 + s1 - s2) + 1; n->s = s1; }
            else { n->p = std::max(p2, p1 + s2 - s1) + 1; n->s = s2; }
            break;
        case Op::Mul: n->p = p1 + p2; n->s = s1 + s2; break;
        case Op::Div: n->p = std::max(p1 - p2 + s2 + 5, 1); n->s = s1 + 4; break;
        case Op::Mod:
            if (s1 != 0 || s2 != 0) { err = "% needs integer (scale 0) operands (P:L1063-1067)"; return 1; }
            n->p = p2; n->s = 0;
            break;
        default: break;
        }
    }
    }
    n->L = limbs_for_precision(n->p);
    return 0;
}

int sum_precision(int p, long long n_global) {
    int k = 0;
    long long t = 1;
    while (t < n_global) { t *= 10; ++k; }
    return p + k;
}

std::string canonical(const Node *n) {
    switch (n->op) {
    case Op::Col: return "c" + std::to_string(n->col + 1);
    case Op::Lit: return "L" + n->lit.to_dec() + "e-" + std::to_string(n->s);
    case Op::Neg: return "(-" + canonical(n->l.get()) + ")";
    case Op::Cast: return "cast(" + canonical(n->l.get()) + "," + std::to_string(n->p) + "," + std::to_string(n->s) + ")";
    default: break;
    }
    const char *o = n->op == Op::Add ? "+" : n->op == Op::Sub ? "-" : n->op == Op::Mul ? "*" : n->op == Op::Div ? "/" : "%";
    return "(" + canonical(n->l.get()) + o + canonical(n->r.get()) + ")";
}

namespace {

struct Konst {   // exact decimal constant: (-1)^neg * mant * 10^-scale
    HBig mant;
    int scale = 0;
    bool neg = false;
    bool is_zero() const { return mant.is_zero(); }
    bool is_one() const { return !neg && scale >= 0 && HBig::cmp(mant, HBig::pow10(scale)) == 0; }
    bool is_minus_one() const { return neg && HBig::cmp(mant, HBig::pow10(scale)) == 0; }
};

Konst kmul(const Konst &a, const Konst &b) {
    Konst r;
    r.mant = HBig::mul(a.mant, b.mant);
    r.scale = a.scale + b.scale;
    r.neg = (a.neg != b.neg) && !r.mant.is_zero();
    return r;
}
Konst kadd(const Konst &a, const Konst &b) {
    const int s = std::max(a.scale, b.scale);
    HBig x = HBig::mul(a.mant, HBig::pow10(s - a.scale)), y = HBig::mul(b.mant, HBig::pow10(s - b.scale));
    Konst r;
    r.scale = s;
    if (a.neg == b.neg) { r.mant = HBig::add(x, y); r.neg = a.neg; }
    else if (HBig::cmp(x, y) >= 0) { r.mant = HBig::sub(x, y); r.neg = a.neg; }
    else { r.mant = HBig::sub(y, x); r.neg = b.neg; }
    if (r.mant.is_zero()) r.neg = false;
    return r;
}
// drop trailing zero fraction digits (a constant is typed by its value)
Konst knorm(Konst k) {
    while (k.scale > 0) {
        uint32_t rem;
        HBig q = k.mant.div_small(10, rem);
        if (rem) break;
        k.mant = q;
        --k.scale;
    }
    return k;
}

std::unique_ptr<Node> mk_lit(const Konst &k) {   // non-negative literal node (sign handled by the caller)
    auto n = std::make_unique<Node>();
    n->op = Op::Lit;
    n->lit = k.mant;
    n->s = k.scale;
    n->p = std::max(std::max(k.mant.dec_digits(), k.scale), 1);
    n->L = limbs_for_precision(n->p);
    return n;
}
std::unique_ptr<Node> mk(Op op, std::unique_ptr<Node> l, std::unique_ptr<Node> r = nullptr) {
    auto n = std::make_unique<Node>();
    n->op = op;
    n->l = std::move(l);
    n->r = std::move(r);
    return n;
}
std::unique_ptr<Node> clone(const Node *n) {
    auto c = std::make_unique<Node>();
    c->op = n->op; c->col = n->col; c->lit = n->lit; c->p = n->p; c->s = n->s; c->L = n->L;
    if (n->l) c->l = clone(n->l.get());
    if (n->r) c->r = clone(n->r.get());
    return c;
}
bool has_divmod(const Node *n) {
    if (!n) return false;
    if (n->op == Op::Div || n->op == Op::Mod) return true;
    return has_divmod(n->l.get()) || has_divmod(n->r.get());
}
std::unique_ptr<Node> cast_to(std::unique_ptr<Node> x, int p, int s) {
    if (x->p == p && x->s == s) return x;
    auto c = mk(Op::Cast, std::move(x));
    c->p = p;
    c->s = s;
    c->L = limbs_for_precision(p);
    return c;
}

struct Term {
    bool neg = false;
    Konst k;                                   // constant factor (mant 1, scale 0 if none)
    std::vector<std::unique_ptr<Node>> f;      // optimised non-constant factors
    bool divmod = false;
};

std::unique_ptr<Node> opt(const Node *n, const std::vector<ColType> &cols, std::string &err);

void collect_product(const Node *n, Term &t, const std::vector<ColType> &cols, std::string &err) {
    switch (n->op) {
    case Op::Mul: collect_product(n->l.get(), t, cols, err); collect_product(n->r.get(), t, cols, err); return;
    case Op::Neg: t.neg = !t.neg; collect_product(n->l.get(), t, cols, err); return;
    case Op::Lit: { Konst k; k.mant = n->lit; k.scale = n->s; t.k = kmul(t.k, k); return; }
    default: {
        if (has_divmod(n)) t.divmod = true;
        t.f.push_back(opt(n, cols, err));
        return;
    }
    }
}
void collect_sum(const Node *n, bool neg, std::vector<Term> &terms, const std::vector<ColType> &cols, std::string &err) {
    switch (n->op) {
    case Op::Add: collect_sum(n->l.get(), neg, terms, cols, err); collect_sum(n->r.get(), neg, terms, cols, err); return;
    case Op::Sub: collect_sum(n->l.get(), neg, terms, cols, err); collect_sum(n->r.get(), !neg, terms, cols, err); return;
    case Op::Neg: collect_sum(n->l.get(), !neg, terms, cols, err); return;
    default: {
        Term t;
        t.k.mant = HBig(1);
        collect_product(n, t, cols, err);
        t.neg = t.neg != neg;
        terms.push_back(std::move(t));
        return;
    }
    }
}

std::unique_ptr<Node> build_product(Term &t, const std::vector<ColType> &cols, std::string &err, bool &negate) {
    // sign of the term = t.neg xor sign of the constant
    negate = t.neg != t.k.neg;
    Konst mag = knorm(t.k);
    mag.neg = false;
    std::unique_ptr<Node> acc;
    for (auto &f : t.f) acc = acc ? mk(Op::Mul, std::move(acc), std::move(f)) : std::move(f);
    if (!acc) return mk_lit(mag);                       // pure constant
    if (!mag.is_one()) acc = mk(Op::Mul, std::move(acc), mk_lit(mag));   // shortcut 1*a
    type_tree(acc.get(), cols, err);
    return acc;
}

std::unique_ptr<Node> opt(const Node *n, const std::vector<ColType> &cols, std::string &err) {
    if (n->op == Op::Col || n->op == Op::Lit) return clone(n);
    if (n->op == Op::Div || n->op == Op::Mod || n->op == Op::Cast) {
        // the operands of / and % keep their original types: the quotient's
        // prescale 10^(s2+4), result scale s1+4 and declared precision depend on them
        auto oc = [&](const Node *ch) {
            auto o = opt(ch, cols, err);
            type_tree(o.get(), cols, err);
            if (o->s > ch->s) o = clone(ch);   // never needed: optimisation only lowers scales
            return cast_to(std::move(o), ch->p, ch->s);
        };
        auto c = mk(n->op, oc(n->l.get()), n->r ? oc(n->r.get()) : nullptr);
        c->p = n->p; c->s = n->s; c->L = n->L;
        if (n->op == Op::Cast) { c->p = n->p; c->s = n->s; }
        type_tree(c.get(), cols, err);
        c->p = n->p; c->s = n->s; c->L = n->L;    // keep the unoptimised type of the node
        return c;
    }
    // additive / multiplicative region: n-ary sum of product terms
    std::vector<Term> terms;
    collect_sum(n, false, terms, cols, err);
    // constant pre-calculation: all pure-constant terms into one; drop x0 terms without / or %
    Konst ksum;
    ksum.mant = HBig();
    std::vector<Term> rest;
    for (auto &t : terms) {
        if (t.f.empty()) {
            Konst k = t.k;
            if (t.neg) k.neg = !k.neg && !k.is_zero();
            ksum = kadd(ksum, k);
        } else if (t.k.is_zero() && !t.divmod) {
            continue;                                     // shortcut: 0*a
        } else {
            rest.push_back(std::move(t));
        }
    }
    // build every product term, then schedule by scale (ascending)
    struct Built { std::unique_ptr<Node> node; bool neg; };
    std::vector<Built> built;
    for (auto &t : rest) {
        bool ng = false;
        auto b = build_product(t, cols, err, ng);
        built.push_back({std::move(b), ng});
    }
    std::stable_sort(built.begin(), built.end(), [](const Built &a, const Built &b) { return a.node->s < b.node->s; });
    std::unique_ptr<Node> acc;
    bool acc_neg = false;   // acc holds -value when acc_neg (only before a positive term is found)
    for (auto &b : built) {
        if (!acc) { acc = std::move(b.node); acc_neg = b.neg; continue; }
        if (acc_neg && !b.neg) { acc = mk(Op::Sub, std::move(b.node), std::move(acc)); acc_neg = false; }
        else if (acc_neg == b.neg) acc = mk(Op::Add, std::move(acc), std::move(b.node));
        else acc = mk(Op::Sub, std::move(acc), std::move(b.node));
        type_tree(acc.get(), cols, err);
    }
    ksum = knorm(ksum);
    if (!ksum.is_zero() || !acc) {
        if (!acc) {
            acc = mk_lit(Konst{ksum.mant, ksum.scale, false});
            acc_neg = ksum.neg;
        } else {
            // a constant is aligned at compile time to the scale it is added at
            Konst kk = ksum;
            const bool kneg = kk.neg;
            kk.neg = false;
            if (acc->s > kk.scale) { kk.mant = HBig::mul(kk.mant, HBig::pow10(acc->s - kk.scale)); kk.scale = acc->s; }
            auto lit = mk_lit(kk);
            lit->s = kk.scale;
            lit->p = std::max(std::max(kk.mant.dec_digits(), kk.scale), 1);
            lit->L = limbs_for_precision(lit->p);
            if (acc_neg && !kneg) { acc = mk(Op::Sub, std::move(lit), std::move(acc)); acc_neg = false; }
            else if (acc_neg == kneg) acc = mk(Op::Add, std::move(acc), std::move(lit));
            else acc = mk(Op::Sub, std::move(acc), std::move(lit));
        }
    }
    if (acc_neg) acc = mk(Op::Neg, std::move(acc));
    type_tree(acc.get(), cols, err);
    return acc;
}

}  // namespace

std::unique_ptr<Node> optimize(const Node *root, const std::vector<ColType> &cols) {
    std::string err;
    auto o = opt(root, cols, err);
    if (!err.empty() || !o) return clone(root);
    type_tree(o.get(), cols, err);
    if (!err.empty() || o->s > root->s) return clone(root);
    // same value; present it in the unoptimised type (exact upward alignment)
    auto r = cast_to(std::move(o), root->p, root->s);
    type_tree(r.get(), cols, err);
    if (!err.empty()) return clone(root);
    return r;
}

bool uses_divmod(const Node *n) {
    if (!n) return false;
    if (n->op == Op::Div || n->op == Op::Mod) return true;
    return uses_divmod(n->l.get()) || uses_divmod(n->r.get());
}

int max_limbs(const Node *n) {
    if (!n) return 0;
    return std::max(n->L, std::max(max_limbs(n->l.get()), max_limbs(n->r.get())));
}

void used_columns(const Node *n, std::vector<bool> &used) {
    if (!n) return;
    if (n->op == Op::Col) used[(size_t)n->col] = true;
    used_columns(n->l.get(), used);
    used_columns(n->r.get(), used);
}

}  // namespace uph
