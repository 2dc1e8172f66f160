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
    default: break;
    }
    const char *o = n->op == Op::Add ? "+" : n->op == Op::Sub ? "-" : n->op == Op::Mul ? "*" : n->op == Op::Div ? "/" : "%";
    return "(" + canonical(n->l.get()) + o + canonical(n->r.get()) + ")";
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
