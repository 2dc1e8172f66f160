// expr.h -- expression front end of libup (product code): parser, typing,
// limb sizing (rows a1/a2).  Independent of the oracle's parser.
#pragma once
#include <memory>
#include <string>
#include <vector>

#include "hbig.h"

namespace uph {

enum class Op { Col, Lit, Add, Sub, Mul, Div, Mod, Neg, Cast };

struct Node {
    Op op = Op::Lit;
    int col = -1;         // Op::Col: 0-based column index
    HBig lit;             // Op::Lit: mantissa (non-negative) at scale s
    int p = 0, s = 0, L = 0;
    std::unique_ptr<Node> l, r;
};

// Lb > 0: the column is stored in the compact byte layout (the paper's
// cDecimal): Lb bytes per row, row-major; Q: limb quads (up.h
// UP_LAYOUT_QUADS); else limb planes
struct ColType { int p, s, limbs; int Lb = 0; bool Q = false; };

// Parse "c1*c2 - c3/c4" (SQL precedence, left-assoc, unary -, parentheses,
// literals typed by value: 1.23 -> DECIMAL(3,2), 10 -> DECIMAL(2,0),
// P:L1302-1305 §III-D2).  Returns nullptr and sets err on failure.
std::unique_ptr<Node> parse_expr(const std::string &src, int ncols, std::string &err);

// Bottom-up typing (§III-B3, readings Q3/Q5/Q7):
//  +/-: (max(p_hi, p_lo + s_hi - s_lo) + 1, s_hi)   x: (p1+p2, s1+s2)
//  /  : (max(p1 - p2 + s2 + 5, 1), s1 + 4)          %: (p2, 0), integers only
//  unary -: unchanged.  Returns an up_status code (0 = ok).
int type_tree(Node *n, const std::vector<ColType> &cols, std::string &err);

// SUM precision p + ceil(log10 N) (reading Q9)
int sum_precision(int p, long long n_global);

// canonical text of a typed tree (cache key component)
std::string canonical(const Node *n);

// Expression optimiser (§III-D): alignment scheduling (- as
// unary negation, + collapsed to n-ary, terms ordered by scale, rebuilt as a
// binary tree) and constant pre-calculation / shortcuts (constants folded per
// level, +a / 0+a / 1*a removed).  Value-preserving: +, -, * are exact, and
// the operands of / and % keep their original types (Cast), so every row's
// value -- including every truncation and every flag -- is unchanged; the
// root is cast back to the unoptimised (p,s) (reading Q12).
std::unique_ptr<Node> optimize(const Node *typed_root, const std::vector<ColType> &cols);

bool uses_divmod(const Node *n);
int max_limbs(const Node *n);
void used_columns(const Node *n, std::vector<bool> &used);

}  // namespace uph
