// codegen.h -- kernel specialisation (row a2).
#pragma once
#include <string>
#include <vector>

#include "expr.h"

namespace uph {

// __launch_bounds__(threads[, UP_MINBLOCKS]) -- the env knob trades registers
// for occupancy in experiments (part of the source, so of the cache key)
std::string launch_bounds(int threads, int min_blocks = 0);
std::string mul_variant_define();

struct GenOpts {
    bool sum = false;   // fused SUM (true) or per-row column output (false)
    int LA = 0;         // SUM limbs
    int cmp = 0;        // > 0: WHERE predicate sign(root) <op> 0 (CmpOp), rows that fail get id -1 in P.out
};
// comparison operators of up_filter (the root is lhs - rhs)
enum CmpOp { CMP_LT = 1, CMP_LE, CMP_GT, CMP_GE, CMP_EQ, CMP_NE };

struct GenInfo {
    int rows_per_thread = 1;
    int ws_slots = 0;
    int dyn_smem = 0;        // dynamic shared memory per block (bytes)
    int threads = 256;
    int rows_per_block = 0;  // > 0: rows handled per block-iteration (warp-per-row kernels)
    bool pdl = false;        // kernel waits (griddepcontrol.wait) before touching its SUM workspace
};

std::string gen_expr_kernel(const Node *root, const std::vector<ColType> &cols, const GenOpts &opt, GenInfo &info);
// row contraction of SUM(ci*cj) (see codegen.cpp)
struct SplitTerm {
    int sign, col_a, col_b;
};
std::string gen_contract_kernel(int La, int Lb, int LA, int sign, int col_a, int col_b, GenInfo &info);
bool split_sum_terms(const Node *root, const std::vector<ColType> &cols, int min_products,
                     std::vector<SplitTerm> &prods, std::unique_ptr<Node> &rest, int &rest_scale);
// wide SUM regime (warp per row); "" if the expression does not fit it
std::string gen_wide_sum_kernel(const Node *root, const std::vector<ColType> &cols, int LA, GenInfo &info);

// grouped aggregation (NEXT-4): SUM / MIN / MAX / AVG of expressions per group
enum AggKind { AGG_SUM = 0, AGG_MIN = 1, AGG_MAX = 2, AGG_AVG = 3 };
struct AggItem {
    int kind;
    const Node *root;   // typed (optimised) expression
    int LA;             // SUM limbs (SUM / AVG)
    int Lr;             // result limbs
    long long off;      // u32 offset of this aggregate's [G][Lr] block in the packed output
};
// mm_words: u32 words of one block's MIN/MAX record (x G x grid = scratch)
std::string gen_group_agg_kernel(const std::vector<AggItem> &aggs, const std::vector<ColType> &cols, int G,
                                 GenInfo &info, int &mm_words);

// modexp / sin_taylor specialisations (special.cpp)
struct ModexpPlan {
    int n = 0;          // modulus limbs
    int Lb = 0;         // base column limbs
    int Lout = 0;       // output limbs
    int LA = 0;         // SUM limbs (sum variant)
};
std::string gen_modexp_kernel(const HBig &N, const HBig &e, const ModexpPlan &plan, bool sum, std::string &err);
std::string gen_sin_kernel(int P, int p, int s, int Lx, int Lout, int LA, bool sum, int &lanes_per_row, std::string &err,
                           int *smem_per_thread = nullptr, bool *is_v3 = nullptr);
// per-operator kernels with TPI lanes per row (tpi.cpp, NEXT-3); op: 0 + 1 - 2 * 3 /
struct TpiInfo {
    int rows_per_block = 0, dyn_smem = 0;
};
std::string gen_tpi_kernel(int op, const ColType &ta, const ColType &tb, const Node *root, int G, bool nr_div,
                           TpiInfo &info, std::string &err);
// skewed-band sine (sin_band.cpp): one warp per block, R = 32 / G rows per warp
struct SinBandInfo {
    int G = 0, rows_per_block = 0, smem = 0, ws_slots = 0, delta = 0, W = 0;
};
std::string gen_sin_kernel_band(int P, int p, int s, int Lout, int LA, bool sum, int G_req, SinBandInfo &info,
                                std::string &err);

}  // namespace uph
