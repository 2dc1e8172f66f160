"""The expression optimiser (NEXT-1: alignment scheduling + constant
pre-calculation, §III-D) reproduces the rewrites the paper prints
(Figs. 6, 7, 10, 12), on the host; on the GPU, optimised kernels are
bit-identical to the oracle (which never optimises) and to UP_NO_OPT kernels."""
import pytest

import oracle
from paper_conf_icde_lixylz24_b200 import up

# (expr, types, expected optimised canonical form) -- citations per row
PAPER_REWRITES = [
    # Fig. 12: 1+a+2+11 -> 14+a, 14 held at a's scale 10 ("DECIMAL(12,10)")
    ("1+c1+2+11", [(12, 10)], "cast((c1+L140000000000e-10),15,10) : (15,10)"),
    # Fig. 12: 1+a+2-3 -> a (no kernel arithmetic left)
    ("1+c1+2-3", [(12, 10)], "cast(c1,15,10) : (15,10)"),
    # Fig. 12: 0.25 x (a+b) x 4 -> a+b
    ("0.25*(c1+c2)*4", [(12, 2), (12, 2)], "cast((c1+c2),16,4) : (16,4)"),
    # Fig. 6: a + b x c + d - e, 3 alignments -> 1 (same-scale terms first)
    ("c1+c2*c3+c4-c5", [(12, 2), (12, 5), (12, 5), (12, 2), (12, 2)],
     "cast((((c1+c4)-c5)+(c2*c3)),27,10) : (27,10)"),
    # Fig. 10: a+b+a+a+a+a+a with a at scale 1, b at scale 11: one alignment
    ("c1+c2+c1+c1+c1+c1+c1", [(12, 1), (18, 11)], "((((((c1+c1)+c1)+c1)+c1)+c1)+c2) : (28,11)"),
    # Fig. 7: 1+a+b x (5+c-5)+d+1.23: 0+c -> c, 1+1.23 = 2.23 pre-aligned
    ("1+c1+c2*(5+c3-5)+c4+1.23", [(12, 2), (12, 1), (12, 3), (12, 2)],
     "cast((((c1+c4)+(c2*c3))+L22300e-4),29,4) : (29,4)"),
]


@pytest.mark.parametrize("expr,types,want", PAPER_REWRITES, ids=[r[0] for r in PAPER_REWRITES])
def test_paper_rewrites(expr, types, want):
    assert up.expr_optimized(expr, types) == want


def test_divisions_keep_their_operand_types():
    # / and % truncate: their operands are cast back to the unoptimised types
    got = up.expr_optimized("(0.25*(c1+c2)*4)/c3", [(12, 2), (12, 2), (9, 1)])
    assert got == "(cast((c1+c2),16,4)/c3) : (13,8)"
    # 0 x (a/b) keeps the division (its divide-by-zero flag must still fire)
    assert "/" in up.expr_optimized("0*(c1/c2)+c1", [(5, 1), (5, 1)])


GPU_CASES = [(e, t) for e, t, _ in PAPER_REWRITES] + [
    ("(0.25*(c1+c2)*4)/c3", [(12, 2), (12, 2), (9, 1)]),
    ("-c1-c2+0-c1*1", [(15, 3), (14, 7)]),
    ("c1*2*0.5 - c2*(-3)", [(20, 4), (11, 0)]),
]


@pytest.mark.gpu
@pytest.mark.parametrize("expr,types", GPU_CASES, ids=[c[0] for c in GPU_CASES])
def test_optimised_kernels_match_oracle(expr, types, monkeypatch):
    from tests import gpu_util as G
    lead = [k for k in range(len(types)) if f"/c{k + 1}" in expr.replace(" ", "")]
    host = G.gen_cols(1500, types, config=8, nonzero_lead_cols=lead)
    ocols = G.to_oracle(host, types)
    want_rows = oracle.eval_rows(expr, ocols, strict=False)
    want_sum = None
    try:
        want_sum = oracle.eval_sum(expr, ocols)[0]
    except oracle.OracleError:
        pass
    c = G.ctx()
    gcols = G.to_gpu(host, types)
    out = c.eval_expr(expr, gcols)
    try:
        c.check()
    except up.UpError:
        pass
    got = c.column_to_strings(out)
    for g, w in zip(got, want_rows):
        if not w.startswith("E"):
            assert g == w
    if want_sum is not None:
        got_sum, _, _ = G.gpu_sum_string(expr, gcols)
        assert got_sum == want_sum
