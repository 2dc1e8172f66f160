"""Paper-literal Query 5: sin(x) as the SQL polynomial
c1 - c1^3/6 + c1^5/120 - ... with 2..11 terms over DECIMAL(9,8) inputs, typed
by the paper's rules (T10: 2 terms -> DECIMAL(32,28), 11 -> DECIMAL(185,172)),
through up_eval_expr / up_sum_expr, bit-exact vs the oracle.  (Accuracy vs
the true sine is context only -- see tools/query5_mae.py.)"""
import math

import pytest

import oracle
from gen import synth
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def q5(terms):
    e = "c1"
    for k in range(1, terms):
        n = 2 * k + 1
        e += (" - " if k % 2 else " + ") + "*".join(["c1"] * n) + "/" + str(math.factorial(n))
    return e


@pytest.mark.parametrize("terms", [2, 3, 5, 8, 11])
@pytest.mark.parametrize("mu", [0.01, 0.78, 1.56])
def test_query5_literal(terms, mu):
    mag, neg = synth.normal_decimal(300, mu, 0.01, 8, config=5, column=3)
    expr = q5(terms)
    ocol = oracle.Column(9, 8, mag, neg)
    c = G.ctx()
    col = c.column_from_host_bin(9, 8, mag, neg)
    P, S = c.expr_type(expr, [col])
    assert (P, S) == oracle.expr_type(expr, [ocol])
    out = c.eval_expr(expr, [col])
    c.check()
    assert c.column_to_strings(out) == oracle.eval_rows(expr, [ocol])
    got, _, _ = G.gpu_sum_string(expr, [col])
    assert got == oracle.eval_sum(expr, [ocol])[0]
