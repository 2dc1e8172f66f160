"""GPU parity of the wide SUM regime (warp per row, rows a10/a11): cfg3's
SUM(c1*c2 - c3/c4) at DECIMAL(200,50) / (500,75) / (1000,100) and other
linear combinations of column, product and quotient terms, vs the oracle."""
import os

import numpy as np
import pytest

import oracle
from gen import synth
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def _sum(expr, types, n, lead=(), seed=synth.SEED):
    host = G.gen_cols(n, types, config=3, nonzero_lead_cols=lead, seed=seed)
    want, P, S = oracle.eval_sum(expr, G.to_oracle(host, types), threads=8)
    got, gP, gS = G.gpu_sum_string(expr, G.to_gpu(host, types))
    assert (gP, gS) == (P, S)
    return got, want


@pytest.mark.parametrize("p,s", [(200, 50), (500, 75), (1000, 100)])
@pytest.mark.parametrize("n", [1, 9, 1000])
def test_cfg3_wide_sum_parity(p, s, n):
    got, want = _sum("c1*c2 - c3/c4", [(p, s)] * 4, n, lead=(3,))
    assert got == want


@pytest.mark.parametrize("expr,types,lead", [
    ("c1*c2 + c3", [(300, 20), (300, 40), (330, 60)], ()),
    ("-c1*c1 - c2/c3 + c1", [(400, 10), (380, 5), (350, 100)], (2,)),
    ("c1/c2 - c3*c4", [(450, 0), (300, 0), (420, 30), (400, 30)], (1,)),
    ("c1*c2", [(600, 200), (300, 100)], ()),
])
def test_wide_linear_combinations(expr, types, lead):
    got, want = _sum(expr, types, 777, lead=lead)
    assert got == want


def test_wide_edge_values_and_flags():
    c = G.ctx()
    p = 400
    big = str(10 ** p - 1)
    vals1 = [big, "-" + big, "0", "1", "-1", big]
    vals2 = ["-" + big, big, big, "7", "-" + big, "0"]
    ga = c.column_from_strings(p, 0, vals1)
    gb = c.column_from_strings(p, 0, vals2)
    oa, ob = oracle.Column(p, 0, strings=vals1), oracle.Column(p, 0, strings=vals2)
    from paper_conf_icde_lixylz24_b200 import up
    res = c.sum_expr("c1*c2 - c2", [ga, gb])
    c.check()
    assert up.result_to_string(res, 0) == oracle.eval_sum("c1*c2 - c2", [oa, ob])[0]
    # division by zero in one row sets the flag
    c.sum_expr("c1/c2", [ga, gb])
    with pytest.raises(up.UpError) as ei:
        c.check()
    assert ei.value.name in ("DIVZERO", "OVERFLOW")


def test_wide_and_per_thread_paths_agree(monkeypatch):
    """p=200 sits on the regime boundary: the per-thread fused kernel
    (UP_NO_WIDE) and the wide kernel must give the same bits."""
    types = [(200, 50)] * 4
    host = G.gen_cols(500, types, config=3, nonzero_lead_cols=(3,), seed=7)
    from paper_conf_icde_lixylz24_b200 import up
    c1 = up.Context(0)
    a, _, _ = (None, None, None)
    cols = [c1.column_from_host_bin(p, s, m, g) for (m, g), (p, s) in zip(host, types)]
    P, S, LA = c1.sum_type("c1*c2 - c3/c4", cols)
    wide = up.result_to_string(c1.sum_expr("c1*c2 - c3/c4", cols), S)
    c1.check()
    monkeypatch.setenv("UP_NO_WIDE", "1")
    c2 = up.Context(0)
    cols2 = [c2.column_from_host_bin(p, s, m, g) for (m, g), (p, s) in zip(host, types)]
    narrow = up.result_to_string(c2.sum_expr("c1*c2 - c3/c4", cols2), S)
    c2.check()
    assert wide == narrow


@pytest.mark.parametrize("expr,types,lead", [
    ("c1*c2 - c3/c4", [(200, 50)] * 4, (3,)),
    ("c1*c2", [(120, 30), (90, 20)], ()),
    ("-c1*c2 + c3*c1 - c2", [(150, 10), (150, 10), (140, 10)], ()),
    ("c1*c2 - c3/c4", [(1000, 100)] * 4, (3,)),
])
@pytest.mark.parametrize("radix", ["tc", "r28", "r32"])
def test_split_sum_matches_unsplit_and_oracle(expr, types, lead, radix, monkeypatch):
    """Row-contraction SUM (products as carry-save column sums over rows, signs
    by correction terms) + fused rest kernel + combine == oracle == UP_NO_SPLIT,
    for the tensor-core contraction (default, contract_tc.cu) and the CUDA-core
    ones (UP_NO_TC: 32-bit, radix-2^28 with UP_CONTRACT28)."""
    n = 300 if types[0][0] >= 1000 else 2000
    monkeypatch.setenv("UP_SPLIT", "1")
    if radix != "tc":
        monkeypatch.setenv("UP_NO_TC", "1")
    if radix == "r28":
        monkeypatch.setenv("UP_CONTRACT28", "1")
    host = G.gen_cols(n, types, config=3, nonzero_lead_cols=lead, seed=11)
    want, P, S = oracle.eval_sum(expr, G.to_oracle(host, types), threads=8)
    from paper_conf_icde_lixylz24_b200 import up
    c = up.Context(0)
    cols = [c.column_from_host_bin(p, s, m, g) for (m, g), (p, s) in zip(host, types)]
    got = up.result_to_string(c.sum_expr(expr, cols), S)
    c.check()
    assert got == want
    monkeypatch.delenv("UP_SPLIT")
    monkeypatch.setenv("UP_NO_SPLIT", "1")
    c2 = up.Context(0)
    cols2 = [c2.column_from_host_bin(p, s, m, g) for (m, g), (p, s) in zip(host, types)]
    assert up.result_to_string(c2.sum_expr(expr, cols2), S) == want


@pytest.mark.parametrize("p", [200, 1000])
@pytest.mark.parametrize("radix", ["tc", "r28", "r32"])
def test_split_contraction_extreme_values(p, radix, monkeypatch):
    """All-nines magnitudes (every 28-bit digit near 2^28 - 1, the column-sum
    bound) with mixed signs over many rows per thread: SUM(c1*c2) by the
    row contraction (tensor cores, both CUDA-core radices) == exact Python value."""
    monkeypatch.setenv("UP_SPLIT", "1")
    if radix != "tc":
        monkeypatch.setenv("UP_NO_TC", "1")
    if radix == "r28":
        monkeypatch.setenv("UP_CONTRACT28", "1")
    import numpy as np
    from paper_conf_icde_lixylz24_b200 import up
    n = 5000 if p == 200 else 600
    big = 10 ** p - 1
    vals1 = [big if i % 3 else -big for i in range(n)]
    vals2 = [-big if i % 5 == 0 else big for i in range(n)]
    def words(vals):
        w = (big.bit_length() + 31) // 32
        mag = np.zeros((n, w), np.uint32); neg = np.zeros(n, np.uint8)
        for i, v in enumerate(vals):
            a = abs(v)
            for j in range(w):
                mag[i, j] = (a >> (32 * j)) & 0xFFFFFFFF
            neg[i] = v < 0
        return mag, neg
    c = up.Context(0)
    cols = [c.column_from_host_bin(p, 10, *words(vals1)), c.column_from_host_bin(p, 10, *words(vals2))]
    P, S, LA = c.sum_type("c1*c2", cols)
    got = up.result_to_string(c.sum_expr("c1*c2", cols), S)
    c.check()
    want = sum(a * b for a, b in zip(vals1, vals2))
    assert got == up._fmt(want, S)
