"""GPU parity of SUMs over wide numbers (rows a6/a7/a10/a11) vs the oracle.

Which kernel runs (up_host.cpp::expr_kernel / up_sum_expr):
* top-level column products of a SUM take the tensor-core row contraction
  (contract_tc.cu) and the rest runs in the per-thread fused kernel (one row
  per thread, up to 256 limbs) -- cfg3 at DECIMAL(200,50) / (500,75) /
  (1000,100) and the linear combinations below;
* numbers of >= 257 limbs (p >= ~2470 digits) take the warp-per-row wide
  regime (up_wide.cuh, codegen.cpp::gen_wide_sum_kernel): a warp owns one
  row, operands staged in shared memory -- test_warp_per_row_* below reach it
  (the kernel source is checked to be the wide one)."""
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


@pytest.mark.parametrize("expr,types,lead", [
    ("c1*c2 - c3/c4", [(200, 50)] * 4, (3,)),
    ("c1*c2", [(120, 30), (90, 20)], ()),
    ("-c1*c2 + c3*c1 - c2", [(150, 10), (150, 10), (140, 10)], ()),
    ("c1*c2 - c3/c4", [(1000, 100)] * 4, (3,)),
])
@pytest.mark.parametrize("radix", ["tc", "r32"])
def test_split_sum_matches_unsplit_and_oracle(expr, types, lead, radix, monkeypatch):
    """Row-contraction SUM (products as carry-save column sums over rows, signs
    by correction terms) + fused rest kernel + combine == oracle == UP_NO_SPLIT,
    for the tensor-core contraction (default, contract_tc.cu) and the CUDA-core
    one (UP_NO_TC, also taken beyond 2^31 rows per call)."""
    n = 300 if types[0][0] >= 1000 else 2000
    monkeypatch.setenv("UP_SPLIT", "1")
    if radix != "tc":
        monkeypatch.setenv("UP_NO_TC", "1")
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
@pytest.mark.parametrize("radix", ["tc", "r32"])
def test_split_contraction_extreme_values(p, radix, monkeypatch):
    """All-nines magnitudes with mixed signs over many rows per thread:
    SUM(c1*c2) by the row contraction (tensor cores, CUDA cores) == exact Python value."""
    monkeypatch.setenv("UP_SPLIT", "1")
    if radix != "tc":
        monkeypatch.setenv("UP_NO_TC", "1")
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
    got = G.limbs_int(c.sum_expr("c1*c2", cols))
    c.check()
    assert got == sum(a * b for a, b in zip(vals1, vals2))   # mantissas at scale S


def _wide_source(expr, types, n):
    from paper_conf_icde_lixylz24_b200 import up
    return up.gen_source("sum", expr, types, n)


@pytest.mark.parametrize("expr,types,lead,env", [
    ("c1+c2", [(2500, 10), (2480, 300)], (), None),
    ("c1 - c2 + c1", [(2600, 0), (2600, 0)], (), None),
    ("c1/c2 - c3", [(2500, 0), (30, 0), (2490, 4)], (1,), None),
    ("c1*c2 - c3", [(1300, 5), (1250, 7), (2000, 12)], (), "UP_NO_SPLIT"),
])
@pytest.mark.parametrize("n", [1, 9, 300])
def test_warp_per_row_wide_regime_parity(expr, types, lead, env, n, monkeypatch):
    """>= 257-limb SUM terms: the warp-per-row kernel (up_wide.cuh) vs the oracle."""
    if env:
        monkeypatch.setenv(env, "1")
    assert "wide SUM regime" in _wide_source(expr, types, n)
    got, want = _sum(expr, types, n, lead=lead, seed=n + 5)
    assert got == want


def test_warp_per_row_wide_regime_extremes():
    """all-nines magnitudes with mixed signs (full carry ripple through 270
    limbs) and a divide-by-zero row raising the sticky flag"""
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    p = 2600
    big = str(10 ** p - 1)
    v1 = [big, "-" + big, big, "0", "1", big, "-1"]
    v2 = [big, big, "-" + big, big, "-" + big, "0", "-1"]
    assert "wide SUM regime" in _wide_source("c1 - c2 + c1", [(p, 0), (p, 0)], len(v1))
    g = [c.column_from_strings(p, 0, v1), c.column_from_strings(p, 0, v2)]
    o = [oracle.Column(p, 0, strings=v1), oracle.Column(p, 0, strings=v2)]
    res = c.sum_expr("c1 - c2 + c1", g)
    c.check()
    assert up.result_to_string(res, 0) == oracle.eval_sum("c1 - c2 + c1", o)[0]
    # 20-digit divisors (nonzero leading digit, reading Q5: no typed-quotient overflow) and one zero
    dv = [str(10 ** 19 + 7), str(3 * 10 ** 19), "0", str(10 ** 20 - 1), str(10 ** 19), str(2 * 10 ** 19 + 1), "-" + str(10 ** 19 + 3)]
    d = [c.column_from_strings(p, 0, v1), c.column_from_strings(20, 0, dv)]
    c.sum_expr("c1/c2", d)
    with pytest.raises(up.UpError) as ei:
        c.check()
    assert ei.value.name == "DIVZERO"
