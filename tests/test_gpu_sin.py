"""GPU parity for the fixed-point Taylor sine sin_P(x) (row a9, reading Q13;
Query 5 inputs P:L2229-2239): bit-exact vs the oracle at every P regime
(one lane per row, and 4/8/32-lane groups = warp-cooperative, row a10)."""
import numpy as np
import pytest

import oracle
from gen import synth
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def _x(n, mu, col=1):
    return synth.normal_decimal(n, mu, 0.01, 8, config=5, column=col)


@pytest.mark.parametrize("P,n", [(8, 300), (20, 300), (60, 300), (100, 200), (500, 130), (1000, 40), (5000, 40)])
@pytest.mark.parametrize("mu", [0.01, 0.78, 1.56])
def test_sin_rows_parity(P, n, mu):
    mag, neg = _x(n, mu)
    c = G.ctx()
    x = c.column_from_host_bin(9, 8, mag, neg)
    out = c.sin_taylor(x, P)
    c.check()
    got = c.column_to_strings(out)
    want = oracle.sin_rows(oracle.Column(9, 8, mag, neg), P)
    assert got == want


def test_sin_20000_digits_rows():
    """32-lane groups, 8 rows per 256-thread block: 10 rows = one full block + a ragged one"""
    mag, neg = _x(10, 0.78)
    c = G.ctx()
    out = c.sin_taylor(c.column_from_host_bin(9, 8, mag, neg), 20000)
    c.check()
    assert c.column_to_strings(out) == oracle.sin_rows(oracle.Column(9, 8, mag, neg), 20000)


@pytest.mark.parametrize("p,s,vals", [
    (1, 0, ["0", "1", "3", "-2", "9"]),
    (2, 0, None),
    (3, 2, ["0.00", "1.00", "-3.14", "9.99", "0.01"]),
    (9, 9, ["0.000000001", "-0.999999999", "0.5"]),
    (9, 8, ["0", "-0.00000001", "3.14159265", "-9.99999999"]),
])
def test_sin_edge_inputs(p, s, vals):
    c = G.ctx()
    if vals is None:   # |x| may reach 10^(p-s) > 10: outside the GPU domain (reading Q20)
        from paper_conf_icde_lixylz24_b200.up import UpError
        with pytest.raises(UpError) as ei:
            c.sin_taylor(c.column_from_strings(p, s, ["12"]), 30)
        assert ei.value.name == "UNSUPPORTED"
        return
    for P in (max(s, 1), 40, 300):
        out = c.sin_taylor(c.column_from_strings(p, s, vals), P)
        c.check()
        assert c.column_to_strings(out) == oracle.sin_rows(oracle.Column(p, s, strings=vals), P), (p, s, P)


@pytest.mark.parametrize("P,n", [(30, 5000), (500, 300), (2000, 40), (5000, 70), (20000, 17)])
def test_sin_sum_parity(P, n):
    """Fused SUM(sin_P) vs the oracle in every kernel regime: one row per
    thread (P <= ~1800), 8-lane groups (P = 5000: 32 rows per block, 70 rows =
    two full blocks + a ragged third) and 32-lane groups (P = 20000: 8 rows per
    block, 17 rows = two full blocks + one row)."""
    mag, neg = _x(n, 0.78, col=2)
    c = G.ctx()
    res = c.sin_taylor_sum(c.column_from_host_bin(9, 8, mag, neg), P)
    c.check()
    from paper_conf_icde_lixylz24_b200 import up
    assert up.result_to_string(res, P) == oracle.sin_sum(oracle.Column(9, 8, mag, neg), P, threads=8)


def test_sin_odd_symmetry_on_gpu():
    mag, neg = _x(64, 0.01)      # ~16% negatives
    c = G.ctx()
    a = c.column_to_strings(c.sin_taylor(c.column_from_host_bin(9, 8, mag, neg), 200))
    b = c.column_to_strings(c.sin_taylor(c.column_from_host_bin(9, 8, mag, 1 - neg), 200))
    c.check()
    for u, v, m in zip(a, b, mag[:, 0]):
        if m == 0:
            assert u == v
        else:
            assert u == ("-" + v if not v.startswith("-") else v[1:])


@pytest.mark.parametrize("P,n", [(8, 100), (20, 200), (300, 50), (1000, 12), (1700, 4)])
@pytest.mark.parametrize("pst", [(9, 8), (8, 7), (3, 2), (1, 0)])
def test_sin_register_sum_variant(P, n, pst):
    """The default kernel for W <= 200 limbs (t in shared memory, S in
    registers, one division pass per term: 64-bit 2-by-1 steps on limb
    pairs, one 3-by-2 step first for an odd limb count; 32-bit 2-by-1 steps
    while D_k < 2^32) against the oracle: scales whose constant shift is a
    right shift (s = 8, 7), a left shift (s = 2) or absent with no constant
    divisor (s = 0); row counts and P give odd and even limb counts."""
    p, s = pst
    mag, neg = synth.uniform_decimal(n, p, 5, 4)
    c = G.ctx()
    x = c.column_from_host_bin(p, s, mag, neg)
    out = c.sin_taylor(x, P)
    c.check()
    assert c.column_to_strings(out) == oracle.sin_rows(oracle.Column(p, s, mag, neg), P)
    from paper_conf_icde_lixylz24_b200 import up
    res = c.sin_taylor_sum(x, P)
    c.check()
    assert up.result_to_string(res, P) == oracle.sin_sum(oracle.Column(p, s, mag, neg), P, threads=8)


@pytest.mark.parametrize("lanes", [1, 2, 8, 32])
@pytest.mark.parametrize("P,n", [(8, 100), (60, 300), (300, 70), (1000, 40)])
@pytest.mark.parametrize("pst", [(9, 8), (8, 7), (3, 2), (1, 0), (9, 9)])
def test_sin_band_kernel_every_shape(lanes, P, n, pst, monkeypatch):
    """The skewed-band kernel (sin_band.cpp; default for W > 200 limbs) forced
    at every P and scale shape: 2s = 16 (the complement trick for negative
    terms), 2s = 14 / 4 / 0 / 18 (general scaled adds, digit drops at
    different term parities, whole-digit normalisation shifts sd = 1 for
    s <= 6), G lanes per row from 1 to 32, rows spanning several warps."""
    monkeypatch.setenv("UP_SIN_BAND_G", str(lanes))
    p, s = pst
    if s > P:
        pytest.skip("s > P is outside sin_taylor's domain (reading Q20)")
    mag, neg = synth.uniform_decimal(n, p, 5, 6)
    c = G.ctx()
    x = c.column_from_host_bin(p, s, mag, neg)
    out = c.sin_taylor(x, P)
    c.check()
    assert c.column_to_strings(out) == oracle.sin_rows(oracle.Column(p, s, mag, neg), P)
    from paper_conf_icde_lixylz24_b200 import up
    res = c.sin_taylor_sum(x, P)
    c.check()
    assert up.result_to_string(res, P) == oracle.sin_sum(oracle.Column(p, s, mag, neg), P, threads=8)
