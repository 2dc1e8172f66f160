"""GPU parity of the per-operator TPI kernels (up_eval_tpi, SURVEY NEXT-3;
the paper's multi-threading arithmetic, Fig. 13)
against the oracle, row by row: + - * at TPI 1..32 over the paper's LEN
ladder (result limbs 2..32), limb-plane and compact (Listing 3 group loads)
inputs, mixed scales (alignment products), negative operands, ragged row
counts; / at TPI 1 by long division and by Newton-Raphson, including
divide-by-zero and typed-quotient overflow rows (flags as up_eval_expr)."""
import numpy as np
import pytest

import oracle
from tests import gpu_util as G

pytestmark = pytest.mark.gpu

# operand (p, s) pairs whose + / * results span LEN 2 .. 32
ADD_TYPES = [((17, 5), (14, 2)), ((37, 0), (37, 0)), ((75, 20), (70, 3)), ((152, 30), (152, 31)), ((306, 9), (300, 0))]
MUL_TYPES = [((9, 2), (9, 3)), ((19, 0), (19, 4)), ((38, 10), (38, 0)), ((76, 5), (77, 6)), ((153, 7), (154, 0))]


def _run(op, ta, tb, tpi, n, compact=(False, False), div_algo="long", seed=3):
    types = [ta, tb]
    lead = [1] if op == "/" else []
    host = G.gen_cols(n, types, config=12, nonzero_lead_cols=lead, seed=seed)
    c = G.ctx()
    cols = [c.column_from_host_bin(p, s, m, g, layout="compact" if cp else "planes")
            for (m, g), (p, s), cp in zip(host, types, compact)]
    out = c.eval_tpi(op, cols[0], cols[1], tpi, div_algo)
    err = None
    try:
        c.check()
    except Exception as e:  # noqa: BLE001
        err = e
    want = oracle.eval_rows(f"c1{op}c2", G.to_oracle(host, types), strict=False)
    got = c.column_to_strings(out)
    bad = [w for w in want if w.startswith("E")]
    assert (err is not None) == bool(bad)
    for g_, w in zip(got, want):
        if not w.startswith("E"):
            assert g_ == w, (op, ta, tb, tpi, g_, w)


@pytest.mark.parametrize("tpi", [1, 2, 4, 8, 16, 32])
@pytest.mark.parametrize("types", ADD_TYPES, ids=lambda t: f"{t[0][0]}x{t[1][0]}")
@pytest.mark.parametrize("op", ["+", "-"])
def test_tpi_add_sub(op, types, tpi):
    _run(op, types[0], types[1], tpi, 1031)


@pytest.mark.parametrize("tpi", [1, 2, 4, 8, 16, 32])
@pytest.mark.parametrize("types", MUL_TYPES, ids=lambda t: f"{t[0][0]}x{t[1][0]}")
def test_tpi_mul(types, tpi):
    _run("*", types[0], types[1], tpi, 1031)


@pytest.mark.parametrize("tpi", [1, 4, 8, 32])
@pytest.mark.parametrize("op", ["+", "*"])
def test_tpi_compact_inputs(op, tpi):
    """Listing 3's group loads of compact rows (mixed with a limb-plane operand)."""
    ta, tb = ((64, 32), (60, 10)) if op == "+" else ((64, 32), (40, 10))
    _run(op, ta, tb, tpi, 2049, compact=(True, False))
    _run(op, ta, tb, tpi, 517, compact=(True, True), seed=4)


@pytest.mark.parametrize("div_algo", ["long", "newton"])
@pytest.mark.parametrize("types", [((17, 2), (9, 0)), ((37, 5), (9, 3)), ((60, 5), (25, 3)), ((75, 10), (38, 2)),
                                   ((200, 50), (200, 50)), ((306, 10), (153, 4)), ((400, 0), (30, 0))],
                         ids=lambda t: f"{t[0][0]}over{t[1][0]}")
def test_tpi_divide(types, div_algo):
    _run("/", types[0], types[1], 1, 777, div_algo=div_algo)


@pytest.mark.parametrize("div_algo", ["long", "newton"])
def test_tpi_divide_edges_and_flags(div_algo):
    """divisors with leading zero limbs, 1, equal operands, all-nines, a zero
    divisor (DIVZERO) and a typed-quotient overflow (reading Q5)"""
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    p = 60
    big = str(10 ** p - 1)
    va = [big, "-" + big, "12345678901234567890123", "1", "0", big, "-7", big]
    vb = ["1", "-3", "12345678901234567890123", big, big, str(10 ** 30 + 1), "2", "-" + str(10 ** 59)]
    a, b = c.column_from_strings(p, 0, va), c.column_from_strings(p, 0, vb)
    out = c.eval_tpi("/", a, b, 1, div_algo)
    try:
        c.check()
    except up.UpError:
        pass
    want = oracle.eval_rows("c1/c2", [oracle.Column(p, 0, strings=va), oracle.Column(p, 0, strings=vb)], strict=False)
    for g_, w in zip(c.column_to_strings(out), want):
        if not w.startswith("E"):
            assert g_ == w
    z = c.column_from_strings(p, 0, ["5", "0"])
    c.eval_tpi("/", c.column_from_strings(p, 0, ["1", "2"]), z, 1, div_algo)
    with pytest.raises(up.UpError) as ei:
        c.check()
    assert ei.value.name == "DIVZERO"


def test_tpi_division_needs_one_lane():
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    a = c.column_from_strings(20, 0, ["1"])
    with pytest.raises(up.UpError) as ei:
        c.eval_tpi("/", a, a, 4)
    assert ei.value.name == "UNSUPPORTED"
