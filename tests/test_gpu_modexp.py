"""GPU parity for X^e mod N (row a8): up_modexp / up_modexp_sum vs the oracle
(and Python pow as a second, independent check), plus the paper's literal
Query 4 (c1*c1%N*c1%N) through the expression path."""
import numpy as np
import pytest

import oracle
from gen import synth
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def test_textbook_rsa_on_gpu():
    c = G.ctx()
    col = c.column_from_strings(4, 0, ["65", "0", "1", "3232", "2790"])
    out = c.modexp(col, 17, 3233)
    c.check()
    got = c.column_to_strings(out)
    assert got[0] == "2790"
    assert got == [str(pow(int(v), 17, 3233)) for v in ["65", "0", "1", "3232", "2790"]]
    back = c.modexp(c.column_from_strings(4, 0, ["2790"]), 2753, 3233)
    c.check()
    assert c.column_to_strings(back) == ["65"]


@pytest.mark.parametrize("bits", [64, 256, 512, 1024, 1034, 2048])
@pytest.mark.parametrize("e", [3, 65537])
@pytest.mark.parametrize("radix", ["r28", "r32"])
def test_modexp_parity(bits, e, radix, monkeypatch):
    """Both Montgomery kernels: radix 2^28 (default up to 64 32-bit limbs,
    the base in shared memory beyond 40; 1034 bits puts 4N right under
    R = 2^1036) and the 32-bit CIOS (UP_MONT32=1, and every modulus wider
    than 64 limbs)."""
    if radix == "r32":
        monkeypatch.setenv("UP_MONT32", "1")
    elif bits > 64 * 32:
        pytest.skip("radix 2^28 kernel only up to 64 limbs")
    N, p, q = synth.rsa_modulus(bits)
    n = 333
    mag, neg = synth.rsa_messages(n, N)
    d = len(str(N))
    c = G.ctx()
    col = c.column_from_host_bin(d, 0, mag, neg)
    out = c.modexp(col, e, N)
    c.check()
    got = c.column_to_strings(out)
    want = oracle.modexp_rows(oracle.Column(d, 0, mag, neg), e, N)
    assert got == want
    assert [int(g) for g in got[:20]] == [pow(m, e, N) for m in synth.to_ints(mag, neg)[:20]]


def test_modexp_base_wider_than_modulus_is_reduced():
    N, p, q = synth.rsa_modulus(128)
    d = len(str(N))
    pb = 2 * d + 3                        # base values up to ~N^2 * 1000
    mag, neg = synth.uniform_decimal(200, pb, 4, 7, signed=False)
    c = G.ctx()
    out = c.modexp(c.column_from_host_bin(pb, 0, mag, neg), 65537, N)
    c.check()
    assert c.column_to_strings(out) == [str(pow(m, 65537, N)) for m in synth.to_ints(mag, neg)]


def test_modexp_sum_parity():
    N, p, q = synth.rsa_modulus(512)
    d = len(str(N))
    n = 1001
    mag, neg = synth.rsa_messages(n, N)
    c = G.ctx()
    res = c.modexp_sum(c.column_from_host_bin(d, 0, mag, neg), 65537, N)
    c.check()
    from paper_conf_icde_lixylz24_b200 import up
    got = up.result_to_string(res, 0)
    assert got == oracle.modexp_sum(oracle.Column(d, 0, mag, neg), 65537, N, threads=4)


def test_modexp_exponent_edge_cases_and_flags():
    c = G.ctx()
    col = c.column_from_strings(3, 0, ["5", "96", "0"])
    assert c.column_to_strings(c.modexp(col, 0, 97)) == ["1", "1", "1"]
    assert c.column_to_strings(c.modexp(col, 1, 97)) == ["5", "96", "0"]
    c.check()
    from paper_conf_icde_lixylz24_b200.up import UpError
    neg = c.column_from_strings(3, 0, ["-5"])
    c.modexp(neg, 3, 97)
    with pytest.raises(UpError) as ei:
        c.check()
    assert ei.value.name == "INVAL"
    with pytest.raises(UpError) as ei:
        c.modexp(col, 3, 98)
    assert ei.value.name == "UNSUPPORTED"


@pytest.mark.parametrize("p", [17, 35])
def test_query4_literal_expression(p):
    """Query 4 verbatim, N a DECIMAL constant of precision p+1."""
    N, _, _ = synth.rsa_modulus(56 if p == 17 else 116)
    Ns = str(N)
    assert len(Ns) <= p + 1
    mag, neg = synth.uniform_decimal(500, p, 4, 1, signed=False)
    expr = f"c1 * c1 % {Ns} * c1 % {Ns}"
    c = G.ctx()
    out = c.eval_expr(expr, [c.column_from_host_bin(p, 0, mag, neg)])
    c.check()
    got = c.column_to_strings(out)
    assert got == oracle.eval_rows(expr, [oracle.Column(p, 0, mag, neg)])
    assert [int(g) for g in got[:10]] == [pow(m, 3, N) for m in synth.to_ints(mag, neg)[:10]]
