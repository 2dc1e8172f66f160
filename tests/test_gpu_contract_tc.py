"""GPU parity of the tensor-core row contraction (csrc/contract_tc.cu):
SUM(c1*c2) as one u8 x u8 -> s32 integer GEMM over the rows on tcgen05
(kind::i8), exact.  Shapes cover one M tile, several M tiles, a sign digit
alone in its own M tile (4La + 1 = 129), two N tiles (4Lb + 1 > 256), two
N groups (4Lb + 1 > 512), La != Lb; row counts cover empty, ragged tails and
mid-run accumulator drains (UP_TC_RBLOCKS=1: > 32768 rows per CTA).  Expected
values are exact Python integers from the same host inputs."""
import random

import numpy as np
import pytest

from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def _words(vals, p):
    w = ((10 ** p - 1).bit_length() + 31) // 32
    n = len(vals)
    mag = np.zeros((n, w), np.uint32)
    neg = np.zeros(n, np.uint8)
    for i, v in enumerate(vals):
        a = abs(v)
        for j in range(w):
            mag[i, j] = (a >> (32 * j)) & 0xFFFFFFFF
        neg[i] = v < 0
    return mag, neg


def _vals(n, p, rng, mode):
    M = 10 ** p - 1
    if mode == "max":
        return [M if i % 3 else -M for i in range(n)]
    out = []
    for i in range(n):
        r = rng.random()
        if r < 0.05:
            v = M
        elif r < 0.08:
            v = 0
        elif r < 0.12:
            v = rng.randrange(min(2 ** 32, M + 1))
        else:
            v = rng.randrange(M + 1)
        out.append(v if rng.random() < 0.5 else -v)
    return out


def _check(p1, p2, n, mode, seed, s1=3, s2=7):
    from paper_conf_icde_lixylz24_b200 import up
    rng = random.Random(seed)
    a, b = _vals(n, p1, rng, mode), _vals(n, p2, rng, "max" if mode == "max" else "rand")
    c = up.Context(0)
    cols = [c.column_from_host_bin(p1, s1, *_words(a, p1)), c.column_from_host_bin(p2, s2, *_words(b, p2))]
    P, S, LA = c.sum_type("c1*c2", cols)
    got = G.limbs_int(c.sum_expr("c1*c2", cols))
    c.check()
    assert got == sum(x * y for x, y in zip(a, b)), (p1, p2, n, mode)   # mantissas at scale S: exact integers


@pytest.mark.parametrize("p1,p2", [(90, 90), (200, 200), (300, 120), (305, 305), (500, 500), (1000, 1000),
                                   (1300, 700), (700, 1300), (9, 1000), (1000, 9), (38, 300)])
@pytest.mark.parametrize("n", [1, 129, 3001])
def test_tc_contraction_shapes(p1, p2, n, monkeypatch):
    monkeypatch.setenv("UP_SPLIT", "1")
    _check(p1, p2, n, "rand", seed=p1 * 31 + p2 + n)


@pytest.mark.parametrize("p", [200, 1000])
def test_tc_contraction_extremes(p, monkeypatch):
    monkeypatch.setenv("UP_SPLIT", "1")
    _check(p, p, 4000, "max", seed=p)


def test_tc_contraction_mid_run_drains(monkeypatch):
    """one row block: every CTA accumulates > 32768 rows, so the s32 TMEM
    accumulator is drained mid-run (several times) -- still exact with
    all-nines digits (each drain window at the s32 bound's order)"""
    monkeypatch.setenv("UP_SPLIT", "1")
    monkeypatch.setenv("UP_TC_RBLOCKS", "1")
    _check(120, 120, 100_000, "max", seed=1)
    _check(120, 100, 70_001, "rand", seed=2)


def test_tc_contraction_empty(monkeypatch):
    monkeypatch.setenv("UP_SPLIT", "1")
    from paper_conf_icde_lixylz24_b200 import up
    c = up.Context(0)
    cols = [c.column_from_host_bin(200, 2, np.zeros((0, 21), np.uint32)),
            c.column_from_host_bin(200, 2, np.zeros((0, 21), np.uint32))]
    P, S, LA = c.sum_type("c1*c2", cols)
    assert G.limbs_int(c.sum_expr("c1*c2", cols)) == 0


def test_tc_two_products_and_signs(monkeypatch):
    """two top-level products (two contractions sharing the workspace, one
    negated) plus a rest term, vs exact Python"""
    monkeypatch.setenv("UP_SPLIT", "1")
    from paper_conf_icde_lixylz24_b200 import up
    rng = random.Random(7)
    n, p = 2500, 250
    cols_v = [_vals(n, p, rng, "rand") for _ in range(4)]
    c = up.Context(0)
    cols = [c.column_from_host_bin(p, 0, *_words(v, p)) for v in cols_v]
    expr = "c1*c2 - c3*c4 + c1"
    P, S, LA = c.sum_type(expr, cols)
    got = G.limbs_int(c.sum_expr(expr, cols))
    c.check()
    a, b, x, y = cols_v
    assert got == sum(a[i] * b[i] - x[i] * y[i] + a[i] for i in range(n))
