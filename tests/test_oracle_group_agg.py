"""Pins for oracle.group_aggregate / oracle.agg_type against
things fixed outside the oracle: the paper's aggregate typing rules
 written as closed forms, brute force with Python Fraction on
the generator's raw integers (not via the oracle's per-row evaluator), and
invariants (SUM over groups = ungrouped SUM, MIN(x) = -MAX(-x), AVG of a
constant column)."""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
from gen import synth


def _ceil_log10(N):
    k = 0
    while 10 ** k < N:
        k += 1
    return k


@pytest.mark.parametrize("p,s,N", [(12, 2, 6_000_000), (5, 0, 1), (38, 10, 10), (38, 10, 11), (200, 50, 12_500_000)])
def test_aggregate_typing_closed_forms(p, s, N):
    # MAX/MIN keep the expression's precision
    assert oracle.agg_type("MIN", p, s, N) == (p, s)
    assert oracle.agg_type("MAX", p, s, N) == (p, s)
    # SUM is p + ceil(log10 N)
    assert oracle.agg_type("SUM", p, s, N) == (p + _ceil_log10(N), s)
    # P:L1076-1080 + the division rule P:L1049-1058 with the divisor
    # DECIMAL(ceil(log10 N)+1, 0): (p+c) - (c+1) + 0 + 5 = p + 4, s + 0 + 4
    assert oracle.agg_type("AVG", p, s, N) == (p + 4, s + 4)


def test_hand_example_with_filter_and_empty_group():
    vals = ["1.00", "2.00", "2.00", "-1.00", "-2.00", "-2.00", "7.00"]
    g = [0, 0, 0, 1, 1, 1, -1]          # last row filtered out, group 2 empty
    res, counts, types = oracle.group_aggregate(
        [("SUM", "c1"), ("AVG", "c1"), ("MIN", "c1"), ("MAX", "c1")],
        [oracle.Column(5, 2, strings=vals)], g, 3)
    assert counts == [3, 3, 0]
    assert res[0] == ["5.00", "-5.00", "0.00"]
    # 5/3 = 1.6666..., truncated toward zero at scale 2 + 4
    assert res[1] == ["1.666666", "-1.666666", "0.000000"]
    assert res[2] == ["1.00", "-2.00", "0.00"]
    assert res[3] == ["2.00", "-1.00", "0.00"]
    assert types == [(6, 2), (9, 6), (5, 2), (5, 2)]


def _frac_str(x: Fraction, s: int) -> str:
    q = abs(x) * 10 ** s
    v = q.numerator // q.denominator       # truncation toward zero
    a = str(v).rjust(s + 1, "0") if s else str(v)
    a = (a[:-s] + "." + a[-s:]) if s else a
    return ("-" if x < 0 and v else "") + a


def test_brute_force_fraction_products_grouped():
    n, G = 3000, 5
    types = [(20, 4), (9, 3)]
    cols, ints = [], []
    for k, (p, s) in enumerate(types):
        mag, neg = synth.uniform_decimal(n, p, config=7, column=k + 1)
        cols.append(oracle.Column(p, s, mag, neg))
        ints.append([Fraction(v, 10 ** s) for v in synth.to_ints(mag, neg)])
    gid = (np.arange(n) * 7919) % (G + 1) - 1          # includes -1 (filtered)
    res, counts, _ = oracle.group_aggregate(
        [("SUM", "c1*c2"), ("AVG", "c1*c2"), ("MIN", "c1*c2"), ("MAX", "c2"), ("AVG", "c2")], cols, gid, G)
    for g in range(G):
        rows = [i for i in range(n) if gid[i] == g]
        assert counts[g] == len(rows)
        prod = [ints[0][i] * ints[1][i] for i in rows]      # exact, scale 4 + 3
        c2 = [ints[1][i] for i in rows]
        assert res[0][g] == _frac_str(sum(prod), 7)
        assert res[1][g] == _frac_str(sum(prod) / len(rows), 11)
        assert res[2][g] == _frac_str(min(prod), 7)
        assert res[3][g] == _frac_str(max(c2), 3)
        assert res[4][g] == _frac_str(sum(c2) / len(rows), 7)


def test_invariants_against_ungrouped_sum_and_negation():
    n = 2000
    mag, neg = synth.uniform_decimal(n, 30, config=7, column=9)
    col = oracle.Column(30, 6, mag, neg)
    gid = np.arange(n) % 3
    res, counts, _ = oracle.group_aggregate([("SUM", "c1"), ("MIN", "c1"), ("MAX", "-c1")], [col], gid, 3)
    total, _, _ = oracle.eval_sum("c1", [col])
    # SUM is linear: the groups' sums add up to the ungrouped SUM (orc_eval_sum)
    assert oracle.add_strings(res[0], 40, 6) == total
    # MIN(x) = -MAX(-x)
    for a, b in zip(res[1], res[2]):
        assert Fraction(a) == -Fraction(b)


def test_avg_of_constant_and_count_one():
    col = oracle.Column(9, 3, strings=["-123456.789"] * 9 + ["5.000"])
    res, counts, _ = oracle.group_aggregate([("AVG", "c1")], [col], [0] * 9 + [1], 2)
    assert res[0] == ["-123456.7890000", "5.0000000"]
    assert counts == [9, 1]
