"""Pins for the oracle's WHERE comparison and GROUP BY ids (SURVEY A22/K10,
NEXT-4; Sec. II-C: DECIMAL comparison operators, used to sort for
grouping).  Pinned by brute force on the mantissas (value = m 10^-s, so two
values compare as m_a 10^(S - s_a) vs m_b 10^(S - s_b) at a common scale S),
Python tuple sorting, closed forms and the paper's own 0.1 + 0.2 = 0.3."""
import numpy as np
import pytest

import oracle
from gen import synth


def _col(vals, p, s):
    """Column from signed Python-int mantissas."""
    n = len(vals)
    w = max(1, (max(abs(v) for v in vals).bit_length() + 31) // 32) if n else 1
    mag = np.zeros((n, w), np.uint32)
    neg = np.zeros(n, np.uint8)
    for i, v in enumerate(vals):
        a = abs(v)
        for j in range(w):
            mag[i, j] = (a >> (32 * j)) & 0xFFFFFFFF
        neg[i] = v < 0
    return oracle.Column(p, s, mag, neg)


def test_filter_closed_forms_paper_example():
    # 0.1 + 0.2 = 0.3 exactly (the paper's motivating example)
    a, b = _col([1, 1, 1], 2, 1), _col([2, 2, 3], 2, 1)
    assert oracle.filter_ids("c1 + c2", "=", "0.3", [a, b]) == [0, 0, -1]
    assert oracle.filter_ids("c1 + c2", ">", "0.3", [a, b]) == [-1, -1, 0]
    # 1/3 at the division rule's scale s1 + 4 truncates to 0.3333 (reading Q4)
    one, three = _col([1], 1, 0), _col([3], 1, 0)
    assert oracle.filter_ids("c1 / c2", "=", "0.3333", [one, three]) == [0]
    assert oracle.filter_ids("c1 / c2", "<", "0.33334", [one, three]) == [0]
    # equal values at different scales: 1.5 = 1.50
    assert oracle.filter_ids("c1", "=", "c2", [_col([15], 2, 1), _col([150], 3, 2)]) == [0]


@pytest.mark.parametrize("op", oracle.CMP_OPS)
def test_filter_brute_force_mixed_scales(op):
    r = np.random.default_rng(7)
    n = 300
    va = [int(x) for x in r.integers(-10 ** 6, 10 ** 6, n)]
    vb = [int(x) for x in r.integers(-10 ** 4, 10 ** 4, n)]
    vb[::7] = [a // 100 if a >= 0 else -((-a) // 100) for a in va[::7]]   # some equal values
    a, b = _col(va, 7, 3), _col(vb, 5, 1)
    want = []
    for x, y in zip(va, vb):   # compare at the common scale 3: y * 10^2
        X, Y = x, y * 100
        ok = {"<": X < Y, "<=": X <= Y, ">": X > Y, ">=": X >= Y, "=": X == Y, "==": X == Y,
              "<>": X != Y, "!=": X != Y}[op]
        want.append(0 if ok else -1)
    assert oracle.filter_ids("c1", op, "c2", [a, b]) == want
    # AND semantics: already-excluded rows stay excluded
    pre = [-1 if i % 5 == 0 else 0 for i in range(n)]
    got = oracle.filter_ids("c1", op, "c2", [a, b], pre)
    assert got == [-1 if (i % 5 == 0 or w < 0) else 0 for i, w in enumerate(want)]


def test_group_ids_single_key_brute_force():
    m, g = synth.uniform_decimal(2000, 2, 9, 1)
    col = oracle.Column(2, 1, m, g)
    vals = synth.to_ints(m, g)
    ids, ng, first = oracle.group_ids([col])
    distinct = sorted(set(vals))
    assert ng == len(distinct)
    assert ids == [distinct.index(v) for v in vals]
    assert first == [vals.index(v) for v in distinct]
    # order-preserving: key_i < key_j  <=>  id_i < id_j
    for i in range(0, 2000, 37):
        for j in range(0, 2000, 41):
            assert (vals[i] < vals[j]) == (ids[i] < ids[j])


def test_group_ids_multi_key_and_exclusion():
    r = np.random.default_rng(3)
    n = 500
    k1 = [int(x) for x in r.integers(-3, 3, n)]
    k2 = [int(x) for x in r.integers(-2, 2, n)]
    pre = [-1 if x % 9 == 0 else 0 for x in range(n)]
    ids, ng, first = oracle.group_ids([_col(k1, 2, 0), _col(k2, 3, 2)], pre)
    tuples = sorted({(a, b) for a, b, e in zip(k1, k2, pre) if e >= 0})
    assert ng == len(tuples)
    for i in range(n):
        assert ids[i] == (-1 if pre[i] < 0 else tuples.index((k1[i], k2[i])))
    for gi, t in enumerate(tuples):
        assert first[gi] == min(i for i in range(n) if pre[i] >= 0 and (k1[i], k2[i]) == t)


def test_group_ids_degenerate():
    c = _col([5, 5, 5], 1, 0)
    assert oracle.group_ids([c]) == ([0, 0, 0], 1, [0])
    assert oracle.group_ids([c], [-1, -1, -1]) == ([-1, -1, -1], 0, [])
    z = _col([0, -0, 0], 1, 0)            # -0 is 0 (reading Q10)
    assert oracle.group_ids([z])[1] == 1
