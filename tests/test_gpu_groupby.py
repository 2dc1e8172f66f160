"""GPU parity of up_filter (WHERE with DECIMAL comparison operators) and
up_group_ids (GROUP BY DECIMAL keys via sorting), SURVEY A22/K10 / NEXT-4
(Sec. II-C), against oracle.filter_ids / oracle.group_ids element
by element: every operator, mixed scales, quotients, narrow (4 rows per
thread) and per-thread regimes with ragged tails, multi-column and wide keys,
negative keys, exclusion, degenerate sizes; then the whole
WHERE -> GROUP BY -> aggregate pipeline against the oracle."""
import numpy as np
import pytest

import oracle
from gen import synth
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("op", ["<", "<=", ">", ">=", "=", "<>"])
@pytest.mark.parametrize("lhs,rhs,types,n", [
    ("c1", "c2", [(4, 1), (3, 2)], 1001),                      # narrow, mixed scales, ragged tail
    ("c1", "c2", [(2, 1), (3, 2)], 1001),                      # many equal values
    ("c1 * c2", "c1 + 1.5", [(9, 2), (8, 3)], 777),
    ("c1 / c2", "c3", [(20, 5), (12, 3), (6, 4)], 503),         # quotient (Knuth D), per-thread regime
    ("c1 * c2 - c3", "0", [(60, 10), (50, 20), (100, 30)], 301),   # wide
])
def test_filter_parity(op, lhs, rhs, types, n):
    import torch
    host = G.gen_cols(n, types, config=11, nonzero_lead_cols=(1,) if "/" in lhs else ())
    if op in ("=", "<>") and lhs == "c1":
        # force equal values on a third of the rows: c2 := c1 rounded to 1 fraction digit -> scale 2
        m1, g1 = host[0]
        v1 = synth.to_ints(m1, g1)
        m2, g2 = host[1]
        v2 = synth.to_ints(m2, g2)
        v2 = [(a * 10 if i % 3 == 0 and abs(a) < 100 else b) for i, (a, b) in enumerate(zip(v1, v2))]
        host[1] = _words(v2, 1)
    c = G.ctx()
    g = G.to_gpu(host, types)
    pre = np.where(np.arange(n) % 11 == 0, -1, 0).astype(np.int32)
    ids = c.filter(lhs, op, rhs, g, torch.as_tensor(pre, device="cuda"))
    c.check()
    want = oracle.filter_ids(lhs, op, rhs, G.to_oracle(host, types), pre.tolist())
    assert ids.cpu().tolist() == want


def _words(vals, w):
    mag = np.zeros((len(vals), w), np.uint32)
    neg = np.zeros(len(vals), np.uint8)
    for i, v in enumerate(vals):
        a = abs(v)
        for j in range(w):
            mag[i, j] = (a >> (32 * j)) & 0xFFFFFFFF
        neg[i] = v < 0
    return mag, neg


@pytest.mark.parametrize("types,n,excl", [
    ([(2, 1)], 5000, 0.0),            # ~199 distinct values, many duplicates
    ([(2, 1)], 4097, 0.2),            # with excluded rows
    ([(1, 0), (2, 2)], 3000, 0.1),    # two key columns, lexicographic
    ([(40, 5)], 1000, 0.0),           # wide (5-limb) keys: all distinct
    ([(12, 2), (1, 0), (30, 0)], 2500, 0.05),
])
def test_group_ids_parity(types, n, excl):
    import torch
    host = G.gen_cols(n, types, config=12)
    if types[0][0] >= 12:              # few distinct leading keys: reuse values
        m, g = host[0]
        v = synth.to_ints(m, g)
        host[0] = _words([v[i % 37] for i in range(n)], m.shape[1])
    r = np.random.default_rng(5)
    pre = np.where(r.random(n) < excl, -1, 0).astype(np.int32)
    c = G.ctx()
    g = G.to_gpu(host, types)
    ids, ng, first = c.group_ids(g, torch.as_tensor(pre, device="cuda"), first=True)
    want, wng, wfirst = oracle.group_ids(G.to_oracle(host, types), pre.tolist())
    assert ng == wng
    assert ids.cpu().tolist() == want
    assert first.cpu().tolist() == wfirst


def test_group_ids_degenerate():
    import torch
    c = G.ctx()
    one = c.column_from_strings(3, 1, ["-1.5"])
    ids, ng = c.group_ids([one])
    assert ng == 1 and ids.cpu().tolist() == [0]
    col = c.column_from_strings(3, 1, ["1.0", "-0.0", "0.0", "-1.0"])
    ids, ng = c.group_ids([col])
    assert ng == 3 and ids.cpu().tolist() == [2, 1, 1, 0]       # -0 = 0 (reading Q10)
    ids, ng = c.group_ids([col], torch.full((4,), -1, dtype=torch.int32, device="cuda"))
    assert ng == 0 and ids.cpu().tolist() == [-1] * 4
    empty = c.column_from_strings(3, 1, [])
    ids, ng = c.group_ids([empty])
    assert ng == 0


def test_where_group_by_aggregate_pipeline():
    """SELECT k, SUM(c2*c3), MIN(c2), MAX(c3), AVG(c2) FROM t WHERE c2 > c3 - 50
    GROUP BY k, all on the GPU, against the oracle's filter -> group ids ->
    group_aggregate."""
    import torch
    from paper_conf_icde_lixylz24_b200 import up
    n = 20000
    types = [(2, 0), (9, 2), (10, 3)]
    host = G.gen_cols(n, types, config=13)
    c = G.ctx()
    g = G.to_gpu(host, types)
    ids = c.filter("c2", ">", "c3 - 50", g)
    ids, ng = c.group_ids([g[0]], ids)
    aggs = [("SUM", "c2*c3"), ("MIN", "c2"), ("MAX", "c3"), ("AVG", "c2")]
    out, counts, layout = c.group_aggregate(aggs, g, ids, ng)
    c.check()
    got, got_counts = up.group_results(out, counts, layout, ng)
    o = G.to_oracle(host, types)
    wids = oracle.filter_ids("c2", ">", "c3 - 50", o)
    wids, wng, _ = oracle.group_ids([o[0]], wids)
    assert ng == wng and ids.cpu().tolist() == wids
    want, wcounts, _ = oracle.group_aggregate(aggs, o, wids, wng)
    assert got_counts == wcounts
    assert got == want
