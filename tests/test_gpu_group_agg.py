"""GPU parity of up_group_aggregate (grouped SUM / MIN / MAX /
AVG with the paper's aggregate typing) against
oracle.group_aggregate, element by element, on seeded inputs: the TPC-H Q1
shape, wide types with products and quotients, one group and
many groups, filtered rows, empty groups, extreme values."""
import numpy as np
import pytest

import oracle
from gen import synth
from tests import gpu_util as G

pytestmark = pytest.mark.gpu

Q1_AGGS = [("SUM", "c1"), ("SUM", "c2"), ("SUM", "c2*(1-c3)"), ("SUM", "c2*(1-c3)*(1+c4)"),
           ("AVG", "c1"), ("AVG", "c2"), ("AVG", "c3")]


def _gid(n, n_groups, seed, filtered=0.1):
    r = np.random.default_rng(seed)
    g = r.integers(0, n_groups, n).astype(np.int32)
    g[r.random(n) < filtered] = -1
    return g


def _check(aggs, host, types, gid, n_groups, n_global=0):
    import torch
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    gcols = G.to_gpu(host, types)
    dg = torch.as_tensor(gid, device="cuda") if gid is not None else None
    out, counts, layout = c.group_aggregate(aggs, gcols, dg, n_groups, n_global)
    c.check()
    got, got_counts = up.group_results(out, counts, layout, n_groups)
    want, want_counts, want_types = oracle.group_aggregate(aggs, G.to_oracle(host, types), gid, n_groups, n_global)
    assert [(p, s) for p, s, _, _ in layout] == want_types
    assert got_counts == want_counts
    for a, (g_a, w_a) in enumerate(zip(got, want)):
        assert g_a == w_a, f"aggregate {a} {aggs[a]}"
    return out


@pytest.mark.parametrize("n", [1, 31, 10007])
def test_tpch_q1_shape(n):
    types = [(12, 2), (12, 2), (3, 2), (3, 2)]
    host = G.gen_cols(n, types, config=8)
    _check(Q1_AGGS, host, types, _gid(n, 4, n), 4)


@pytest.mark.parametrize("types,lead", [([(60, 10), (45, 5)], (1,)), ([(150, 30), (140, 20)], (1,))])
def test_all_kinds_wide(types, lead):
    n = 3001
    host = G.gen_cols(n, types, config=8, nonzero_lead_cols=lead, seed=5)
    aggs = [(k, e) for e in ("c1*c2", "c1/c2", "c1-c2") for k in ("SUM", "MIN", "MAX", "AVG")]
    _check(aggs, host, types, _gid(n, 7, 3), 7)


def test_one_group_null_ids_and_n_global():
    types = [(30, 6)]
    host = G.gen_cols(4099, types, config=8, seed=9)
    _check([("SUM", "c1"), ("MIN", "c1"), ("MAX", "c1"), ("AVG", "c1")], host, types, None, 1, n_global=10 ** 9)


def test_many_groups():
    types = [(18, 4), (9, 2)]
    n = 40000
    host = G.gen_cols(n, types, config=8, seed=11)
    _check([("SUM", "c1+c2"), ("MAX", "c1*c2"), ("AVG", "c2")], host, types, _gid(n, 250, 4), 250)


def test_extremes_all_filtered_and_empty_groups():
    from paper_conf_icde_lixylz24_b200 import up
    p = 38
    big = str(10 ** p - 1)
    vals = [big, "-" + big] * 40 + ["0", "-1", "1"]
    n = len(vals)
    c = G.ctx()
    col = c.column_from_strings(p, 0, vals)
    ocol = oracle.Column(p, 0, strings=vals)
    import torch
    for gid, ng in ((np.zeros(n, np.int32), 3), (np.full(n, -1, np.int32), 2), (np.arange(n, dtype=np.int32) % 2, 2)):
        aggs = [("SUM", "c1"), ("MIN", "c1"), ("MAX", "c1"), ("AVG", "c1"), ("MIN", "-c1")]
        out, counts, layout = c.group_aggregate(aggs, [col], torch.as_tensor(gid, device="cuda"), ng)
        c.check()
        got, gc = up.group_results(out, counts, layout, ng)
        want, wc, _ = oracle.group_aggregate(aggs, [ocol], gid, ng)
        assert gc == wc and got == want


def test_bad_group_id_sets_flag():
    import torch
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    col = c.column_from_strings(5, 0, ["1", "2", "3"])
    gid = torch.tensor([0, 5, 1], dtype=torch.int32, device="cuda")
    c.group_aggregate([("SUM", "c1")], [col], gid, 2)
    with pytest.raises(up.UpError) as ei:
        c.check()
    assert ei.value.name == "INVAL"


def test_repeat_launches_are_deterministic():
    types = [(12, 2), (12, 2), (3, 2), (3, 2)]
    n = 50000
    host = G.gen_cols(n, types, config=8, seed=13)
    gid = _gid(n, 4, 7)
    a = _check(Q1_AGGS + [("MIN", "c2*(1-c3)"), ("MAX", "c1")], host, types, gid, 4)
    b = _check(Q1_AGGS + [("MIN", "c2*(1-c3)"), ("MAX", "c1")], host, types, gid, 4)
    assert bool((a == b).all())


@pytest.mark.parametrize("nranks", [2, 3, 5])
@pytest.mark.parametrize("case", ["q1", "wide"])
def test_multi_rank_group_combine(nranks, case):
    """Row shards' group_aggregate(partial=True) (AVG as SUM, global-N typing),
    concatenated rank-major as an all-gather would, merged by up_group_combine
    == the oracle's whole-table aggregates (includes groups empty on some
    ranks: with 7 groups and 200 rows over 5 shards)."""
    import torch
    from paper_conf_icde_lixylz24_b200 import up
    if case == "q1":
        types, aggs, n, ng = [(12, 2), (12, 2), (3, 2), (3, 2)], Q1_AGGS + [("MIN", "c1"), ("MAX", "c2*(1-c3)")], 6007, 4
        host = G.gen_cols(n, types, config=8)
    else:
        types, n, ng = [(60, 10), (45, 5)], 200, 7
        aggs = [(k, e) for e in ("c1*c2", "c1/c2") for k in ("SUM", "MIN", "MAX", "AVG")]
        host = G.gen_cols(n, types, config=8, nonzero_lead_cols=(1,), seed=11)
    gid = _gid(n, ng, 17)
    c = G.ctx()
    parts, cnts = [], []
    for r in range(nranks):
        lo, hi = n * r // nranks, n * (r + 1) // nranks
        sh = [(m[lo:hi], g[lo:hi]) for m, g in host]
        gcols = G.to_gpu(sh, types) if hi > lo else [c.column_from_host_bin(p, s, np.zeros((0, 1), np.uint32))
                                                      for p, s in types]
        dg = torch.as_tensor(np.ascontiguousarray(gid[lo:hi]), device="cuda")
        o, k, _ = c.group_aggregate(aggs, gcols, dg if hi > lo else None, ng, n, partial=True) if hi > lo else \
            (None, None, None)
        if o is None:
            continue
        parts.append(o)
        cnts.append(k)
    out, counts, layout = c.group_combine(aggs, G.to_gpu(host, types), torch.cat(parts), torch.cat(cnts), len(parts),
                                          ng, n)
    c.check()
    got, got_counts = up.group_results(out, counts, layout, ng)
    want, want_counts, want_types = oracle.group_aggregate(aggs, G.to_oracle(host, types), gid, ng, n)
    assert [(p, s) for p, s, _, _ in layout] == want_types
    assert got_counts == want_counts
    for a, (g_a, w_a) in enumerate(zip(got, want)):
        assert g_a == w_a, f"aggregate {a} {aggs[a]}"
