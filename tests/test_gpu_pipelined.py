"""Pipelined SUM launches (up_set_pipelined: programmatic dependent launch of
the fused SUM kernels).  Back-to-back SUMs over resident columns are enqueued
with no synchronisation between them -- each kernel's CTAs may start while
the previous one finishes and wait for it before touching the shared SUM
workspace -- and every result must still equal the oracle's.  Mixes kernels
with different workspace widths, the compact layout, the tensor-core split
SUM (its rest kernel follows the contraction kernel) and repeats of the same
query, so a workspace / ticket / result hand-over bug would show."""
import pytest

import oracle
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def _oracle_sum(expr, host, types):
    return oracle.eval_sum(expr, G.to_oracle(host, types), threads=8)[0]


def test_back_to_back_pipelined_sums_match_oracle():
    import torch
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    n = 300_001
    t2 = [(35, 5), (32, 2)]
    t1 = [(17, 5), (14, 2)]
    t3 = [(60, 10), (40, 5)]
    h2, h1, h3 = G.gen_cols(n, t2, config=2), G.gen_cols(n, t1, config=1), G.gen_cols(n, t3, config=9)
    g2, g1, g3 = G.to_gpu(h2, t2), G.to_gpu(h1, t1), G.to_gpu(h3, t3)
    g2c = [c.column_from_host_bin(p, s, m, g, layout="compact") for (m, g), (p, s) in zip(h2, t2)]
    queries = [("c1+c2", g2, h2, t2), ("c1+c2", g2, h2, t2), ("c1-c2", g1, h1, t1), ("c1*c2", g3, h3, t3),
               ("c1+c2", g2c, h2, t2), ("c1+c2", g2, h2, t2), ("c1*c2-c2", g3, h3, t3), ("c1", g1, h1, t1)]
    want = {}
    for expr, _, h, t in queries:
        key = (expr, id(h))
        if key not in want:
            want[key] = _oracle_sum(expr, h, t)
    c.set_pipelined(True)
    try:
        outs = []
        for rep in range(3):
            for expr, g, h, t in queries:
                P, S, LA = c.sum_type(expr, g)
                o = torch.full((LA,), -1, dtype=torch.int32, device="cuda")
                c.sum_expr(expr, g, out=o)          # no sync between the launches
                outs.append((o, S, (expr, id(h))))
        c.check()
        for o, S, key in outs:
            assert up.result_to_string(o, S) == want[key]
    finally:
        c.set_pipelined(False)


def test_pipelined_split_sum_matches_oracle():
    """cfg3's shape: tensor-core contraction, then the pipelined rest kernel."""
    import torch
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    n = 40_003
    t = [(200, 50)] * 4
    h = G.gen_cols(n, t, config=3, nonzero_lead_cols=(3,))
    g = G.to_gpu(h, t)
    expr = "c1*c2 - c3/c4"
    want = _oracle_sum(expr, h, t)
    c.set_pipelined(True)
    try:
        P, S, LA = c.sum_type(expr, g)
        outs = [torch.zeros(LA, dtype=torch.int32, device="cuda") for _ in range(4)]
        for o in outs:
            c.sum_expr(expr, g, out=o)
        c.check()
        assert all(up.result_to_string(o, S) == want for o in outs)
    finally:
        c.set_pipelined(False)
