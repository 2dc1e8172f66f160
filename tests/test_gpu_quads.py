"""GPU parity of limb-quad columns (up.h UP_LAYOUT_QUADS: four limbs of a row
per 16 bytes, the sign flag in limb L).  The layout exists so that SUM(c_a*c_b)
feeds the tensor cores straight from TMA copies (contract_tc.cu
k_contract_tq: the schoolbook product of P:L576-607 with the row sum of
P:L1069-1080 moved inside it, as a u8 x u8 -> s32 GEMM over the rows); every
generated kernel reads it too.  Covered: ingestion / read-back round trip,
the quad contraction against exact Python integers (one / several M tiles, a
sign digit in its own quad, two N tiles, two N groups, La != Lb, ragged tails,
empty input, mid-run drains with double-buffered and single TMEM
accumulators), cfg3's SUM(c1*c2 - c3/c4) and per-row eval against the oracle,
mixed layouts in one expression, and the entry points that refuse quads."""
import random

import numpy as np
import pytest

import oracle
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def _words(vals, p):
    w = ((10 ** p - 1).bit_length() + 31) // 32
    mag = np.zeros((len(vals), w), np.uint32)
    neg = np.zeros(len(vals), np.uint8)
    for i, v in enumerate(vals):
        a = abs(v)
        for j in range(w):
            mag[i, j] = (a >> (32 * j)) & 0xFFFFFFFF
        neg[i] = v < 0
    return mag, neg


def _vals(n, p, rng, mode="rand"):
    M = 10 ** p - 1
    if mode == "max":
        return [M if i % 3 else -M for i in range(n)]
    out = []
    for _ in range(n):
        r = rng.random()
        v = M if r < 0.05 else 0 if r < 0.08 else rng.randrange(min(2 ** 32, M + 1)) if r < 0.12 else rng.randrange(M + 1)
        out.append(v if rng.random() < 0.5 else -v)
    return out


@pytest.mark.parametrize("p", [9, 17, 38, 200, 300, 1000])
@pytest.mark.parametrize("n", [1, 5, 1027])
def test_quads_round_trip(p, n):
    rng = random.Random(p * 7 + n)
    vals = _vals(n, p, rng)
    c = G.ctx()
    col = c.column_from_host_bin(p, 2, *_words(vals, p), layout="quads")
    assert col.data.shape[0] == (col.limbs + 4) // 4
    assert c.column_to_ints(col) == vals
    # the stored words: limbs in two's complement, the sign flag at limb L, zero padding
    q = col.data.cpu().numpy().astype(np.uint32)
    L = col.limbs
    for i in (0, n - 1):
        words = [int(q[j // 4, i, j % 4]) for j in range(4 * q.shape[0])]
        v = vals[i] % (1 << (32 * L))
        assert words[:L] == [(v >> (32 * j)) & 0xFFFFFFFF for j in range(L)]
        assert words[L] == (1 if vals[i] < 0 else 0) and not any(words[L + 1:])


def _contract(p1, p2, n, mode, seed):
    rng = random.Random(seed)
    a, b = _vals(n, p1, rng, mode), _vals(n, p2, rng, "max" if mode == "max" else "rand")
    c = G.ctx()
    cols = [c.column_from_host_bin(p1, 3, *_words(a, p1), layout="quads"),
            c.column_from_host_bin(p2, 7, *_words(b, p2), layout="quads")]
    got = G.limbs_int(c.sum_expr("c1*c2", cols))
    c.check()
    assert got == sum(x * y for x, y in zip(a, b)), (p1, p2, n, mode)


# shapes: Ga = ceil((La + 1) / 4) quads; (90: L 10 -> 3 quads), (200: 21 -> 6), (300: 32 -> 9 quads: the sign
# flag alone in quad 8 = a second M tile), (305: 32), (500: 52 -> 14), (1000: 104 -> 27 quads: two N tiles),
# (1300: 135 -> 34 quads: two N groups), (9: one limb)
@pytest.mark.parametrize("p1,p2", [(90, 90), (200, 200), (300, 120), (305, 305), (500, 500), (1000, 1000),
                                   (1300, 700), (700, 1300), (9, 1000), (1000, 9), (38, 300)])
@pytest.mark.parametrize("n", [1, 129, 3001])
def test_quad_contraction_shapes(p1, p2, n, monkeypatch):
    monkeypatch.setenv("UP_SPLIT", "1")
    _contract(p1, p2, n, "rand", seed=p1 * 31 + p2 + n)


@pytest.mark.parametrize("p", [200, 1000])
def test_quad_contraction_extremes(p, monkeypatch):
    monkeypatch.setenv("UP_SPLIT", "1")
    _contract(p, p, 4000, "max", seed=p)


@pytest.mark.parametrize("p", [200, 1000])
def test_quad_contraction_mid_run_drains(p, monkeypatch):
    """one row block: the CTA accumulates 70000 rows, i.e. 3 accumulation
    windows of <= 32768 rows -- p = 200 alternates two TMEM accumulators
    (W = 96 columns each), p = 1000 reuses one (W = 432): the MMA issuer
    waits for the drain of the window before"""
    monkeypatch.setenv("UP_SPLIT", "1")
    monkeypatch.setenv("UP_TC_RBLOCKS", "1")
    _contract(p, p, 70000, "max", seed=p + 1)
    _contract(p, p, 70001, "rand", seed=p + 2)


def test_quad_contraction_empty():
    c = G.ctx()
    empty = np.zeros((0, 1), np.uint32)
    cols = [c.column_from_host_bin(200, 0, empty, layout="quads"), c.column_from_host_bin(200, 0, empty, layout="quads")]
    assert G.limbs_int(c.sum_expr("c1*c2", cols)) == 0
    c.check()


CFG3 = [(200, 50), (500, 75), (1000, 100)]


@pytest.mark.parametrize("lays", ["qqqq", "qqpp"])
@pytest.mark.parametrize("serial", [False, True], ids=["side-stream", "serial"])
@pytest.mark.parametrize("ps", CFG3, ids=lambda t: f"p{t[0]}")
@pytest.mark.parametrize("n", [1, 1000, 4099])
def test_cfg3_sum_quads(ps, n, serial, lays, monkeypatch):
    """cfg3's SUM(c1*c2 - c3/c4) with c1, c2 in quads (tensor-core contraction
    on the ctx side stream beside the fused top-limb division, or both on one
    stream with UP_SERIAL_SPLIT; c3, c4 quads or planes -- the bench's "mixed")
    == the oracle"""
    if serial:
        monkeypatch.setenv("UP_SERIAL_SPLIT", "1")
    types = [ps] * 4
    host = G.gen_cols(n, types, config=3, nonzero_lead_cols=(3,))
    want, P, S = oracle.eval_sum("c1*c2 - c3/c4", G.to_oracle(host, types), n=n, threads=8)
    c = G.ctx()
    layout = {"q": "quads", "p": "planes"}
    gcols = [c.column_from_host_bin(p, s, m, g, layout=layout[lays[k]]) for k, ((m, g), (p, s)) in enumerate(zip(host, types))]
    got, gP, gS = G.gpu_sum_string("c1*c2 - c3/c4", gcols)
    assert (gP, gS) == (P, S)
    assert got == want


def test_cfg3_quads_back_to_back_pipelined():
    """K split SUMs back to back on one stream with pipelined (PDL) launches:
    the contraction, the rest kernel and the combine of consecutive steps
    share the partials buffer and the workspace -- every result must be the
    oracle's"""
    import torch
    types = [(200, 50)] * 4
    n = 70001
    host = G.gen_cols(n, types, config=3, nonzero_lead_cols=(3,))
    want, P, S = oracle.eval_sum("c1*c2 - c3/c4", G.to_oracle(host, types), n=n, threads=8)
    c = G.ctx()
    gcols = [c.column_from_host_bin(p, s, m, g, layout="quads") for (m, g), (p, s) in zip(host, types)]
    from paper_conf_icde_lixylz24_b200 import up
    _, S2, LA = c.sum_type("c1*c2 - c3/c4", gcols)
    outs = [torch.empty(LA, dtype=torch.int32, device="cuda") for _ in range(6)]
    c.set_pipelined(True)
    try:
        for o in outs:
            c.sum_expr("c1*c2 - c3/c4", gcols, out=o)
        c.check()
    finally:
        c.set_pipelined(False)
    assert all(up.result_to_string(o, S) == want for o in outs)


CASES = [
    ("c1+c2", [(17, 5), (14, 2)], ["quads", "quads"]),             # narrow regime: 4 rows per thread
    ("c1+c2", [(35, 5), (32, 2)], ["quads", "planes"]),
    ("c1*c2 - c3/c4", [(200, 50)] * 4, ["quads"] * 4),            # top-limb division over quads
    ("c1*c2 - c3/c4", [(200, 50)] * 4, ["quads", "planes", "planes", "quads"]),
    ("c1/c2 + c3", [(30, 4), (11, 2), (20, 6)], ["quads", "quads", "compact"]),
    ("c1 % c2", [(25, 0), (13, 0)], ["quads", "quads"]),
]


@pytest.mark.parametrize("case", CASES, ids=lambda c: c[0].replace(" ", "") + "@" + "".join(x[0] for x in c[2]))
def test_quads_eval_parity(case):
    expr, types, lays = case
    n = 2053
    lead = [k for k in range(len(types)) if f"/c{k + 1}" in expr.replace(" ", "") or f"%c{k + 1}" in expr.replace(" ", "")]
    host = G.gen_cols(n, types, nonzero_lead_cols=lead)
    want = oracle.eval_rows(expr, G.to_oracle(host, types), strict=False)
    c = G.ctx()
    gcols = [c.column_from_host_bin(p, s, m, g, layout=l) for (m, g), (p, s), l in zip(host, types, lays)]
    out = c.eval_expr(expr, gcols)
    try:
        c.check()
    except Exception:
        pass
    got = c.column_to_strings(out)
    for g, w in zip(got, want):
        if not w.startswith("E"):
            assert g == w
    sgot, sP, sS = None, None, None
    if not any(w.startswith("E") for w in want):
        sgot, sP, sS = G.gpu_sum_string(expr, gcols)
        swant, P, S = oracle.eval_sum(expr, G.to_oracle(host, types), n=n, threads=4)
        assert (sP, sS) == (P, S) and sgot == swant


def test_quads_compact_ingest_and_readback():
    """the paper's compact rows -> quads -> compact rows and ints"""
    from paper_conf_icde_lixylz24_b200 import up
    rng = random.Random(5)
    p, n = 200, 777
    vals = _vals(n, p, rng)
    c = G.ctx()
    planes = c.column_from_host_bin(p, 0, *_words(vals, p))
    comp = c.column_to_compact(planes)
    q = c.column_from_compact(p, 0, comp, n=n, layout="quads")
    assert c.column_to_ints(q) == vals
    assert bytes(c.column_to_compact(q)) == bytes(comp)
    assert q.layout == up.LAYOUT_QUADS
    import torch   # the device-buffer entry point (up_column_from_device_compact) into quads
    qd = c.column_from_compact(p, 0, torch.from_numpy(comp).cuda(), n=n, layout="quads")
    assert c.column_to_ints(qd) == vals


def test_quads_refused_where_unsupported():
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    x = c.column_from_host_bin(300, 0, *_words([5, 7], 300), layout="quads")
    with pytest.raises(up.UpError):
        c.modexp(x, 3, 2 ** 521 - 1)
    with pytest.raises(up.UpError):
        c.eval_tpi("+", x, x, tpi=4)
    with pytest.raises(up.UpError):
        c.group_aggregate([("SUM", "c1")], [x])


@pytest.mark.parametrize("op", ["<", "=", ">="])
@pytest.mark.parametrize("lhs,rhs,types,n", [
    ("c1", "c2", [(4, 1), (3, 2)], 1001),                        # narrow: 4 rows per thread
    ("c1 / c2", "c3", [(200, 50), (200, 50), (6, 4)], 503),       # top-limb division over quads
    ("c1 * c2 - c3", "0", [(60, 10), (50, 20), (100, 30)], 301),
])
def test_quads_filter_parity(op, lhs, rhs, types, n):
    """WHERE over quad columns (up_filter reads quads like planes) == the oracle"""
    import torch
    host = G.gen_cols(n, types, config=11, nonzero_lead_cols=(1,) if "/" in lhs else ())
    c = G.ctx()
    g = [c.column_from_host_bin(p, s, m, ng, layout="quads") for (m, ng), (p, s) in zip(host, types)]
    pre = np.where(np.arange(n) % 11 == 0, -1, 0).astype(np.int32)
    ids = c.filter(lhs, op, rhs, g, torch.as_tensor(pre, device="cuda"))
    c.check()
    assert ids.cpu().tolist() == oracle.filter_ids(lhs, op, rhs, G.to_oracle(host, types), pre.tolist())
