"""GPU parity of compact-resident columns (the paper's cDecimal
rows, Fig. 4, read in place by the fused kernels: Listing 1's
"expand" step).  Every case evaluates the same seeded columns held
in the compact layout (up.h UP_LAYOUT_COMPACT), and where mixed, some in limb
planes, against the oracle -- SUM and per-row eval, 4-rows-per-thread and
1-row-per-thread kernels, ragged tails (not a multiple of the 256 R-row tile),
empty and one-row columns, and the edge magnitudes 10^p - 1."""
import numpy as np
import pytest

import oracle
from tests import gpu_util as G

pytestmark = pytest.mark.gpu

CASES = [
    ("c1+c2", [(17, 5), (14, 2)], [True, True]),          # cfg1 types (Lb 8 / 7)
    ("c1+c2", [(35, 5), (32, 2)], [True, True]),          # cfg2 types (Lb 15 / 14)
    ("c1+c2", [(35, 5), (32, 2)], [True, False]),         # mixed layouts
    ("c1*c2 - c2", [(12, 3), (9, 1)], [True, True]),
    ("c1/c2 + c3", [(30, 4), (11, 2), (20, 6)], [True, True, False]),   # 1 row per thread (division)
    ("c1 % c2", [(25, 0), (13, 0)], [True, True]),
    ("-c1*c1 + c2", [(60, 10), (70, 20)], [True, True]),   # wide-ish numbers (L 7 / 8 -> products 15 limbs)
]


def _cols(host, types, compact):
    c = G.ctx()
    return [c.column_from_host_bin(p, s, m, g, layout="compact" if cp else "planes")
            for (m, g), (p, s), cp in zip(host, types, compact)]


@pytest.mark.parametrize("case", CASES, ids=lambda c: c[0].replace(" ", "") + "@" + "".join("c" if x else "p" for x in c[2]))
@pytest.mark.parametrize("n", [0, 1, 1023, 1025, 4099])
def test_compact_sum_parity(case, n):
    expr, types, compact = case
    lead = [k for k in range(len(types)) if f"/c{k + 1}" in expr.replace(" ", "") or f"%c{k + 1}" in expr.replace(" ", "")]
    host = G.gen_cols(n, types, nonzero_lead_cols=lead)
    want, P, S = oracle.eval_sum(expr, G.to_oracle(host, types), n=n, threads=4)
    if n == 0:
        gcols = [G.ctx().column_from_host_bin(p, s, np.zeros((0, 1), np.uint32), layout="compact" if cp else "planes")
                 for (p, s), cp in zip(types, compact)]
    else:
        gcols = _cols(host, types, compact)
    got, gP, gS = G.gpu_sum_string(expr, gcols)
    assert (gP, gS) == (P, S)
    assert got == want


@pytest.mark.parametrize("case", CASES, ids=lambda c: c[0].replace(" ", "") + "@" + "".join("c" if x else "p" for x in c[2]))
def test_compact_eval_parity(case):
    expr, types, compact = case
    n = 2053
    lead = [k for k in range(len(types)) if f"/c{k + 1}" in expr.replace(" ", "") or f"%c{k + 1}" in expr.replace(" ", "")]
    host = G.gen_cols(n, types, nonzero_lead_cols=lead)
    want = oracle.eval_rows(expr, G.to_oracle(host, types), strict=False)
    c = G.ctx()
    out = c.eval_expr(expr, _cols(host, types, compact))
    try:
        c.check()
    except Exception:  # noqa: BLE001 -- overflow rows are compared only where valid
        pass
    got = c.column_to_strings(out)
    for g, w in zip(got, want):
        if not w.startswith("E"):
            assert g == w


@pytest.mark.parametrize("p", [9, 17, 18, 19, 35, 38, 77])
def test_compact_edge_magnitudes_round_trip_and_sum(p):
    """10^p - 1 (every magnitude bit up to the sign bit), signs, zero: the
    in-kernel expand must agree with the planes path bit for bit."""
    c = G.ctx()
    big = str(10 ** p - 1)
    vals = [big, "-" + big, "0", "1", "-1", big, str(2 ** 32 - 1)[:p], "-" + big] * 37
    cc = c.column_from_strings(p, 0, vals, layout="compact")
    cp = c.column_from_strings(p, 0, vals)
    assert c.column_to_strings(cc) == c.column_to_strings(cp) == oracle.eval_rows("c1", [oracle.Column(p, 0, strings=vals)])
    from paper_conf_icde_lixylz24_b200 import up
    want = oracle.eval_sum("c1 + c1", [oracle.Column(p, 0, strings=vals)])[0]
    assert up.result_to_string(c.sum_expr("c1 + c1", [cc]), 0) == want
    assert c.column_to_strings(c.eval_expr("c1 - 1", [cc])) == oracle.eval_rows("c1 - 1", [oracle.Column(p, 0, strings=vals)])


def test_compact_in_place_ingest_and_range_flag():
    """up_column_from_host_compact into a compact column copies the rows in
    place (no planes) and still raises RANGE for a magnitude >= 10^p."""
    from gen import synth
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    types = [(35, 5), (32, 2)]
    host = G.gen_cols(3001, types)
    rows = [synth.to_compact(m, g, p) for (m, g), (p, s) in zip(host, types)]
    cols = [c.column_from_compact(p, s, r, layout="compact") for r, (p, s) in zip(rows, types)]
    c.check()
    assert np.array_equal(c.column_to_compact(cols[0]), rows[0])
    got, _, _ = G.gpu_sum_string("c1+c2", cols)
    assert got == oracle.eval_sum("c1+c2", G.to_oracle(host, types))[0]
    bad = rows[1].copy()
    bad[:14] = 0xFF
    bad[13] = 0x7F       # row 0: magnitude 2^111 - 1 >= 10^32, positive
    c.column_from_compact(32, 2, bad, layout="compact")
    with pytest.raises(up.UpError) as ei:
        c.check()
    assert ei.value.name == "RANGE"


def test_compact_unsupported_entry_points():
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    x = c.column_from_strings(9, 8, ["0.5"], layout="compact")
    with pytest.raises(up.UpError) as ei:
        c.sin_taylor(x, 20)
    assert ei.value.name == "UNSUPPORTED"


@pytest.mark.parametrize("layout", ["planes", "quads", "compact"])
def test_chunked_host_compact_ingestion(layout):
    """up_column_from_host_compact pipelines large inputs in chunks (the copy of
    chunk k+1 beside the conversion of chunk k, 256-row chunk boundaries): a
    9M-row column (8 chunks) must equal the one-kernel device ingestion byte
    for byte, and a range error in a middle chunk must still raise RANGE."""
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    c = G.ctx()
    n, p, s = 9_000_003, 35, 5
    mag, neg = gdev.uniform_decimal(n, p, 2, 1)
    ref = c.column_from_device_bin(p, s, mag, neg)
    del mag, neg
    rows = c.column_to_compact(ref)
    col = c.column_from_compact(p, s, torch.from_numpy(rows).pin_memory(), n=n, layout=layout)
    c.check()
    assert np.array_equal(c.column_to_compact(col), rows)
    got, _, _ = G.gpu_sum_string("c1", [col])
    want, _, _ = G.gpu_sum_string("c1", [ref])
    assert got == want
    Lb = up.compact_bytes(p)
    bad = rows.copy()
    r = 4_500_001                                   # inside the 5th of 8 chunks
    bad[r * Lb:(r + 1) * Lb] = 0xFF
    bad[(r + 1) * Lb - 1] = 0x7F                    # magnitude 2^119 - 1 >= 10^35, positive
    c.column_from_compact(p, s, torch.from_numpy(bad).pin_memory(), n=n, layout=layout)
    with pytest.raises(up.UpError) as ei:
        c.check()
    assert ei.value.name == "RANGE"
