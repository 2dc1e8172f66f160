"""Compact byte-aligned rows (the paper's cDecimal, Fig. 4):
Lb = ceil((1 + p log2 10)/8) bytes, magnitude little-endian, sign in the top
bit of the last byte.  Host pins against the paper's printed bytes and sizes
(tests/golden/paper_examples.txt C1-C4); GPU round trips through the C ABI."""
import os

import numpy as np
import pytest

import oracle
from gen import synth
from paper_conf_icde_lixylz24_b200 import up

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_examples.txt")


def golden_compact():
    rows = []
    for line in open(GOLDEN):
        if line.startswith("C"):
            f = [x.strip() for x in line.split("|")]
            rows.append((f[0], int(f[1]), int(f[2]), int(f[3]), bytes.fromhex(f[4].replace(" ", ""))))
    return rows


@pytest.mark.parametrize("row", golden_compact(), ids=lambda r: r[0])
def test_paper_compact_bytes(row):
    tid, p, m, Lb, want = row
    assert synth.compact_bytes(p) == Lb
    assert up.compact_bytes(p) == Lb
    W = max(1, (abs(m).bit_length() + 31) // 32)
    mag = np.array([synth.int_to_words(abs(m), W)], dtype=np.uint32)
    neg = np.array([1 if m < 0 else 0], dtype=np.uint8)
    assert bytes(synth.to_compact(mag, neg, p)) == want


def test_compact_size_formula_matches_paper_expression():
    import math
    for p in range(1, 400):
        assert up.compact_bytes(p) == math.ceil((1 + p * math.log2(10)) / 8) == synth.compact_bytes(p)


@pytest.mark.gpu
@pytest.mark.parametrize("p,s,n", [(10, 2, 1), (35, 5, 257), (32, 2, 1000), (200, 50, 33), (17, 5, 4099)])
def test_compact_round_trip_and_sum(p, s, n):
    from tests import gpu_util as G
    mag, neg = synth.uniform_decimal(n, p, 7, 1)
    cb = synth.to_compact(mag, neg, p)
    c = G.ctx()
    col = c.column_from_compact(p, s, cb)
    c.check()
    assert c.column_to_ints(col) == synth.to_ints(mag, neg)
    canon_neg = (neg & mag.any(axis=1)).astype(np.uint8)   # no negative zero on the way back
    assert np.array_equal(c.column_to_compact(col), synth.to_compact(mag, canon_neg, p))
    res = c.sum_expr("c1", [col])
    c.check()
    assert up.result_to_string(res, s) == oracle.eval_sum("c1", [oracle.Column(p, s, mag, neg)])[0]


@pytest.mark.gpu
def test_compact_paper_example_decodes():
    from tests import gpu_util as G
    c = G.ctx()
    col = c.column_from_compact(10, 2, np.frombuffer(bytes([0x7B, 0, 0, 0, 0x80]), dtype=np.uint8).copy())
    c.check()
    assert c.column_to_strings(col) == ["-1.23"]
