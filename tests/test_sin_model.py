"""The band sine's word-level plan (tools/sin_model.py: Horner long division
over non-normalised product digits, 32-bit digits with 3-by-2 steps or 64-bit
chunks with 2-by-1 steps, bit offsets, drops, masks, the scaled running sum)
against the Q13 definition written out with Python integers.  This checks
the kernel's arithmetic plan, not the kernel (the GPU tests do that)."""
import os
import random
import sys

import pytest

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
import sin_model  # noqa: E402


def q13(m, s, P):
    t, k, S = abs(m) * 10 ** (P - s), 1, 0
    while t:
        S += t if k % 2 else -t
        t = t * m * m // (10 ** (2 * s) * (2 * k) * (2 * k + 1))
        k += 1
    return -S if m < 0 else S


@pytest.mark.parametrize("chunk64", [False, True])
@pytest.mark.parametrize("s", [0, 1, 2, 5, 7, 8, 9])
def test_band_plan_matches_q13(s, chunk64):
    rng = random.Random(s * 7 + chunk64)
    lim = 10 ** (s + 1) - 1          # p - s <= 1: |x| < 10
    ms = [0, 1, -1, lim, -lim, 10 ** s, 10 ** s - 1] + [rng.randrange(-lim, lim + 1) for _ in range(12)]
    for P in (max(s, 1), 20, 97, 300):
        for m in ms:
            got, _ = sin_model.sin_row(m, s, P, chunk64=chunk64)
            assert got == q13(m, s, P), (m, s, P, chunk64)


def test_mg_2by1_64_exhaustive_edges():
    rng = random.Random(5)
    for _ in range(2000):
        d = rng.randrange(1 << 63, 1 << 64)
        v = sin_model.mg_reciprocal_2by1_64(d)
        u1 = rng.choice([0, d - 1, rng.randrange(d)])
        u0 = rng.choice([0, (1 << 64) - 1, rng.randrange(1 << 64)])
        q, r = sin_model.mg_div_2by1_64(u1, u0, d, v)
        assert (q, r) == divmod((u1 << 64) | u0, d)
