"""The top-limb division decision's word-level plan (tools/divtop_model.py:
Moller-Granlund 3-by-2 quotient limbs on the normalised divisor window, the
Alg. 6 reciprocal, the dividend shifted on the fly, at most one add-back)
against Python's integer // and %: every decided window must give the exact
quotient and remainder.  This checks the kernel's arithmetic plan, not the
kernel (tests/test_gpu_divtop.py does)."""
import os
import sys

import pytest

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
import divtop_model  # noqa: E402


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_divtop_plan_exact(seed):
    assert divtop_model.run(iters=4000, seed=seed) > 1000


def test_recip_3by2_definition():
    B = 1 << 32
    for d1 in (1 << 31, (1 << 31) + 1, B - 1, 0x9E3779B9):
        for d0 in (0, 1, B - 1, 0x7F4A7C15):
            assert divtop_model.recip_3by2(d1, d0) == ((1 << 96) - 1) // ((d1 << 32) | d0) - B
