"""Quick tensor-core contraction check (csrc/contract_tc.cu): SUM(c1*c2) vs
exact Python integers on a few shapes, each printed as it finishes."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("UP_SPLIT", "1")
from tests.test_gpu_contract_tc import _check  # noqa: E402

for p1, p2, n in [(200, 200, 1000), (90, 90, 129), (1000, 1000, 300), (305, 305, 500), (1300, 700, 200)]:
    t = time.time()
    try:
        _check(p1, p2, n, "rand", seed=1)
        print("ok", p1, p2, n, round(time.time() - t, 2), flush=True)
    except AssertionError as e:
        print("MISMATCH", p1, p2, n, str(e)[:300], flush=True)
