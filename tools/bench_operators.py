#!/usr/bin/env python
"""Per-operator kernels a+b, a*b, a/b at the paper's result widths LEN 2..32
(result precision 18/38/76/153/307), 10M rows, column output --
the B200 analogue of the paper's Fig. 13 kernel experiment (P:L1880-1946,
there with TPI 1..32 on an A6000).  Here every kernel is the per-thread
specialised one (TPI = 1); CUDA events, L2 flushed before each run.
One JSON line per (operator, LEN)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# operand precisions chosen so the RESULT has the paper's LEN
CASES = {
    "a+b": {2: (17, 17), 4: (37, 37), 8: (75, 75), 16: (152, 152), 32: (306, 306)},
    "a*b": {2: (9, 9), 4: (19, 19), 8: (38, 38), 16: (76, 77), 32: (153, 154)},
    "a/b": {2: (17, 9), 4: (37, 9), 8: (75, 38), 16: (152, 76), 32: (306, 153)},
}
EXPR = {"a+b": "c1+c2", "a*b": "c1*c2", "a/b": "c1/c2"}


def main():
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    gdev.build()
    ctx = up.Context(0)
    n = int(os.environ.get("ROWS", "10000000"))
    flush = torch.empty(int(256e6) // 4, dtype=torch.int32, device="cuda")
    for op, table in CASES.items():
        for LEN, (pa, pb) in table.items():
            mag1, neg1 = gdev.uniform_decimal(n, pa, 11, 1)
            mag2, neg2 = gdev.uniform_decimal(n, pb, 11, 2, nonzero_lead=True)
            a = ctx.column_from_device_bin(pa, 0, mag1, neg1)
            b = ctx.column_from_device_bin(pb, 0, mag2, neg2)
            out = ctx.eval_expr(EXPR[op], [a, b])
            for _ in range(3):
                ctx.eval_expr(EXPR[op], [a, b], out=out)
            try:
                ctx.check()
            except up.UpError:
                pass
            ts = []
            for _ in range(7):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                ctx.eval_expr(EXPR[op], [a, b], out=out)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = sorted(ts)[len(ts) // 2]
            print(json.dumps({"op": op, "LEN": up.limbs(out.p), "result_type": [out.p, out.s],
                              "operands": [pa, pb], "rows": n, "ms": ms, "Mtuples_per_s": n / ms / 1e3}),
                  flush=True)
            del a, b, out, mag1, neg1, mag2, neg2
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
