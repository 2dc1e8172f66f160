#!/usr/bin/env python
"""Kernel time with and without the expression optimiser (NEXT-1, P:L1781-1878
§IV-C: alignment scheduling Fig. 10, constant construction Fig. 11, constant
pre-calculation Fig. 12) on synthetic 10M-row columns, column output (as the
paper measures), CUDA events, L2 flushed between runs.  One JSON line per
expression."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CASES = [
    # Fig. 10: a at scale 1, b at scale 11, LEN 2 and LEN 32 result widths
    ("fig10 LEN2 a+b+a", "c1+c2+c1", [(6, 1), (17, 11)]),
    ("fig10 LEN32 a+b+a+a+a+a+a", "c1+c2+c1+c1+c1+c1+c1", [(290, 1), (300, 11)]),
    # Fig. 11: constant construction 1+a, a at scale 10
    ("fig11 1+a LEN8", "1+c1", [(70, 10)]),
    # Fig. 12: constant pre-calculation
    ("fig12 1+a+2+11", "1+c1+2+11", [(30, 10)]),
    ("fig12 1+a+2-3", "1+c1+2-3", [(30, 10)]),
    ("fig12 0.25*(a+b)*4", "0.25*(c1+c2)*4", [(30, 10), (30, 10)]),
]


def main():
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    gdev.build()
    ctx = up.Context(0)
    n = int(os.environ.get("ROWS", "10000000"))
    flush = torch.empty(int(256e6) // 4, dtype=torch.int32, device="cuda")
    for name, expr, types in CASES:
        cols = []
        for k, (p, s) in enumerate(types):
            mag, neg = gdev.uniform_decimal(n, p, 10, k + 1)
            cols.append(ctx.column_from_device_bin(p, s, mag, neg))
        res = {}
        for mode in ("opt", "noopt"):
            if mode == "noopt":
                os.environ["UP_NO_OPT"] = "1"
            else:
                os.environ.pop("UP_NO_OPT", None)
            out = ctx.eval_expr(expr, cols)
            for _ in range(3):
                ctx.eval_expr(expr, cols, out=out)
            ctx.check()
            ts = []
            for _ in range(10):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                ctx.eval_expr(expr, cols, out=out)
                b.record()
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            res[mode] = sorted(ts)[len(ts) // 2]
            res[mode + "_result_row0"] = ctx.column_to_strings(out)[:1] if n < 100 else None
        os.environ.pop("UP_NO_OPT", None)
        print(json.dumps({"case": name, "expr": expr, "types": types, "rows": n,
                          "optimised": up.expr_optimized(expr, types), "ms_opt": res["opt"],
                          "ms_noopt": res["noopt"], "saving": 1 - res["opt"] / res["noopt"]}), flush=True)


if __name__ == "__main__":
    main()
