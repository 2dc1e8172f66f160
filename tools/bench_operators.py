#!/usr/bin/env python
"""Per-operator kernels a+b, a*b, a/b at the paper's result widths LEN 2..32
(result precision 18/38/76/153/307), 10M rows, column output --
the B200 analogue of the paper's Fig. 13 kernel experiment (P:L1880-1946,
TPI 1/4/8/16/32 on an A6000).  Kernels: the fused per-thread expression
kernel (up_eval_expr, "fused") and the per-operator TPI kernels
(up_eval_tpi, tpi = 1..32); division: long division and Newton-Raphson at
TPI 1.  Operands in limb planes (LAYOUT=planes) or the paper's compact rows
(LAYOUT=compact, Listing 3 group loads).  CUDA events, L2 flushed before each
run, median of 7.  One JSON line per (operator, LEN, kernel)."""
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
OP = {"a+b": "+", "a*b": "*", "a/b": "/"}


def main():
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    gdev.build()
    ctx = up.Context(0)
    n = int(os.environ.get("ROWS", "10000000"))
    layout = os.environ.get("LAYOUT", "planes")
    flush = torch.empty(int(256e6) // 4, dtype=torch.int32, device="cuda")

    def timed(fn):
        for _ in range(3):
            fn()
        try:
            ctx.check()
        except up.UpError:
            pass
        ts = []
        for _ in range(7):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        try:
            ctx.check()
        except up.UpError:
            pass
        return sorted(ts)[len(ts) // 2]

    for op, table in CASES.items():
        for LEN, (pa, pb) in table.items():
            mag1, neg1 = gdev.uniform_decimal(n, pa, 11, 1)
            mag2, neg2 = gdev.uniform_decimal(n, pb, 11, 2, nonzero_lead=True)
            a = ctx.column_from_device_bin(pa, 0, mag1, neg1, layout=layout)
            b = ctx.column_from_device_bin(pb, 0, mag2, neg2, layout=layout)
            out = up.Column(*ctx.expr_type(f"c1{OP[op]}c2", [a, b]), n)
            kernels = [("fused", lambda: ctx.eval_expr(f"c1{OP[op]}c2", [a, b], out=out))]
            if op == "a/b":
                for alg in ("long", "newton"):
                    kernels.append((f"tpi1-{alg}", lambda alg=alg: ctx.eval_tpi("/", a, b, 1, alg, out=out)))
            else:
                for t in (1, 4, 8, 16, 32):
                    kernels.append((f"tpi{t}", lambda t=t: ctx.eval_tpi(OP[op], a, b, t, out=out)))
            for name, fn in kernels:
                try:
                    ms = timed(fn)
                except up.UpError as e:
                    print(json.dumps({"op": op, "LEN": LEN, "kernel": name, "error": str(e)[:200]}), flush=True)
                    continue
                print(json.dumps({"op": op, "LEN": up.limbs(out.p), "kernel": name, "layout": layout,
                                  "result_type": [out.p, out.s], "operands": [pa, pb], "rows": n, "ms": round(ms, 4),
                                  "Mtuples_per_s": round(n / ms / 1e3, 1)}), flush=True)
            del a, b, out, mag1, neg1, mag2, neg2
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
