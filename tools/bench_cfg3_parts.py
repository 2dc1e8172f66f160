#!/usr/bin/env python
"""Where the time of cfg3 goes: SUM(c1*c2), SUM(c3/c4) and the whole
SUM(c1*c2 - c3/c4) timed separately at p = 200 / 500 / 1000 (SURVEY §8d
cfg3 inputs), each with the row-contraction split on and off.  CUDA events
on the launching stream, 8 back-to-back calls per event pair, median of 5
after 3 warm-ups.  One JSON line per
(p, expression, split)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SCALE = {200: 50, 500: 75, 1000: 100}
ROWS = {200: 12_500_000, 500: 2_000_000, 1000: 1_000_000}


def main():
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    gdev.build()
    ctx = up.Context(0)
    ps = [int(x) for x in os.environ.get("PS", "200,500,1000").split(",")]
    exprs = os.environ.get("EXPRS", "c1*c2;c3/c4;c1*c2 - c3/c4").split(";")
    for p in ps:
        s, n = SCALE[p], int(os.environ.get("ROWS", ROWS[p]))
        cols = []
        for k in range(4):
            mag, neg = gdev.uniform_decimal(n, p, 3, k + 1, nonzero_lead=(k == 3))
            cols.append(ctx.column_from_device_bin(p, s, mag, neg))
            del mag, neg
        for expr in exprs:
            for split in ("auto", "off"):
                if split == "off":
                    os.environ["UP_NO_SPLIT"] = "1"
                else:
                    os.environ.pop("UP_NO_SPLIT", None)
                for _ in range(3):
                    ctx.sum_expr(expr, cols)
                ctx.check()
                ts = []
                for _ in range(5):
                    # 8 back-to-back calls per event pair: host launch overhead is
                    # hidden behind the queued kernels (as in bench.py's K steps)
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    for _ in range(8):
                        r = ctx.sum_expr(expr, cols)
                    e1.record()
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1) / 8)
                ms = sorted(ts)[len(ts) // 2]
                print(json.dumps({"p": p, "s": s, "expr": expr, "split": split, "rows": n, "ms": round(ms, 4),
                                  "Mtuples_per_s": round(n / ms / 1e3, 2), "result_head": str(r)[:24]}), flush=True)
        os.environ.pop("UP_NO_SPLIT", None)
        del cols
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
