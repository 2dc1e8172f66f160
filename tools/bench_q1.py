#!/usr/bin/env python
"""TPC-H Q1-shaped grouped aggregation on B200 (the paper's
Fig. 14b workload): 4 DECIMAL columns, 2 expressions, 7
DECIMAL aggregates + COUNT(*), GROUP BY (l_returnflag, l_linestatus), one
launch of up_group_aggregate.

Synthetic lineitem (no TPC-H data here; recipe in DESIGN.md):
  * "orig": all columns DECIMAL(12,2) as in the paper's original-Q1 run:
    l_quantity 1..50, l_extendedprice = quantity x retail price
    (900.00..2099.00), l_discount 0.00..0.10, l_tax 0.00..0.08 (TPC-H
    value ranges), groups A/F, N/F, N/O, R/F with TPC-H-like frequencies
    (0.247 / 0.007 / 0.493 / 0.253) and ~1.5% of rows removed by the shipdate
    filter (group id -1);
  * "LEN k": l_quantity / l_extendedprice widened to DECIMAL(P,2) with
    uniform values so that SUM(charge) needs k words (the paper's LEN axis),
    l_discount / l_tax stay DECIMAL(3,2).
Timing: CUDA events, median of 7 runs, L2 flushed (256 MB write) before each.
Roofline: algorithmic bytes = column bytes + 4 B group id per row."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

AGGS = [("SUM", "c1"), ("SUM", "c2"), ("SUM", "c2*(1-c3)"), ("SUM", "c2*(1-c3)*(1+c4)"),
        ("AVG", "c1"), ("AVG", "c2"), ("AVG", "c3")]
# LEN -> precision of l_quantity / l_extendedprice
WIDTHS = {"orig": 12, 2: 18, 4: 38, 8: 76, 16: 153, 32: 307}   # the paper's ladder


def hbm_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"])
    except (OSError, KeyError):
        pass
    return 6549.4


def make_lineitem(n, P, ctx, key_orig):
    import torch
    from gen import device as gdev
    from gen import synth
    seed = synth.SEED
    z = torch.zeros(n, dtype=torch.uint8, device="cuda")
    if key_orig:
        q, _ = gdev.uniform_range(seed, synth.stream_id(10, 1), n, 1, 50, signed=False)
        r, _ = gdev.uniform_range(seed, synth.stream_id(10, 2), n, 90000, 209900, signed=False)
        q = q[:, 0].to(torch.int64)
        qty = (q * 100).to(torch.int32).view(n, 1)
        price = (q * r[:, 0].to(torch.int64)).to(torch.int32).view(n, 1)
        c1 = ctx.column_from_device_bin(12, 2, qty.contiguous(), z)
        c2 = ctx.column_from_device_bin(12, 2, price.contiguous(), z)
    else:
        m1, _ = gdev.uniform_decimal(n, P, 10, 1, signed=False)
        m2, _ = gdev.uniform_decimal(n, P, 10, 2, signed=False)
        c1 = ctx.column_from_device_bin(P, 2, m1, z)
        c2 = ctx.column_from_device_bin(P, 2, m2, z)
    d, _ = gdev.uniform_range(seed, synth.stream_id(10, 3), n, 0, 10, signed=False)
    t, _ = gdev.uniform_range(seed, synth.stream_id(10, 4), n, 0, 8, signed=False)
    dp = 12 if key_orig else 3
    c3 = ctx.column_from_device_bin(dp, 2, d.contiguous(), z)
    c4 = ctx.column_from_device_bin(dp, 2, t.contiguous(), z)
    u, _ = gdev.uniform_range(seed, synth.stream_id(10, 5), n, 0, 9999, signed=False)
    u = u[:, 0]
    gid = torch.full((n,), 2, dtype=torch.int32, device="cuda")       # N/O
    gid[u < 2470] = 0                                                 # A/F
    gid[(u >= 2470) & (u < 2540)] = 1                                 # N/F
    gid[(u >= 2540) & (u < 5070)] = 3                                 # R/F
    gid[u >= 9850] = -1                                               # shipdate filter
    return [c1, c2, c3, c4], gid


def main():
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    gdev.build()
    ctx = up.Context(0)
    n = int(os.environ.get("ROWS", "60000000"))
    peak = hbm_peak()
    flush = torch.empty(int(256e6) // 4, dtype=torch.int32, device="cuda")
    lens = os.environ.get("LENS", "orig,2,4,8,16,32").split(",")
    for key in lens:
        k = key if key == "orig" else int(key)
        P = WIDTHS[k]
        cols, gid = make_lineitem(n, P, ctx, key == "orig")
        out, counts, layout = ctx.group_aggregate(AGGS, cols, gid, 4)
        ctx.check()
        ts = []
        for it in range(10):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ctx.group_aggregate(AGGS, cols, gid, 4, out=out, counts=counts)
            e1.record()
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(e0.elapsed_time(e1))
        ctx.check()
        ms = sorted(ts)[len(ts) // 2]
        nbytes = n * (sum(c.limbs for c in cols) * 4 + 4)
        res, cnt = up.group_results(out, counts, layout, 4)
        print(json.dumps({"workload": "tpch_q1_shape", "LEN": key, "cols": [[c.p, c.s] for c in cols],
                          "sum_charge_limbs": layout[3][2], "rows": n, "ms": ms,
                          "rows_per_s": n / ms * 1e3, "GBps": nbytes / ms / 1e6,
                          "hbm_frac": nbytes / ms / 1e6 / peak, "counts": cnt,
                          "sum_qty": res[0], "avg_disc": res[6]}), flush=True)
        del cols, gid, out, counts
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
