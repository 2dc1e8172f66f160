#!/usr/bin/env python
"""WHERE -> GROUP BY DECIMAL key -> aggregates on B200 (SURVEY NEXT-4, A22/K10:
P:L730-734 compares DECIMAL values to sort for grouping).

    SELECT k, SUM(c2*c3), MIN(c2), MAX(c3), AVG(c2), COUNT(*)
    FROM t WHERE c2 > c3 - 50 GROUP BY k

Synthetic columns (device generator, seeded): k DECIMAL(kp,1) uniform (about
2*10^kp distinct keys... capped by kp), c2 DECIMAL(9,2), c3 DECIMAL(10,3),
n rows.  Three calls, each timed with CUDA events (median of 5, after 2
warm-ups): up_filter (one fused kernel), up_group_ids (stable LSD radix sort
over the key limbs + run heads + scan + scatter; synchronises to return the
group count), up_group_aggregate (one kernel).  One JSON line per
configuration."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from gen import device as gdev
    from gen import synth
    from paper_conf_icde_lixylz24_b200 import up
    gdev.build()
    ctx = up.Context(0)
    for n, kp in ((10_000_000, 2), (10_000_000, 1), (50_000_000, 2)):
        z = torch.zeros(n, dtype=torch.uint8, device="cuda")
        mk, gk = gdev.uniform_decimal(n, kp, 14, 1)
        m2, g2 = gdev.uniform_decimal(n, 9, 14, 2)
        m3, g3 = gdev.uniform_decimal(n, 10, 14, 3)
        cols = [ctx.column_from_device_bin(kp, 1 if kp > 1 else 0, mk, gk),
                ctx.column_from_device_bin(9, 2, m2, g2), ctx.column_from_device_bin(10, 3, m3, g3)]
        aggs = [("SUM", "c2*c3"), ("MIN", "c2"), ("MAX", "c3"), ("AVG", "c2")]
        times = {"filter": [], "group_ids": [], "aggregate": []}
        ng = 0
        for it in range(7):
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            torch.cuda.synchronize()
            ev[0].record()
            ids = ctx.filter("c2", ">", "c3 - 50", cols)
            ev[1].record()
            ids, ng = ctx.group_ids([cols[0]], ids)
            ev[2].record()
            out, counts, layout = ctx.group_aggregate(aggs, cols, ids, ng)
            ev[3].record()
            torch.cuda.synchronize()
            if it >= 2:
                for k, (a, b) in zip(times, zip(ev[:-1], ev[1:])):
                    times[k].append(a.elapsed_time(b))
        ctx.check()
        med = {k: statistics.median(v) for k, v in times.items()}
        tot = sum(med.values())
        print(json.dumps({"query": "SELECT k, SUM(c2*c3), MIN(c2), MAX(c3), AVG(c2) WHERE c2 > c3-50 GROUP BY k",
                          "rows": n, "key_type": [kp, cols[0].s], "groups": ng,
                          "ms": {k: round(v, 4) for k, v in med.items()}, "total_ms": round(tot, 4),
                          "rows_per_s": n / (tot * 1e-3)}), flush=True)
        del cols, ids, out, counts, mk, gk, m2, g2, m3, g3, z
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
