#!/usr/bin/env python
"""Where does a cfg2 step's time go?  Host cost of one up_sum_expr call, and
the per-step time of SUM(c1+c2) over 10M rows (a) as bench.py times it
(events around every step), (b) K back-to-back launches between two events,
(c) replayed from a CUDA graph of one step, (d) a CUDA graph of 20 steps.
Run once with UP_PDL unset and once with UP_PDL=1 (programmatic dependent
launch of the SUM kernel).  One JSON line per measurement."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    gdev.build()
    ctx = up.Context(0)
    rows = int(os.environ.get("ROWS", "10000000"))
    K = 200
    tag = {"pdl": bool(os.environ.get("UP_PDL")), "rows": rows}
    cols = []
    for k, (p, s) in enumerate([(35, 5), (32, 2)]):
        mag, neg = gdev.uniform_decimal(rows, p, 2, k + 1)
        cols.append(ctx.column_from_device_bin(p, s, mag, neg))
    _, _, LA = ctx.sum_type("c1+c2", cols)
    out = torch.zeros(LA, dtype=torch.int32, device="cuda")
    st = torch.cuda.current_stream()

    def step():
        ctx.sum_expr("c1+c2", cols, out=out)

    for _ in range(2000):
        step()
    torch.cuda.synchronize()
    ref = up.result_to_string(out, 5)

    # host cost per call on a tiny column (GPU never the limit)
    small = []
    for k, (p, s) in enumerate([(35, 5), (32, 2)]):
        mag, neg = gdev.uniform_decimal(4096, p, 2, k + 1)
        small.append(ctx.column_from_device_bin(p, s, mag, neg))
    o2 = torch.zeros(LA, dtype=torch.int32, device="cuda")
    for _ in range(100):
        ctx.sum_expr("c1+c2", small, out=o2)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(2000):
        ctx.sum_expr("c1+c2", small, out=o2)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    print(json.dumps(dict(tag, what="host_us_per_sum_expr_call", value=round((t1 - t0) / 2000 * 1e6, 2))), flush=True)

    def ev():
        return torch.cuda.Event(enable_timing=True)

    # (a) bench-style: events around each step
    for rep in range(3):
        sev = [(ev(), ev()) for _ in range(K)]
        torch.cuda.synchronize()
        for i in range(K):
            sev[i][0].record(st)
            step()
            sev[i][1].record(st)
        torch.cuda.synchronize()
        ms = sum(a.elapsed_time(b) for a, b in sev) / K
        print(json.dumps(dict(tag, what="a_events_per_step_us", value=round(ms * 1e3, 2))), flush=True)
    # (b) K launches between two events
    for rep in range(3):
        e0, e1 = ev(), ev()
        torch.cuda.synchronize()
        e0.record(st)
        for i in range(K):
            step()
        e1.record(st)
        torch.cuda.synchronize()
        print(json.dumps(dict(tag, what="b_back_to_back_us", value=round(e0.elapsed_time(e1) / K * 1e3, 2))), flush=True)
    # (c) graph of one step, replayed K times
    g = torch.cuda.CUDAGraph()
    s2 = torch.cuda.Stream()
    s2.wait_stream(st)
    with torch.cuda.stream(s2):
        step()
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s2):
            step()
    torch.cuda.synchronize()
    for rep in range(3):
        e0, e1 = ev(), ev()
        torch.cuda.synchronize()
        e0.record(st)
        for i in range(K):
            g.replay()
        e1.record(st)
        torch.cuda.synchronize()
        print(json.dumps(dict(tag, what="c_graph1_replay_us", value=round(e0.elapsed_time(e1) / K * 1e3, 2))), flush=True)
    # (d) graph of 20 steps
    g20 = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s2):
        with torch.cuda.graph(g20, stream=s2):
            for _ in range(20):
                step()
    torch.cuda.synchronize()
    for rep in range(3):
        e0, e1 = ev(), ev()
        torch.cuda.synchronize()
        e0.record(st)
        for i in range(K // 20):
            g20.replay()
        e1.record(st)
        torch.cuda.synchronize()
        print(json.dumps(dict(tag, what="d_graph20_replay_us", value=round(e0.elapsed_time(e1) / K * 1e3, 2))), flush=True)
    ctx.check()
    assert up.result_to_string(out, 5) == ref, "result changed"
    print(json.dumps(dict(tag, what="result_unchanged", value=True)), flush=True)


if __name__ == "__main__":
    main()
