#!/usr/bin/env python
"""Probe: can cfg3's two kernels share the SMs?  Times, on quad columns of
cfg3 (DECIMAL(200,50) x 4, 12.5M rows): the tensor-core contraction
SUM(c1*c2) alone, the rest SUM(c3/c4) alone, the two back to back on one
stream, the two on two streams from two contexts (separate workspaces), and
the library's split step.  Prints one JSON line.  Measurement tool only (no
product code path).  Round-2 result (profiles/r02_s28, r02_s31): two streams
0.69-0.90 ms vs 0.80-0.86 back to back, varying from run to run with the
block placement -- the library keeps the kernels on one stream.

    python tools/probe_overlap.py [--rows N] [--reps K]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=12_500_000)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--p", type=int, default=200)
    ap.add_argument("--rest-layout", default="quads", help="layout of c3, c4 (the division's columns)")
    a = ap.parse_args()
    s = {200: 50, 500: 75, 1000: 100}[a.p]
    c1, c2 = up.Context(0), up.Context(0)
    cols = []
    for k in range(4):
        mag, neg = gdev.uniform_decimal(a.rows, a.p, 3, k + 1, nonzero_lead=(k == 3))
        cols.append(c1.column_from_device_bin(a.p, s, mag, neg, layout="quads" if k < 2 else a.rest_layout))
        del mag, neg
    c1.check()
    n = a.rows
    o1 = torch.empty(64, dtype=torch.int32, device="cuda")
    o2 = torch.empty(64, dtype=torch.int32, device="cuda")
    o3 = torch.empty(64, dtype=torch.int32, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def tc(ctx=c1, st=None):
        ctx.sum_expr("c1*c2", cols[:2], n, out=o1, stream=st)

    def rest(ctx=c1, st=None):
        ctx.sum_expr("c1/c2", cols[2:], n, out=o2, stream=st)

    def both_serial():
        tc(); rest()

    def both_streams():
        cur = torch.cuda.current_stream()
        s1.wait_stream(cur); s2.wait_stream(cur)
        tc(c1, s1); rest(c2, s2)
        cur.wait_stream(s1); cur.wait_stream(s2)

    def split():
        c1.sum_expr("c1*c2 - c3/c4", cols, n, out=o3)

    def split_on_stream():   # the library's split, called on a created (non-legacy) stream
        cur = torch.cuda.current_stream()
        s2.wait_stream(cur)
        c1.sum_expr("c1*c2 - c3/c4", cols, n, out=o3, stream=s2)
        cur.wait_stream(s2)

    def t(fn):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return round(e0.elapsed_time(e1) / a.reps, 4)

    r = {"p": a.p, "rows": n, "rest_layout": a.rest_layout, "tc_ms": t(tc), "rest_ms": t(rest), "serial_ms": t(both_serial),
         "two_streams_ms": t(both_streams), "split_step_ms": t(split), "split_on_stream_ms": t(split_on_stream)}
    print(json.dumps(r))


if __name__ == "__main__":
    main()
