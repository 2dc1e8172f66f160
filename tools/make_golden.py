#!/usr/bin/env python
"""Write tests/golden/fullsize_sums.json: the ORACLE's SUM for every bench
workload at its full BASELINE size, so the GPU tests can compare the CUDA path
at full size without re-running hours of oracle work on the GPU box.

This script calls only `gen/` (seeded input generation, no method arithmetic)
and `oracle/` (the CPU checker): no value in the file comes from libup or any
CUDA code.  Inputs are the host twins of the generators bench.py uses
(gen/synth.py; the device twin is bit-identical, tests/test_gpu_parity.py::
test_device_generator_matches_host_twin).  Rows are generated and summed in
chunks (each chunk typed with the GLOBAL row count, P:L1075 reading Q9) and the
chunk sums are added by the oracle's exact adder.

    python tools/make_golden.py [--only NAME[,NAME]] [--threads T]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from gen import synth  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "fullsize_sums.json")
CHUNK = 1 << 22

# name -> workload (the bench.py configs at their BASELINE / SURVEY §8d sizes)
ENTRIES = {
    "cfg1_2p30": dict(kind="expr", config=1, expr="c1+c2", types=[(17, 5), (14, 2)], rows=1 << 30),
    "cfg2_10M": dict(kind="expr", config=2, expr="c1+c2", types=[(35, 5), (32, 2)], rows=10_000_000),
    "cfg2_2p30": dict(kind="expr", config=2, expr="c1+c2", types=[(35, 5), (32, 2)], rows=1 << 30),
    "cfg3_p200": dict(kind="expr", config=3, expr="c1*c2 - c3/c4", types=[(200, 50)] * 4, rows=12_500_000,
                      lead=[3]),
    "cfg3_p500": dict(kind="expr", config=3, expr="c1*c2 - c3/c4", types=[(500, 75)] * 4, rows=12_500_000,
                      lead=[3]),
    "cfg3_p1000": dict(kind="expr", config=3, expr="c1*c2 - c3/c4", types=[(1000, 100)] * 4, rows=12_500_000,
                       lead=[3]),
    "cfg4_1024_e65537": dict(kind="modexp", bits=1024, e=65537, rows=10_000_000),
    "cfg4_1024_e3": dict(kind="modexp", bits=1024, e=3, rows=10_000_000),
    "cfg4_2048_e65537": dict(kind="modexp", bits=2048, e=65537, rows=10_000_000),
    "cfg5_P500": dict(kind="sin", P=500, mu=0.78, rows=1_000_000),
    "cfg5_P1000": dict(kind="sin", P=1000, mu=0.78, rows=1_000_000),
    "cfg5_P5000": dict(kind="sin", P=5000, mu=0.78, rows=1_000_000),
    "cfg5_P20000_100k": dict(kind="sin", P=20000, mu=0.78, rows=100_000),
}


def chunk_sum(e, lo, hi, threads):
    n = hi - lo
    if e["kind"] == "expr":
        cols = []
        for k, (p, s) in enumerate(e["types"]):
            m, g = synth.uniform_decimal(n, p, e["config"], k + 1, row0=lo, nonzero_lead=(k in e.get("lead", ())))
            cols.append(oracle.Column(p, s, m, g))
        v, P, S = oracle.eval_sum(e["expr"], cols, n_global=e["rows"], threads=threads)
        return v, P, S
    if e["kind"] == "modexp":
        N, _, _ = synth.rsa_modulus(e["bits"])
        m, g = synth.rsa_messages(n, N, row0=lo)
        v = oracle.modexp_sum(oracle.Column(len(str(N)), 0, m, g), e["e"], N, threads=threads)
        P = len(str(N)) + len(str(e["rows"] - 1))   # p + ceil(log10 N) for N > 1 rows (reading Q9)
        return v, P, 0
    m, g = synth.normal_decimal(n, e["mu"], 0.01, 8, config=5, column=0, row0=lo)
    v = oracle.sin_sum(oracle.Column(9, 8, m, g), e["P"], threads=threads)
    return v, None, e["P"]


def run(name, e, threads):
    t0 = time.time()
    parts, P, S = [], None, None
    chunk = CHUNK if e["kind"] == "expr" else 1 << 20
    for lo in range(0, e["rows"], chunk):
        hi = min(e["rows"], lo + chunk)
        v, P, S = chunk_sum(e, lo, hi, threads)
        parts.append(v)
        print(f"  {name}: rows {hi}/{e['rows']} ({time.time() - t0:.0f} s)", flush=True)
    if e["kind"] == "expr":
        P2 = P
    elif e["kind"] == "modexp":
        P2 = P
    else:
        P2 = e["P"] + 1 + len(str(e["rows"] - 1))
    total = parts[0] if len(parts) == 1 else oracle.add_strings(parts, P2, S)
    return {"sum": total, "p": P2, "s": S, "rows": e["rows"], "workload": {k: v for k, v in e.items()},
            "oracle_seconds": round(time.time() - t0, 1), "threads": threads}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="")
    ap.add_argument("--threads", type=int, default=len(os.sched_getaffinity(0)))
    a = ap.parse_args()
    sys.set_int_max_str_digits(0)
    data = json.load(open(OUT)) if os.path.exists(OUT) else {}
    data["_about"] = ("Oracle SUMs at full bench sizes, written by tools/make_golden.py (gen/ + oracle/ only; "
                      "no CUDA). Each entry's 'workload' is the bench.py config it checks.")
    names = a.only.split(",") if a.only else list(ENTRIES)
    for name in names:
        print(f"{name} ...", flush=True)
        data[name] = run(name, ENTRIES[name], a.threads)
        with open(OUT + ".tmp", "w") as f:
            json.dump(data, f, indent=1, sort_keys=True)
        os.replace(OUT + ".tmp", OUT)
        print(f"{name}: {data[name]['sum'][:60]}... in {data[name]['oracle_seconds']} s", flush=True)


if __name__ == "__main__":
    main()
