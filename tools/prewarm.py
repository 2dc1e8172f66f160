#!/usr/bin/env python
"""Pre-compile (NVRTC, sm_100a, no GPU needed) the specialised kernels the
bench and the heavier tests use into libup's on-disk cubin cache, so GPU runs
do not spend their time in NVRTC.  Purely a compile-time cache.

    python tools/prewarm.py [--jobs 8]
"""
import argparse
import os
import sys
from concurrent.futures import ProcessPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def sources():
    from gen import synth
    from paper_conf_icde_lixylz24_b200 import up
    out = []
    for ws in (1, 2, 4, 8):
        out.append(up.gen_source("sum", "c1+c2", [(17, 5), (14, 2)], 1_000_000 * ws))
        out.append(up.gen_source("sum", "c1+c2", [(35, 5), (32, 2)], 10_000_000 * ws))
        out.append(up.gen_source("sum", "c1*c2 - c3/c4", [(200, 50)] * 4, 12_500_000 * ws))
        for bits in (1024, 2048):
            N, _, _ = synth.rsa_modulus(bits)
            out.append(up.gen_modexp_source(65537, N, len(str(N)), True, 10_000_000 * ws))
        for P in (500, 1000, 5000, 20000):
            out.append(up.gen_sin_source(P, 9, 8, True, 1_000_000 * ws))
    for bits in (1024, 2048):
        N, _, _ = synth.rsa_modulus(bits)
        for e in (3, 65537):
            out.append(up.gen_modexp_source(e, N, len(str(N)), False, 1))
            out.append(up.gen_modexp_source(e, N, len(str(N)), True, 10_000_000))
    N, _, _ = synth.rsa_modulus(512)
    out.append(up.gen_modexp_source(65537, N, len(str(N)), True, 1001))
    for P in (500, 1000, 5000, 20000):
        out.append(up.gen_sin_source(P, 9, 8, False, 1))
    out.append(up.gen_sin_source(2000, 9, 8, True, 40))
    out.append(up.gen_sin_source(500, 9, 8, True, 300))
    # heavier kernels of the GPU test-suite (exact sources: LA depends on the row count)
    for bits, n in ((1024, 333), (512, 333), (256, 333), (64, 333)):
        N, _, _ = synth.rsa_modulus(bits)
        for e in (3, 65537):
            out.append(up.gen_modexp_source(e, N, len(str(N)), False, n))
    # the slowest compiles of the suite: 2048-bit Montgomery kernels (radix 2^28 default,
    # and the 32-bit CIOS that test_modexp_parity forces with UP_MONT32)
    N, _, _ = synth.rsa_modulus(2048)
    for e in (3, 65537):
        out.append(up.gen_modexp_source(e, N, len(str(N)), False, 333))
    os.environ["UP_MONT32"] = "1"
    for bits in (1024, 1034, 2048):
        N, _, _ = synth.rsa_modulus(bits)
        for e in (3, 65537):
            out.append(up.gen_modexp_source(e, N, len(str(N)), False, 333))
    del os.environ["UP_MONT32"]
    N, _, _ = synth.rsa_modulus(1034)
    for e in (3, 65537):
        out.append(up.gen_modexp_source(e, N, len(str(N)), False, 333))
    N, _, _ = synth.rsa_modulus(1024)
    out.append(up.gen_modexp_source(65537, N, len(str(N)), True, 10_000_000))
    out.append(up.gen_modexp_source(65537, N, len(str(N)), False, 10_000_000))
    for p, s in ((200, 50), (500, 75), (1000, 100)):
        for n in (1, 9, 1000, 300, 2000, 500):
            out.append(up.gen_source("sum", "c1*c2 - c3/c4", [(p, s)] * 4, n))
    out.append(up.gen_source("sum", "c1*c2 - c3/c4", [(200, 50)] * 4, 12_500_000))
    out.append(up.gen_source("sum", "c1+c2", [(35, 5), (32, 2)], 10_000_000))
    import math
    def q5(terms):
        e = "c1"
        for k in range(1, terms):
            m = 2 * k + 1
            e += (" - " if k % 2 else " + ") + "*".join(["c1"] * m) + "/" + str(math.factorial(m))
        return e
    for terms in (2, 3, 5, 8, 11):
        out.append(up.gen_source("eval", q5(terms), [(9, 8)], 300))
        out.append(up.gen_source("sum", q5(terms), [(9, 8)], 300))
    for P in (1000,):
        out.append(up.gen_sin_source(P, 9, 8, True, 1_000_000))
        out.append(up.gen_sin_source(P, 9, 8, False, 1_000_000))
    # TPC-H Q1-shaped grouped aggregation (tools/bench_q1.py, 60M rows)
    q1 = [("SUM", "c1"), ("SUM", "c2"), ("SUM", "c2*(1-c3)"), ("SUM", "c2*(1-c3)*(1+c4)"),
          ("AVG", "c1"), ("AVG", "c2"), ("AVG", "c3")]
    out.append(up.gen_group_agg_source(q1, [(12, 2)] * 4, 4, 60_000_000))
    for P in (18, 38, 76, 153, 307):
        out.append(up.gen_group_agg_source(q1, [(P, 2), (P, 2), (3, 2), (3, 2)], 4, 60_000_000))
    return list(dict.fromkeys(out))


def _one(src):
    from paper_conf_icde_lixylz24_b200 import up
    up.jit_prewarm(src)
    return len(src)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--jobs", type=int, default=os.cpu_count())
    a = ap.parse_args()
    srcs = sources()
    with ProcessPoolExecutor(a.jobs) as ex:
        for _ in ex.map(_one, srcs):
            pass
    print(f"prewarmed {len(srcs)} kernels")


if __name__ == "__main__":
    main()
