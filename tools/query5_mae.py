#!/usr/bin/env python
"""Mean absolute error of the paper-literal Query 5 (2..11 terms) and of
sin_P against the true sine (mpmath, 300 digits) on the three input
distributions of P:L2229-2239 (the paper used GMP to 287 digits).
CPU-side context only (values come from the oracle, which the GPU matches bit
for bit)."""
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import mpmath

import oracle
from gen import synth


def q5(terms):
    e = "c1"
    for k in range(1, terms):
        n = 2 * k + 1
        e += (" - " if k % 2 else " + ") + "*".join(["c1"] * n) + "/" + str(math.factorial(n))
    return e


def main():
    mpmath.mp.dps = 300
    n = 200
    for mu in (0.01, 0.78, 1.56):
        mag, neg = synth.normal_decimal(n, mu, 0.01, 8, config=5, column=3)
        col = oracle.Column(9, 8, mag, neg)
        xs = [mpmath.mpf(v) / 10 ** 8 for v in synth.to_ints(mag, neg)]
        truth = [mpmath.sin(x) for x in xs]
        for terms in (2, 3, 5, 8, 11):
            rows = oracle.eval_rows(q5(terms), [col])
            mae = sum(abs(mpmath.mpf(r) - t) for r, t in zip(rows, truth)) / n
            print(json.dumps({"mu": mu, "query5_terms": terms, "mae": float(mae)}))
        for P in (50, 200):
            rows = oracle.sin_rows(col, P)
            mae = sum(abs(mpmath.mpf(r) - t) for r, t in zip(rows, truth)) / n
            print(json.dumps({"mu": mu, "sin_P": P, "mae": float(mae)}))


if __name__ == "__main__":
    main()
