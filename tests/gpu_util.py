"""Shared helpers for the GPU parity tests: build the same seeded columns for
the CUDA path (libup, via the C ABI) and for the oracle."""
from __future__ import annotations

import numpy as np

import oracle
from gen import synth

_CTX = None


def ctx():
    global _CTX
    if _CTX is None:
        from paper_conf_icde_lixylz24_b200 import up
        _CTX = up.Context(0)
    return _CTX


def gen_cols(n, types, config=9, nonzero_lead_cols=(), seed=synth.SEED):
    """host (mag, neg) per column, uniform magnitudes."""
    out = []
    for k, (p, s) in enumerate(types):
        mag, neg = synth.uniform_decimal(n, p, config, k + 1, seed=seed, nonzero_lead=(k in nonzero_lead_cols))
        out.append((mag, neg))
    return out


def to_gpu(host_cols, types):
    c = ctx()
    return [c.column_from_host_bin(p, s, mag, neg) for (mag, neg), (p, s) in zip(host_cols, types)]


def to_oracle(host_cols, types):
    return [oracle.Column(p, s, mag, neg) for (mag, neg), (p, s) in zip(host_cols, types)]


def gpu_sum_string(expr, gcols, n_global=0):
    from paper_conf_icde_lixylz24_b200 import up
    c = ctx()
    P, S, LA = c.sum_type(expr, gcols, n_global)
    res = c.sum_expr(expr, gcols, n_global)
    c.check()
    return up.result_to_string(res, S), P, S


def int_rows_to_strings(vals, s):
    from paper_conf_icde_lixylz24_b200.up import _fmt
    return [_fmt(v, s) for v in vals]
