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
    """Mantissas at scale s -> "[-]int.frac" input strings (test-local)."""
    out = []
    for v in vals:
        a = str(abs(v))
        if s:
            a = a.rjust(s + 1, "0")
            a = a[:-s] + "." + a[-s:]
        out.append(("-" if v < 0 else "") + a)
    return out


def limbs_int(limb_tensor) -> int:
    """Two's-complement little-endian 32-bit limbs (device tensor or list) ->
    Python int, written here so expected values never pass through libup's
    own formatter or converters."""
    vals = limb_tensor.detach().cpu().tolist() if hasattr(limb_tensor, "detach") else list(limb_tensor)
    v = 0
    for x in reversed(vals):
        v = (v << 32) | (int(x) & 0xFFFFFFFF)
    if vals and int(vals[-1]) & 0x80000000:
        v -= 1 << (32 * len(vals))
    return v
