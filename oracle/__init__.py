"""CPU oracle for the UltraPrecise DECIMAL hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_icde_lixylz24_b200`` never imports it and shares
no code with it.  The arithmetic lives in ``oracle/updec.c`` (plain C,
base-10^9 sign-magnitude bignum); this module only builds and marshals.

Every oracle function is pinned by ``tests/test_oracle_*.py`` against closed
forms, the paper's worked examples (``tests/golden/``), textbook RSA values,
and brute force with Python ``int`` / ``decimal`` on small inputs.  Parity
status per function is listed in DESIGN.md ("Oracle pins").
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "updec.c")
_LIB = os.path.join(_HERE, "liboracle.so")

STATUS = {0: "OK", 1: "INVAL", 2: "RANGE", 3: "OVERFLOW", 4: "DIVZERO", 5: "NOMEM"}


class OracleError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        super().__init__(f"oracle error {STATUS.get(code, code)} {what}")
        self.code = code
        self.name = STATUS.get(code, str(code))


def build(force: bool = False) -> str:
    """Compile oracle/updec.c into oracle/liboracle.so (plain gcc -O2)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread",
                               "-Wall", "-Wno-unused-function", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        c = ctypes
        PI = c.POINTER(c.c_int)
        PPU32 = c.POINTER(c.c_void_p)
        _lib.orc_expr_type.argtypes = [c.c_char_p, c.c_int, PI, PI, PI, PI]
        _lib.orc_sum_type.argtypes = [c.c_int, c.c_int, c.c_int64, PI, PI]
        _lib.orc_eval_rows.argtypes = [c.c_char_p, c.c_int, PI, PI, PI, PPU32, PPU32, PPU32,
                                       c.c_int64, c.c_char_p, c.c_size_t]
        _lib.orc_eval_sum.argtypes = [c.c_char_p, c.c_int, PI, PI, PI, PPU32, PPU32, PPU32,
                                      c.c_int64, c.c_int64, c.c_int, c.c_char_p, c.c_size_t, PI, PI]
        _lib.orc_modexp_rows.argtypes = [c.c_char_p, c.c_char_p, c.c_int, c.c_int, c.c_void_p,
                                         c.c_void_p, PPU32, c.c_int64, c.c_char_p, c.c_size_t]
        _lib.orc_modexp_sum.argtypes = [c.c_char_p, c.c_char_p, c.c_int, c.c_int, c.c_void_p,
                                        c.c_void_p, c.c_int64, c.c_int, c.c_char_p, c.c_size_t]
        _lib.orc_sin_rows.argtypes = [c.c_int, c.c_int, c.c_int, c.c_int, c.c_void_p, c.c_void_p,
                                      PPU32, c.c_int64, c.c_char_p, c.c_size_t]
        _lib.orc_sin_sum.argtypes = [c.c_int, c.c_int, c.c_int, c.c_int, c.c_void_p, c.c_void_p,
                                     c.c_int64, c.c_int, c.c_char_p, c.c_size_t]
        _lib.orc_add_strings.argtypes = [PPU32, c.c_int, c.c_int, c.c_int, c.c_char_p, c.c_size_t]
    return _lib


def _ints(xs):
    return (ctypes.c_int * max(1, len(xs)))(*xs)


def _ptrs(arrs):
    return (ctypes.c_void_p * max(1, len(arrs)))(*[a.ctypes.data if a is not None else None for a in arrs])


def _strs(strs):
    enc = [s.encode() for s in strs]
    arr = (ctypes.c_char_p * max(1, len(enc)))(*enc)
    return ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p)), (arr, enc)


class Column:
    """A column in the generator's host format: magnitude words (n x w, uint32,
    little-endian words) + negative flags (n, uint8), or decimal strings."""

    def __init__(self, p: int, s: int, mag: Optional[np.ndarray] = None,
                 neg: Optional[np.ndarray] = None, strings: Optional[Sequence[str]] = None):
        self.p, self.s = p, s
        if strings is not None:
            self.strings = list(strings)
            self.n = len(self.strings)
            self.mag = self.neg = None
            self.w = 0
        else:
            self.mag = np.ascontiguousarray(mag, dtype=np.uint32)
            self.n, self.w = self.mag.shape
            self.neg = (np.ascontiguousarray(neg, dtype=np.uint8) if neg is not None
                        else np.zeros(self.n, np.uint8))
            self.strings = None

    def head(self, k: int) -> "Column":
        if self.strings is not None:
            return Column(self.p, self.s, strings=self.strings[:k])
        return Column(self.p, self.s, self.mag[:k], self.neg[:k])


def _cols_args(cols: Sequence[Column]):
    n = cols[0].n if cols else 1
    p = _ints([c.p for c in cols]); s = _ints([c.s for c in cols]); w = _ints([c.w for c in cols])
    if cols and cols[0].strings is not None:
        flat = [cols[k].strings[i] for i in range(n) for k in range(len(cols))]
        sp, keep = _strs(flat)
        return n, p, s, w, _ptrs([]), _ptrs([]), sp, keep
    keep = [c.mag for c in cols] + [c.neg for c in cols]
    return n, p, s, w, _ptrs([c.mag for c in cols]), _ptrs([c.neg for c in cols]), None, keep


def _out_buf(n_rows: int, digits: int):
    return ctypes.create_string_buffer(max(64, (digits + 8) * max(n_rows, 1) + 16))


def expr_type(expr: str, cols: Sequence[Column]):
    P, S = ctypes.c_int(), ctypes.c_int()
    e = lib().orc_expr_type(expr.encode(), len(cols), _ints([c.p for c in cols]),
                            _ints([c.s for c in cols]), ctypes.byref(P), ctypes.byref(S))
    if e:
        raise OracleError(e, expr)
    return P.value, S.value


def sum_type(p: int, s: int, n_global: int):
    P, S = ctypes.c_int(), ctypes.c_int()
    lib().orc_sum_type(p, s, n_global, ctypes.byref(P), ctypes.byref(S))
    return P.value, S.value


def eval_rows(expr: str, cols: Sequence[Column], n: Optional[int] = None, strict: bool = True):
    """Canonical decimal string of expr for every row ("E<code>" for a failing row)."""
    n_, p, s, w, mags, negs, strs, keep = _cols_args(cols)
    n = n_ if n is None else n
    P, _ = expr_type(expr, cols)
    buf = _out_buf(n, P + 4)
    e = lib().orc_eval_rows(expr.encode(), len(cols), p, s, w, mags, negs, strs, n, buf, len(buf))
    if e and (strict or e == 5):
        raise OracleError(e, expr)
    return buf.value.decode().split("\n")[:n]


def eval_sum(expr: str, cols: Sequence[Column], n: Optional[int] = None,
             n_global: int = 0, threads: int = 1):
    """SELECT SUM(expr): (canonical string, P, S)."""
    n_, p, s, w, mags, negs, strs, keep = _cols_args(cols)
    n = n_ if n is None else n
    P0, _ = expr_type(expr, cols)
    buf = _out_buf(1, P0 + 40)
    oP, oS = ctypes.c_int(), ctypes.c_int()
    e = lib().orc_eval_sum(expr.encode(), len(cols), p, s, w, mags, negs, strs, n, n_global,
                           threads, buf, len(buf), ctypes.byref(oP), ctypes.byref(oS))
    if e:
        raise OracleError(e, expr)
    return buf.value.decode(), oP.value, oS.value


def modexp_rows(col: Column, exponent: int, modulus: int, n: Optional[int] = None):
    n = col.n if n is None else n
    keep = None
    if col.strings is not None:
        sp, keep = _strs(col.strings[:n])
        mag = neg = None
    else:
        sp, mag, neg = None, col.mag.ctypes.data, col.neg.ctypes.data
    buf = _out_buf(n, len(str(modulus)) + 2)
    e = lib().orc_modexp_rows(str(exponent).encode(), str(modulus).encode(), col.p, col.w,
                              mag, neg, sp, n, buf, len(buf))
    if e:
        raise OracleError(e, "modexp")
    return buf.value.decode().split("\n")[:n]


def modexp_sum(col: Column, exponent: int, modulus: int, n: Optional[int] = None, threads: int = 1):
    n = col.n if n is None else n
    buf = _out_buf(1, len(str(modulus)) + 24)
    e = lib().orc_modexp_sum(str(exponent).encode(), str(modulus).encode(), col.p, col.w,
                             col.mag.ctypes.data, col.neg.ctypes.data, n, threads, buf, len(buf))
    if e:
        raise OracleError(e, "modexp_sum")
    return buf.value.decode()


def sin_rows(col: Column, P: int, n: Optional[int] = None):
    n = col.n if n is None else n
    keep = None
    if col.strings is not None:
        sp, keep = _strs(col.strings[:n])
        mag = neg = None
    else:
        sp, mag, neg = None, col.mag.ctypes.data, col.neg.ctypes.data
    buf = _out_buf(n, P + 8)
    e = lib().orc_sin_rows(P, col.p, col.s, col.w, mag, neg, sp, n, buf, len(buf))
    if e:
        raise OracleError(e, "sin")
    return buf.value.decode().split("\n")[:n]


def sin_sum(col: Column, P: int, n: Optional[int] = None, threads: int = 1):
    n = col.n if n is None else n
    buf = _out_buf(1, P + 24)
    e = lib().orc_sin_sum(P, col.p, col.s, col.w, col.mag.ctypes.data, col.neg.ctypes.data,
                          n, threads, buf, len(buf))
    if e:
        raise OracleError(e, "sin_sum")
    return buf.value.decode()


def add_strings(values: Sequence[str], p: int, s: int) -> str:
    sp, keep = _strs(values)
    buf = _out_buf(1, p + 4)
    e = lib().orc_add_strings(sp, len(values), p, s, buf, len(buf))
    if e:
        raise OracleError(e, "add_strings")
    return buf.value.decode()


AGG_KINDS = ("SUM", "MIN", "MAX", "AVG")


def _scaled_int(txt: str, s: int) -> int:
    neg = txt.startswith("-")
    t = txt[1:] if neg else txt
    ip, _, fp = t.partition(".")
    v = int(ip + fp.ljust(s, "0")[:s]) if s else int(ip)
    return -v if neg else v


def _fmt_scaled(v: int, s: int) -> str:
    a = str(abs(v))
    if s:
        a = a.rjust(s + 1, "0")
        a = a[:-s] + "." + a[-s:]
    return ("-" if v < 0 else "") + a


def agg_type(kind: str, p: int, s: int, n_global: int):
    """Result type of an aggregate over n_global tuples, P:L1069-1080 (Sec. III-B):
    MAX/MIN keep the expression's precision; SUM is p + ceil(log10 N) (orc_sum_type);
    AVG follows the SUM rule and then the division rule (p1-p2+s2+5, s1+4),
    P:L1049-1058, with the divisor converted to DECIMAL(ceil(log10 N)+1, 0)."""
    if kind in ("MIN", "MAX"):
        return p, s
    ps, ss = sum_type(p, s, n_global)
    if kind == "SUM":
        return ps, ss
    if kind == "AVG":
        p2, s2 = (ps - p) + 1, 0          # ceil(log10 N) = ps - p
        return ps - p2 + s2 + 5, ss + 4
    raise ValueError(kind)


def group_aggregate(aggs, cols: Sequence[Column], group=None, n_groups: int = 1, n_global: int = 0):
    """SELECT agg(expr), ... GROUP BY g, written out row by row (Python ints on
    the oracle's exact per-row values, orc_eval_rows).  Rows with g < 0 are
    excluded (a WHERE filter).  AVG = trunc(SUM * 10^(s2+4) / COUNT) with s2 = 0
    (the division of P:L1049-1058 by COUNT as DECIMAL(ceil(log10 N)+1, 0),
    truncation toward zero, reading Q4).  An empty group reports 0 (SQL NULL,
    see its count).  Returns ([[string per group] per aggregate], counts, types)."""
    n = cols[0].n
    N = n_global or n
    gid = np.zeros(n, np.int64) if group is None else np.asarray(group, dtype=np.int64)
    counts = [0] * n_groups
    for g in gid.tolist():
        if 0 <= g < n_groups:
            counts[g] += 1
    results, types = [], []
    for kind, expr in aggs:
        P, S = expr_type(expr, cols)
        rows = eval_rows(expr, cols, strict=False)
        acc = [None] * n_groups
        for r, g in zip(rows, gid.tolist()):
            if not 0 <= g < n_groups:
                continue
            if r.startswith("E"):
                raise OracleError(int(r[1:] or 1), expr)
            v = _scaled_int(r, S)
            a = acc[g]
            if kind in ("SUM", "AVG"):
                acc[g] = v if a is None else a + v
            elif kind == "MIN":
                acc[g] = v if a is None or v < a else a
            else:
                acc[g] = v if a is None or v > a else a
        tp, ts = agg_type(kind, P, S, N)
        out = []
        for g in range(n_groups):
            a = acc[g]
            if a is None:
                out.append(_fmt_scaled(0, ts))
            elif kind == "AVG":
                q = abs(a) * 10 ** 4 // counts[g]
                out.append(_fmt_scaled(-q if a < 0 else q, ts))
            else:
                out.append(_fmt_scaled(a, ts))
        results.append(out)
        types.append((tp, ts))
    return results, counts, types


CMP_OPS = ("<", "<=", ">", ">=", "=", "==", "<>", "!=")


def _cmp(a, b, op: str) -> bool:
    return {"<": a < b, "<=": a <= b, ">": a > b, ">=": a >= b, "=": a == b, "==": a == b,
            "<>": a != b, "!=": a != b}[op]


def filter_ids(lhs: str, op: str, rhs: str, cols: Sequence[Column], ids=None):
    """WHERE lhs <op> rhs (the DECIMAL comparison operators of
    P:L730-734).  Each side is evaluated exactly by the oracle (orc_eval_rows,
    the paper's typing and truncation) and the two VALUES are compared as
    exact rationals (each side's mantissa over 10^scale), written out row by
    row.  Returns ids with -1 for every row whose predicate is false (rows
    already negative stay negative).  Rows with an evaluation error raise."""
    from fractions import Fraction
    n = cols[0].n
    out = [0] * n if ids is None else [int(v) for v in ids]
    _, sl = expr_type(lhs, cols)
    _, sr = expr_type(rhs, cols)
    a_rows = eval_rows(lhs, cols, strict=False)
    b_rows = eval_rows(rhs, cols, strict=False)
    for i, (a, b) in enumerate(zip(a_rows, b_rows)):
        if a.startswith("E") or b.startswith("E"):
            raise OracleError(1, f"row {i}: evaluation error")
        va = Fraction(_scaled_int(a, sl), 10 ** sl)
        vb = Fraction(_scaled_int(b, sr), 10 ** sr)
        if not _cmp(va, vb, op):
            out[i] = -1
    return out


def group_ids(keys: Sequence[Column], ids=None):
    """GROUP BY keys (DECIMAL values compared to
    sort for grouping), written out plainly: every included row's key tuple
    (exact values, first key most significant) is collected, the distinct
    tuples are sorted ascending (Python's sort: a library primitive), and each
    row gets the index of its tuple.  Rows with a negative id on input are
    excluded and keep -1.  Returns (ids, n_groups, first) with first[g] the
    smallest row index of group g."""
    from fractions import Fraction
    n = keys[0].n
    base = [0] * n if ids is None else [int(v) for v in ids]
    vals = []
    for col in keys:
        rows = eval_rows("c1", [col], strict=True)
        vals.append([Fraction(_scaled_int(r, col.s), 10 ** col.s) for r in rows])
    tuples = [tuple(v[i] for v in vals) for i in range(n)]
    distinct = sorted({tuples[i] for i in range(n) if base[i] >= 0})
    index = {t: g for g, t in enumerate(distinct)}
    out = [-1] * n
    first = [None] * len(distinct)
    for i in range(n):
        if base[i] < 0:
            continue
        g = index[tuples[i]]
        out[i] = g
        if first[g] is None:
            first[g] = i
    return out, len(distinct), first
