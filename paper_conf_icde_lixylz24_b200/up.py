"""Thin Python binding of libup.so (include/up.h): argument marshalling only.

Every step of the hot path runs in libup's CUDA kernels; PyTorch supplies
device memory, streams and process groups.  There is no CPU fallback: if the
extension is missing, importing/using this module raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import List, Optional, Sequence

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libup.so")

STATUS = {0: "OK", 1: "INVAL", 2: "RANGE", 3: "OVERFLOW", 4: "DIVZERO", 5: "NOMEM",
          6: "CUDA", 7: "NVRTC", 8: "UNSUPPORTED"}


class UpError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"libup {STATUS.get(code, code)}: {msg}")
        self.code = code
        self.name = STATUS.get(code, str(code))


class up_column(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("ld", ctypes.c_int64), ("p", ctypes.c_int32),
                ("s", ctypes.c_int32), ("limbs", ctypes.c_int32), ("layout", ctypes.c_int32),
                ("data", ctypes.c_void_p)]


_lib = None
EXPORTS = ["up_last_error", "up_ctx_create", "up_ctx_destroy", "up_limbs", "up_quads", "up_ld", "up_sum_precision",
           "up_column_from_host_bin", "up_column_from_device_bin", "up_column_from_host",
           "up_column_to_host_bin", "up_expr_type", "up_eval_expr", "up_sum_type", "up_sum_expr",
           "up_sum", "up_sum_combine", "up_modexp", "up_modexp_sum_type", "up_modexp_sum",
           "up_sin_taylor", "up_sin_taylor_sum", "up_check", "up_format_decimal", "up_launch_count",
           "up_jit_ms", "up_gen_source", "up_nvrtc_compile", "up_gen_modexp_source", "up_jit_prewarm", "up_gen_sin_source", "up_compact_bytes",
           "up_column_from_host_compact", "up_column_from_device_compact", "up_column_to_host_compact",
           "up_expr_optimized", "up_gen_contract_source", "up_agg_type", "up_group_aggregate",
           "up_gen_group_agg_source", "up_filter", "up_group_ids", "up_group_combine", "up_eval_tpi",
           "up_gen_tpi_source", "up_set_pipelined"]

AGG = {"SUM": 0, "MIN": 1, "MAX": 2, "AVG": 3}


def lib():
    """Load libup.so (raises if it has not been built: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_icde_lixylz24_b200.build`")
    L = ctypes.CDLL(LIB_PATH)
    c = ctypes
    P = c.c_void_p
    PC = c.POINTER(up_column)
    L.up_last_error.restype = c.c_char_p
    L.up_limbs.argtypes = [c.c_int32]; L.up_limbs.restype = c.c_int32
    L.up_ld.argtypes = [c.c_int64]; L.up_ld.restype = c.c_int64
    L.up_quads.argtypes = [c.c_int32]; L.up_quads.restype = c.c_int32
    L.up_sum_precision.argtypes = [c.c_int32, c.c_int64]; L.up_sum_precision.restype = c.c_int32
    L.up_ctx_create.argtypes = [c.c_int, c.POINTER(P)]
    L.up_ctx_destroy.argtypes = [P]
    L.up_set_pipelined.argtypes = [P, c.c_int]
    L.up_column_from_host_bin.argtypes = [P, P, c.c_int32, P, PC, P]
    L.up_column_from_device_bin.argtypes = [P, P, c.c_int32, P, PC, P]
    L.up_column_from_host.argtypes = [P, c.POINTER(c.c_char_p), PC, P]
    L.up_column_to_host_bin.argtypes = [P, PC, P, P, P]
    L.up_expr_type.argtypes = [P, c.c_char_p, PC, c.c_int, c.POINTER(c.c_int32), c.POINTER(c.c_int32)]
    L.up_eval_expr.argtypes = [P, c.c_char_p, PC, c.c_int, PC, P]
    L.up_sum_type.argtypes = [P, c.c_char_p, PC, c.c_int, c.c_int64, c.POINTER(c.c_int32),
                              c.POINTER(c.c_int32), c.POINTER(c.c_int32)]
    L.up_sum_expr.argtypes = [P, c.c_char_p, PC, c.c_int, c.c_int64, P, P]
    L.up_sum.argtypes = [P, PC, c.c_int64, P, P]
    L.up_sum_combine.argtypes = [P, P, c.c_int32, c.c_int32, P, P]
    L.up_modexp.argtypes = [P, PC, c.c_char_p, c.c_char_p, PC, P]
    L.up_modexp_sum_type.argtypes = [P, c.c_char_p, c.c_int64, c.POINTER(c.c_int32), c.POINTER(c.c_int32)]
    L.up_modexp_sum.argtypes = [P, PC, c.c_char_p, c.c_char_p, c.c_int64, P, P]
    L.up_sin_taylor.argtypes = [P, PC, c.c_int32, PC, P]
    L.up_sin_taylor_sum.argtypes = [P, PC, c.c_int32, c.c_int64, P, P]
    L.up_check.argtypes = [P, P]
    L.up_format_decimal.argtypes = [P, c.c_int32, c.c_int32, c.c_char_p, c.c_size_t]
    L.up_launch_count.argtypes = [P]; L.up_launch_count.restype = c.c_uint64
    L.up_jit_ms.argtypes = [P]; L.up_jit_ms.restype = c.c_double
    L.up_gen_source.argtypes = [c.c_char_p, c.c_char_p, PC, c.c_int, c.c_int64, c.c_char_p, c.c_size_t]
    L.up_nvrtc_compile.argtypes = [c.c_char_p, c.c_char_p, c.c_char_p, c.c_size_t]
    L.up_jit_prewarm.argtypes = [c.c_char_p]
    L.up_compact_bytes.argtypes = [c.c_int32]; L.up_compact_bytes.restype = c.c_int32
    L.up_expr_optimized.argtypes = [c.c_char_p, PC, c.c_int, c.c_char_p, c.c_size_t]
    L.up_gen_contract_source.argtypes = [c.c_int32, c.c_int32, c.c_int32, c.c_int, c.c_char_p, c.c_size_t]
    L.up_column_from_host_compact.argtypes = [P, P, PC, P]
    L.up_column_from_device_compact.argtypes = [P, P, PC, P]
    L.up_column_to_host_compact.argtypes = [P, PC, P, P]
    L.up_gen_sin_source.argtypes = [c.c_int32, c.c_int32, c.c_int32, c.c_int, c.c_int64, c.c_char_p, c.c_size_t]
    PI32 = c.POINTER(c.c_int32)
    L.up_agg_type.argtypes = [c.c_char_p, c.c_int32, PC, c.c_int, c.c_int64, PI32, PI32, PI32]
    L.up_group_aggregate.argtypes = [P, c.c_int32, PI32, c.POINTER(c.c_char_p), PC, c.c_int, P, c.c_int32,
                                     c.c_int64, P, P, P]
    L.up_gen_group_agg_source.argtypes = [c.c_int32, PI32, c.POINTER(c.c_char_p), PC, c.c_int, c.c_int32,
                                          c.c_int64, c.c_char_p, c.c_size_t]
    L.up_filter.argtypes = [P, c.c_char_p, c.c_char_p, c.c_char_p, PC, c.c_int, P, P]
    L.up_group_ids.argtypes = [P, PC, c.c_int, P, c.POINTER(c.c_int64), P, P]
    L.up_eval_tpi.argtypes = [P, c.c_char_p, PC, PC, c.c_int32, c.c_int32, PC, P]
    L.up_gen_tpi_source.argtypes = [c.c_char_p, PC, c.c_int32, c.c_int32, c.c_char_p, c.c_size_t]
    L.up_group_combine.argtypes = [P, c.c_int32, PI32, c.POINTER(c.c_char_p), PC, c.c_int, c.c_int32, c.c_int64, P,
                                   c.c_int32, P, P, P, P]
    L.up_gen_modexp_source.argtypes = [c.c_char_p, c.c_char_p, c.c_int32, c.c_int, c.c_int64, c.c_char_p, c.c_size_t]
    _lib = L
    return L


def _chk(code: int):
    if code != 0:
        raise UpError(code, lib().up_last_error().decode(errors="replace"))


def limbs(p: int) -> int:
    return lib().up_limbs(p)


def compact_bytes(p: int) -> int:
    return lib().up_compact_bytes(p)


def quads(p: int) -> int:
    return lib().up_quads(p)


def ld_for(n: int) -> int:
    return lib().up_ld(n)


def sum_precision(p: int, n_global: int) -> int:
    return lib().up_sum_precision(p, n_global)


def _stream_ptr(stream) -> Optional[int]:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


LAYOUT_PLANES, LAYOUT_COMPACT, LAYOUT_QUADS = 0, 1, 2
_LAYOUTS = {"planes": LAYOUT_PLANES, "compact": LAYOUT_COMPACT, "quads": LAYOUT_QUADS}


class Column:
    """A DECIMAL(p,s) column on the GPU.  layout "planes": `limbs`
    two's-complement limb planes in a torch int32 tensor (limbs, ld);
    layout "compact": the paper's compact byte rows (Lb = compact_bytes(p)
    bytes per row, up.h UP_LAYOUT_COMPACT) in a uint8 tensor padded to 16 bytes;
    layout "quads": limb quads (up.h UP_LAYOUT_QUADS), an int32 tensor
    (quads(p), ld, 4)."""

    def __init__(self, p: int, s: int, n: int, device="cuda", data=None, layout: str = "planes"):
        import torch
        self.p, self.s, self.n = p, s, n
        self.limbs = limbs(p)
        self.layout = _LAYOUTS[layout]
        if self.layout == LAYOUT_COMPACT:
            self.ld = compact_bytes(p)
            if data is None:
                data = torch.empty(((n * self.ld + 15) // 16) * 16 + 16, dtype=torch.uint8, device=device)
        elif self.layout == LAYOUT_QUADS:
            self.ld = ld_for(n)
            if data is None:
                data = torch.empty((quads(p), max(self.ld, 4), 4), dtype=torch.int32, device=device)
        else:
            self.ld = ld_for(n)
            if data is None:
                data = torch.empty((self.limbs, max(self.ld, 4)), dtype=torch.int32, device=device)
        self.data = data

    def desc(self) -> up_column:
        return up_column(self.n, self.ld, self.p, self.s, self.limbs, self.layout, self.data.data_ptr())

    def rows(self, r0: int, r1: int) -> "Column":
        """Rows [r0, r1) as a column sharing this one's memory (same ld; r0 a
        multiple of 4, of 16 for compact rows, keeps the 16-byte alignment)."""
        if not 0 <= r0 <= r1 <= self.n:
            raise ValueError("bad row range")
        v = Column.__new__(Column)
        v.p, v.s, v.n, v.limbs, v.layout, v.ld = self.p, self.s, r1 - r0, self.limbs, self.layout, self.ld
        if self.layout == LAYOUT_COMPACT:
            v.data = self.data[r0 * self.ld:]
        elif self.layout == LAYOUT_QUADS:
            v.data = self.data[:, r0:, :]
        else:
            v.data = self.data[:, r0:]
        if v.data.data_ptr() % 16:
            raise ValueError("row view not 16-byte aligned")
        return v

    @property
    def type(self):
        return (self.p, self.s)


def _descs(cols: Sequence[Column]):
    arr = (up_column * max(1, len(cols)))()
    for i, c in enumerate(cols):
        arr[i] = c.desc()
    return arr


def format_decimal(limbs_u32: Sequence[int], s: int) -> str:
    """Canonical string of a two's-complement limb vector (libup's formatter)."""
    n = len(limbs_u32)
    arr = (ctypes.c_uint32 * n)(*[int(x) & 0xFFFFFFFF for x in limbs_u32])
    buf = ctypes.create_string_buffer(n * 10 + s + 8)
    _chk(lib().up_format_decimal(arr, n, s, buf, len(buf)))
    return buf.value.decode()


def limbs_to_int(limbs_u32: Sequence[int]) -> int:
    v = 0
    for x in reversed(list(limbs_u32)):
        v = (v << 32) | (int(x) & 0xFFFFFFFF)
    n = len(limbs_u32)
    if n and (int(limbs_u32[-1]) & 0x80000000):
        v -= 1 << (32 * n)
    return v


class Context:
    """One libup context (kernel cache, SUM workspace, staging) on one device."""

    def __init__(self, device: int = 0):
        import torch
        torch.cuda.init()
        torch.cuda.set_device(device)
        self.device = device
        h = ctypes.c_void_p()
        _chk(lib().up_ctx_create(device, ctypes.byref(h)))
        self.h = h

    def close(self):
        if self.h:
            lib().up_ctx_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_pipelined(self, on: bool = True):
        """Programmatic dependent launch of the fused SUM kernels (up.h
        up_set_pipelined): back-to-back SUMs over resident columns overlap.
        The kernel right before such a SUM on its stream must not write the
        SUM's input columns."""
        _chk(lib().up_set_pipelined(self.h, 1 if on else 0))

    # ------------------------------------------------------------------ info
    @property
    def launches(self) -> int:
        return lib().up_launch_count(self.h)

    @property
    def jit_ms(self) -> float:
        return lib().up_jit_ms(self.h)

    # ------------------------------------------------------------------ columns
    def column_from_host_bin(self, p: int, s: int, mag, neg=None, stream=None, out: Optional[Column] = None,
                             layout: str = "planes"):
        """mag: (n, W) uint32 host array (numpy or pinned torch); neg: (n,) uint8."""
        import numpy as np
        import torch
        if isinstance(mag, np.ndarray):
            n, W = mag.shape
            mag_ptr = mag.ctypes.data
            neg_ptr = neg.ctypes.data if neg is not None else None
        else:
            n, W = mag.shape
            mag_ptr = mag.data_ptr()
            neg_ptr = neg.data_ptr() if neg is not None else None
        col = out if out is not None else Column(p, s, n, layout=layout)
        d = col.desc()
        _chk(lib().up_column_from_host_bin(self.h, mag_ptr, W, neg_ptr, ctypes.byref(d), _stream_ptr(stream)))
        return col

    def column_from_device_bin(self, p: int, s: int, d_mag, d_neg=None, stream=None, out: Optional[Column] = None,
                               layout: str = "planes"):
        """d_mag: (n, W) int32/uint32 CUDA tensor; d_neg: (n,) uint8 CUDA tensor."""
        n, W = d_mag.shape
        col = out if out is not None else Column(p, s, n, layout=layout)
        d = col.desc()
        _chk(lib().up_column_from_device_bin(self.h, d_mag.data_ptr(), W,
                                             d_neg.data_ptr() if d_neg is not None else None,
                                             ctypes.byref(d), _stream_ptr(stream)))
        return col

    def column_from_compact(self, p: int, s: int, data, n: Optional[int] = None, stream=None,
                            out: Optional[Column] = None, layout: str = "planes"):
        """Compact rows: numpy uint8 / pinned torch uint8 (host) or a CUDA uint8 tensor."""
        import numpy as np
        Lb = compact_bytes(p)
        if isinstance(data, np.ndarray):
            n = data.size // Lb if n is None else n
            ptr, dev = data.ctypes.data, False
        else:
            n = data.numel() // Lb if n is None else n
            ptr, dev = data.data_ptr(), data.is_cuda
        col = out if out is not None else Column(p, s, n, layout=layout)
        d = col.desc()
        fn = lib().up_column_from_device_compact if dev else lib().up_column_from_host_compact
        _chk(fn(self.h, ptr, ctypes.byref(d), _stream_ptr(stream)))
        return col

    def column_to_compact(self, col: Column, stream=None):
        import numpy as np
        out = np.zeros(max(1, col.n * compact_bytes(col.p)), dtype=np.uint8)
        d = col.desc()
        _chk(lib().up_column_to_host_compact(self.h, ctypes.byref(d), out.ctypes.data, _stream_ptr(stream)))
        return out[: col.n * compact_bytes(col.p)]

    def column_from_strings(self, p: int, s: int, values: Sequence[str], stream=None, layout: str = "planes"):
        col = Column(p, s, len(values), layout=layout)
        arr = (ctypes.c_char_p * max(1, len(values)))(*[v.encode() for v in values])
        d = col.desc()
        _chk(lib().up_column_from_host(self.h, arr, ctypes.byref(d), _stream_ptr(stream)))
        return col

    def column_to_ints(self, col: Column, stream=None) -> List[int]:
        import numpy as np
        mag = np.zeros((max(col.n, 1), col.limbs), dtype=np.uint32)
        neg = np.zeros(max(col.n, 1), dtype=np.uint8)
        d = col.desc()
        _chk(lib().up_column_to_host_bin(self.h, ctypes.byref(d), mag.ctypes.data, neg.ctypes.data,
                                         _stream_ptr(stream)))
        out = []
        for i in range(col.n):
            v = 0
            for x in reversed(mag[i].tolist()):
                v = (v << 32) | x
            out.append(-v if neg[i] else v)
        return out

    def column_to_strings(self, col: Column, stream=None) -> List[str]:
        """Canonical decimal strings of every row (libup's formatter)."""
        import numpy as np
        mag = np.zeros((max(col.n, 1), col.limbs + 1), dtype=np.uint32)   # +1: keep magnitudes non-negative
        neg = np.zeros(max(col.n, 1), dtype=np.uint8)
        tmp = np.zeros((max(col.n, 1), col.limbs), dtype=np.uint32)
        d = col.desc()
        _chk(lib().up_column_to_host_bin(self.h, ctypes.byref(d), tmp.ctypes.data, neg.ctypes.data,
                                         _stream_ptr(stream)))
        mag[:, :col.limbs] = tmp
        out = []
        buf = ctypes.create_string_buffer((col.limbs + 1) * 10 + col.s + 8)
        for i in range(col.n):
            row = np.ascontiguousarray(mag[i])
            _chk(lib().up_format_decimal(row.ctypes.data, col.limbs + 1, col.s, buf, len(buf)))
            v = buf.value.decode()
            out.append("-" + v if neg[i] and v.strip("0.") else v)
        return out

    # ------------------------------------------------------------------ expressions
    def expr_type(self, expr: str, cols: Sequence[Column]):
        P, S = ctypes.c_int32(), ctypes.c_int32()
        _chk(lib().up_expr_type(self.h, expr.encode(), _descs(cols), len(cols), ctypes.byref(P), ctypes.byref(S)))
        return P.value, S.value

    def eval_expr(self, expr: str, cols: Sequence[Column], out: Optional[Column] = None, stream=None) -> Column:
        p, s = self.expr_type(expr, cols)
        if out is None:
            out = Column(p, s, cols[0].n)
        d = out.desc()
        _chk(lib().up_eval_expr(self.h, expr.encode(), _descs(cols), len(cols), ctypes.byref(d), _stream_ptr(stream)))
        return out

    def sum_type(self, expr: str, cols: Sequence[Column], n_global: int = 0):
        P, S, LA = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
        _chk(lib().up_sum_type(self.h, expr.encode(), _descs(cols), len(cols), n_global,
                               ctypes.byref(P), ctypes.byref(S), ctypes.byref(LA)))
        return P.value, S.value, LA.value

    def sum_expr(self, expr: str, cols: Sequence[Column], n_global: int = 0, out=None, stream=None):
        """SELECT SUM(expr): returns the device tensor of LA two's-complement limbs."""
        if out is None:     # (typing parses the expression: only when the caller has no buffer)
            import torch
            _, _, LA = self.sum_type(expr, cols, n_global)
            out = torch.empty(LA, dtype=torch.int32, device=cols[0].data.device)
        _chk(lib().up_sum_expr(self.h, expr.encode(), _descs(cols), len(cols), n_global, out.data_ptr(),
                               _stream_ptr(stream)))
        return out

    def sum_combine(self, partials, la: int, out=None, stream=None):
        """partials: (nranks * la) int32 CUDA tensor (e.g. an all-gather output)."""
        import torch
        nranks = partials.numel() // la
        if out is None:
            out = torch.empty(la, dtype=torch.int32, device=partials.device)
        _chk(lib().up_sum_combine(self.h, partials.data_ptr(), nranks, la, out.data_ptr(), _stream_ptr(stream)))
        return out

    def modexp(self, base: Column, exponent: int, modulus: int, out: Optional[Column] = None, stream=None):
        if out is None:
            out = Column(len(str(modulus)), 0, base.n)
        d = out.desc()
        bd = base.desc()
        _chk(lib().up_modexp(self.h, ctypes.byref(bd), str(exponent).encode(), str(modulus).encode(),
                             ctypes.byref(d), _stream_ptr(stream)))
        return out

    def modexp_sum_type(self, modulus: int, n_global: int):
        P, LA = ctypes.c_int32(), ctypes.c_int32()
        _chk(lib().up_modexp_sum_type(self.h, str(modulus).encode(), n_global, ctypes.byref(P), ctypes.byref(LA)))
        return P.value, LA.value

    def modexp_sum(self, base: Column, exponent: int, modulus: int, n_global: int = 0, out=None, stream=None):
        import torch
        _, LA = self.modexp_sum_type(modulus, n_global or base.n)
        if out is None:
            out = torch.empty(LA, dtype=torch.int32, device=base.data.device)
        bd = base.desc()
        _chk(lib().up_modexp_sum(self.h, ctypes.byref(bd), str(exponent).encode(), str(modulus).encode(),
                                 n_global, out.data_ptr(), _stream_ptr(stream)))
        return out

    def sin_taylor(self, x: Column, P: int, out: Optional[Column] = None, stream=None):
        if out is None:
            out = Column(P + 1, P, x.n)
        d, xd = out.desc(), x.desc()
        _chk(lib().up_sin_taylor(self.h, ctypes.byref(xd), P, ctypes.byref(d), _stream_ptr(stream)))
        return out

    def sin_taylor_sum(self, x: Column, P: int, n_global: int = 0, out=None, stream=None):
        import torch
        LA = limbs(sum_precision(P + 1, n_global or x.n))
        if out is None:
            out = torch.empty(LA, dtype=torch.int32, device=x.data.device)
        xd = x.desc()
        _chk(lib().up_sin_taylor_sum(self.h, ctypes.byref(xd), P, n_global, out.data_ptr(), _stream_ptr(stream)))
        return out

    def group_aggregate(self, aggs: Sequence[tuple], cols: Sequence[Column], group=None, n_groups: int = 1,
                        n_global: int = 0, out=None, counts=None, stream=None, partial: bool = False):
        """SELECT agg(expr), ... GROUP BY group in one launch (include/up.h
        up_group_aggregate).  aggs: [(kind, expr)], kind in AGG's keys.
        Returns (packed int32 device tensor, int64 device counts, layout) where
        layout[a] = (p, s, limbs, offset) and aggregate a of group g occupies
        out[offset + g*limbs : offset + (g+1)*limbs].  partial=True: each AVG
        is computed as its SUM (the state up_group_combine merges across ranks)."""
        import torch
        if partial:
            aggs = [("SUM" if k == "AVG" else k, e) for k, e in aggs]
        layout, off = [], 0
        for kind, expr in aggs:
            p, s, L = agg_type(kind, expr, [(c.p, c.s) for c in cols], n_global or cols[0].n)
            layout.append((p, s, L, off))
            off += n_groups * L
        dev = cols[0].data.device
        if out is None:
            out = torch.empty(max(off, 1), dtype=torch.int32, device=dev)
        if counts is None:
            counts = torch.empty(n_groups, dtype=torch.int64, device=dev)
        kinds, exprs = _agg_args(aggs)
        _chk(lib().up_group_aggregate(self.h, len(aggs), kinds, exprs, _descs(cols), len(cols),
                                      group.data_ptr() if group is not None else None, n_groups, n_global,
                                      out.data_ptr(), counts.data_ptr(), _stream_ptr(stream)))
        return out, counts, layout

    def group_combine(self, aggs: Sequence[tuple], cols: Sequence[Column], parts, counts, nranks: int,
                      n_groups: int = 1, n_global: int = 0, out=None, counts_out=None, stream=None):
        """Merge nranks gathered group_aggregate(partial=True) outputs (parts:
        int32 device tensor, rank-major; counts: int64 device tensor nranks x
        n_groups) into the final aggregates (include/up.h up_group_combine).
        Returns (packed int32 device tensor, int64 counts, layout) like group_aggregate."""
        import torch
        N = n_global or cols[0].n
        layout, off = [], 0
        for kind, expr in aggs:
            p, s, L = agg_type(kind, expr, [(c.p, c.s) for c in cols], N)
            layout.append((p, s, L, off))
            off += n_groups * L
        dev = parts.device
        if out is None:
            out = torch.empty(max(off, 1), dtype=torch.int32, device=dev)
        if counts_out is None:
            counts_out = torch.empty(n_groups, dtype=torch.int64, device=dev)
        kinds, exprs = _agg_args(aggs)
        _chk(lib().up_group_combine(self.h, len(aggs), kinds, exprs, _descs(cols), len(cols), n_groups, N,
                                    parts.data_ptr(), nranks, counts.data_ptr(), out.data_ptr(), counts_out.data_ptr(),
                                    _stream_ptr(stream)))
        return out, counts_out, layout

    def eval_tpi(self, op: str, a: Column, b: Column, tpi: int = 1, div_algo: str = "long", out: Optional[Column] = None,
                 stream=None) -> Column:
        """a <op> b per row with tpi lanes per row (include/up.h up_eval_tpi);
        div_algo "long" (Knuth D) or "newton" (Newton-Raphson) for "/"."""
        p, s = self.expr_type(f"c1{op}c2", [a, b])
        if out is None:
            out = Column(p, s, a.n)
        d, ad, bd = out.desc(), a.desc(), b.desc()
        _chk(lib().up_eval_tpi(self.h, op.encode(), ctypes.byref(ad), ctypes.byref(bd), tpi,
                               1 if div_algo == "newton" else 0, ctypes.byref(d), _stream_ptr(stream)))
        return out

    def filter(self, lhs: str, op: str, rhs: str, cols: Sequence[Column], ids=None, stream=None):
        """WHERE lhs <op> rhs (include/up.h up_filter): rows whose predicate is
        false get id -1 in `ids` (int32 device tensor, created as zeros when
        None); returns ids.  Successive calls AND their predicates."""
        import torch
        if ids is None:
            ids = torch.zeros(cols[0].n, dtype=torch.int32, device=cols[0].data.device)
        _chk(lib().up_filter(self.h, lhs.encode(), op.encode(), rhs.encode(), _descs(cols), len(cols),
                             ids.data_ptr(), _stream_ptr(stream)))
        return ids

    def group_ids(self, keys: Sequence[Column], ids=None, first: bool = False, stream=None):
        """GROUP BY keys (include/up.h up_group_ids): dense group ids in ascending
        key order written into `ids` (rows already negative stay excluded).
        Returns (ids, n_groups[, first_row int64 tensor of the groups' smallest row])."""
        import torch
        dev = keys[0].data.device
        if ids is None:
            ids = torch.zeros(keys[0].n, dtype=torch.int32, device=dev)
        f = torch.empty(max(keys[0].n, 1), dtype=torch.int64, device=dev) if first else None
        ng = ctypes.c_int64(0)
        _chk(lib().up_group_ids(self.h, _descs(keys), len(keys), ids.data_ptr(), ctypes.byref(ng),
                                f.data_ptr() if f is not None else None, _stream_ptr(stream)))
        return (ids, ng.value, f[:ng.value]) if first else (ids, ng.value)

    def check(self, stream=None):
        _chk(lib().up_check(self.h, _stream_ptr(stream)))


def _agg_args(aggs):
    kinds = (ctypes.c_int32 * len(aggs))(*[AGG[k] for k, _ in aggs])
    exprs = (ctypes.c_char_p * len(aggs))(*[e.encode() for _, e in aggs])
    return kinds, exprs


def _type_descs(types: Sequence[tuple], n: int = 1):
    arr = (up_column * max(1, len(types)))()
    for i, (p, s) in enumerate(types):
        arr[i] = up_column(n, ld_for(n), p, s, limbs(p), 0, None)
    return arr


def agg_type(kind: str, expr: str, types: Sequence[tuple], n_global: int):
    """(p, s, limbs) of an aggregate over n_global tuples (no GPU)."""
    p, s, L = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    _chk(lib().up_agg_type(expr.encode(), AGG[kind], _type_descs(types), len(types), n_global,
                           ctypes.byref(p), ctypes.byref(s), ctypes.byref(L)))
    return p.value, s.value, L.value


def group_results(out, counts, layout, n_groups: int):
    """Packed group_aggregate output -> ([[string per group] per aggregate], [count per group])."""
    host = out.detach().cpu().tolist()
    res = []
    for p, s, L, off in layout:
        res.append([format_decimal(host[off + g * L: off + (g + 1) * L], s) for g in range(n_groups)])
    return res, [int(x) for x in counts.detach().cpu().tolist()]


def _fmt(v: int, s: int) -> str:
    sign = "-" if v < 0 else ""
    a = str(abs(v))
    if s == 0:
        return sign + a
    a = a.rjust(s + 1, "0")
    return sign + a[:-s] + "." + a[-s:]


def result_to_string(limb_tensor, s: int) -> str:
    """Device/host limb tensor of a SUM result -> canonical decimal string."""
    vals = limb_tensor.detach().cpu().tolist() if hasattr(limb_tensor, "detach") else list(limb_tensor)
    return format_decimal(vals, s)


# ---------------------------------------------------------------------- diagnostics
def gen_source(variant: str, expr: str, types: Sequence[tuple], n_global: int = 1,
               compact: Optional[Sequence[bool]] = None, layouts: Optional[Sequence[str]] = None) -> str:
    """Generated kernel source (no GPU); compact[i]: column i in the compact
    layout; layouts[i]: "planes" / "compact" / "quads"."""
    arr = (up_column * max(1, len(types)))()
    for i, (p, s) in enumerate(types):
        lay = layouts[i] if layouts else ("compact" if compact and compact[i] else "planes")
        if lay == "compact":
            arr[i] = up_column(n_global, compact_bytes(p), p, s, limbs(p), LAYOUT_COMPACT, None)
        elif lay == "quads":
            arr[i] = up_column(n_global, ld_for(n_global), p, s, limbs(p), LAYOUT_QUADS, None)
        else:
            arr[i] = up_column(n_global, ld_for(n_global), p, s, limbs(p), 0, None)
    buf = ctypes.create_string_buffer(1 << 24)
    _chk(lib().up_gen_source(variant.encode(), expr.encode(), arr, len(types), n_global, buf, len(buf)))
    return buf.value.decode()


def gen_tpi_source(op: str, types: Sequence[tuple], tpi: int = 1, div_algo: str = "long",
                   compact: Optional[Sequence[bool]] = None) -> str:
    arr = (up_column * 2)()
    for i, (p, s) in enumerate(types):
        if compact and compact[i]:
            arr[i] = up_column(1, compact_bytes(p), p, s, limbs(p), LAYOUT_COMPACT, None)
        else:
            arr[i] = up_column(1, 4, p, s, limbs(p), 0, None)
    buf = ctypes.create_string_buffer(1 << 22)
    _chk(lib().up_gen_tpi_source(op.encode(), arr, tpi, 1 if div_algo == "newton" else 0, buf, len(buf)))
    return buf.value.decode()


def gen_modexp_source(exponent: int, modulus: int, base_p: int, sum: bool = False, n_global: int = 1) -> str:
    buf = ctypes.create_string_buffer(1 << 24)
    _chk(lib().up_gen_modexp_source(str(exponent).encode(), str(modulus).encode(), base_p, int(sum), n_global,
                                    buf, len(buf)))
    return buf.value.decode()


def gen_sin_source(P: int, p: int = 9, s: int = 8, sum: bool = False, n_global: int = 1) -> str:
    buf = ctypes.create_string_buffer(1 << 24)
    _chk(lib().up_gen_sin_source(P, p, s, int(sum), n_global, buf, len(buf)))
    return buf.value.decode()


def expr_optimized(expr: str, types: Sequence[tuple]) -> str:
    """Canonical text of the optimised expression tree (no GPU)."""
    arr = (up_column * max(1, len(types)))()
    for i, (p, s) in enumerate(types):
        arr[i] = up_column(1, 4, p, s, limbs(p), 0, None)
    buf = ctypes.create_string_buffer(1 << 16)
    _chk(lib().up_expr_optimized(expr.encode(), arr, len(types), buf, len(buf)))
    return buf.value.decode()


def gen_contract_source(La: int, Lb: int, LA: int, sign: int = 1) -> str:
    buf = ctypes.create_string_buffer(1 << 20)
    _chk(lib().up_gen_contract_source(La, Lb, LA, sign, buf, len(buf)))
    return buf.value.decode()


def gen_group_agg_source(aggs: Sequence[tuple], types: Sequence[tuple], n_groups: int, n_global: int) -> str:
    kinds, exprs = _agg_args(aggs)
    buf = ctypes.create_string_buffer(1 << 24)
    _chk(lib().up_gen_group_agg_source(len(aggs), kinds, exprs, _type_descs(types, n_global), len(types),
                                       n_groups, n_global, buf, len(buf)))
    return buf.value.decode()


def jit_prewarm(src: str):
    _chk(lib().up_jit_prewarm(src.encode()))


def nvrtc_compile(src: str, cubin_path: Optional[str] = None) -> str:
    log = ctypes.create_string_buffer(1 << 16)
    code = lib().up_nvrtc_compile(src.encode(), cubin_path.encode() if cubin_path else None, log, len(log))
    if code:
        raise UpError(code, lib().up_last_error().decode() + "\n" + log.value.decode(errors="replace"))
    return log.value.decode(errors="replace")
