"""Device-side generation through gen/libupgen.so (the CUDA twin of
gen/synth.py).  Input generation only -- no method arithmetic."""
from __future__ import annotations

import ctypes
import os
import subprocess

from . import synth

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen_kernels.cu")
LIB_PATH = os.path.join(_HERE, "libupgen.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < os.path.getmtime(_SRC):
        tmp = LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-lineinfo", "-Xcompiler", "-fPIC", "-shared", "-cudart", "static", _SRC, "-o", tmp])
        os.replace(tmp, LIB_PATH)
    return LIB_PATH


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run gen.device.build()")
        _lib = ctypes.CDLL(LIB_PATH)
        _lib.upgen_uniform.argtypes = [ctypes.c_uint64, ctypes.c_longlong, ctypes.c_longlong, ctypes.c_int,
                                       ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                       ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
    return _lib


def uniform_range(seed: int, stream_id: int, n: int, lo: int, hi: int, signed: bool = True, row0: int = 0,
                  device="cuda", cuda_stream=None):
    """Device twin of synth.uniform_range: returns (mag int32[n, W], neg uint8[n]) CUDA tensors."""
    import numpy as np
    import torch
    nbits = hi.bit_length()
    W = (nbits + 31) // 32
    topmask = ((1 << (nbits - 32 * (W - 1))) - 1) if nbits % 32 else 0xFFFFFFFF
    key = synth.stream_key(seed, stream_id)
    lo_w = torch.from_numpy(synth.int_to_words(lo, W).view(np.int32).copy()).to(device)
    hi_w = torch.from_numpy(synth.int_to_words(hi, W).view(np.int32).copy()).to(device)
    mag = torch.empty((max(n, 1), W), dtype=torch.int32, device=device)
    neg = torch.empty(max(n, 1), dtype=torch.uint8, device=device)
    fail = torch.zeros(1, dtype=torch.int32, device=device)
    st = cuda_stream if cuda_stream is not None else torch.cuda.current_stream().cuda_stream
    rc = lib().upgen_uniform(key, row0, n, W, topmask, lo_w.data_ptr(), hi_w.data_ptr(), int(signed),
                             mag.data_ptr(), neg.data_ptr(), fail.data_ptr(), st)
    if rc:
        raise RuntimeError(f"upgen_uniform failed ({rc})")
    if int(fail.item()):
        raise RuntimeError("device generator: rejection sampling did not converge")
    return mag[:n], neg[:n]


def uniform_decimal(n: int, p: int, config: int, column: int, seed: int = synth.SEED, row0: int = 0,
                    nonzero_lead: bool = False, signed: bool = True, device="cuda"):
    lo = 10 ** (p - 1) if nonzero_lead else 0
    return uniform_range(seed, synth.stream_id(config, column), n, lo, 10 ** p - 1, signed, row0, device)
