"""Seeded synthetic inputs shaped like the paper's workloads (host side).

This module holds NONE of the method's arithmetic: it only draws random
integers.  It serves both the oracle and the CUDA path.  Its device twin is
``gen/gen_kernels.cu`` (``libupgen.so``), which implements the SAME
counter-based generator, so a device-generated column is bit-identical to
the host one (checked by ``tests/test_gpu_parity.py::test_device_generator``).

Counter-based draw (both sides):
    key(seed, stream)       = mix64(seed * GOLD + stream)
    word(key, row, att, j)  = low32( mix64(key ^ mix64((row << 32) | (att << 10) | j)) )
with mix64 the SplitMix64 finaliser.  A value of W words uses words
j = 0..W-1 of attempt ``att`` (top word masked to bitlen(hi)); it is accepted
when lo <= v <= hi (rejection sampling: uniform on [lo, hi]); the sign is
bit 0 of word j = W of the accepted attempt.  Seeds/streams: SURVEY §8(d)
(seed 20240513, stream = 64*config + column).

Distributions (SURVEY §8c readings Q14-Q16, "randomly generated"):
  * uniform_decimal: magnitude uniform on [0, 10^p - 1], uniform sign;
  * divisor columns: magnitude in [10^(p-1), 10^p - 1] (reading Q5);
  * series: mantissa a + i*d (closed-form SUM pin);
  * normal_decimal: round-half-even(N(mu, sigma) * 10^s) (trig);
  * rsa_modulus / messages (Query 4, reading Q15).
"""
from __future__ import annotations

import numpy as np

SEED = 20240513
GOLD = 0x9E3779B97F4A7C15
M64 = (1 << 64) - 1


def stream_id(config: int, column: int) -> int:
    return 64 * config + column


def _mix64_np(z: np.ndarray) -> np.ndarray:
    z = z.astype(np.uint64, copy=True)
    z ^= z >> np.uint64(30)
    z *= np.uint64(0xBF58476D1CE4E5B9)
    z ^= z >> np.uint64(27)
    z *= np.uint64(0x94D049BB133111EB)
    z ^= z >> np.uint64(31)
    return z


def _mix64_int(z: int) -> int:
    z &= M64
    z ^= z >> 30
    z = (z * 0xBF58476D1CE4E5B9) & M64
    z ^= z >> 27
    z = (z * 0x94D049BB133111EB) & M64
    z ^= z >> 31
    return z


def stream_key(seed: int, stream: int) -> int:
    return _mix64_int((seed * GOLD + stream) & M64)


def _words(key: int, rows: np.ndarray, att: int, j: int) -> np.ndarray:
    ctr = (rows.astype(np.uint64) << np.uint64(32)) | np.uint64((att << 10) | j)
    return (_mix64_np(np.uint64(key) ^ _mix64_np(ctr)) & np.uint64(0xFFFFFFFF)).astype(np.uint32)


def int_to_words(v: int, w: int) -> np.ndarray:
    return np.array([(v >> (32 * j)) & 0xFFFFFFFF for j in range(w)], dtype=np.uint32)


def words_to_int(row) -> int:
    v = 0
    for j in reversed(range(len(row))):
        v = (v << 32) | int(row[j])
    return v


def _ge(a: np.ndarray, bound: np.ndarray) -> np.ndarray:
    """row-wise a >= bound for (m, W) word arrays vs a (W,) constant."""
    res = np.ones(a.shape[0], dtype=bool)       # equal so far -> >=
    decided = np.zeros(a.shape[0], dtype=bool)
    for j in reversed(range(a.shape[1])):
        gt = (a[:, j] > bound[j]) & ~decided
        lt = (a[:, j] < bound[j]) & ~decided
        res[lt] = False
        res[gt] = True
        decided |= gt | lt
    return res


def uniform_range(seed: int, stream: int, n: int, lo: int, hi: int, signed: bool = True,
                  row0: int = 0, max_attempts: int = 4096):
    """n values with magnitude uniform on [lo, hi] (rejection on bitlen(hi)).
    Returns (mag uint32[n, W], neg uint8[n]) with W = ceil(bitlen(hi)/32)."""
    assert 0 <= lo <= hi and hi > 0
    nbits = hi.bit_length()
    W = (nbits + 31) // 32
    topmask = np.uint32((1 << (nbits - 32 * (W - 1))) - 1) if nbits % 32 else np.uint32(0xFFFFFFFF)
    key = stream_key(seed, stream)
    lo_w, hi_w = int_to_words(lo, W), int_to_words(hi, W)
    mag = np.zeros((n, W), dtype=np.uint32)
    neg = np.zeros(n, dtype=np.uint8)
    pending = np.arange(n, dtype=np.int64)
    for att in range(max_attempts):
        if pending.size == 0:
            break
        rows = pending + row0
        cand = np.empty((pending.size, W), dtype=np.uint32)
        for j in range(W):
            cand[:, j] = _words(key, rows, att, j)
        cand[:, W - 1] &= topmask
        ok = _ge(cand, lo_w) & ~_gt(cand, hi_w)
        acc = pending[ok]
        mag[acc] = cand[ok]
        if signed:
            neg[acc] = (_words(key, rows[ok], att, W) & np.uint32(1)).astype(np.uint8)
        pending = pending[~ok]
    if pending.size:
        raise RuntimeError("generator: rejection sampling did not converge")
    return mag, neg


def _gt(a: np.ndarray, bound: np.ndarray) -> np.ndarray:
    """row-wise a > bound."""
    res = np.zeros(a.shape[0], dtype=bool)
    decided = np.zeros(a.shape[0], dtype=bool)
    for j in reversed(range(a.shape[1])):
        gt = (a[:, j] > bound[j]) & ~decided
        lt = (a[:, j] < bound[j]) & ~decided
        res[gt] = True
        decided |= gt | lt
    return res


def uniform_decimal(n: int, p: int, config: int, column: int, seed: int = SEED, row0: int = 0,
                    nonzero_lead: bool = False, signed: bool = True):
    """DECIMAL(p, .) column: |mantissa| uniform on [0, 10^p-1] (or [10^(p-1), 10^p-1])."""
    lo = 10 ** (p - 1) if nonzero_lead else 0
    return uniform_range(seed, stream_id(config, column), n, lo, 10 ** p - 1, signed, row0)


def series(n: int, a: int, d: int, w: int, row0: int = 0):
    """mantissas a + i*d (i = row0..row0+n-1), sign-magnitude words."""
    vals = [a + (row0 + i) * d for i in range(n)]
    mag = np.zeros((n, w), dtype=np.uint32)
    neg = np.zeros(n, dtype=np.uint8)
    for i, v in enumerate(vals):
        mag[i] = int_to_words(abs(v), w)
        neg[i] = 1 if v < 0 else 0
    return mag, neg


def normal_decimal(n: int, mu: float, sigma: float, s: int, config: int, column: int,
                   seed: int = SEED, row0: int = 0):
    """round-half-even(N(mu, sigma) * 10^s) as a one-word sign-magnitude column
    (Box-Muller on two counter-based 32-bit uniforms).  Host-only."""
    key = stream_key(seed, stream_id(config, column))
    rows = np.arange(row0, row0 + n, dtype=np.int64)
    u1 = (_words(key, rows, 0, 0).astype(np.float64) + 1.0) / 4294967296.0   # (0, 1]
    u2 = _words(key, rows, 0, 1).astype(np.float64) / 4294967296.0          # [0, 1)
    z = np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)
    m = np.rint((mu + sigma * z) * (10.0 ** s)).astype(np.int64)
    if np.any(np.abs(m) >= 2 ** 32):
        raise ValueError("normal_decimal: value does not fit one word")
    mag = np.abs(m).astype(np.uint32).reshape(n, 1)
    neg = (m < 0).astype(np.uint8)
    return mag, neg


def _next_prime(x: int) -> int:
    import sympy
    return int(sympy.nextprime(x))


def rsa_modulus(bits: int, seed: int = SEED, config: int = 4):
    """N = p*q with p, q primes of bits/2 bits, the top two bits set (reading Q15)."""
    half = bits // 2
    out = []
    for idx in (0, 1):
        key = stream_key(seed, stream_id(config, 60 + idx))
        words = [int(_words(key, np.array([bits]), 0, j)[0]) for j in range((half + 31) // 32)]
        r = words_to_int(words) & ((1 << half) - 1)
        r |= (3 << (half - 2)) | 1
        out.append(_next_prime(r))
    p, q = out
    N = p * q
    assert N.bit_length() == bits
    return N, p, q


def rsa_messages(n: int, N: int, config: int = 4, column: int = 0, seed: int = SEED, row0: int = 0):
    """messages uniform on [0, N-1], non-negative."""
    return uniform_range(seed, stream_id(config, column), n, 0, N - 1, signed=False, row0=row0)


def to_ints(mag: np.ndarray, neg: np.ndarray):
    """Python ints from sign-magnitude words (test helper)."""
    out = []
    for i in range(mag.shape[0]):
        v = words_to_int(mag[i])
        out.append(-v if neg[i] else v)
    return out


def compact_bytes(p: int) -> int:
    """Lb = ceil((1 + p log2 10) / 8): bitlen(10^p - 1) + 1 sign bit."""
    return ((10 ** p - 1).bit_length() + 1 + 7) // 8


def to_compact(mag: np.ndarray, neg: np.ndarray, p: int) -> np.ndarray:
    """Pack sign-magnitude words into the paper's compact rows (Fig. 4):
    Lb bytes per row, magnitude little-endian, sign in the top bit of the last
    byte.  Pure re-packing of the generator's output (no arithmetic)."""
    Lb = compact_bytes(p)
    n, W = mag.shape
    raw = np.ascontiguousarray(mag, dtype="<u4").view(np.uint8).reshape(n, 4 * W)
    out = np.zeros((n, Lb), dtype=np.uint8)
    k = min(Lb, 4 * W)
    out[:, :k] = raw[:, :k]
    out[:, Lb - 1] |= (np.asarray(neg, dtype=np.uint8) & 1) << 7
    return out.reshape(-1)
