#!/usr/bin/env python
"""Word-level Python model of the skewed-band sin_P kernel (special.cpp
gen_sin_kernel_band), used to validate its arithmetic before/alongside the
CUDA code.  It is NOT the oracle: it mirrors the kernel's 32-bit digit steps
(Horner long division with non-normalised product digits, Moller-Granlund
3-by-2 quotient steps against a normalised 64-bit divisor, the bit offset o_k
that absorbs the 2^(2s) factor of 10^(2s), digit drops, the low-bit mask, the
scaled carry-save running sum) so a mistake in that plan shows up as a
mismatch against the Q13 definition (tests/test_sin_model.py); term_divide64
is the same division on 64-bit chunks (the band kernel's digit pairs).

Per row, x = m 10^-s (|m| < 10^9, 2s < 32), X2 = m^2,
D_k = 5^(2s) (2k)(2k+1), 10^(2s) (2k)(2k+1) = 2^(2s) D_k.
Y_k = t_k 2^(o_k) (o_1 = 0); term k computes Q = floor(Y_k X2 / D_k) as a
Horner long division MS -> LS over the digit stream of V = Y_k X2 2^sh
(sh = clz64(D_k), D~ = D_k 2^sh normalised), then with o' = o_k + 2s:
Y_(k+1) = (Q with its low o' bits cleared) / B^[o' >= 32],  o_(k+1) = o' mod 32
(floor composition: t_(k+1) = floor(Q / 2^o')).  S = sum (-1)^(k-1) t_k is
accumulated as S 2^c = sum (-1)^(k-1) Y_k 2^(c - o_k) in 64-bit slots.
"""
from __future__ import annotations

M32 = (1 << 32) - 1
B = 1 << 32


def mg_reciprocal_3by2(d: int) -> int:
    """v = floor((B^3 - 1) / d) - B for a normalised 64-bit d (MG Alg. 6 result)."""
    assert d >> 63 == 1
    return (B ** 3 - 1) // d - B


def mg_div_3by2(u2, u1, u0, d1, d0, v):
    """Moller-Granlund 2011, Algorithm 5: (q, r1, r0) with q = floor((u2,u1,u0)/(d1,d0)),
    requires (u2,u1) < (d1,d0), d1 >= 2^31.  All arithmetic on 32-bit words."""
    q = v * u2 + ((u2 << 32) | u1)
    q1, q0 = (q >> 32) & M32, q & M32
    r1 = (u1 - q1 * d1) & M32
    t = d0 * q1
    r = (((r1 << 32) | u0) - t - ((d1 << 32) | d0)) & ((1 << 64) - 1)
    r1, r0 = r >> 32, r & M32
    q1 = (q1 + 1) & M32
    if r1 >= q0:
        q1 = (q1 - 1) & M32
        r = (r + ((d1 << 32) | d0)) & ((1 << 64) - 1)
    if r >= ((d1 << 32) | d0):
        q1 += 1
        r -= (d1 << 32) | d0
    return q1, r


def digits(v: int, n: int):
    return [(v >> (32 * i)) & M32 for i in range(n)]


def from_digits(ds) -> int:
    v = 0
    for x in reversed(ds):
        v = (v << 32) | x
    return v


def term_divide(Y, X2, D, n_out):
    """One term: Horner MS->LS over V = Y X2 2^sh with the kernel's digit
    recurrences; returns the quotient digits q_0..q_(n_out-1) (Q < B^n_out)
    and whether the rare 'top >= D~' path was taken."""
    sh = 64 - D.bit_length()
    sd, sb = divmod(sh, 32)
    Dn = D << sh
    d1, d0 = Dn >> 32, Dn & M32
    v = mg_reciprocal_3by2(Dn)
    x0, x1 = X2 & M32, X2 >> 32
    n = len(Y)
    def prod(i):                       # y_i X2 = p0 + p1 B + p2 B^2 (y_i < B, X2 < 2^60)
        y = Y[i] if 0 <= i < n else 0
        a = y * x0
        b = y * x1 + (a >> 32)
        return a & M32, b & M32, b >> 32
    def A(i):                          # non-normalised product digit (< 3B)
        return prod(i)[0] + prod(i - 1)[1] + prod(i - 2)[2]
    def Vdig(i):                       # digit i of V = sum A_j B^j 2^sh: (lo32, carry)
        j = i - sd
        hi = (A(j) << sb) & M32
        lo = A(j - 1) >> (32 - sb)      # sb = 0: the high part of the digit below
        t = hi + lo
        return t & M32, t >> 32
    top = n + 3 + sd                    # V digits at positions >= top are zero
    R = 0                               # remainder, already in the normalised (x 2^sh) frame
    q = [0] * max(n_out, top + 1)
    rare = False
    for i in range(top, -1, -1):
        u0, c = Vdig(i)
        # Horner: digit j's carry c belongs to position i+1, already consumed -> add to R
        T = R + c
        if T >= Dn:                     # quotient digit would be >= B: the rare path
            rare = True
            T -= Dn
            # +1 to the previously emitted digit (position i+1), ripple upward
            j = i + 1
            while True:
                q[j] += 1
                if q[j] < B:
                    break
                q[j] = 0
                j += 1
        qi, R = mg_div_3by2(T >> 32, T & M32, u0, d1, d0, v)
        q[i] = qi
    return q[:n_out], rare


M64 = (1 << 64) - 1
C64 = 1 << 64


def mg_reciprocal_2by1_64(d: int) -> int:
    """v = floor((C^2 - 1) / d) - C for a normalised 64-bit d (MG 2011, 2-by-1)."""
    assert d >> 63 == 1
    return (C64 * C64 - 1) // d - C64


def mg_div_2by1_64(u1, u0, d, v):
    """Moller-Granlund 2011, Algorithm 4 on 64-bit words: (q, r), u1 < d."""
    assert u1 < d
    q = v * u1 + ((u1 << 64) | u0)
    q1, q0 = (q >> 64) & M64, q & M64
    q1 = (q1 + 1) & M64
    r = (u0 - q1 * d) & M64
    if r > q0:
        q1 = (q1 - 1) & M64
        r = (r + d) & M64
    if r >= d:
        q1 += 1
        r -= d
    return q1, r


def term_divide64(Y, X2, D, n_out):
    """The 64-bit-chunk variant (sin_band.cpp, band64): chunks c_m = y_2m +
    y_(2m+1) B, c_m X2 = L_m + H_m C (C = 2^64), A_m = L_m + H_(m-1) (65
    bits, no carry travels), V_m = lo64(A_m << sh) + (A_(m-1) >> (64 - sh))
    (sh = clz64(D), 0..63; carry <= 1 into the position above: Horner, added
    to R), one 2-by-1 step on 64-bit words per chunk.  Returns 32-bit
    quotient digits."""
    sh = 64 - D.bit_length()
    Dn = D << sh
    v = mg_reciprocal_2by1_64(Dn)
    n = len(Y)
    nc = (n + 1) // 2
    def chunk(m):
        if m < 0 or m >= nc:
            return 0
        lo = Y[2 * m] if 2 * m < n else 0
        hi = Y[2 * m + 1] if 2 * m + 1 < n else 0
        return lo | (hi << 32)
    def LH(m):
        pr = chunk(m) * X2
        return pr & M64, pr >> 64
    def A(m):
        return LH(m)[0] + LH(m - 1)[1]          # < 2^64 + 2^60
    def Vc(m):
        t = ((A(m) << sh) & M64) + (A(m - 1) >> (64 - sh))
        assert t >> 64 <= 1
        return t & M64, t >> 64
    top = nc + 2
    R = 0
    q = [0] * (top + 2)
    rare = False
    for m in range(top, -1, -1):
        u0, c = Vc(m)
        T = R + c
        assert T < C64
        if T >= Dn:
            rare = True
            T -= Dn
            j = m + 1
            while True:
                q[j] += 1
                if q[j] < C64:
                    break
                q[j] = 0
                j += 1
        q[m], R = mg_div_2by1_64(T, u0, Dn, v)
    out = []
    for x in q:
        out += [x & M32, x >> 32]
    out += [0] * max(0, n_out - len(out))
    return out[:n_out], rare


def sin_row(m: int, s: int, P: int, c_scale=None, check=True, chunk64=False):
    """sin_P(m 10^-s) per the kernel's plan; returns the integer mantissa at scale P."""
    X2 = m * m
    W = (abs(m) * 10 ** (P - s)).bit_length() // 32 + 3
    Y = digits(abs(m) * 10 ** (P - s), W)
    o = 0
    os_ = sorted({(2 * s * k) % 32 for k in range(64)})
    c = max(os_) if c_scale is None else c_scale
    Sacc = 0                            # S * 2^c
    k = 1
    rare_any = False
    while any(Y):
        Yv = from_digits(Y)
        sign = 1 if k % 2 == 1 else -1
        Sacc += sign * (Yv << (c - o))
        D = 5 ** (2 * s) * (2 * k) * (2 * k + 1)
        assert D < 1 << 64
        q, rare = (term_divide64 if chunk64 else term_divide)(Y, X2, D, len(Y) + 2)
        rare_any |= rare
        if check:
            assert from_digits(q) == (Yv * X2) // D
        o2 = o + 2 * s
        drop = 1 if o2 >= 32 else 0
        o = o2 - 32 * drop
        Ynew = q[drop:]
        Ynew[0] &= ~((1 << o) - 1) & M32
        while len(Ynew) > 1 and Ynew[-1] == 0:
            Ynew.pop()
        Y = Ynew
        if check:
            assert from_digits(Y) == ((from_digits(q) >> o2) << o)
        k += 1
    assert Sacc % (1 << c) == 0
    S = Sacc >> c
    return (-S if m < 0 else S), rare_any


def sin_q13(m: int, s: int, P: int) -> int:
    t, k, S = abs(m) * 10 ** (P - s), 1, 0
    while t:
        S += t if k % 2 else -t
        t = t * m * m // (10 ** (2 * s) * (2 * k) * (2 * k + 1))
        k += 1
    return -S if m < 0 else S


if __name__ == "__main__":
    import random
    rng = random.Random(1)
    for P in (8, 30, 200):
        for s in (0, 2, 8):
            for _ in range(20):
                m = rng.randrange(-(10 ** (s + 1)) + 1, 10 ** (s + 1))
                for c64 in (False, True):
                    got, _ = sin_row(m, s, P, chunk64=c64)
                    assert got == sin_q13(m, s, P), (m, s, P, c64)
    print("model == Q13")
