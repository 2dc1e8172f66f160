"""Word-level model of the top-limb division decision (up_dev.cuh
div_top_decide): q0 = floor(ah C / vh) by Moller-Granlund 3-by-2 steps on the
normalised window (reciprocal from Alg. 6, dividend shifted on the fly, one
add-back at most), then the exactness test q0 <= R, R + C < vh.  The model
asserts q0 and R against Python's // and % wherever it decides; it checks
the kernel's arithmetic plan, not the kernel (tests/test_gpu_divtop.py does).

    python tools/divtop_model.py        # 20000 random windows
"""
import random
B = 1 << 32
M = B - 1

def recip_word(d1):
    """floor((2^64 - 1) / d1) - 2^32 the way the kernel computes it: the
    correctly rounded double reciprocal (Python's 1.0 / d1, as __drcp_rn),
    scaled by 2^64, truncated, then an exact integer fix-up"""
    q = int((1.0 / d1) * 2.0 ** 64)
    p = q * d1
    top = (1 << 64) - 1
    if p > top: q -= 1; p -= d1
    if p > top: q -= 1; p -= d1
    if top - p >= d1: q += 1
    assert q == top // d1
    return q - B

def recip_3by2(d1, d0):
    v = recip_word(d1)
    p = (d1 * v) % B
    p = (p + d0) % B
    if p < d0:
        v -= 1
        if p >= d1:
            v -= 1; p -= d1
        p = (p - d1) % B
    t = v * d0; t1, t0 = t >> 32, t & M
    p = (p + t1) % B
    if p < t1:
        v -= 1
        if (p, t0) >= (d1, d0):
            v -= 1
    return v % B

def div3by2(u2, u1, u0, d1, d0, v):
    q = v * u2 + ((u2 << 32) | u1)
    q1, q0 = (q >> 32) % B, q & M
    r1 = (u1 - q1 * d1) % B
    dd = (d1 << 32) | d0
    r = (((r1 << 32) | u0) - d0 * q1 - dd) % (1 << 64)
    q1 = (q1 + 1) % B
    if (r >> 32) >= q0:
        q1 = (q1 - 1) % B; r = (r + dd) % (1 << 64)
    if r >= dd:
        q1 += 1; r -= dd
    return q1, r >> 32, r & M

def limbs(x, n): return [(x >> (32 * i)) & M for i in range(n)]
def val(l): return sum(w << (32 * i) for i, w in enumerate(l))

def decide(ah, vh, c, NQ):
    NAH, T, NC = len(ah), len(vh), len(c)
    if vh[T - 1] == 0: return None
    NU = NAH + NC
    uh = limbs(val(ah) * val(c), NU)
    sh = 32 - vh[T - 1].bit_length()
    vn = limbs(val(vh) << sh, T)
    NN = NU + 1
    un = limbs(val(uh) << sh, NN)
    R = [un[NQ + i] if NQ + i < NN else 0 for i in range(T)]
    if any(un[k] for k in range(NQ + T, NN)) or not val(R) < val(vn):
        return None
    d1, d0 = vn[T - 1], vn[T - 2]
    v = recip_3by2(d1, d0)
    q = [0] * NQ
    for j in range(NQ - 1, -1, -1):
        if R[T - 1] == d1 and R[T - 2] == d0:
            return None
        qh, r1, r0 = div3by2(R[T - 1], R[T - 2], R[T - 3] if T >= 3 else un[j], d1, d0, v)
        src = ([un[j]] + R[:T - 3])[:T - 2]
        nr = [0] * T
        cy, br = 0, 0
        for i in range(T - 2):
            p = qh * vn[i] + cy; cy = p >> 32
            d = src[i] - (p & M) - br
            nr[i] = d % B; br = 1 if d < 0 else 0
        top = (r1 << 32) | r0
        s = cy + br
        t = (top - s) % (1 << 64)
        nr[T - 2], nr[T - 1] = t & M, t >> 32
        if top < s:
            qh -= 1
            x = val(nr) + val(vn)
            nr = limbs(x, T)
        R = nr
        q[j] = qh
    Rt = val(R) >> sh
    Q = val(q)
    assert Q == val(uh) // val(vh) and Rt == val(uh) % val(vh), "mismatch"
    return Q, (Q <= Rt) and (Rt + val(c) < val(vh))

def run(iters=20000, seed=1):
  rng = random.Random(seed)
  n = 0
  for it in range(iters):
      T = rng.choice([2, 3, 4, 7, 8])
      NC = rng.randrange(1, T)
      NQ = rng.randrange(1, T + 1)
      NAH = rng.choice([T - 1, T, T + 1])
      ah = [rng.getrandbits(32) for _ in range(NAH)]
      vh = [rng.getrandbits(32) for _ in range(T)]
      mode = rng.random()
      if mode < 0.1: vh[T - 1] = rng.getrandbits(rng.randrange(1, 33)) or 1
      if mode > 0.9: vh = [M] * T
      if 0.5 < mode < 0.55: ah = [M] * NAH
      if 0.55 < mode < 0.6: vh[T - 1] = 1 << 31; vh[:T - 1] = [0] * (T - 1)
      c = [rng.getrandbits(32) for _ in range(NC)]
      if rng.random() < 0.3: c = limbs(10 ** rng.randrange(1, 32 * NC * 3 // 10 + 1), NC)
      r = decide(ah, vh, c, NQ)
      if r is not None: n += 1
  return n


if __name__ == "__main__":
    print("ok", run())
