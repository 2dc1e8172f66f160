"""Pins for the CPU oracle (oracle/updec.c) against things other than itself:
the paper's worked examples (tests/golden/paper_examples.txt), closed forms,
textbook RSA, Python's exact rational/integer arithmetic on small inputs,
invariants (division identity, odd symmetry), and an accuracy bound against
mpmath.  None of these re-call oracle code for the expected value."""
import math
import os
import random
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import Column, OracleError
from gen import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def dec(s: str) -> Fraction:
    return Fraction(s)


def parse_golden(name):
    rows = []
    for line in open(os.path.join(GOLDEN, name)):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        f = [x.strip() for x in line.split("|")]
        if len(f) == 6 and f[0].startswith("T"):      # expression examples (C* rows: tests/test_compact_codec.py)
            rows.append(f)
    return rows


@pytest.mark.parametrize("row", parse_golden("paper_examples.txt"), ids=lambda r: r[0])
def test_paper_examples(row):
    tid, expr, types, values, rtype, result = row
    if types == "-":
        cols = [Column(1, 0, strings=["0"])]  # unused column; literal-only expression
    else:
        cols = [Column(int(t.split(",")[0]), int(t.split(",")[1]), strings=[v])
                for t, v in zip(types.split(";"), values.split(";"))]
    P, S = oracle.expr_type(expr, cols)
    want_p, want_s = map(int, rtype.split(","))
    if tid != "T7":   # T7's DECIMAL(3,2) is the paper's value-based re-typing after folding
        assert (P, S) == (want_p, want_s)
    assert dec(oracle.eval_rows(expr, cols)[0]) == dec(result)


def test_point_one_plus_point_two():
    """0.1 + 0.2 = 0.3 exactly (the binary-float counter-example, §II-A)."""
    c = [Column(2, 1, strings=["0.1"]), Column(2, 1, strings=["0.2"])]
    assert oracle.eval_rows("c1+c2", c) == ["0.3"]
    assert oracle.expr_type("c1+c2", c) == (3, 1)


def test_canonical_format_and_negative_zero():
    c = [Column(5, 3, strings=["-0.000"]), Column(5, 3, strings=["0.5"])]
    assert oracle.eval_rows("c1", c) == ["0.000"]
    assert oracle.eval_rows("c1*c2", c) == ["0.000000"]
    assert oracle.eval_rows("-c2", c) == ["-0.500"]
    assert oracle.eval_rows("c2-c2", c) == ["0.000"]


def test_query5_typing():
    """T10: Query 5 typed by P:L1044-1062: 2 terms -> (32,28), 11 -> (185,172)."""
    def q5(terms):
        e = "c1"
        for k in range(1, terms):
            n = 2 * k + 1
            e += (" - " if k % 2 else " + ") + "*".join(["c1"] * n) + "/" + str(math.factorial(n))
        return e
    x = [Column(9, 8, strings=["0.78000000"])]
    assert oracle.expr_type(q5(2), x) == (32, 28)
    assert oracle.expr_type(q5(11), x) == (185, 172)


def test_typing_rules_by_hand():
    """+/- (max(p1,p2+s1-s2)+1, s1); x (p1+p2, s1+s2); / (p1-p2+s2+5, s1+4); % (p2, 0)."""
    c = [Column(17, 5, strings=["0"]), Column(14, 2, strings=["0"])]
    assert oracle.expr_type("c1+c2", c) == (18, 5)
    assert oracle.expr_type("c2+c1", c) == (18, 5)     # reading Q3 (symmetric)
    c = [Column(35, 5, strings=["0"]), Column(32, 2, strings=["0"])]
    assert oracle.expr_type("c1+c2", c) == (36, 5)
    c = [Column(200, 50, strings=["0"])] * 4
    assert oracle.expr_type("c1*c2", c) == (400, 100)
    assert oracle.expr_type("c3/c4", c) == (55, 54)
    assert oracle.expr_type("c1*c2 - c3/c4", c) == (401, 100)
    c = [Column(17, 0, strings=["0"]), Column(18, 0, strings=["1"])]
    assert oracle.expr_type("c1%c2", c) == (18, 0)
    with pytest.raises(OracleError):
        oracle.expr_type("c1%c2", [Column(5, 1, strings=["0"]), Column(5, 0, strings=["1"])])
    # SUM: p + ceil(log10 N)  (reading Q9)
    assert oracle.sum_type(18, 5, 1_000_000) == (24, 5)
    assert oracle.sum_type(18, 5, 2 ** 30) == (28, 5)
    assert oracle.sum_type(36, 5, 10_000_000) == (43, 5)
    assert oracle.sum_type(36, 5, 1) == (36, 5)
    assert oracle.sum_type(36, 5, 11) == (38, 5)


def test_arithmetic_series_sum_closed_form():
    """SUM over mantissas a + i*d equals N*a + d*N(N-1)/2 (closed form)."""
    N, a, d = 20000, -123456789012345, 987654321
    mag, neg = synth.series(N, a, d, 2)
    col = Column(17, 5, mag, neg)
    got, P, S = oracle.eval_sum("c1", [col], threads=4)
    want = N * a + d * N * (N - 1) // 2
    assert dec(got) == Fraction(want, 10 ** 5)
    assert (P, S) == (17 + 5, 5)


def test_sum_of_two_series_columns_with_alignment():
    N = 5000
    m1, n1 = synth.series(N, -10 ** 16 + 7, 3 * 10 ** 12, 2)
    m2, n2 = synth.series(N, 10 ** 13 - 1, -2 * 10 ** 9 - 1, 2)
    cols = [Column(17, 5, m1, n1), Column(14, 2, m2, n2)]
    got, P, S = oracle.eval_sum("c1+c2", cols, threads=3)
    s1 = N * (-10 ** 16 + 7) + 3 * 10 ** 12 * N * (N - 1) // 2
    s2 = N * (10 ** 13 - 1) + (-2 * 10 ** 9 - 1) * N * (N - 1) // 2
    assert dec(got) == Fraction(s1, 10 ** 5) + Fraction(s2, 10 ** 2)


# ---------------------------------------------------------------------------
# brute force with Python's exact rationals (an independent evaluator)
# ---------------------------------------------------------------------------
def _tokenize(e):
    toks, i = [], 0
    while i < len(e):
        ch = e[i]
        if ch == " ":
            i += 1
        elif ch in "+-*/%()":
            toks.append(ch); i += 1
        elif ch == "c":
            j = i + 1
            while j < len(e) and e[j].isdigit():
                j += 1
            toks.append(e[i:j]); i = j
        else:
            j = i
            while j < len(e) and (e[j].isdigit() or e[j] == "."):
                j += 1
            toks.append(e[i:j]); i = j
    return toks


def brute_eval(expr, types, values):
    """Exact rational evaluation; division truncates toward zero at scale s1+4
    (P:L1049-1058), % is the truncated remainder.  Returns
    (value, scale) with the scale computed from the paper's rules."""
    toks = _tokenize(expr)
    pos = [0]

    def peek():
        return toks[pos[0]] if pos[0] < len(toks) else None

    def take():
        t = toks[pos[0]]; pos[0] += 1; return t

    def primary():
        t = take()
        if t == "(":
            v = add(); take(); return v
        if t == "-":
            v, s = primary_unary_after_minus()
            return v, s
        if t.startswith("c"):
            k = int(t[1:]) - 1
            return Fraction(values[k]), types[k][1]
        frac = t.split(".")[1] if "." in t else ""
        return Fraction(t), len(frac)

    def primary_unary_after_minus():
        v, s = primary()
        return -v, s

    def mul():
        v, s = primary()
        while peek() in ("*", "/", "%"):
            op = take()
            w, s2 = primary()
            if op == "*":
                v, s = v * w, s + s2
            elif op == "/":
                q = v / w
                scale = 10 ** (s + 4)
                mant = abs(q.numerator * scale) // q.denominator   # trunc toward zero
                v, s = Fraction(mant if q >= 0 else -mant, scale), s + 4
            else:
                a, b = int(v), int(w)
                r = abs(a) % abs(b)
                v, s = Fraction(r if a >= 0 else -r), 0
        return v, s

    def add():
        v, s = mul()
        while peek() in ("+", "-"):
            op = take()
            w, s2 = mul()
            v, s = (v + w if op == "+" else v - w), max(s, s2)
        return v, s

    return add()


def _rand_value(rng, p, s, edge=False):
    if edge:
        m = rng.choice([0, 1, 10 ** p - 1, 10 ** (p - 1), 2 ** min(32, int(p * 3.3)) - 1,
                        (10 ** p - 1) // 2])
        m = min(m, 10 ** p - 1)
    else:
        m = rng.randrange(10 ** rng.randint(1, p))
    if rng.random() < 0.5:
        m = -m
    return _fmt(m, s)


def _fmt(m, s):
    sign = "-" if m < 0 else ""
    a = str(abs(m)).rjust(s + 1, "0")
    return sign + (a if s == 0 else a[:-s] + "." + a[-s:])


EXPRS = ["c1+c2", "c1-c2", "c2-c1", "c1*c2", "c1/c2", "-c1+c2*c1", "(c1+c2)*(c1-c2)",
         "c1*c2-c3/c4", "c1/c2/c3", "c1+c2+c3+c4", "c1*1.5+0.25", "c3-c1*c2*c4",
         "c1/(c2+c3)", "-(c1/c4)"]


@pytest.mark.parametrize("expr", EXPRS)
def test_brute_force_expressions(expr):
    rng = random.Random(hash(expr) & 0xFFFF)
    for trial in range(60):
        types = []
        for k in range(4):
            p = rng.randint(1, 40)
            s = rng.randint(0, p)
            types.append((p, s))
        vals = [_rand_value(rng, p, s, edge=(trial % 5 == 0)) for p, s in types]
        cols = [Column(p, s, strings=[v]) for (p, s), v in zip(types, vals)]
        try:
            got = oracle.eval_rows(expr, cols)[0]
        except OracleError as e:
            # only division/modulo may fail: divide by zero, or the Q5 overflow
            assert e.name in ("DIVZERO", "OVERFLOW")
            if e.name == "OVERFLOW":
                P, S = oracle.expr_type(expr, cols)
                assert "/" in expr
            else:
                assert any(Fraction(v) == 0 for v in vals[1:]) or "/" in expr
            continue
        want, ws = brute_eval(expr, types, vals)
        assert dec(got) == want, (expr, types, vals, got, want)
        P, S = oracle.expr_type(expr, cols)
        assert S == ws
        assert len(got.split(".")[1]) == S if S else "." not in got


@pytest.mark.parametrize("terms", [2, 3, 5, 8, 11])
def test_query5_literal_brute_force(terms):
    """Paper-literal Query 5 (the SQL Taylor polynomial of sin
    with 2..11 terms over DECIMAL(9,8) x): the oracle's rows equal the exact
    rational evaluation with the paper's per-division truncation (brute_eval),
    and every row lies within the truncation budget of the exact polynomial
    sum_k (-1)^k x^(2k+1)/(2k+1)!: term k's division truncates at scale
    8(2k+1)+4, so |row - poly| < sum_k 10^-(8(2k+1)+4); with 11
    terms the polynomial is within x^23/23! (+ float rounding) of sin x."""
    rng = random.Random(terms)
    xs = []
    for mu in (0.01, 0.78, 1.56):
        mag, neg = synth.normal_decimal(12, mu, 0.01, 8, config=5, column=3)
        xs += [(-int(m[0]) if g else int(m[0])) for m, g in zip(mag, neg)]
    xs += [0, 1, -1, 10 ** 9 - 1, -(10 ** 9 - 1), rng.randrange(10 ** 9)]
    vals = [_fmt(m, 8) for m in xs]
    e = "c1"
    for k in range(1, terms):
        n = 2 * k + 1
        e += (" - " if k % 2 else " + ") + "*".join(["c1"] * n) + "/" + str(math.factorial(n))
    col = Column(9, 8, strings=vals)
    got = oracle.eval_rows(e, [col])
    P, S = oracle.expr_type(e, [col])
    for v, g in zip(vals, got):
        want, ws = brute_eval(e, [(9, 8)], [v])
        assert ws == S and dec(g) == want, (terms, v, g, want)
        x = Fraction(v)
        poly = sum(Fraction((-1) ** k) * x ** (2 * k + 1) / math.factorial(2 * k + 1) for k in range(terms))
        assert abs(dec(g) - poly) < sum(Fraction(1, 10 ** (8 * (2 * k + 1) + 4)) for k in range(1, terms))
        if terms == 11:
            assert abs(poly - Fraction(math.sin(float(x)))) <= abs(x) ** 23 / math.factorial(23) + Fraction(1, 10 ** 15)


def test_modulo_brute_force():
    rng = random.Random(7)
    for _ in range(300):
        p1, p2 = rng.randint(1, 60), rng.randint(1, 60)
        a = rng.randrange(10 ** p1) * rng.choice([1, -1])
        b = rng.randrange(1, 10 ** p2) * rng.choice([1, -1])
        cols = [Column(p1, 0, strings=[str(a)]), Column(p2, 0, strings=[str(b)])]
        r = abs(a) % abs(b)
        want = r if a >= 0 else -r
        assert int(oracle.eval_rows("c1%c2", cols)[0]) == want
        assert oracle.expr_type("c1%c2", cols) == (p2, 0)


def test_division_identity_and_paths():
    """Q*|B| <= |A|*10^(s2+4) < (Q+1)*|B|, for 1-digit, 1-word and multi-word divisors."""
    rng = random.Random(11)
    for _ in range(400):
        p1, s1 = rng.randint(1, 80), 0
        p2 = rng.choice([1, 2, 9, 10, 19, 20, 40, 80])
        s2 = rng.randint(0, min(p2, 6))
        s1 = rng.randint(0, min(p1, 6))
        a = rng.randrange(10 ** p1)
        b = rng.randrange(max(1, 10 ** (p2 - 1)), 10 ** p2)
        cols = [Column(p1, s1, strings=[_fmt(a, s1)]), Column(p2, s2, strings=[_fmt(b, s2)])]
        try:
            q = oracle.eval_rows("c1/c2", cols)[0]
        except OracleError as e:
            assert e.name == "OVERFLOW"
            continue
        Q = int(q.replace(".", ""))
        A = a * 10 ** (s2 + 4)
        assert Q * b <= A < (Q + 1) * b


def test_division_by_zero_and_overflow_flags():
    cols = [Column(5, 0, strings=["7"]), Column(5, 0, strings=["0"])]
    with pytest.raises(OracleError) as ei:
        oracle.eval_rows("c1/c2", cols)
    assert ei.value.name == "DIVZERO"
    with pytest.raises(OracleError) as ei:
        oracle.eval_rows("c1%c2", cols)
    assert ei.value.name == "DIVZERO"
    # reading Q5: (4,2)/(4,1) typed (6,6) but 1.23/1.1 = 1.118181 needs 7 digits
    cols = [Column(4, 2, strings=["1.23"]), Column(4, 1, strings=["1.1"])]
    with pytest.raises(OracleError) as ei:
        oracle.eval_rows("c1/c2", cols)
    assert ei.value.name == "OVERFLOW"
    cols = [Column(4, 2, strings=["1.23"]), Column(4, 1, strings=["100.1"])]
    assert oracle.eval_rows("c1/c2", cols) == ["0.012287"]   # 1.23/100.1 = 0.0122877...


def test_range_rejection():
    with pytest.raises(OracleError) as ei:
        oracle.eval_rows("c1", [Column(3, 1, strings=["100.0"])])
    assert ei.value.name == "RANGE"
    with pytest.raises(OracleError):
        oracle.eval_rows("c1", [Column(5, 1, strings=["1.25"])])


def test_full_carry_ripple():
    """(10^p - 1)^2 = 10^(2p) - 2*10^p + 1 and 0xFF..F word patterns."""
    for p in (9, 18, 19, 38, 77, 154, 308):
        v = str(10 ** p - 1)
        cols = [Column(p, 0, strings=[v]), Column(p, 0, strings=["-" + v])]
        assert int(oracle.eval_rows("c1*c2", cols)[0]) == -(10 ** (2 * p) - 2 * 10 ** p + 1)
        assert int(oracle.eval_rows("c1-c2", cols)[0]) == 2 * (10 ** p - 1)
    for w in (1, 2, 3, 5, 8):
        v = 2 ** (32 * w) - 1
        p = len(str(v))
        cols = [Column(p, 0, strings=[str(v)]), Column(p, 0, strings=["1"])]
        assert int(oracle.eval_rows("c1+c2", cols)[0]) == v + 1
        cols = [Column(p, 0, strings=[str(v + 1 - 1)]), Column(p, 0, strings=[str(v)])]
        assert int(oracle.eval_rows("c1/c2", cols)[0].replace(".", "")) == 10 ** 4


def test_binary_column_input_matches_string_input():
    mag, neg = synth.uniform_decimal(64, 35, config=2, column=1)
    col = Column(35, 5, mag, neg)
    ints = synth.to_ints(mag, neg)
    strs = [_fmt(v, 5) for v in ints]
    assert oracle.eval_rows("c1", [col]) == [oracle.eval_rows("c1", [Column(35, 5, strings=[s])])[0] for s in strs]
    assert [dec(x) for x in oracle.eval_rows("c1", [col])] == [Fraction(v, 10 ** 5) for v in ints]


def test_sum_threads_and_shard_combine():
    """Sum of k shard sums = whole-column sum; thread count does not matter."""
    n = 3000
    m1, n1 = synth.uniform_decimal(n, 35, 2, 1)
    m2, n2 = synth.uniform_decimal(n, 32, 2, 2)
    cols = [Column(35, 5, m1, n1), Column(32, 2, m2, n2)]
    whole, P, S = oracle.eval_sum("c1+c2", cols, threads=1)
    assert oracle.eval_sum("c1+c2", cols, threads=7)[0] == whole
    ints1, ints2 = synth.to_ints(m1, n1), synth.to_ints(m2, n2)
    assert dec(whole) == sum(Fraction(a, 10 ** 5) + Fraction(b, 10 ** 2) for a, b in zip(ints1, ints2))
    parts = []
    for r in range(4):
        lo, hi = n * r // 4, n * (r + 1) // 4
        sh = [Column(35, 5, m1[lo:hi], n1[lo:hi]), Column(32, 2, m2[lo:hi], n2[lo:hi])]
        parts.append(oracle.eval_sum("c1+c2", sh, n_global=n)[0])
    assert oracle.add_strings(parts, P, S) == whole


# ---------------------------------------------------------------------------
# modexp (Query 4)
# ---------------------------------------------------------------------------
def test_textbook_rsa():
    """n = 61*53 = 3233, e = 17, m = 65 -> c = 2790; d = 2753 decrypts to 65."""
    c = oracle.modexp_rows(Column(4, 0, strings=["65"]), 17, 3233)
    assert c == ["2790"]
    assert oracle.modexp_rows(Column(4, 0, strings=["2790"]), 2753, 3233) == ["65"]


def test_modexp_matches_python_pow_and_round_trip():
    N, p, q = synth.rsa_modulus(256)
    e = 65537
    d = pow(e, -1, (p - 1) * (q - 1))
    mag, neg = synth.rsa_messages(40, N)
    col = Column(len(str(N)), 0, mag, neg)
    ms = synth.to_ints(mag, neg)
    cs = oracle.modexp_rows(col, e, N)
    assert [int(x) for x in cs] == [pow(m, e, N) for m in ms]
    back = oracle.modexp_rows(Column(len(str(N)), 0, strings=cs), d, N)
    assert [int(x) for x in back] == ms
    assert oracle.modexp_rows(col, 3, N) == [str(pow(m, 3, N)) for m in ms]


def test_modexp_fermat_and_edge_cases():
    q = 1000000007
    for a in (2, 3, 12345, q - 1):
        assert oracle.modexp_rows(Column(10, 0, strings=[str(a)]), q - 1, q) == ["1"]
    assert oracle.modexp_rows(Column(10, 0, strings=["0"]), 3, 97) == ["0"]
    assert oracle.modexp_rows(Column(10, 0, strings=["500"]), 3, 97) == [str(pow(500, 3, 97))]  # x >= N
    assert oracle.modexp_rows(Column(10, 0, strings=["5"]), 0, 97) == ["1"]


# ---------------------------------------------------------------------------
# sin_P
# ---------------------------------------------------------------------------
def test_sin_zero_and_odd_symmetry():
    assert oracle.sin_rows(Column(9, 8, strings=["0"]), 50) == ["0." + "0" * 50]
    for x in ("0.01000000", "0.78123456", "1.56999999", "3.14159265"):
        a = oracle.sin_rows(Column(9, 8, strings=[x]), 120)[0]
        b = oracle.sin_rows(Column(9, 8, strings=["-" + x]), 120)[0]
        assert b == "-" + a


@pytest.mark.parametrize("P", [30, 100, 500])
def test_sin_accuracy_bound_vs_mpmath(P):
    """|sin_P(x) - sin(x)| <= (K+1) 10^-P with K the number of terms (truncation
    error <= 1 ulp per term plus the Taylor remainder < 1 ulp)."""
    import mpmath
    mpmath.mp.dps = P + 60
    mag, neg = synth.normal_decimal(12, 0.78, 0.01, 8, config=5, column=0)
    col = Column(9, 8, mag, neg)
    got = oracle.sin_rows(col, P)
    for g, m in zip(got, synth.to_ints(mag, neg)):
        x = mpmath.mpf(m) / 10 ** 8
        err = abs(mpmath.mpf(g) - mpmath.sin(x))
        K = 0
        t, k = abs(m) * 10 ** (P - 8), 1
        while t:                         # count terms only (bound, not the value)
            K += 1
            t = t * m * m // (10 ** 16 * (2 * k) * (2 * k + 1)); k += 1
        assert err <= (K + 1) * mpmath.mpf(10) ** (-P), (P, g)


def test_sin_small_P_matches_decimal_context():
    """For tiny P the recurrence must agree with sin computed by Python's decimal
    module (exact Taylor to 60 digits) within the (K+1) ulp bound and be within
    1 ulp of a direct truncated evaluation for x = 0.5."""
    import decimal
    decimal.getcontext().prec = 80
    x = decimal.Decimal("0.5")
    s, t, k = decimal.Decimal(0), x, 1
    while abs(t) > decimal.Decimal(10) ** -75:
        s += t
        t = -t * x * x / ((2 * k) * (2 * k + 1)); k += 1
    got = decimal.Decimal(oracle.sin_rows(Column(9, 8, strings=["0.50000000"]), 20)[0])
    assert abs(got - s) <= decimal.Decimal(10) ** -20 * 12


def _sin_q13_python(m: int, s: int, P: int) -> str:
    """Reading Q13 written out with Python ints, term by
    term in the order the definition states: t_1 = |m| 10^(P-s),
    t_(k+1) = floor(t_k m^2 / (10^(2s) (2k)(2k+1))), stop at t = 0,
    S = sum (-1)^(k-1) t_k, result sign(m) S at scale P.  Independent of
    oracle/updec.c (base-10^9 C); the canonical string has exactly P fraction
    digits and no "-0"."""
    t, k, S = abs(m) * 10 ** (P - s), 1, 0
    while t:
        S += t if k % 2 == 1 else -t
        t = t * m * m // (10 ** (2 * s) * (2 * k) * (2 * k + 1))
        k += 1
    v = -S if m < 0 else S
    sign = "-" if v < 0 else ""
    a = str(abs(v)).rjust(P + 1, "0")
    return sign + a[:-P] + "." + a[-P:]


@pytest.mark.parametrize("P", [8, 57, 300, 1000])
@pytest.mark.parametrize("mu", [0.01, 0.78, 1.56])
@pytest.mark.parametrize("s", [0, 2, 8])
def test_sin_bits_match_q13_python_int_brute_force(P, mu, s):
    """Pins the BITS of oracle.sin_rows (the accuracy tests above pin only the
    value to within (K+1) ulps): a floor->round or floor->ceil slip, a dropped
    term or a wrong sign in the recurrence fails here.  Query 5's inputs are
    x ~ N(mu, 0.01^2) with mu in {0.01, 0.78, 1.56} (§IV, reading
    Q14), here rounded to scale s in {0, 2, 8} (p = s + 1 digits, |x| < 10)."""
    n = 25
    mag, neg = synth.normal_decimal(n, mu, 0.01, s, config=5, column=7)
    col = Column(s + 1, s, mag, neg)
    got = oracle.sin_rows(col, P)
    want = [_sin_q13_python(m, s, P) for m in synth.to_ints(mag, neg)]
    assert got == want


def test_sin_bits_q13_edge_values():
    """Boundary mantissas: zero, one ulp, the largest DECIMAL(9,8) magnitude
    (|x| just below 10), and negative values."""
    vals = ["0", "0.00000001", "-0.00000001", "9.99999999", "-9.99999999", "3.14159265", "-1.57079633"]
    ms = [int(v.replace(".", "")) for v in vals]
    for P in (8, 40, 333):
        got = oracle.sin_rows(Column(9, 8, strings=vals), P)
        assert got == [_sin_q13_python(m, 8, P) for m in ms], P
