/*
 * oracle/updec.c -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.
 *
 * A plain, slow, obviously-correct CPU implementation of the DECIMAL(p,s)
 * semantics of UltraPrecise (Li et al., ICDE 2024, /root/reference/PAPER.md,
 * cited below as "P:L<line> §<section>").  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_icde_lixylz24_b200/csrc); neither includes the other.
 *
 * Representation (independent of the GPU's two's-complement binary limbs):
 *   sign-magnitude, magnitude in base 10^9 digits, little-endian, no leading
 *   zero digits; zero is always non-negative.
 * Every operation is the schoolbook definition:
 *   +/-   P:L530-574 §II-B (align to the larger scale by x10^k, signed add)
 *   *     P:L576-594 §II-B (elementary-school product)
 *   /     P:L609-656 §II-B, §III-B3: Q = trunc(|A|*10^(s2+4)/|B|)
 *         (reading Q4: truncation toward zero), computed by Knuth long
 *         division in base 10^9 (the paper's binary search finds the same
 *         floor quotient).
 *   %     P:L1063-1067 §III-B3: integer operands only, type (p2,0),
 *         truncated remainder with the dividend's sign (reading Q7).
 *   SUM   P:L1069-1080 §III-B3: type (p + ceil(log10 N), s) (reading Q9).
 *   modexp  P:L2124-2154 §IV (Query 4, X^e mod N), square-and-multiply with
 *         a % after every product.
 *   sin_P   SURVEY §8c-Q13 (fixed-point truncated Taylor recurrence for the
 *         trig workload of P:L2197-2249 §IV).
 * Typing rules: §III-B3 plus readings Q3 (symmetric +/-),
 * Q5 (division overflow flagged), literal typing P:L1302-1305 §III-D2.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>
#include <ctype.h>
#include <pthread.h>
#include <time.h>

#define BASE 1000000000u

/* status codes: identical numeric values to the product's up_status, but
 * defined here independently (the oracle includes no product header). */
enum { O_OK = 0, O_E_INVAL = 1, O_E_RANGE = 2, O_E_OVERFLOW = 3,
       O_E_DIVZERO = 4, O_E_NOMEM = 5 };

/* ------------------------------------------------------------------ */
/* base-10^9 sign-magnitude big integer                                */
/* ------------------------------------------------------------------ */
typedef struct { int neg; int n; uint32_t *d; } obig;   /* value = (-1)^neg * sum d[i]*B^i */

static obig big_zero(void) { obig r = {0, 0, NULL}; return r; }
static void big_free(obig *a) { free(a->d); a->d = NULL; a->n = 0; a->neg = 0; }
static uint32_t *dalloc(int n) { return (uint32_t *)calloc((size_t)(n > 0 ? n : 1), sizeof(uint32_t)); }
static void big_trim(obig *a) {
    while (a->n > 0 && a->d[a->n - 1] == 0) a->n--;
    if (a->n == 0) a->neg = 0;                 /* no negative zero (Q10) */
}
static obig big_copy(const obig *a) {
    obig r; r.neg = a->neg; r.n = a->n; r.d = dalloc(a->n);
    if (a->n) memcpy(r.d, a->d, sizeof(uint32_t) * (size_t)a->n);
    return r;
}
static obig big_from_u64(uint64_t v) {
    obig r; r.neg = 0; r.d = dalloc(3); r.n = 0;
    while (v) { r.d[r.n++] = (uint32_t)(v % BASE); v /= BASE; }
    return r;
}
/* |a| vs |b| : -1, 0, 1 ; compares from the most significant digit */
static int mag_cmp(const obig *a, const obig *b) {
    if (a->n != b->n) return a->n < b->n ? -1 : 1;
    for (int i = a->n - 1; i >= 0; i--)
        if (a->d[i] != b->d[i]) return a->d[i] < b->d[i] ? -1 : 1;
    return 0;
}
/* |a| + |b| : least- to most-significant digit with carry */
static obig mag_add(const obig *a, const obig *b) {
    int n = (a->n > b->n ? a->n : b->n) + 1;
    obig r; r.neg = 0; r.d = dalloc(n); r.n = n;
    uint32_t carry = 0;
    for (int i = 0; i < n; i++) {
        uint64_t t = (uint64_t)carry + (i < a->n ? a->d[i] : 0) + (i < b->n ? b->d[i] : 0);
        r.d[i] = (uint32_t)(t % BASE); carry = (uint32_t)(t / BASE);
    }
    big_trim(&r); return r;
}
/* |a| - |b| with |a| >= |b| */
static obig mag_sub(const obig *a, const obig *b) {
    obig r; r.neg = 0; r.d = dalloc(a->n); r.n = a->n;
    int64_t borrow = 0;
    for (int i = 0; i < a->n; i++) {
        int64_t t = (int64_t)a->d[i] - (i < b->n ? b->d[i] : 0) - borrow;
        if (t < 0) { t += BASE; borrow = 1; } else borrow = 0;
        r.d[i] = (uint32_t)t;
    }
    big_trim(&r); return r;
}
/* signed add: the signs choose add vs subtract; magnitudes are compared to
 * pick the minuend (§II-B) */
static obig big_add(const obig *a, const obig *b) {
    obig r;
    if (a->neg == b->neg) { r = mag_add(a, b); r.neg = a->neg; }
    else {
        int c = mag_cmp(a, b);
        if (c >= 0) { r = mag_sub(a, b); r.neg = a->neg; }
        else        { r = mag_sub(b, a); r.neg = b->neg; }
    }
    big_trim(&r); return r;
}
static obig big_neg(const obig *a) { obig r = big_copy(a); r.neg = !a->neg; big_trim(&r); return r; }
static obig big_sub(const obig *a, const obig *b) { obig nb = big_neg(b); obig r = big_add(a, &nb); big_free(&nb); return r; }
/* schoolbook product: word k collects all a_i*b_j with i+j = k */
static obig big_mul(const obig *a, const obig *b) {
    if (a->n == 0 || b->n == 0) return big_zero();
    int n = a->n + b->n;
    obig r; r.neg = a->neg ^ b->neg; r.d = dalloc(n); r.n = n;
    for (int i = 0; i < a->n; i++) {
        uint64_t carry = 0;
        for (int j = 0; j < b->n; j++) {
            uint64_t t = (uint64_t)a->d[i] * b->d[j] + r.d[i + j] + carry;
            r.d[i + j] = (uint32_t)(t % BASE); carry = t / BASE;
        }
        int k = i + b->n;
        while (carry) { uint64_t t = r.d[k] + carry; r.d[k] = (uint32_t)(t % BASE); carry = t / BASE; k++; }
    }
    big_trim(&r); return r;
}
static obig mag_mul_small(const obig *a, uint32_t m) {   /* |a| * m, m < B */
    obig r; r.neg = 0; r.d = dalloc(a->n + 1); r.n = a->n + 1;
    uint64_t carry = 0;
    for (int i = 0; i < a->n; i++) { uint64_t t = (uint64_t)a->d[i] * m + carry; r.d[i] = (uint32_t)(t % BASE); carry = t / BASE; }
    r.d[a->n] = (uint32_t)carry;
    big_trim(&r); return r;
}
/* |a| / m, m < B, most- to least-significant digit */
static obig mag_div_small(const obig *a, uint32_t m, uint32_t *rem) {
    obig q; q.neg = 0; q.d = dalloc(a->n); q.n = a->n;
    uint64_t r = 0;
    for (int i = a->n - 1; i >= 0; i--) { uint64_t t = r * BASE + a->d[i]; q.d[i] = (uint32_t)(t / m); r = t % m; }
    if (rem) *rem = (uint32_t)r;
    big_trim(&q); return q;
}
/* Magnitude long division |u| = q*|v| + r, 0 <= r < |v|, v != 0.
 * Knuth, TAOCP vol.2 4.3.1 Algorithm D, in base 10^9. */
static void mag_divmod(const obig *u, const obig *v, obig *q, obig *r) {
    if (mag_cmp(u, v) < 0) { *q = big_zero(); *r = big_copy(u); r->neg = 0; return; }
    if (v->n == 1) {
        uint32_t rr; *q = mag_div_small(u, v->d[0], &rr);
        *r = big_from_u64(rr); return;
    }
    int n = v->n, m = u->n - v->n;
    uint32_t f = BASE / (v->d[n - 1] + 1);               /* D1 normalise */
    obig un = mag_mul_small(u, f), vn = mag_mul_small(v, f);
    uint32_t *U = dalloc(m + n + 1);
    memcpy(U, un.d, sizeof(uint32_t) * (size_t)un.n);
    uint32_t *V = vn.d;                                  /* vn.n == n, V[n-1] >= B/2 */
    obig Q; Q.neg = 0; Q.d = dalloc(m + 1); Q.n = m + 1;
    for (int j = m; j >= 0; j--) {                        /* D2..D7 */
        uint64_t num = (uint64_t)U[j + n] * BASE + U[j + n - 1];
        uint64_t qhat = num / V[n - 1], rhat = num % V[n - 1];
        while (qhat >= BASE || qhat * V[n - 2] > rhat * BASE + U[j + n - 2]) {
            qhat--; rhat += V[n - 1];
            if (rhat >= BASE) break;
        }
        int64_t borrow = 0; uint64_t carry = 0;           /* D4 multiply and subtract */
        for (int i = 0; i < n; i++) {
            uint64_t p = qhat * V[i] + carry;
            carry = p / BASE;
            int64_t t = (int64_t)U[i + j] - (int64_t)(p % BASE) - borrow;
            if (t < 0) { t += BASE; borrow = 1; } else borrow = 0;
            U[i + j] = (uint32_t)t;
        }
        int64_t t = (int64_t)U[j + n] - (int64_t)carry - borrow;
        if (t < 0) {                                      /* D6 add back */
            U[j + n] = (uint32_t)(t + BASE);
            qhat--;
            uint32_t c = 0;
            for (int i = 0; i < n; i++) {
                uint64_t s = (uint64_t)U[i + j] + V[i] + c;
                U[i + j] = (uint32_t)(s % BASE); c = (uint32_t)(s / BASE);
            }
            U[j + n] = (uint32_t)(((uint64_t)U[j + n] + c) % BASE);
        } else U[j + n] = (uint32_t)t;
        Q.d[j] = (uint32_t)qhat;
    }
    big_trim(&Q);
    obig R; R.neg = 0; R.n = n; R.d = U; big_trim(&R);  /* D8 unnormalise */
    uint32_t dummy; *r = mag_div_small(&R, f, &dummy);
    *q = Q;
    big_free(&R); big_free(&un); big_free(&vn);
}
static obig big_pow10(int k) {
    obig r; r.neg = 0; r.n = k / 9 + 1; r.d = dalloc(r.n);
    uint32_t v = 1; for (int i = 0; i < k % 9; i++) v *= 10;
    r.d[k / 9] = v; return r;
}
/* x * 10^k, k >= 0: the upward alignment of P:L540-553 */
static obig big_scale_up(const obig *a, int k) {
    obig t = big_pow10(k); obig r = big_mul(a, &t); big_free(&t); return r;
}
static int big_is_zero(const obig *a) { return a->n == 0; }
/* |a| < 10^p ? (the DECIMAL(p,s) range, Eq.1 P:L443 with reading Q2) */
static int big_fits(const obig *a, int p) {
    obig t = big_pow10(p); int ok = mag_cmp(a, &t) < 0; big_free(&t); return ok;
}
/* binary magnitude words (little-endian uint32) -> base 10^9 (Horner). */
static obig big_from_words(const uint32_t *w, int nw, int neg) {
    obig acc = big_zero();
    for (int j = nw - 1; j >= 0; j--) {
        obig t1 = mag_mul_small(&acc, 65536u); obig t2 = mag_mul_small(&t1, 65536u);
        obig add = big_from_u64(w[j]); obig t3 = mag_add(&t2, &add);
        big_free(&acc); big_free(&t1); big_free(&t2); big_free(&add); acc = t3;
    }
    acc.neg = neg; big_trim(&acc); return acc;
}
/* parse an unsigned decimal integer string of digits */
static obig big_from_digits(const char *s, int len) {
    obig r; r.neg = 0; r.n = len / 9 + 1; r.d = dalloc(r.n);
    int di = 0;
    for (int end = len; end > 0; end -= 9, di++) {
        int beg = end - 9 < 0 ? 0 : end - 9; uint32_t v = 0;
        for (int i = beg; i < end; i++) v = v * 10 + (uint32_t)(s[i] - '0');
        r.d[di] = v;
    }
    big_trim(&r); return r;
}
/* decimal digits of |a| (no sign) into buf; returns length */
static int big_digits(const obig *a, char *buf) {
    if (a->n == 0) { buf[0] = '0'; buf[1] = 0; return 1; }
    int len = sprintf(buf, "%u", a->d[a->n - 1]);
    for (int i = a->n - 2; i >= 0; i--) len += sprintf(buf + len, "%09u", a->d[i]);
    return len;
}
/* canonical "[-]int.frac" with exactly s fractional digits */
static char *big_format(const obig *a, int s) {
    size_t cap = (size_t)a->n * 9 + (size_t)(s > 0 ? s : 0) + 8;
    char *dig = (char *)malloc(cap), *out = (char *)malloc(cap + 4);
    int len = big_digits(a, dig);
    char *o = out;
    if (a->neg && a->n) *o++ = '-';
    if (s <= 0) { memcpy(o, dig, (size_t)len); o[len] = 0; }
    else if (len > s) { memcpy(o, dig, (size_t)(len - s)); o += len - s; *o++ = '.'; memcpy(o, dig + len - s, (size_t)s); o[s] = 0; }
    else { *o++ = '0'; *o++ = '.'; for (int i = 0; i < s - len; i++) *o++ = '0'; memcpy(o, dig, (size_t)len); o[len] = 0; }
    free(dig); return out;
}
/* parse "[-]ddd[.ddd]" into the mantissa at scale s (Eq.1: value = i*10^-s).
 * O_E_RANGE if it has more than s fractional digits (only trailing zeros
 * would be exact; we reject any) or the mantissa needs more than p digits. */
static int big_parse_at_scale(const char *str, int p, int s, obig *out) {
    while (*str == ' ') str++;
    int neg = 0;
    if (*str == '-' || *str == '+') { neg = (*str == '-'); str++; }
    const char *ip = str; int il = 0;
    while (isdigit((unsigned char)ip[il])) il++;
    const char *fp = ""; int fl = 0;
    if (ip[il] == '.') { fp = ip + il + 1; while (isdigit((unsigned char)fp[fl])) fl++; if (fp[fl] != 0 && fp[fl] != ' ') return O_E_INVAL; }
    else if (ip[il] != 0 && ip[il] != ' ') return O_E_INVAL;
    if (il == 0 && fl == 0) return O_E_INVAL;
    if (fl > s) return O_E_RANGE;
    char *buf = (char *)malloc((size_t)(il + s + 2));
    memcpy(buf, ip, (size_t)il); memcpy(buf + il, fp, (size_t)fl);
    for (int i = fl; i < s; i++) buf[il + i] = '0';
    obig m = big_from_digits(buf, il + s); free(buf);
    m.neg = neg; big_trim(&m);
    if (!big_fits(&m, p)) { big_free(&m); return O_E_RANGE; }
    *out = m; return O_OK;
}

/* ------------------------------------------------------------------ */
/* expression front end: parser + typing (§III-B3)        */
/* ------------------------------------------------------------------ */
enum { N_COL, N_LIT, N_ADD, N_SUB, N_MUL, N_DIV, N_MOD, N_NEG };
typedef struct onode {
    int kind, col; int p, s;
    obig lit;                          /* literal mantissa at scale s */
    struct onode *l, *r;
} onode;

typedef struct { const char *s; int pos; int err; int ncols; const int *cp, *cs; } oparser;

static void skipws(oparser *P) { while (P->s[P->pos] == ' ' || P->s[P->pos] == '\t') P->pos++; }
static onode *mknode(int kind, onode *l, onode *r) {
    onode *n = (onode *)calloc(1, sizeof(onode)); n->kind = kind; n->l = l; n->r = r; return n;
}
static void free_tree(onode *n) {
    if (!n) return;
    free_tree(n->l); free_tree(n->r); big_free(&n->lit); free(n);
}
static onode *p_expr(oparser *P);
static onode *p_primary(oparser *P) {
    skipws(P);
    char c = P->s[P->pos];
    if (c == '(') {
        P->pos++; onode *e = p_expr(P); skipws(P);
        if (P->s[P->pos] != ')') { P->err = 1; free_tree(e); return NULL; }
        P->pos++; return e;
    }
    if (c == 'c' || c == 'C') {
        P->pos++; int k = 0, nd = 0;
        while (isdigit((unsigned char)P->s[P->pos])) { k = k * 10 + (P->s[P->pos] - '0'); P->pos++; nd++; }
        if (nd == 0 || k < 1 || k > P->ncols) { P->err = 1; return NULL; }
        onode *n = mknode(N_COL, NULL, NULL); n->col = k - 1; return n;
    }
    if (isdigit((unsigned char)c) || c == '.') {
        int st = P->pos, il = 0, fl = 0;
        while (isdigit((unsigned char)P->s[P->pos])) { P->pos++; il++; }
        if (P->s[P->pos] == '.') { P->pos++; while (isdigit((unsigned char)P->s[P->pos])) { P->pos++; fl++; } }
        if (il + fl == 0) { P->err = 1; return NULL; }
        /* literal typing, §III-D2: 1.23 -> DECIMAL(3,2), 10 -> DECIMAL(2,0) */
        char *buf = (char *)malloc((size_t)(il + fl + 1));
        memcpy(buf, P->s + st, (size_t)il); memcpy(buf + il, P->s + st + il + (fl ? 1 : 0), (size_t)fl);
        onode *n = mknode(N_LIT, NULL, NULL);
        n->lit = big_from_digits(buf, il + fl); free(buf);
        char *dg = (char *)malloc((size_t)n->lit.n * 9 + 4); int nd = big_digits(&n->lit, dg); free(dg);
        n->s = fl; n->p = nd > fl ? nd : fl; if (n->p < 1) n->p = 1;
        return n;
    }
    P->err = 1; return NULL;
}
static onode *p_unary(oparser *P) {
    skipws(P);
    if (P->s[P->pos] == '-') { P->pos++; onode *a = p_unary(P); if (!a) return NULL; return mknode(N_NEG, a, NULL); }
    if (P->s[P->pos] == '+') { P->pos++; return p_unary(P); }
    return p_primary(P);
}
static onode *p_term(oparser *P) {
    onode *a = p_unary(P); if (!a) return NULL;
    for (;;) {
        skipws(P); char c = P->s[P->pos];
        int k = c == '*' ? N_MUL : c == '/' ? N_DIV : c == '%' ? N_MOD : -1;
        if (k < 0) return a;
        P->pos++; onode *b = p_unary(P); if (!b) { free_tree(a); return NULL; }
        a = mknode(k, a, b);
    }
}
static onode *p_expr(oparser *P) {
    onode *a = p_term(P); if (!a) return NULL;
    for (;;) {
        skipws(P); char c = P->s[P->pos];
        int k = c == '+' ? N_ADD : c == '-' ? N_SUB : -1;
        if (k < 0) return a;
        P->pos++; onode *b = p_term(P); if (!b) { free_tree(a); return NULL; }
        a = mknode(k, a, b);
    }
}
static int imax(int a, int b) { return a > b ? a : b; }
/* bottom-up typing, §III-B3 (readings Q3, Q5, Q7 in DESIGN.md) */
static int type_tree(onode *n, const int *cp, const int *cs) {
    int e;
    switch (n->kind) {
    case N_COL: n->p = cp[n->col]; n->s = cs[n->col]; return O_OK;
    case N_LIT: return O_OK;
    case N_NEG: if ((e = type_tree(n->l, cp, cs))) return e; n->p = n->l->p; n->s = n->l->s; return O_OK;
    default: break;
    }
    if ((e = type_tree(n->l, cp, cs)) || (e = type_tree(n->r, cp, cs))) return e;
    int p1 = n->l->p, s1 = n->l->s, p2 = n->r->p, s2 = n->r->s;
    switch (n->kind) {
    case N_ADD: case N_SUB:
        /* DECIMAL(max(p1, p2+s1-s2)+1, s1) for s1 >= s2; symmetric otherwise */
        if (s1 >= s2) { n->p = imax(p1, p2 + s1 - s2) + 1; n->s = s1; }
        else          { n->p = imax(p2, p1 + s2 - s1) + 1; n->s = s2; }
        return O_OK;
    case N_MUL: n->p = p1 + p2; n->s = s1 + s2; return O_OK;
    case N_DIV: n->p = imax(p1 - p2 + s2 + 5, 1); n->s = s1 + 4; return O_OK;
    case N_MOD: if (s1 != 0 || s2 != 0) return O_E_INVAL; n->p = p2; n->s = 0; return O_OK;
    }
    return O_E_INVAL;
}
static int parse_typed(const char *expr, int ncols, const int *cp, const int *cs, onode **out) {
    oparser P = {expr, 0, 0, ncols, cp, cs};
    onode *t = p_expr(&P); skipws(&P);
    if (!t || P.err || expr[P.pos] != 0) { free_tree(t); return O_E_INVAL; }
    int e = type_tree(t, cp, cs);
    if (e) { free_tree(t); return e; }
    *out = t; return O_OK;
}

/* evaluate node n for one row; vals[k] = mantissa of column k at its scale */
static int eval_node(const onode *n, const obig *vals, obig *out) {
    obig a, b; int e;
    switch (n->kind) {
    case N_COL: *out = big_copy(&vals[n->col]); return O_OK;
    case N_LIT: *out = big_copy(&n->lit); return O_OK;
    case N_NEG: if ((e = eval_node(n->l, vals, &a))) return e; *out = big_neg(&a); big_free(&a); return O_OK;
    default: break;
    }
    if ((e = eval_node(n->l, vals, &a))) return e;
    if ((e = eval_node(n->r, vals, &b))) { big_free(&a); return e; }
    int s1 = n->l->s, s2 = n->r->s;
    obig r = big_zero(); e = O_OK;
    switch (n->kind) {
    case N_ADD: case N_SUB: {
        /* align the smaller scale upward by x10^(s_hi - s_lo) */
        obig aa = s1 < s2 ? big_scale_up(&a, s2 - s1) : big_copy(&a);
        obig bb = s2 < s1 ? big_scale_up(&b, s1 - s2) : big_copy(&b);
        r = n->kind == N_ADD ? big_add(&aa, &bb) : big_sub(&aa, &bb);
        big_free(&aa); big_free(&bb); break;
    }
    case N_MUL: r = big_mul(&a, &b); break;
    case N_DIV: {
        if (big_is_zero(&b)) { e = O_E_DIVZERO; break; }
        /* Q = trunc(|A| * 10^(s2+4) / |B|), sign = xor (Q4) */
        obig ua = big_scale_up(&a, s2 + 4), rr; ua.neg = 0;
        obig ub = big_copy(&b); ub.neg = 0;
        mag_divmod(&ua, &ub, &r, &rr);
        r.neg = a.neg ^ b.neg; big_trim(&r);
        big_free(&ua); big_free(&ub); big_free(&rr); break;
    }
    case N_MOD: {
        if (big_is_zero(&b)) { e = O_E_DIVZERO; break; }
        obig ua = big_copy(&a), ub = big_copy(&b), q; ua.neg = 0; ub.neg = 0;
        mag_divmod(&ua, &ub, &q, &r);
        r.neg = a.neg; big_trim(&r);                     /* sign of the dividend (Q7) */
        big_free(&ua); big_free(&ub); big_free(&q); break;
    }
    }
    big_free(&a); big_free(&b);
    if (e) { big_free(&r); return e; }
    if (!big_fits(&r, n->p)) { big_free(&r); return O_E_OVERFLOW; }   /* |v| >= 10^p */
    *out = r; return O_OK;
}

/* ------------------------------------------------------------------ */
/* column input: binary sign-magnitude rows (the generator's format)   */
/* or decimal strings                                                  */
/* ------------------------------------------------------------------ */
typedef struct {
    int ncols; const int *p, *s, *w;            /* per column: precision, scale, words per row */
    const uint32_t *const *mag;                  /* mag[k] : n * w[k] words, row-major */
    const uint8_t *const *neg;                   /* neg[k] : n bytes (or NULL) */
    const char *const *str;                      /* alternative: str[row*ncols + k] */
} ocols;

static int load_row(const ocols *C, int64_t row, obig *vals) {
    for (int k = 0; k < C->ncols; k++) {
        if (C->str) {
            int e = big_parse_at_scale(C->str[row * C->ncols + k], C->p[k], C->s[k], &vals[k]);
            if (e) { for (int j = 0; j < k; j++) big_free(&vals[j]); return e; }
        } else {
            vals[k] = big_from_words(C->mag[k] + row * C->w[k], C->w[k], C->neg && C->neg[k] ? C->neg[k][row] : 0);
            if (!big_fits(&vals[k], C->p[k])) { for (int j = 0; j <= k; j++) big_free(&vals[j]); return O_E_RANGE; }
        }
    }
    return O_OK;
}

static int ceil_log10(int64_t N) {      /* smallest k with 10^k >= N ; N <= 1 -> 0 (reading Q9) */
    int k = 0; int64_t t = 1;
    while (t < N) { t *= 10; k++; }
    return k;
}

/* ---- threaded SUM driver (static row blocks, exact in-order combine) ---- */
typedef struct {
    const onode *tree; const ocols *C; int64_t r0, r1; obig acc; int err;
    int mode; /* 0 = expr, 1 = modexp, 2 = sin */
    const obig *mod_e, *mod_n; int sin_P;
} ojob;

static int row_value(ojob *J, int64_t i, obig *v);

static void *sum_worker(void *arg) {
    ojob *J = (ojob *)arg; J->acc = big_zero(); J->err = O_OK;
    for (int64_t i = J->r0; i < J->r1; i++) {
        obig v; int e = row_value(J, i, &v);
        if (e) { J->err = e; return NULL; }
        obig t = big_add(&J->acc, &v); big_free(&J->acc); big_free(&v); J->acc = t;
    }
    return NULL;
}
static int run_sum(ojob *proto, int64_t n, int nthreads, obig *out) {
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    if ((int64_t)nthreads > n) nthreads = n > 0 ? (int)n : 1;
    ojob *J = (ojob *)calloc((size_t)nthreads, sizeof(ojob));
    pthread_t *th = (pthread_t *)calloc((size_t)nthreads, sizeof(pthread_t));
    for (int t = 0; t < nthreads; t++) {
        J[t] = *proto; J[t].r0 = n * t / nthreads; J[t].r1 = n * (t + 1) / nthreads;
        if (nthreads == 1) sum_worker(&J[t]); else pthread_create(&th[t], NULL, sum_worker, &J[t]);
    }
    int err = O_OK; obig acc = big_zero();
    for (int t = 0; t < nthreads; t++) {
        if (nthreads > 1) pthread_join(th[t], NULL);
        if (J[t].err && !err) err = J[t].err;
        obig s = big_add(&acc, &J[t].acc); big_free(&acc); big_free(&J[t].acc); acc = s;
    }
    free(J); free(th);
    if (err) { big_free(&acc); return err; }
    *out = acc; return O_OK;
}

/* ------------------------------------------------------------------ */
/* modexp: X^e mod N (Query 4): square-and-multiply,     */
/* every product reduced by % (the long division above).               */
/* ------------------------------------------------------------------ */
static int modexp_one(const obig *x, const obig *E, const obig *N, obig *out) {
    if (x->neg) return O_E_INVAL;
    if (big_is_zero(N) || N->neg) return O_E_INVAL;
    obig q, base; mag_divmod(x, N, &q, &base); big_free(&q);     /* x >= N is reduced first (Q15) */
    /* binary digits of E, most significant first */
    obig e = big_copy(E); int nbits = 0; unsigned char *bits = (unsigned char *)malloc((size_t)e.n * 30 + 8);
    while (!big_is_zero(&e)) { uint32_t rb; obig h = mag_div_small(&e, 2, &rb); bits[nbits++] = (unsigned char)rb; big_free(&e); e = h; }
    big_free(&e);
    obig one = big_from_u64(1), r, tmp;
    mag_divmod(&one, N, &q, &r); big_free(&q); big_free(&one);   /* r = 1 mod N */
    for (int i = nbits - 1; i >= 0; i--) {
        obig sq = big_mul(&r, &r); big_free(&r);
        mag_divmod(&sq, N, &q, &r); big_free(&q); big_free(&sq);
        if (bits[i]) {
            obig pr = big_mul(&r, &base); big_free(&r);
            mag_divmod(&pr, N, &q, &tmp); big_free(&q); big_free(&pr); r = tmp;
        }
    }
    free(bits); big_free(&base);
    *out = r; return O_OK;
}

/* ------------------------------------------------------------------ */
/* sin_P(x): x = m_x*10^-s (s <= P, |x| < 10),           */
/* t_1 = |m_x|*10^(P-s), t_{k+1} = floor(t_k*m_x^2 / (10^(2s)*(2k)(2k+1))),  */
/* S = sum_k (-1)^(k-1) t_k until t = 0, result sign(m_x)*S at scale P.  */
/* ------------------------------------------------------------------ */
static int sin_one(const obig *mx, int s, int P, obig *out) {
    if (s > P || s < 0) return O_E_INVAL;
    obig ax = big_copy(mx); ax.neg = 0;
    obig X2 = big_mul(&ax, &ax);
    obig den0 = big_pow10(2 * s);
    obig t = big_scale_up(&ax, P - s);
    obig S = big_zero();
    for (int64_t k = 1; !big_is_zero(&t); k++) {
        obig nS = (k & 1) ? big_add(&S, &t) : big_sub(&S, &t);
        big_free(&S); S = nS;
        obig num = big_mul(&t, &X2);
        obig kk = big_from_u64((uint64_t)(2 * k) * (uint64_t)(2 * k + 1));
        obig den = big_mul(&den0, &kk);
        obig q, r; mag_divmod(&num, &den, &q, &r);
        big_free(&num); big_free(&kk); big_free(&den); big_free(&r); big_free(&t);
        t = q;
    }
    S.neg = S.neg ^ mx->neg; big_trim(&S);
    big_free(&ax); big_free(&X2); big_free(&den0); big_free(&t);
    *out = S; return O_OK;
}

static int row_value(ojob *J, int64_t i, obig *v) {
    obig vals[64]; int e;
    if ((e = load_row(J->C, i, vals))) return e;
    if (J->mode == 0) e = eval_node(J->tree, vals, v);
    else if (J->mode == 1) e = modexp_one(&vals[0], J->mod_e, J->mod_n, v);
    else e = sin_one(&vals[0], J->C->s[0], J->sin_P, v);
    for (int k = 0; k < J->C->ncols; k++) big_free(&vals[k]);
    return e;
}

/* ------------------------------------------------------------------ */
/* exported C API (ctypes; see oracle/__init__.py)                      */
/* ------------------------------------------------------------------ */
static int put_str(char *out, size_t outlen, const char *s) {
    size_t l = strlen(s);
    if (l + 1 > outlen) return O_E_NOMEM;
    memcpy(out, s, l + 1); return O_OK;
}

int orc_expr_type(const char *expr, int ncols, const int *p, const int *s, int *P, int *S) {
    onode *t; int e = parse_typed(expr, ncols, p, s, &t); if (e) return e;
    *P = t->p; *S = t->s; free_tree(t); return O_OK;
}

int orc_sum_type(int p, int s, int64_t n_global, int *P, int *S) {
    *P = p + ceil_log10(n_global); *S = s; return O_OK;
}

static int make_cols(ocols *C, int ncols, const int *p, const int *s, const int *w,
                     const uint32_t *const *mag, const uint8_t *const *neg, const char *const *str) {
    C->ncols = ncols; C->p = p; C->s = s; C->w = w; C->mag = mag; C->neg = neg; C->str = str;
    return ncols <= 64 ? O_OK : O_E_INVAL;
}

/* one canonical decimal string per row, '\n'-separated; a row whose
 * evaluation fails is written as "E<code>". Returns the first error code. */
static int rows_common(ojob *proto, int64_t n, int out_s, char *out, size_t outlen) {
    size_t pos = 0; int first = O_OK;
    for (int64_t i = 0; i < n; i++) {
        obig v; char tmp[16]; char *str; int e = row_value(proto, i, &v);
        if (e) { if (!first) first = e; snprintf(tmp, sizeof tmp, "E%d", e); str = tmp; }
        else { str = big_format(&v, out_s); big_free(&v); }
        size_t l = strlen(str);
        if (pos + l + 2 > outlen) { if (str != tmp) free(str); return O_E_NOMEM; }
        memcpy(out + pos, str, l); pos += l; out[pos++] = '\n';
        if (str != tmp) free(str);
    }
    out[pos] = 0; return first;
}

int orc_eval_rows(const char *expr, int ncols, const int *p, const int *s, const int *w,
                  const uint32_t *const *mag, const uint8_t *const *neg, const char *const *str,
                  int64_t n, char *out, size_t outlen) {
    ocols C; if (make_cols(&C, ncols, p, s, w, mag, neg, str)) return O_E_INVAL;
    onode *t; int e = parse_typed(expr, ncols, p, s, &t); if (e) return e;
    ojob J; memset(&J, 0, sizeof J); J.tree = t; J.C = &C; J.mode = 0;
    e = rows_common(&J, n, t->s, out, outlen);
    free_tree(t); return e;
}

int orc_eval_sum(const char *expr, int ncols, const int *p, const int *s, const int *w,
                 const uint32_t *const *mag, const uint8_t *const *neg, const char *const *str,
                 int64_t n, int64_t n_global, int nthreads, char *out, size_t outlen, int *outP, int *outS) {
    ocols C; if (make_cols(&C, ncols, p, s, w, mag, neg, str)) return O_E_INVAL;
    onode *t; int e = parse_typed(expr, ncols, p, s, &t); if (e) return e;
    ojob J; memset(&J, 0, sizeof J); J.tree = t; J.C = &C; J.mode = 0;
    obig acc; e = run_sum(&J, n, nthreads, &acc);
    int P = t->p + ceil_log10(n_global > 0 ? n_global : n), S = t->s;
    free_tree(t);
    if (e) return e;
    if (!big_fits(&acc, P)) { big_free(&acc); return O_E_OVERFLOW; }
    char *str_ = big_format(&acc, S); big_free(&acc);
    e = put_str(out, outlen, str_); free(str_);
    if (outP) *outP = P;
    if (outS) *outS = S;
    return e;
}

static int parse_uint(const char *str, obig *out) {
    int l = 0; while (isdigit((unsigned char)str[l])) l++;
    if (l == 0 || str[l] != 0) return O_E_INVAL;
    *out = big_from_digits(str, l); return O_OK;
}

int orc_modexp_rows(const char *exponent, const char *modulus, int p, int w,
                    const uint32_t *mag, const uint8_t *neg, const char *const *str,
                    int64_t n, char *out, size_t outlen) {
    int s = 0; ocols C; const uint32_t *mags[1] = {mag}; const uint8_t *negs[1] = {neg};
    make_cols(&C, 1, &p, &s, &w, mags, neg ? negs : NULL, str);
    obig E, N; if (parse_uint(exponent, &E)) return O_E_INVAL;
    if (parse_uint(modulus, &N)) { big_free(&E); return O_E_INVAL; }
    ojob J; memset(&J, 0, sizeof J); J.C = &C; J.mode = 1; J.mod_e = &E; J.mod_n = &N;
    int e = rows_common(&J, n, 0, out, outlen);
    big_free(&E); big_free(&N); return e;
}

int orc_modexp_sum(const char *exponent, const char *modulus, int p, int w,
                   const uint32_t *mag, const uint8_t *neg, int64_t n, int nthreads,
                   char *out, size_t outlen) {
    int s = 0; ocols C; const uint32_t *mags[1] = {mag}; const uint8_t *negs[1] = {neg};
    make_cols(&C, 1, &p, &s, &w, mags, neg ? negs : NULL, NULL);
    obig E, N; if (parse_uint(exponent, &E)) return O_E_INVAL;
    if (parse_uint(modulus, &N)) { big_free(&E); return O_E_INVAL; }
    ojob J; memset(&J, 0, sizeof J); J.C = &C; J.mode = 1; J.mod_e = &E; J.mod_n = &N;
    obig acc; int e = run_sum(&J, n, nthreads, &acc);
    big_free(&E); big_free(&N);
    if (e) return e;
    char *s_ = big_format(&acc, 0); big_free(&acc);
    e = put_str(out, outlen, s_); free(s_); return e;
}

int orc_sin_rows(int P, int p, int s, int w, const uint32_t *mag, const uint8_t *neg,
                 const char *const *str, int64_t n, char *out, size_t outlen) {
    ocols C; const uint32_t *mags[1] = {mag}; const uint8_t *negs[1] = {neg};
    make_cols(&C, 1, &p, &s, &w, mags, neg ? negs : NULL, str);
    ojob J; memset(&J, 0, sizeof J); J.C = &C; J.mode = 2; J.sin_P = P;
    return rows_common(&J, n, P, out, outlen);
}

int orc_sin_sum(int P, int p, int s, int w, const uint32_t *mag, const uint8_t *neg,
                int64_t n, int nthreads, char *out, size_t outlen) {
    ocols C; const uint32_t *mags[1] = {mag}; const uint8_t *negs[1] = {neg};
    make_cols(&C, 1, &p, &s, &w, mags, neg ? negs : NULL, NULL);
    ojob J; memset(&J, 0, sizeof J); J.C = &C; J.mode = 2; J.sin_P = P;
    obig acc; int e = run_sum(&J, n, nthreads, &acc);
    if (e) return e;
    char *s_ = big_format(&acc, P); big_free(&acc);
    e = put_str(out, outlen, s_); free(s_); return e;
}

/* exact sum of decimal strings at one scale (the multi-rank combine check) */
int orc_add_strings(const char *const *vals, int n, int p, int s, char *out, size_t outlen) {
    obig acc = big_zero();
    for (int i = 0; i < n; i++) {
        obig v; int e = big_parse_at_scale(vals[i], p, s, &v);
        if (e) { big_free(&acc); return e; }
        obig t = big_add(&acc, &v); big_free(&acc); big_free(&v); acc = t;
    }
    char *s_ = big_format(&acc, s); big_free(&acc);
    int e = put_str(out, outlen, s_); free(s_); return e;
}
