/*
 * up.h -- C ABI of libup.so, the B200 (sm_100a) hot path of UltraPrecise
 * (Li, Xiao, Yu, Lee, Zhang, ICDE 2024; /root/reference/PAPER.md, cited as
 * "P:L<line> §<section>").
 *
 * What it computes: column-at-a-time evaluation of fixed-point DECIMAL(p,s)
 * expressions (+ - * / % and unary -, over columns c1..cK and decimal
 * literals) and the exact SUM over them, RSA-style modular exponentiation,
 * and a fixed-point Taylor sine.  Semantics and typing: §II,
 * P:L1028-1080 §III-B3, readings Q1-Q16 in DESIGN.md.
 *
 * Conventions (all entry points):
 *  - Every call returns up_status; nothing throws across the ABI.  On error
 *    up_last_error() returns a thread-local message.
 *  - Pointers named d_* and the up_column.data field are DEVICE pointers;
 *    everything else is host memory.  Device memory passed in is CALLER-owned
 *    (e.g. torch tensors) and never freed by the library; the ctx owns only
 *    its kernel cache, workspaces and staging buffers.
 *  - `stream` is a cudaStream_t (NULL = legacy default stream).  All work is
 *    ordered on it; calls return without synchronising unless stated.
 *  - Data-dependent arithmetic faults (declared-type overflow, divide by
 *    zero, out-of-range input) never abort a kernel: they set a sticky device
 *    flag that up_check() reads (values of the affected rows are unspecified).
 *  - One ctx per host thread / stream (its SUM workspace is not shared-safe).
 */
#ifndef UP_H
#define UP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    UP_OK = 0,
    UP_E_INVAL = 1,        /* bad argument, bad expression, % on non-integers */
    UP_E_RANGE = 2,        /* input value does not fit its DECIMAL(p,s) */
    UP_E_OVERFLOW = 3,     /* a value exceeded its inferred type (reading Q5: only / can) */
    UP_E_DIVZERO = 4,      /* division or modulo by zero (reading Q6) */
    UP_E_NOMEM = 5,
    UP_E_CUDA = 6,         /* CUDA runtime / driver error */
    UP_E_NVRTC = 7,        /* kernel specialisation (JIT) failed */
    UP_E_UNSUPPORTED = 8   /* valid request outside what this build implements */
} up_status;

const char *up_last_error(void);

typedef struct up_ctx up_ctx;

/* Create a context bound to CUDA device `device` (makes it current). */
up_status up_ctx_create(int device, up_ctx **out);
up_status up_ctx_destroy(up_ctx *ctx);

/*
 * Pipelined SUM launches (default off).  When on, the fused SUM kernels of
 * up_sum_expr / up_sum are launched with programmatic dependent launch: their
 * CTAs may start (and stream their input columns) while the previous kernel
 * on the same stream is finishing, and wait for that kernel to complete
 * before touching the context's SUM workspace and d_partial.  Back-to-back
 * aggregation queries over resident columns then overlap one query's ramp
 * with the previous one's tail.  Contract: the kernel immediately before such
 * a SUM on its stream must not write that SUM's input columns (a kernel two
 * or more launches back is fully ordered as usual).  Turn it off around
 * ingestion or evaluation that produces a column a SUM reads next.
 */
up_status up_set_pipelined(up_ctx *ctx, int on);

/*
 * A DECIMAL(p,s) column of n rows as `limbs` limb planes (SURVEY §8a layout):
 * data[j*ld + i] is limb j (little-endian, 32-bit) of row i's mantissa in
 * TWO'S COMPLEMENT, value = mantissa * 10^-s (Eq. 1).  ld >= n is a
 * multiple of 4 and data is 16-byte aligned.  limbs must equal up_limbs(p).
 * Rows n..ld-1 are padding and are never read as values.
 */
typedef struct {
    int64_t n, ld;
    int32_t p, s, limbs, layout;
    uint32_t *data;
} up_column;

/*
 * Column layouts (up_column.layout):
 *  UP_LAYOUT_PLANES  -- limb planes as above (every entry point).
 *  UP_LAYOUT_COMPACT -- the paper's compact byte rows (cDecimal, P:L843-873,
 *     Fig. 4) kept resident on the device: row i is the Lb = up_compact_bytes(p)
 *     bytes at ((uint8_t *)data)[i*Lb], little-endian magnitude, sign in the
 *     top bit of the last byte; ld must equal Lb; data 16-byte aligned and the
 *     allocation at least n*Lb rounded up to 16 bytes (kernels read whole
 *     16-byte vectors).  Read directly (no limb planes materialised) by
 *     up_eval_expr / up_sum_expr / up_sum / up_filter inputs;
 *     ingestion: up_column_from_{host,device}_compact copy the rows in place
 *     (+ range check), the _bin / string calls convert.  Other entry points
 *     return UP_E_UNSUPPORTED for compact inputs.
 */
/*
 *  UP_LAYOUT_QUADS -- limb quads: the limbs grouped four at a time per row,
 *     G = up_quads(p) = ceil((limbs + 1) / 4) quads of ld rows; quad g of row i
 *     is the 16 bytes ((uint32_t *)data)[4*(g*ld + i) .. +4) = limbs 4g..4g+3
 *     (two's complement as in the planes), limb `limbs` holds the SIGN FLAG
 *     (1 for a negative row, else 0) and the limbs above it are 0.  ld >= n,
 *     a multiple of 4; data 16-byte aligned, G*ld*16 bytes.  Why: a 3-D TMA
 *     box of this layout lands in shared memory as the tensor cores' MN-major
 *     core matrices (16 digit bytes x 8 rows) with the sign digit included,
 *     so SUM(c_a*c_b) feeds tcgen05 straight from the copies (SURVEY §8a rows
 *     a6/a11; contract_tc.cu; calls below 2^30 rows -- beyond, the product
 *     stays in the fused per-row kernel).  Read by up_eval_expr / up_sum_expr / up_sum /
 *     up_filter (every generated kernel reads quads with 16-byte loads);
 *     ingestion and read-back convert through limb planes in the ctx scratch.
 *     Other entry points return UP_E_UNSUPPORTED for quad inputs.
 */
enum { UP_LAYOUT_PLANES = 0, UP_LAYOUT_COMPACT = 1, UP_LAYOUT_QUADS = 2 };

/* Limb count L = min{L : 10^p <= 2^(32L-1)} (reading Q1 of P:L821-837 vs
 * reproduces 18/38/76/153/307 <-> 2/4/8/16/32). */
int32_t up_limbs(int32_t p);
/* Quads of a UP_LAYOUT_QUADS column: ceil((up_limbs(p) + 1) / 4). */
int32_t up_quads(int32_t p);
/* ld for n rows (n rounded up to a multiple of 4). */
int64_t up_ld(int64_t n);
/* SUM result precision p + ceil(log10 N), N = n_global (reading Q9). */
int32_t up_sum_precision(int32_t p, int64_t n_global);

/*
 * Column ingestion (row a3).  Sign-magnitude binary input: row i's magnitude
 * is mag[i*mag_words .. +mag_words) (little-endian uint32), its sign neg[i]
 * (nonzero = negative; NULL = all non-negative).  dst must be preset by the
 * caller: n, ld, p, s, limbs, data (device, limbs*ld uint32).  A magnitude
 * >= 10^p sets the RANGE flag (see up_check).
 *   _host_bin: mag/neg are HOST pointers (pinned for async copies); they are
 *              staged through ctx-owned device memory on `stream`; the call
 *              returns after the host buffers may be reused (it synchronises
 *              the stream before returning).
 *   _device_bin: mag/neg are DEVICE pointers (e.g. from the generator).
 *   _host: decimal strings "[-]ddd[.ddd]" (at most s fraction digits, else
 *              UP_E_RANGE); parsed on the host, then as _host_bin.
 */
up_status up_column_from_host_bin(up_ctx *ctx, const uint32_t *mag, int32_t mag_words,
                                  const uint8_t *neg, up_column *dst, void *stream);
up_status up_column_from_device_bin(up_ctx *ctx, const uint32_t *d_mag, int32_t mag_words,
                                    const uint8_t *d_neg, up_column *dst, void *stream);
up_status up_column_from_host(up_ctx *ctx, const char *const *decimals, up_column *dst, void *stream);
/* Column to host as sign-magnitude: mag (n x col->limbs words), neg (n bytes).
 * Synchronises the stream. */
up_status up_column_to_host_bin(up_ctx *ctx, const up_column *col, uint32_t *mag, uint8_t *neg,
                                void *stream);

/*
 * Compact byte-aligned column codec (the paper's cDecimal, Fig. 4):
 * each row is Lb = up_compact_bytes(p) = ceil((1 + p log2 10)/8) bytes, the
 * magnitude little-endian in the low 8*Lb-1 bits and the sign in the top bit
 * of the last byte (-1.23 in DECIMAL(10,2) = {123,0,0,0,0x80}).  Rows are
 * contiguous (row i at bytes[i*Lb]).  _host_: host buffer staged through the
 * ctx (same lifetime rule as _host_bin; inputs of >= 32 MB are copied in up to
 * 8 chunks on a ctx-owned copy stream, each chunk converted / range-checked on
 * `stream` as soon as it lands -- pinned memory makes the copies asynchronous);
 * _device_: device buffer;
 * to_host_compact synchronises the stream.  Range errors set RANGE.
 */
int32_t up_compact_bytes(int32_t p);
up_status up_column_from_host_compact(up_ctx *ctx, const uint8_t *bytes, up_column *dst, void *stream);
up_status up_column_from_device_compact(up_ctx *ctx, const uint8_t *d_bytes, up_column *dst, void *stream);
up_status up_column_to_host_compact(up_ctx *ctx, const up_column *col, uint8_t *bytes, void *stream);

/* Result type of expr over the columns (§III-B3). */
up_status up_expr_type(up_ctx *ctx, const char *expr, const up_column *cols, int ncols,
                       int32_t *p, int32_t *s);

/*
 * Evaluate expr for every row (rows a1-a7, a12): out must be caller-allocated
 * with up_expr_type's (p,s), limbs = up_limbs(p), n = cols[0].n.  The first
 * call for an (expr, column types) pair specialises and JIT-compiles a fused
 * kernel for sm_100a (row a2, §III-B); later calls hit the cache.
 */
up_status up_eval_expr(up_ctx *ctx, const char *expr, const up_column *cols, int ncols,
                       up_column *out, void *stream);

/*
 * SELECT SUM(expr) over this shard's rows (row a11), fused with evaluation.
 * The result type is DECIMAL(p_expr + ceil(log10 n_global), s_expr) with
 * LA = up_limbs(that p) limbs (query with up_sum_type).  d_partial receives LA
 * two's-complement limbs (device).  n_global = rows over all shards (typing
 * only; 0 means cols[0].n).  One kernel launch -- except when a top-level
 * product of two wide columns is split off (SUM is linear): its tensor-core
 * contraction, the fused kernel for the rest of the expression and an exact
 * combine kernel; over limb-quad columns the contraction and the rest run on
 * two ctx-owned streams forked from `stream` and joined back into it before
 * the combine (the call stays ordered on `stream`; UP_SERIAL_SPLIT keeps
 * everything on `stream`).
 */
up_status up_sum_type(up_ctx *ctx, const char *expr, const up_column *cols, int ncols,
                      int64_t n_global, int32_t *p, int32_t *s, int32_t *la);
up_status up_sum_expr(up_ctx *ctx, const char *expr, const up_column *cols, int ncols,
                      int64_t n_global, uint32_t *d_partial, void *stream);
/* SUM of one column: up_sum_expr(ctx, "c1", col, 1, ...). */
up_status up_sum(up_ctx *ctx, const up_column *col, int64_t n_global, uint32_t *d_partial, void *stream);

/*
 * Exact combine of nranks SUM partials (row a13): d_partials holds nranks x la
 * two's-complement limbs (device, rank-major, e.g. an NCCL all-gather
 * output); d_out receives their sum in la limbs.  One kernel launch.
 */
up_status up_sum_combine(up_ctx *ctx, const uint32_t *d_partials, int32_t nranks, int32_t la,
                         uint32_t *d_out, void *stream);

/*
 * Grouped aggregation: SELECT agg_a(expr_a) ... GROUP BY g in
 * ONE kernel launch.  Aggregate typing follows P:L1069-1080 (Sec. III-B):
 *   SUM(e): DECIMAL(p + ceil(log10 N), s)      (as up_sum_type)
 *   MIN(e), MAX(e): DECIMAL(p, s)              (the expression's type)
 *   AVG(e): the SUM rule, then the division rule with the
 *           divisor COUNT converted to DECIMAL(ceil(log10 N)+1, 0), i.e.
 *           DECIMAL(p + 4, s + 4), value trunc(SUM * 10^4 / COUNT)
 *           (truncation toward zero, reading Q4).
 * N = n_global (0 means the local row count): the tuple count of the query.
 * kinds[a] in up_agg_kind; exprs[a] use the up_eval_expr grammar.
 * d_group: device int32 per row (16-byte aligned); rows with a negative id are excluded (a
 *   WHERE filter); ids >= n_groups set the INVAL flag and are excluded; NULL
 *   means one group (n_groups must then be 1).  n_groups is limited by the
 *   shared-memory group records (UNSUPPORTED beyond ~200 KB per block).
 * d_out (device, packed): aggregate a's results for groups 0..n_groups-1,
 *   each up_agg_type(...).limbs two's-complement limbs, aggregates in order;
 *   total sum_a n_groups * limbs_a uint32.
 * d_counts (device): n_groups uint64 row counts (COUNT(*) per group).  An
 *   empty group yields 0 for every aggregate (SQL NULL; see its count).
 * Errors raised by rows of excluded groups are not flagged.  Across ranks:
 * up_group_combine below.
 */
typedef enum { UP_AGG_SUM = 0, UP_AGG_MIN = 1, UP_AGG_MAX = 2, UP_AGG_AVG = 3 } up_agg_kind;
up_status up_agg_type(const char *expr, int32_t kind, const up_column *cols, int ncols, int64_t n_global,
                      int32_t *p, int32_t *s, int32_t *limbs);
up_status up_group_aggregate(up_ctx *ctx, int32_t n_aggs, const int32_t *kinds, const char *const *exprs,
                             const up_column *cols, int ncols, const int32_t *d_group, int32_t n_groups,
                             int64_t n_global, uint32_t *d_out, uint64_t *d_counts, void *stream);

/*
 * Per-operator kernels with TPI threads per instance (the
 * paper's multi-threading arithmetic, Sec. III-E1, Fig. 13):
 * out = a <op> b per row, op "+" "-" "*" "/", with the values, types and
 * flags of up_eval_expr("c1<op>c2").  A group of tpi lanes
 * (1, 2, 4, 8, 16, 32) owns each row: + - * run on every tpi; "/" runs one row
 * per thread (tpi 1) with div_algo 0 = long division (Knuth D, the fused
 * kernels' method) or 1 = Newton-Raphson reciprocal iteration,
 * operands up to 64 limbs.  Inputs: limb planes or compact rows (compact rows
 * are read by the group as in the paper's Listing 3); out: limb planes,
 * caller-allocated with the expression's type.  One kernel launch.
 */
up_status up_eval_tpi(up_ctx *ctx, const char *op, const up_column *a, const up_column *b, int32_t tpi,
                      int32_t div_algo, up_column *out, void *stream);

/*
 * Multi-rank GROUP BY (NEXT-4 with rows a13/e): every rank runs
 * up_group_aggregate over its rows with each AVG replaced by SUM (the
 * combinable partial state of an average; same n_global on every rank), the
 * packed outputs and the counts are all-gathered rank-major (d_parts:
 * nranks x that layout's words, d_counts: nranks x n_groups uint64), then
 * this call writes the final results in up_group_aggregate's layout for the
 * ORIGINAL kinds: SUM = exact sum over ranks; MIN / MAX over the ranks whose
 * group is non-empty; AVG = trunc(|SUM| 10^4 / COUNT) sign(SUM) of the
 * combined SUM and COUNT (reading Q4; COUNT 0 -> 0).
 * d_counts_out (optional): n_groups combined counts.  One kernel launch;
 * aggregates wider than 80 limbs: UP_E_UNSUPPORTED.
 */
up_status up_group_combine(up_ctx *ctx, int32_t n_aggs, const int32_t *kinds, const char *const *exprs,
                           const up_column *cols, int ncols, int32_t n_groups, int64_t n_global,
                           const uint32_t *d_parts, int32_t nranks, const uint64_t *d_counts, uint32_t *d_out,
                           uint64_t *d_counts_out, void *stream);

/*
 * WHERE lhs <op> rhs (the DECIMAL comparison
 * operators of P:L730-734 Sec. II-C).  lhs, rhs: expressions over cols (the
 * up_eval_expr grammar); op: "<" "<=" ">" ">=" "=" ("==") "<>" ("!=").  The
 * comparison is exact: the sign of lhs - rhs evaluated at the type the
 * paper's +/- rule gives the difference (each side keeps its
 * own division truncation, reading Q4).  d_ids: device int32 per row; every
 * row whose predicate is FALSE gets -1, other entries are left unchanged, so
 * successive calls AND their predicates and the array feeds up_group_ids /
 * up_group_aggregate (negative id = excluded).  One fused kernel launch.
 * Rows that raise DIVZERO/OVERFLOW flag it; their predicate is unspecified.
 */
up_status up_filter(up_ctx *ctx, const char *lhs, const char *op, const char *rhs, const up_column *cols,
                    int ncols, int32_t *d_ids, void *stream);

/*
 * GROUP BY key columns (DECIMAL values
 * are compared to sort for grouping).  keys: nkeys DECIMAL columns of n rows
 * each, compared lexicographically (keys[0] most significant), each by its
 * exact value (one column = one scale, so by its mantissa).  d_ids: device
 * int32 per row, IN/OUT: rows with a negative entry on input are excluded
 * (e.g. by up_filter; pass an array of zeros to keep all rows) and stay -1;
 * every other row receives its dense group id, 0 for the smallest key and
 * increasing with the key.  *n_groups (host) = number of groups; the call
 * synchronises the stream to read it.  d_first (device int64, optional,
 * n entries): d_first[g] = the smallest row index of group g, for
 * g < *n_groups.  Implementation (groupby.cu, hand-written): stable LSD
 * radix sort of (key limb, row) pairs, 8-bit digits (tile histograms, a scan
 * of the digit-major counts, a stable scatter), least significant key column
 * and limb first, the top limb's sign bit flipped so two's complement orders
 * as signed; excluded rows sorted last; then an adjacent-difference pass over
 * all limbs, a prefix sum and a scatter.  Scratch: the ctx's persistent scratch
 * buffer (24 bytes per row + sort temporaries), grown on demand (growing it
 * synchronises the device); the call holds the ctx lock throughout.
 */
up_status up_group_ids(up_ctx *ctx, const up_column *keys, int nkeys, int32_t *d_ids, int64_t *n_groups,
                       int64_t *d_first, void *stream);

/*
 * x^e mod N per row (row a8; Query 4 P:L2124-2154 generalised to any e).
 * base: s == 0, values >= 0 (a negative value sets INVAL); values >= N are
 * reduced mod N first.  exponent, modulus: decimal strings, modulus odd and
 * > 1 (even moduli: UP_E_UNSUPPORTED).  out: DECIMAL(digits(N), 0),
 * caller-allocated (p = number of decimal digits of N).  N is converted and
 * its Montgomery constants are derived at specialisation time.
 * up_modexp_sum: fused SUM of the results into d_partial, type
 * DECIMAL(digits(N) + ceil(log10 n_global), 0) (query with up_modexp_sum_type).
 */
up_status up_modexp(up_ctx *ctx, const up_column *base, const char *exponent, const char *modulus,
                    up_column *out, void *stream);
up_status up_modexp_sum_type(up_ctx *ctx, const char *modulus, int64_t n_global,
                             int32_t *p, int32_t *la);
up_status up_modexp_sum(up_ctx *ctx, const up_column *base, const char *exponent, const char *modulus,
                        int64_t n_global, uint32_t *d_partial, void *stream);

/*
 * Fixed-point Taylor sine sin_P(x) per row (row a9, from
 * Query 5 P:L2197-2249): x DECIMAL(p,s) with p <= 9, p - s <= 1 (|x| < 10, else
 * UP_E_UNSUPPORTED), s <= P,
 * t_1 = |m_x| 10^(P-s), t_{k+1} = floor(t_k m_x^2 / (10^(2s) (2k)(2k+1))),
 * result sign(m_x) * sum_k (-1)^(k-1) t_k, type DECIMAL(P+1, P).
 * up_sin_taylor: out caller-allocated DECIMAL(P+1,P).
 * up_sin_taylor_sum: fused SUM, type DECIMAL(P+1+ceil(log10 n_global), P).
 */
up_status up_sin_taylor(up_ctx *ctx, const up_column *x, int32_t P, up_column *out, void *stream);
up_status up_sin_taylor_sum(up_ctx *ctx, const up_column *x, int32_t P, int64_t n_global,
                            uint32_t *d_partial, void *stream);

/* Synchronise the stream and read + clear the sticky device flags:
 * UP_E_OVERFLOW / UP_E_DIVZERO / UP_E_RANGE / UP_E_INVAL (first in that order). */
up_status up_check(up_ctx *ctx, void *stream);

/* Format `limbs` two's-complement limbs (HOST memory) at scale s as the
 * canonical "[-]int.frac" string (exactly s fraction digits, no "-0"). */
up_status up_format_decimal(const uint32_t *limbs, int32_t nlimbs, int32_t s, char *buf, size_t len);

/* Number of kernels this ctx has launched (evidence for gpu_launches). */
uint64_t up_launch_count(up_ctx *ctx);
/* Milliseconds spent in NVRTC specialisation so far (excluded from timing). */
double up_jit_ms(up_ctx *ctx);

/* Diagnostics (no GPU needed).  up_gen_source: the CUDA source the
 * specialiser emits for variant "sum" or "eval" (cols supply types only).
 * up_nvrtc_compile: NVRTC-compile a source for sm_100a (ptxas -v log into
 * `log`; cubin written to cubin_path if non-NULL). */
up_status up_gen_source(const char *variant, const char *expr, const up_column *cols, int ncols,
                        int64_t n_global, char *buf, size_t len);
up_status up_nvrtc_compile(const char *src, const char *cubin_path, char *log, size_t len);
/* The expression after the optimiser (alignment scheduling + constant
 * pre-calculation; value-preserving, root kept at the
 * unoptimised type), as canonical text "tree : (p,s)" (no GPU needed). */
up_status up_expr_optimized(const char *expr, const up_column *cols, int ncols, char *buf, size_t len);
/* Generated row-contraction source for SUM(c1*c2) with La x Lb limbs (sign +1/-1). */
up_status up_gen_contract_source(int32_t La, int32_t Lb, int32_t LA, int sign, char *buf, size_t len);
/* Compile a generated source into the on-disk cubin cache ($UP_JIT_CACHE,
 * else <dir of libup.so>/_jitcache) so a GPU process loads it without NVRTC. */
up_status up_jit_prewarm(const char *src);
/* Generated sin_taylor source for x DECIMAL(p,s) (sum != 0: fused SUM variant). */
up_status up_gen_sin_source(int32_t P, int32_t p, int32_t s, int sum, int64_t n_global, char *buf, size_t len);
/* Generated grouped-aggregation source (arguments as up_group_aggregate). */
up_status up_gen_group_agg_source(int32_t n_aggs, const int32_t *kinds, const char *const *exprs,
                                  const up_column *cols, int ncols, int32_t n_groups, int64_t n_global,
                                  char *buf, size_t len);
/* Generated up_eval_tpi source for cols[0] <op> cols[1] (types / layouts only). */
up_status up_gen_tpi_source(const char *op, const up_column *cols, int32_t tpi, int32_t div_algo, char *buf, size_t len);
/* Generated modexp source for a DECIMAL(base_p,0) base (sum != 0: fused SUM variant). */
up_status up_gen_modexp_source(const char *exponent, const char *modulus, int32_t base_p, int sum,
                               int64_t n_global, char *buf, size_t len);

#ifdef __cplusplus
}
#endif
#endif /* UP_H */
