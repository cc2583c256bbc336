/*
 * oracle.c -- PreScaler CPU ORACLE.  TEST INFRASTRUCTURE ONLY: only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load this.  It shares no code with the CUDA path.
 *
 * Plain, slow, single-threaded C written to be checked against the paper by
 * eye.  Build: gcc -O2 -ffp-contract=off -fno-fast-math (no FMA contraction,
 * no FTZ/DAZ), x86-64 SSE arithmetic (float ops are IEEE single, double ops
 * IEEE double).  Every narrowing conversion goes through the software
 * bit-manipulation converter below, never an FPU conversion instruction.
 *
 * Precision codes: 0 f64, 1 f32, 2 f16 (the paper's), 3 bf16, 4 fp8
 * E4M3, 5 fp8 E5M2 (Blackwell extensions, DESIGN.md
 * readings #28/#29; fp8 objects carry a per-tensor power-of-two scale).
 *
 * What it computes (readings listed in DESIGN.md):
 *   a1 config decode   ("(1+#Conv_Types)^N", order P:293)
 *   a2 input conversion of every memory object to its assigned precision
 *      (device-side conversion, Fig. 3c; memory-object scaling P:55-57)
 *   a3 the precision-scaled application statements (readings R1-R5)
 *   a4 back-conversion of the outputs to their original type
 *   a5 mean-relative-error quality vs the fp64 run and the TOQ test
 *      "Accuracy < TOQ -> fail" (Alg. 1 line 10)
 *
 * Pins (tests/test_oracle_*.py): F16C hardware + numpy over all 2^32 fp32
 * inputs, numpy + AVX512-FP16 on fp64 inputs, paper fixed points
 * (tests/golden/), numpy float64 textbook results for every app, exact-integer
 * invariants for the reduction orders, closed forms for the quality metric.
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ===================================================================== */
/* c-1: software IEEE-754 converter                                      */
/* ===================================================================== */

typedef struct { int ebits, mbits, bias, has_inf; } fmt_t;
/* index = precision code: f64, f32, f16, bf16 (8 exponent, 7 fraction bits),
 * fp8 E4M3 and E5M2 (reading #29).  E4M3 (OCP "fn" variant) has no infinity:
 * its all-ones exponent field is an ordinary binade except fraction 111 = NaN,
 * so its largest finite value is 1.75 * 2^8 = 448; a rounded magnitude above
 * 448 (or an infinite input) becomes NaN.  E5M2 is IEEE-like (max 57344, inf). */
static const fmt_t FMT[6] = { {11, 52, 1023, 1}, {8, 23, 127, 1}, {5, 10, 15, 1}, {8, 7, 127, 1},
                              {4, 3, 7, 0}, {5, 2, 15, 1} };

/* number of significant bits of v (0 for v == 0) */
static int bitlen64(uint64_t v) { return v ? 64 - __builtin_clzll(v) : 0; }

/* Reading #5 (R-NaN): canonical NaN = every bit set except the sign bit. */
static uint64_t canonical_nan(const fmt_t *d) {
  int w = 1 + d->ebits + d->mbits;
  return (w == 64) ? 0x7FFFFFFFFFFFFFFFull : ((1ull << (w - 1)) - 1);
}

uint64_t oracle_convert_bits(uint64_t x, int st, int dt) {
  const fmt_t *s = &FMT[st], *d = &FMT[dt];
  int sw = 1 + s->ebits + s->mbits, dw = 1 + d->ebits + d->mbits;
  uint64_t sign = (x >> (sw - 1)) & 1u;
  uint64_t e = (x >> s->mbits) & ((1ull << s->ebits) - 1);
  uint64_t f = x & ((1ull << s->mbits) - 1);
  uint64_t emax_s = (1ull << s->ebits) - 1, emax_d = (1ull << d->ebits) - 1;
  uint64_t dsign = sign << (dw - 1);
  uint64_t S, K;
  int xexp, E, q, r, emin_d;

  /* step 2: inf / NaN (E4M3 source: only fraction all-ones is NaN, the rest of
   * its top binade is finite; E4M3 destination: no infinity, inf -> NaN) */
  if (e == emax_s && (s->has_inf || f == (1ull << s->mbits) - 1)) {
    if (f == 0 && s->has_inf) return d->has_inf ? (dsign | (emax_d << d->mbits)) : canonical_nan(d);
    return canonical_nan(d);
  }
  /* step 3: signed zero */
  if (e == 0 && f == 0) return dsign;
  /* step 4: value = S * 2^xexp */
  if (e == 0) { S = f; xexp = 1 - s->bias - s->mbits; }
  else        { S = f | (1ull << s->mbits); xexp = (int)e - s->bias - s->mbits; }
  /* step 5: unbiased exponent of the leading bit */
  E = bitlen64(S) - 1 + xexp;
  /* step 7.1: destination quantum exponent (subnormal floor emin_d) */
  emin_d = 1 - d->bias;
  q = (E > emin_d ? E : emin_d) - d->mbits;
  r = q - xexp;
  if (r <= 0) {
    K = S << (-r);                 /* exact (widening, or narrowing w/o loss) */
  } else if (r > bitlen64(S)) {
    K = 0;                         /* below half of the smallest quantum      */
  } else {
    /* step 7.4: round to nearest, ties to even */
    uint64_t rem = S & ((1ull << r) - 1), half = 1ull << (r - 1);
    K = S >> r;
    if (rem > half || (rem == half && (K & 1u))) K++;
  }
  if (K == 0) return dsign;
  /* step 8: encode */
  if (K >= (1ull << d->mbits)) {
    int64_t biased = (int64_t)q + d->mbits + d->bias;
    if (K == (1ull << (d->mbits + 1))) { K >>= 1; biased++; }
    if (!d->has_inf) {   /* E4M3: the top binade is finite up to fraction 110 */
      if (biased > (int64_t)emax_d || (biased == (int64_t)emax_d && K == (1ull << (d->mbits + 1)) - 1))
        return canonical_nan(d);                                           /* overflow -> NaN */
      return dsign | ((uint64_t)biased << d->mbits) | (K - (1ull << d->mbits));
    }
    if (biased >= (int64_t)emax_d) return dsign | (emax_d << d->mbits);   /* overflow -> inf */
    return dsign | ((uint64_t)biased << d->mbits) | (K - (1ull << d->mbits));
  }
  return dsign | K;                /* subnormal (q == emin_d - mbits) */
}

static int is_fp8(int t) { return t == OR_E4M3 || t == OR_E5M2; }

static uint64_t load_bits(const void *p, int t, size_t i) {
  switch (t) {
    case OR_F64: { uint64_t b; memcpy(&b, (const char *)p + 8 * i, 8); return b; }
    case OR_F32: { uint32_t b; memcpy(&b, (const char *)p + 4 * i, 4); return b; }
    case OR_E4M3: case OR_E5M2: return ((const uint8_t *)p)[i];
    default:     { uint16_t b; memcpy(&b, (const char *)p + 2 * i, 2); return b; }
  }
}
static void store_bits(void *p, int t, size_t i, uint64_t b) {
  switch (t) {
    case OR_F64: memcpy((char *)p + 8 * i, &b, 8); break;
    case OR_F32: { uint32_t v = (uint32_t)b; memcpy((char *)p + 4 * i, &v, 4); break; }
    case OR_E4M3: case OR_E5M2: ((uint8_t *)p)[i] = (uint8_t)b; break;
    default:     { uint16_t v = (uint16_t)b; memcpy((char *)p + 2 * i, &v, 2); break; }
  }
}

int oracle_convert(const void *src, int st, void *dst, int dt, size_t n) {
  size_t i;
  if (st < 0 || st > 5 || dt < 0 || dt > 5) return 1;
  if (n && (!src || !dst)) return 1;
  for (i = 0; i < n; i++) {
    uint64_t b = load_bits(src, st, i);
    store_bits(dst, dt, i, st == dt ? b : oracle_convert_bits(b, st, dt));
  }
  return 0;
}

static double bits_to_double(uint64_t b) { double d; memcpy(&d, &b, 8); return d; }
static uint64_t double_to_bits(double d) { uint64_t b; memcpy(&b, &d, 8); return b; }
static uint32_t float_to_bits(float f) { uint32_t b; memcpy(&b, &f, 4); return b; }
static float bits_to_float(uint32_t b) { float f; memcpy(&f, &b, 4); return f; }

/* exact widening of element i of a buffer of type t to double (fp8: the code's
 * own value, without the object's scale) */
static double widen(const void *p, int t, size_t i) {
  uint64_t b = load_bits(p, t, i);
  return bits_to_double(t == OR_F64 ? b : oracle_convert_bits(b, t, OR_F64));
}

/* ---- fp8 per-tensor power-of-two scale (reading #29) ------------------- */
static double fp8_max(int t) { return t == OR_E4M3 ? 448.0 : 57344.0; }

int oracle_fp8_scale_exp(double amax, int t) {
  int k;
  if (!(amax > 0.0)) return 0;
  for (k = ORACLE_FP8_KMIN; k <= ORACLE_FP8_KMAX; k++)
    if (amax <= ldexp(fp8_max(t), k)) return k;   /* ldexp: exact power-of-two scaling */
  return ORACLE_FP8_KMAX;
}
/* q = RNE_fp8(v * 2^-k): the product is exact in double (or, below 2^-1022,
 * far under half the smallest fp8 subnormal, so the code is +-0 either way) */
static uint64_t fp8_encode(double v, int k, int t) {
  return oracle_convert_bits(double_to_bits(ldexp(v, -k)), OR_F64, t);
}
static double fp8_decode(uint64_t q, int k, int t) {
  return ldexp(bits_to_double(oracle_convert_bits(q, t, OR_F64)), k);
}

int oracle_convert_scaled(const void *src, int st, void *dst, int dt, size_t n, int *k_io) {
  size_t i;
  double amax = 0.0;
  int k;
  if (st < 0 || st > 5 || dt < 0 || dt > 5) return 1;
  if (n && (!src || !dst)) return 1;
  if (!is_fp8(st) && !is_fp8(dt)) return oracle_convert(src, st, dst, dt, n);
  if (!k_io) return 1;
  if (!is_fp8(dt)) {                         /* decode: RNE_dst(q * 2^k) */
    for (i = 0; i < n; i++) {
      double v = fp8_decode(load_bits(src, st, i), *k_io, st);
      store_bits(dst, dt, i, dt == OR_F64 ? double_to_bits(v)
                                          : oracle_convert_bits(double_to_bits(v), OR_F64, dt));
    }
    return 0;
  }
  for (i = 0; i < n; i++) {                  /* amax over the finite source values */
    double v = is_fp8(st) ? fp8_decode(load_bits(src, st, i), *k_io, st) : widen(src, st, i);
    if (isfinite(v) && fabs(v) > amax) amax = fabs(v);
  }
  k = oracle_fp8_scale_exp(amax, dt);
  for (i = 0; i < n; i++) {
    double v = is_fp8(st) ? fp8_decode(load_bits(src, st, i), *k_io, st) : widen(src, st, i);
    store_bits(dst, dt, i, fp8_encode(v, k, dt));
  }
  *k_io = k;
  return 0;
}

/* ===================================================================== */
/* c-5: quality                                                          */
/* ===================================================================== */

void oracle_quality_accumulate(const void *out, int ot, const double *ref, size_t n,
                               double *sum_e, double *max_rel, uint64_t *nonfinite) {
  size_t i;
  for (i = 0; i < n; i++) {
    double o = widen(out, ot, i), r = ref[i], e, rel;
    if (!isfinite(o)) (*nonfinite)++;
    if (o == r) { e = 0.0; rel = 0.0; }
    else if (!isfinite(o) || !isfinite(r) || r == 0.0) { e = 1.0; rel = INFINITY; }
    else { rel = fabs(o - r) / fabs(r); e = rel < 1.0 ? rel : 1.0; }
    *sum_e = *sum_e + e;
    if (rel > *max_rel) *max_rel = rel;
  }
}

int oracle_quality(const void *out, int ot, const double *ref, size_t n,
                   oracle_quality_result *res) {
  double s = 0.0, mx = 0.0;
  uint64_t nf = 0;
  if (!res || ot < 0 || ot > 5) return 1;
  oracle_quality_accumulate(out, ot, ref, n, &s, &mx, &nf);
  res->n = n;
  res->mean_rel = n ? s / (double)n : 0.0;
  res->quality = 1.0 - res->mean_rel;
  res->max_rel = mx;
  res->nonfinite = nf;
  return 0;
}

/* ===================================================================== */
/* c-2: configuration codec                                              */
/* ===================================================================== */

/* id = sum_m code(m) * radix^m, object 0 least significant */
int oracle_config_decode_radix(int m, int radix, uint64_t id, int *prec) {
  int i;
  uint64_t space = 1;
  if (radix != 3 && radix != 4 && radix != 6) return 1;
  for (i = 0; i < m; i++) space *= (uint64_t)radix;
  if (m <= 0 || id >= space || !prec) return 1;
  for (i = 0; i < m; i++) { prec[i] = (int)(id % (uint64_t)radix); id /= (uint64_t)radix; }
  return 0;
}

int oracle_config_encode_radix(int m, int radix, const int *prec, uint64_t *id) {
  int i;
  uint64_t v = 0, w = 1;
  if (m <= 0 || !prec || !id || (radix != 3 && radix != 4 && radix != 6)) return 1;
  for (i = 0; i < m; i++) {
    if (prec[i] < 0 || prec[i] >= radix) return 1;
    v += (uint64_t)prec[i] * w;
    w *= (uint64_t)radix;
  }
  *id = v;
  return 0;
}

int oracle_config_decode(int m, uint64_t id, int *prec) { return oracle_config_decode_radix(m, 3, id, prec); }
int oracle_config_encode(int m, const int *prec, uint64_t *id) { return oracle_config_encode_radix(m, 3, prec, id); }

/* ===================================================================== */
/* R1/R2/R4: objects and arithmetic "in T"                               */
/* ===================================================================== */

/* An object stored in precision `type`.  In sampling mode (oracle_sample) an
 * input object may instead be "lazy": element i is RNE_type(src[i]) converted
 * on access from the original f32 data -- the same value a2 would have stored. */
/* An fp8 object (reading #29) also keeps val[i] = the exact current value
 * q_i * 2^k of every element, its scale exponent k, and a dirty flag: stores
 * inside a statement go to val; fp8_commit() at the end of every statement that
 * wrote the object re-quantises the whole object with a fresh per-tensor scale. */
typedef struct { int type; size_t n; void *p; const float *src; double *val; int k, dirty; } obj_t;

static size_t tsize(int t) { return t == OR_F64 ? 8 : (t == OR_F32 ? 4 : (is_fp8(t) ? 1 : 2)); }

/* R1: load = exact widening of the stored element */
static double ld(const obj_t *o, size_t i) {
  if (o->val) return o->val[i];              /* fp8: q_i * 2^k (or this statement's store) */
  if (o->src) {
    uint32_t b;
    memcpy(&b, &o->src[i], 4);
    uint64_t s = o->type == OR_F32 ? b : oracle_convert_bits(b, OR_F32, o->type);
    return bits_to_double(o->type == OR_F64 ? s : oracle_convert_bits(s, o->type, OR_F64));
  }
  return widen(o->p, o->type, i);
}

/* R1: store = RNE from the compute type T to the object's precision.  The
 * value v is exactly representable in T. */
static void st(obj_t *o, size_t i, double v, int T) {
  uint64_t b;
  if (o->val) {                              /* fp8: keep the value in T until the commit */
    o->val[i] = (T == OR_F64) ? v : (double)(float)v;
    o->dirty = 1;
    return;
  }
  if (o->type == OR_F64) { ((double *)o->p)[i] = v; return; }
  if (T == OR_F64) b = oracle_convert_bits(double_to_bits(v), OR_F64, o->type);
  else if (o->type == OR_F32) b = float_to_bits((float)v);        /* exact: v is f32 */
  else b = oracle_convert_bits(float_to_bits((float)v), OR_F32, o->type);   /* f16 / bf16 */
  store_bits(o->p, o->type, i, b);
}

/* Reading #29: end of a statement that wrote fp8 object o -- amax over its
 * finite values, k, then every element re-encoded as RNE_fp8(v * 2^-k). */
static void fp8_commit(obj_t *o) {
  size_t i;
  double amax = 0.0;
  if (!o->val || !o->dirty) return;
  for (i = 0; i < o->n; i++)
    if (isfinite(o->val[i]) && fabs(o->val[i]) > amax) amax = fabs(o->val[i]);
  o->k = oracle_fp8_scale_exp(amax, o->type);
  for (i = 0; i < o->n; i++) {
    uint64_t q = fp8_encode(o->val[i], o->k, o->type);
    store_bits(o->p, o->type, i, q);
    o->val[i] = fp8_decode(q, o->k, o->type);
  }
  o->dirty = 0;
}

/* R2: T = widest of the touched objects, floored at f32 (code 0 = widest; f16,
 * bf16, e4m3 and e5m2, codes 2-5, are all narrower than f32, so they compute in f32) */
static int W2(int a, int b) { int t = a < b ? a : b; return t < OR_F32 ? t : OR_F32; }
static int W3(int a, int b, int c) { return W2(W2(a, b), c); }

/* R4: single correctly rounded IEEE operations in T.  Operands are exactly
 * representable in T, so the (float) casts below are exact. */
static double t_add(int T, double a, double b) {
  return T == OR_F64 ? a + b : (double)((float)a + (float)b);
}
static double t_sub(int T, double a, double b) {
  return T == OR_F64 ? a - b : (double)((float)a - (float)b);
}
static double t_mul(int T, double a, double b) {
  return T == OR_F64 ? a * b : (double)((float)a * (float)b);
}
static double t_div(int T, double a, double b) {
  return T == OR_F64 ? a / b : (double)((float)a / (float)b);
}
static double t_fma(int T, double a, double b, double c) {
  return T == OR_F64 ? fma(a, b, c) : (double)fmaf((float)a, (float)b, (float)c);
}
static double t_sqrt(int T, double a) {
  return T == OR_F64 ? sqrt(a) : (double)sqrtf((float)a);
}
/* R2: scalars are RNE-rounded from their fp64 literal to T */
static double t_lit(int T, double lit) {
  if (T == OR_F64) return lit;
  return (double)bits_to_float((uint32_t)oracle_convert_bits(double_to_bits(lit), OR_F64, OR_F32));
}

/* ===================================================================== */
/* R3 / R5: canonical reduction orders                                   */
/* ===================================================================== */

/* R3: C_ij-style contraction: acc <- fma(a_k, b_k, acc) from +0, k ascending.
 * a(k) = A[ai + k*ask], b(k) = B[bi + k*bsk]. */
static double dot_chain(int T, const obj_t *A, size_t ai, size_t ask,
                        const obj_t *B, size_t bi, size_t bsk, size_t K) {
  double acc = 0.0;
  size_t k;
  for (k = 0; k < K; k++) acc = t_fma(T, ld(A, ai + k * ask), ld(B, bi + k * bsk), acc);
  return acc;
}

/* R5 row-dot: y = sum_j A[row, j] x_j for a row of length n, hierarchically:
 *  - chunk: lane l of a 32-lane slab owns the V = 16 / sizeof(stored A)
 *    consecutive elements j = 32*V*s + l*V + v and runs an fma chain over them
 *    from +0 (v ascending; elements past n are skipped);
 *  - slab s (32*V columns): the 32 lane values combine by xor butterfly with
 *    offsets 16,8,4,2,1 as a + partner;
 *  - tile (ORACLE_ROWDOT_TILE slabs): slab sums added left to right;
 *  - row: tile sums added left to right. */
static double rowdot(int T, const obj_t *A, size_t row0, size_t n, const obj_t *x) {
  double lane[ORACLE_ROWDOT_LANES], nxt[ORACLE_ROWDOT_LANES];
  /* an fp8 matrix is decoded into T before the statement (reading #29), so its
   * lane chunk is that of T */
  size_t V = 16 / (is_fp8(A->type) ? tsize(T) : tsize(A->type)), W = ORACLE_ROWDOT_LANES * V;
  size_t nslab = (n + W - 1) / W, s, v;
  double total = 0.0, tile = 0.0;
  int l, off;
  for (s = 0; s < nslab; s++) {
    for (l = 0; l < ORACLE_ROWDOT_LANES; l++) {
      lane[l] = 0.0;
      for (v = 0; v < V; v++) {
        size_t j = s * W + (size_t)l * V + v;
        if (j < n) lane[l] = t_fma(T, ld(A, row0 + j), ld(x, j), lane[l]);
      }
    }
    for (off = ORACLE_ROWDOT_LANES / 2; off >= 1; off >>= 1) {
      for (l = 0; l < ORACLE_ROWDOT_LANES; l++) nxt[l] = t_add(T, lane[l], lane[l ^ off]);
      memcpy(lane, nxt, sizeof(lane));
    }
    tile = (s % ORACLE_ROWDOT_TILE == 0) ? lane[0] : t_add(T, tile, lane[0]);
    if (s % ORACLE_ROWDOT_TILE == ORACLE_ROWDOT_TILE - 1 || s == nslab - 1)
      total = (s < ORACLE_ROWDOT_TILE) ? tile : t_add(T, total, tile);
  }
  return total;
}

/* R5 column-sum: z_j = sum_i A_ij w_i.  Rows are split into chunks of
 * ORACLE_COLSUM_CHUNK; each chunk runs an fma chain from +0 (i ascending);
 * the chunk partials are added in ascending chunk order (total = p_0 first).
 * mode 0: term fma(A_ij, w_i, p); mode 1: p + A_ij (w ignored);
 * mode 2: d = A_ij - mu_j, fma(d, d, p) (mu = w, indexed by column). */
static double colsum(int T, const obj_t *A, size_t nrows, size_t ncols, size_t j,
                     const obj_t *w, int mode) {
  double total = 0.0, p;
  size_t c0, i;
  for (c0 = 0; c0 < nrows; c0 += ORACLE_COLSUM_CHUNK) {
    size_t c1 = c0 + ORACLE_COLSUM_CHUNK < nrows ? c0 + ORACLE_COLSUM_CHUNK : nrows;
    p = 0.0;
    for (i = c0; i < c1; i++) {
      double a = ld(A, i * ncols + j);
      if (mode == 0) p = t_fma(T, a, ld(w, i), p);
      else if (mode == 1) p = t_add(T, p, a);
      else { double d = t_sub(T, a, ld(w, j)); p = t_fma(T, d, d, p); }
    }
    total = (c0 == 0) ? p : t_add(T, total, p);
  }
  return total;
}

/* ===================================================================== */
/* c-4: applications                                                     */
/* ===================================================================== */

typedef struct {
  const char *kind;
  int nobj, ndims_full;
  const char *names[8];
  int roles[8];
  int outputs[8];
} app_def_t;

/* object order = configuration-id digit order (c-2) */
static const app_def_t APPS[] = {
  {"gemm", 3, 3, {"A", "B", "C"}, {0, 0, 2}, {0, 0, 1}},
  {"2mm", 5, 4, {"A", "B", "C", "D", "E"}, {0, 0, 3, 0, 1}, {0, 0, 0, 0, 1}},
  {"3mm", 7, 5, {"A", "B", "C", "D", "E", "F", "G"}, {0, 0, 0, 0, 3, 3, 1}, {0, 0, 0, 0, 0, 0, 1}},
  {"atax", 4, 2, {"A", "x", "y", "tmp"}, {0, 0, 1, 3}, {0, 0, 1, 0}},
  {"bicg", 5, 2, {"A", "r", "s", "p", "q"}, {0, 0, 1, 0, 1}, {0, 0, 1, 0, 1}},
  {"gesummv", 5, 1, {"A", "B", "x", "y", "tmp"}, {0, 0, 0, 1, 3}, {0, 0, 0, 1, 0}},
  {"corr", 4, 2, {"data", "mean", "stddev", "symmat"}, {2, 3, 3, 1}, {0, 0, 0, 1}},
  {"covar", 3, 2, {"data", "mean", "symmat"}, {2, 3, 1}, {0, 0, 1}},
  {"mvt", 5, 1, {"A", "x1", "x2", "y1", "y2"}, {0, 2, 2, 0, 0}, {0, 1, 1, 0, 0}},
  {"syrk", 2, 2, {"A", "C"}, {0, 2}, {0, 1}},
  {"conv2d", 2, 2, {"A", "B"}, {0, 1}, {0, 1}},
  {"syr2k", 3, 2, {"A", "B", "C"}, {0, 0, 2}, {0, 0, 1}},
  {"conv3d", 2, 3, {"A", "B"}, {0, 1}, {0, 1}},
  {"fdtd2d", 4, 3, {"fict", "ex", "ey", "hz"}, {0, 2, 2, 2}, {0, 1, 1, 1}},
};

static const app_def_t *find_app(const char *kind) {
  size_t i;
  if (!kind) return NULL;
  for (i = 0; i < sizeof(APPS) / sizeof(APPS[0]); i++)
    if (strcmp(APPS[i].kind, kind) == 0) return &APPS[i];
  return NULL;
}

/* expand dims: ndims == 1 means every dimension equals dims[0] */
static int full_dims(const app_def_t *a, const int64_t *dims, int ndims, int64_t *d) {
  int i;
  if (!dims || (ndims != 1 && ndims != a->ndims_full)) return 1;
  for (i = 0; i < a->ndims_full; i++) {
    d[i] = (ndims == 1) ? dims[0] : dims[i];
    if (d[i] <= 0) return 1;
  }
  return 0;
}

static void shapes(const app_def_t *a, const int64_t *d, int64_t rows[8], int64_t cols[8]) {
  int i;
  for (i = 0; i < 8; i++) { rows[i] = 1; cols[i] = 1; }
  if (!strcmp(a->kind, "gemm")) {            /* NI, NJ, NK */
    rows[0] = d[0]; cols[0] = d[2];          /* A NI x NK */
    rows[1] = d[2]; cols[1] = d[1];          /* B NK x NJ */
    rows[2] = d[0]; cols[2] = d[1];          /* C NI x NJ */
  } else if (!strcmp(a->kind, "2mm")) {      /* NI, NJ, NK, NL */
    rows[0] = d[0]; cols[0] = d[2];          /* A NI x NK */
    rows[1] = d[2]; cols[1] = d[1];          /* B NK x NJ */
    rows[2] = d[0]; cols[2] = d[1];          /* C NI x NJ */
    rows[3] = d[1]; cols[3] = d[3];          /* D NJ x NL */
    rows[4] = d[0]; cols[4] = d[3];          /* E NI x NL */
  } else if (!strcmp(a->kind, "3mm")) {      /* NI, NJ, NK, NL, NM */
    rows[0] = d[0]; cols[0] = d[2];          /* A NI x NK */
    rows[1] = d[2]; cols[1] = d[1];          /* B NK x NJ */
    rows[2] = d[1]; cols[2] = d[4];          /* C NJ x NM */
    rows[3] = d[4]; cols[3] = d[3];          /* D NM x NL */
    rows[4] = d[0]; cols[4] = d[1];          /* E NI x NJ */
    rows[5] = d[1]; cols[5] = d[3];          /* F NJ x NL */
    rows[6] = d[0]; cols[6] = d[3];          /* G NI x NL */
  } else if (!strcmp(a->kind, "atax")) {     /* NX, NY */
    rows[0] = d[0]; cols[0] = d[1];          /* A NX x NY */
    cols[1] = d[1];                          /* x NY */
    cols[2] = d[1];                          /* y NY */
    cols[3] = d[0];                          /* tmp NX */
  } else if (!strcmp(a->kind, "bicg")) {     /* NX, NY */
    rows[0] = d[0]; cols[0] = d[1];          /* A NX x NY */
    cols[1] = d[0];                          /* r NX */
    cols[2] = d[1];                          /* s NY */
    cols[3] = d[1];                          /* p NY */
    cols[4] = d[0];                          /* q NX */
  } else if (!strcmp(a->kind, "gesummv")) {  /* N */
    rows[0] = d[0]; cols[0] = d[0];
    rows[1] = d[0]; cols[1] = d[0];
    cols[2] = d[0]; cols[3] = d[0]; cols[4] = d[0];
  } else if (!strcmp(a->kind, "corr")) {     /* N rows, M cols */
    rows[0] = d[0]; cols[0] = d[1];          /* data N x M */
    cols[1] = d[1]; cols[2] = d[1];          /* mean, stddev M */
    rows[3] = d[1]; cols[3] = d[1];          /* symmat M x M */
  } else if (!strcmp(a->kind, "covar")) {    /* N rows, M cols */
    rows[0] = d[0]; cols[0] = d[1];
    cols[1] = d[1];
    rows[2] = d[1]; cols[2] = d[1];
  } else if (!strcmp(a->kind, "mvt")) {      /* N */
    rows[0] = d[0]; cols[0] = d[0];
    cols[1] = d[0]; cols[2] = d[0]; cols[3] = d[0]; cols[4] = d[0];
  } else if (!strcmp(a->kind, "syrk")) {     /* A: N x M, C: M x M */
    rows[0] = d[0]; cols[0] = d[1];
    rows[1] = d[1]; cols[1] = d[1];
  } else if (!strcmp(a->kind, "conv2d")) {   /* NI x NJ */
    rows[0] = d[0]; cols[0] = d[1];
    rows[1] = d[0]; cols[1] = d[1];
  } else if (!strcmp(a->kind, "syr2k")) {    /* A, B: N x M; C: M x M */
    rows[0] = d[0]; cols[0] = d[1];
    rows[1] = d[0]; cols[1] = d[1];
    rows[2] = d[1]; cols[2] = d[1];
  } else if (!strcmp(a->kind, "conv3d")) {   /* NI x (NJ NK) */
    rows[0] = d[0]; cols[0] = d[1] * d[2];
    rows[1] = d[0]; cols[1] = d[1] * d[2];
  } else {                                   /* fdtd2d: TMAX, NX, NY */
    cols[0] = d[0];
    rows[1] = d[1]; cols[1] = d[2];
    rows[2] = d[1]; cols[2] = d[2];
    rows[3] = d[1]; cols[3] = d[2];
  }
}

int oracle_app_objects(const char *kind, const int64_t *dims, int ndims, oracle_object_info *info) {
  const app_def_t *a = find_app(kind);
  int64_t d[8], rows[8], cols[8];
  int m;
  if (!a || full_dims(a, dims, ndims, d)) return -1;
  shapes(a, d, rows, cols);
  if (info) {
    for (m = 0; m < a->nobj; m++) {
      info[m].name = a->names[m];
      info[m].role = a->roles[m];
      info[m].is_output = a->outputs[m];
      info[m].rows = rows[m];
      info[m].cols = cols[m];
    }
  }
  return a->nobj;
}

/* default scalars (reading #18): gemm alpha,beta; gesummv alpha,beta; corr eps */
static double scalar_or(const double *s, int i, double dflt) { return s ? s[i] : dflt; }

static void app_gemm(obj_t *o, const int64_t *d, const double *sc) {
  /* C <- alpha * (A . B) + beta * C   (R3 epilogue r = fma(alpha, acc, beta*C)) */
  size_t NI = d[0], NJ = d[1], NK = d[2], i, j;
  int T = W3(o[0].type, o[1].type, o[2].type);
  double al = t_lit(T, scalar_or(sc, 0, 32412.0)), be = t_lit(T, scalar_or(sc, 1, 2123.0));
  for (i = 0; i < NI; i++)
    for (j = 0; j < NJ; j++) {
      double acc = dot_chain(T, &o[0], i * NK, 1, &o[1], j, NJ, NK);
      double bc = t_mul(T, be, ld(&o[2], i * NJ + j));
      st(&o[2], i * NJ + j, t_fma(T, al, acc, bc), T);
    }
  fp8_commit(&o[2]);
}

/* out[i][j] <- sum_k A[i][k] B[k][j] (no epilogue), R3 order */
static void matmul(obj_t *A, obj_t *B, obj_t *C, size_t NI, size_t NJ, size_t NK) {
  size_t i, j;
  int T = W3(A->type, B->type, C->type);
  for (i = 0; i < NI; i++)
    for (j = 0; j < NJ; j++) st(C, i * NJ + j, dot_chain(T, A, i * NK, 1, B, j, NJ, NK), T);
  fp8_commit(C);
}

static void app_2mm(obj_t *o, const int64_t *d) {
  size_t NI = d[0], NJ = d[1], NK = d[2], NL = d[3];
  matmul(&o[0], &o[1], &o[2], NI, NJ, NK);   /* C <- A . B */
  matmul(&o[2], &o[3], &o[4], NI, NL, NJ);   /* E <- C . D */
}

static void app_3mm(obj_t *o, const int64_t *d) {
  size_t NI = d[0], NJ = d[1], NK = d[2], NL = d[3], NM = d[4];
  matmul(&o[0], &o[1], &o[4], NI, NJ, NK);   /* E <- A . B */
  matmul(&o[2], &o[3], &o[5], NJ, NL, NM);   /* F <- C . D */
  matmul(&o[4], &o[5], &o[6], NI, NL, NJ);   /* G <- E . F */
}

static void app_atax(obj_t *o, const int64_t *d) {
  size_t NX = d[0], NY = d[1], i, j;
  int T1 = W3(o[0].type, o[1].type, o[3].type), T2 = W3(o[0].type, o[3].type, o[2].type);
  for (i = 0; i < NX; i++) st(&o[3], i, rowdot(T1, &o[0], i * NY, NY, &o[1]), T1);  /* tmp <- A x */
  fp8_commit(&o[3]);
  for (j = 0; j < NY; j++) st(&o[2], j, colsum(T2, &o[0], NX, NY, j, &o[3], 0), T2); /* y <- A^T tmp */
  fp8_commit(&o[2]);
}

static void app_bicg(obj_t *o, const int64_t *d) {
  size_t NX = d[0], NY = d[1], i, j;
  int T1 = W3(o[0].type, o[1].type, o[2].type), T2 = W3(o[0].type, o[3].type, o[4].type);
  for (j = 0; j < NY; j++) st(&o[2], j, colsum(T1, &o[0], NX, NY, j, &o[1], 0), T1); /* s <- A^T r */
  fp8_commit(&o[2]);
  for (i = 0; i < NX; i++) st(&o[4], i, rowdot(T2, &o[0], i * NY, NY, &o[3]), T2);  /* q <- A p */
  fp8_commit(&o[4]);
}

static void app_gesummv(obj_t *o, const int64_t *d, const double *sc) {
  size_t N = d[0], i;
  int T1 = W3(o[0].type, o[2].type, o[4].type);   /* tmp <- A x */
  int T2 = W3(o[1].type, o[2].type, o[3].type);   /* y   <- B x */
  int T3 = W2(o[4].type, o[3].type);              /* y   <- alpha tmp + beta y */
  double al = t_lit(T3, scalar_or(sc, 0, 43532.0)), be = t_lit(T3, scalar_or(sc, 1, 12313.0));
  for (i = 0; i < N; i++) st(&o[4], i, rowdot(T1, &o[0], i * N, N, &o[2]), T1);
  fp8_commit(&o[4]);
  for (i = 0; i < N; i++) st(&o[3], i, rowdot(T2, &o[1], i * N, N, &o[2]), T2);
  fp8_commit(&o[3]);
  for (i = 0; i < N; i++)
    st(&o[3], i, t_fma(T3, al, ld(&o[4], i), t_mul(T3, be, ld(&o[3], i))), T3);
  fp8_commit(&o[3]);
}

/* symmetric product sym[j1][j2] = sym[j2][j1] = sum_i X_ij1 X_ij2 (R3),
 * j1 < j2 (diag_one) or j1 <= j2; divided by div if div != 0. */
static void syrk_upper(obj_t *X, obj_t *S, size_t N, size_t M, int diag_one, double div_lit) {
  size_t j1, j2;
  int T = W2(X->type, S->type);
  double dv = div_lit != 0.0 ? t_lit(T, div_lit) : 0.0;
  for (j1 = 0; j1 < M; j1++) {
    if (diag_one) st(S, j1 * M + j1, 1.0, T);
    for (j2 = diag_one ? j1 + 1 : j1; j2 < M; j2++) {
      double acc = dot_chain(T, X, j1, M, X, j2, M, N);
      if (div_lit != 0.0) acc = t_div(T, acc, dv);
      st(S, j1 * M + j2, acc, T);
      st(S, j2 * M + j1, acc, T);
    }
  }
  fp8_commit(S);
}

static void col_mean(obj_t *data, obj_t *mean, size_t N, size_t M) {
  size_t j;
  int T = W2(data->type, mean->type);
  double n = t_lit(T, (double)N);
  for (j = 0; j < M; j++) st(mean, j, t_div(T, colsum(T, data, N, M, j, NULL, 1), n), T);
  fp8_commit(mean);
}

static void app_corr(obj_t *o, const int64_t *d, const double *sc) {
  size_t N = d[0], M = d[1], i, j;
  int T2 = W3(o[0].type, o[1].type, o[2].type), T3 = T2;
  double n2 = t_lit(T2, (double)N), eps = t_lit(T2, scalar_or(sc, 0, 0.005));
  double sqn = t_lit(T3, sqrt((double)N));
  col_mean(&o[0], &o[1], N, M);                                   /* mean */
  for (j = 0; j < M; j++) {                                       /* stddev */
    double s = t_sqrt(T2, t_div(T2, colsum(T2, &o[0], N, M, j, &o[1], 2), n2));
    st(&o[2], j, s <= eps ? 1.0 : s, T2);
  }
  fp8_commit(&o[2]);
  for (i = 0; i < N; i++)                                         /* normalise */
    for (j = 0; j < M; j++) {
      double dd = t_sub(T3, ld(&o[0], i * M + j), ld(&o[1], j));
      st(&o[0], i * M + j, t_div(T3, dd, t_mul(T3, sqn, ld(&o[2], j))), T3);
    }
  fp8_commit(&o[0]);
  syrk_upper(&o[0], &o[3], N, M, 1, 0.0);                         /* symmat */
}

static void app_covar(obj_t *o, const int64_t *d) {
  size_t N = d[0], M = d[1], i, j;
  int T2 = W2(o[0].type, o[1].type);
  col_mean(&o[0], &o[1], N, M);                                   /* mean */
  for (i = 0; i < N; i++)                                         /* centre */
    for (j = 0; j < M; j++)
      st(&o[0], i * M + j, t_sub(T2, ld(&o[0], i * M + j), ld(&o[1], j)), T2);
  fp8_commit(&o[0]);
  syrk_upper(&o[0], &o[2], N, M, 0, (double)N - 1.0);             /* symmat */
}

/* MVT: x1 <- x1 + A y1 (row-dot, R5) ; x2 <- x2 + A^T y2 (column-sum, R5) */
static void app_mvt(obj_t *o, const int64_t *d) {
  size_t N = d[0], i;
  int T1 = W3(o[0].type, o[1].type, o[3].type), T2 = W3(o[0].type, o[2].type, o[4].type);
  for (i = 0; i < N; i++)
    st(&o[1], i, t_add(T1, ld(&o[1], i), rowdot(T1, &o[0], i * N, N, &o[3])), T1);
  fp8_commit(&o[1]);
  for (i = 0; i < N; i++)
    st(&o[2], i, t_add(T2, ld(&o[2], i), colsum(T2, &o[0], N, N, i, &o[4], 0)), T2);
  fp8_commit(&o[2]);
}

/* SYRK (BLAS 'T' form, reading #23): C <- alpha A^T A + beta C over A: N x M,
 * C_j1j2 = fma(alpha, sum_k A_kj1 A_kj2, beta C_j1j2) for j1 <= j2 (R3), mirrored */
static void app_syrk(obj_t *o, const int64_t *d, const double *sc) {
  size_t N = d[0], M = d[1], j1, j2;
  int T = W2(o[0].type, o[1].type);
  double al = t_lit(T, scalar_or(sc, 0, 32412.0)), be = t_lit(T, scalar_or(sc, 1, 2123.0));
  for (j1 = 0; j1 < M; j1++)
    for (j2 = j1; j2 < M; j2++) {
      double acc = dot_chain(T, &o[0], j1, M, &o[0], j2, M, N);
      double r = t_fma(T, al, acc, t_mul(T, be, ld(&o[1], j1 * M + j2)));
      st(&o[1], j1 * M + j2, r, T);
      st(&o[1], j2 * M + j1, r, T);
    }
  fp8_commit(&o[1]);
}

/* 2DCONV (reading #24): B_ij = c11 A(i-1,j-1) + c12 A(i,j-1) + c13 A(i+1,j-1)
 *   + c21 A(i-1,j) + c22 A(i,j) + c23 A(i+1,j) + c31 A(i-1,j+1) + c32 A(i,j+1)
 *   + c33 A(i+1,j+1), each product rounded in T, sums left to right (no
 *   contraction, R4), for 1 <= i < NI-1, 1 <= j < NJ-1; border outputs +0. */
static const double CONV2D_C[9] = {0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10};
static double conv2d_at(int T, const obj_t *A, size_t NJ, size_t i, size_t j) {
  static const int di[9] = {-1, 0, 1, -1, 0, 1, -1, 0, 1};
  static const int dj[9] = {-1, -1, -1, 0, 0, 0, 1, 1, 1};
  double acc = 0.0;
  int k;
  for (k = 0; k < 9; k++) {
    double p = t_mul(T, t_lit(T, CONV2D_C[k]), ld(A, (i + di[k]) * NJ + (j + dj[k])));
    acc = (k == 0) ? p : t_add(T, acc, p);
  }
  return acc;
}
static void app_conv2d(obj_t *o, const int64_t *d) {
  size_t NI = d[0], NJ = d[1], i, j;
  int T = W2(o[0].type, o[1].type);
  for (i = 0; i < NI; i++)
    for (j = 0; j < NJ; j++) {
      int border = (i == 0 || j == 0 || i + 1 >= NI || j + 1 >= NJ);
      st(&o[1], i * NJ + j, border ? 0.0 : conv2d_at(T, &o[0], NJ, i, j), T);
    }
  fp8_commit(&o[1]);
}

/* SYR2K (BLAS 'T' form, reading #25): C <- alpha A^T B + beta C ; C <- alpha B^T A + C
 * (two statements, each an R3 chain and an RNE store of C) over A, B: N x M */
static void app_syr2k(obj_t *o, const int64_t *d, const double *sc) {
  size_t N = d[0], M = d[1], i, j;
  int T = W3(o[0].type, o[1].type, o[2].type);
  double al = t_lit(T, scalar_or(sc, 0, 32412.0)), be = t_lit(T, scalar_or(sc, 1, 2123.0));
  for (i = 0; i < M; i++)
    for (j = 0; j < M; j++) {
      double s1 = dot_chain(T, &o[0], i, M, &o[1], j, M, N);
      st(&o[2], i * M + j, t_fma(T, al, s1, t_mul(T, be, ld(&o[2], i * M + j))), T);
    }
  fp8_commit(&o[2]);
  for (i = 0; i < M; i++)
    for (j = 0; j < M; j++) {
      double s2 = dot_chain(T, &o[1], i, M, &o[0], j, M, N);
      st(&o[2], i * M + j, t_fma(T, al, s2, ld(&o[2], i * M + j)), T);
    }
  fp8_commit(&o[2]);
}

/* 3DCONV (reading #26): 27-point stencil on A[NI][NJ][NK]: the 2DCONV weights on
 * each (j,k)-plane (C9 index (dk+1)*3 + (dj+1)) scaled by g = (0.25, 0.5, 0.25)
 * for di = -1, 0, +1; weights formed in fp64 and RNE-rounded to T; products
 * rounded, summed left to right (di outer, then the 2DCONV order); border +0. */
static double conv3d_at(int T, const obj_t *A, size_t NJ, size_t NK, size_t i, size_t j, size_t k) {
  static const double g[3] = {0.25, 0.5, 0.25};
  double acc = 0.0;
  int p, q;
  for (p = 0; p < 3; p++)
    for (q = 0; q < 9; q++) {
      const int di = p - 1, dj = (q % 3) - 1, dk = (q / 3) - 1;
      double w = t_lit(T, g[p] * CONV2D_C[q]);
      double v = ld(A, ((i + di) * NJ + (j + dj)) * NK + (k + dk));
      double prod = t_mul(T, w, v);
      acc = (p == 0 && q == 0) ? prod : t_add(T, acc, prod);
    }
  return acc;
}
static void app_conv3d(obj_t *o, const int64_t *d) {
  size_t NI = d[0], NJ = d[1], NK = d[2], i, j, k;
  int T = W2(o[0].type, o[1].type);
  for (i = 0; i < NI; i++)
    for (j = 0; j < NJ; j++)
      for (k = 0; k < NK; k++) {
        int border = i == 0 || j == 0 || k == 0 || i + 1 >= NI || j + 1 >= NJ || k + 1 >= NK;
        st(&o[1], (i * NJ + j) * NK + k, border ? 0.0 : conv3d_at(T, &o[0], NJ, NK, i, j, k), T);
      }
  fp8_commit(&o[1]);
}

/* FDTD-2D (reading #27), TMAX steps over ex, ey, hz (NX x NY), each statement a
 * separate pass in its own compute type:
 *   ey[0][j] = fict[t]
 *   ey[i][j] = ey[i][j] - 0.5 (hz[i][j] - hz[i-1][j])            i >= 1
 *   ex[i][j] = ex[i][j] - 0.5 (hz[i][j] - hz[i][j-1])            j >= 1
 *   hz[i][j] = hz[i][j] - 0.7 (ex[i][j+1] - ex[i][j] + ey[i+1][j] - ey[i][j])
 *                                                   i < NX-1, j < NY-1 */
static void app_fdtd2d(obj_t *o, const int64_t *d) {
  size_t TM = d[0], NX = d[1], NY = d[2], t, i, j;
  int T1 = W2(o[0].type, o[2].type), T2 = W2(o[2].type, o[3].type);
  int T3 = W2(o[1].type, o[3].type), T4 = W3(o[3].type, o[1].type, o[2].type);
  double h2 = t_lit(T2, 0.5), h3 = t_lit(T3, 0.5), c4 = t_lit(T4, 0.7);
  for (t = 0; t < TM; t++) {
    for (j = 0; j < NY; j++) st(&o[2], j, ld(&o[0], t), T1);
    fp8_commit(&o[2]);   /* ey[0][j] = fict[t] is its own statement (reading #29) */
    for (i = 1; i < NX; i++)
      for (j = 0; j < NY; j++) {
        double dh = t_sub(T2, ld(&o[3], i * NY + j), ld(&o[3], (i - 1) * NY + j));
        st(&o[2], i * NY + j, t_sub(T2, ld(&o[2], i * NY + j), t_mul(T2, h2, dh)), T2);
      }
    fp8_commit(&o[2]);
    for (i = 0; i < NX; i++)
      for (j = 1; j < NY; j++) {
        double dh = t_sub(T3, ld(&o[3], i * NY + j), ld(&o[3], i * NY + j - 1));
        st(&o[1], i * NY + j, t_sub(T3, ld(&o[1], i * NY + j), t_mul(T3, h3, dh)), T3);
      }
    fp8_commit(&o[1]);
    for (i = 0; i + 1 < NX; i++)
      for (j = 0; j + 1 < NY; j++) {
        double s = t_sub(T4, ld(&o[1], i * NY + j + 1), ld(&o[1], i * NY + j));
        s = t_add(T4, s, ld(&o[2], (i + 1) * NY + j));
        s = t_sub(T4, s, ld(&o[2], i * NY + j));
        st(&o[3], i * NY + j, t_sub(T4, ld(&o[3], i * NY + j), t_mul(T4, c4, s)), T4);
      }
    fp8_commit(&o[3]);
  }
}

static int run_objects(const app_def_t *a, const int64_t *d, const double *sc, obj_t *o) {
  if (!strcmp(a->kind, "syr2k")) { app_syr2k(o, d, sc); return 0; }
  if (!strcmp(a->kind, "conv3d")) { app_conv3d(o, d); return 0; }
  if (!strcmp(a->kind, "fdtd2d")) { app_fdtd2d(o, d); return 0; }
  if (!strcmp(a->kind, "mvt")) { app_mvt(o, d); return 0; }
  if (!strcmp(a->kind, "syrk")) { app_syrk(o, d, sc); return 0; }
  if (!strcmp(a->kind, "conv2d")) { app_conv2d(o, d); return 0; }
  if (!strcmp(a->kind, "gemm")) app_gemm(o, d, sc);
  else if (!strcmp(a->kind, "2mm")) app_2mm(o, d);
  else if (!strcmp(a->kind, "3mm")) app_3mm(o, d);
  else if (!strcmp(a->kind, "atax")) app_atax(o, d);
  else if (!strcmp(a->kind, "bicg")) app_bicg(o, d);
  else if (!strcmp(a->kind, "gesummv")) app_gesummv(o, d, sc);
  else if (!strcmp(a->kind, "corr")) app_corr(o, d, sc);
  else app_covar(o, d);
  return 0;
}

static void free_objects(obj_t *o, int n) {
  int m;
  for (m = 0; m < n; m++) { free(o[m].p); free(o[m].val); }
}

/* a2 + a3 */
static int run_to_objects(const char *kind, const int64_t *dims, int ndims, const double *sc,
                          const int *prec, const float *const *inputs, obj_t *o, const app_def_t **pa,
                          int64_t *d) {
  const app_def_t *a = find_app(kind);
  int64_t rows[8], cols[8];
  int m;
  if (!a || full_dims(a, dims, ndims, d) || !prec) return 1;
  shapes(a, d, rows, cols);
  memset(o, 0, sizeof(obj_t) * 8);
  for (m = 0; m < a->nobj; m++) {
    if (prec[m] < 0 || prec[m] > 5) { free_objects(o, m); return 1; }
    o[m].type = prec[m];
    o[m].n = (size_t)(rows[m] * cols[m]);
    o[m].p = calloc(o[m].n ? o[m].n : 1, tsize(prec[m]));
    if (!o[m].p) { free_objects(o, m); return 1; }
    if (is_fp8(prec[m])) {                              /* reading #29: values + scale */
      o[m].val = (double *)calloc(o[m].n ? o[m].n : 1, sizeof(double));
      if (!o[m].val) { free_objects(o, m + 1); return 1; }
    }
    if (a->roles[m] == 0 || a->roles[m] == 2) {         /* a2: convert orig f32 -> c(m) */
      if (!inputs || !inputs[m]) { free_objects(o, m + 1); return 1; }
      if (is_fp8(prec[m])) {                            /* exact f32 values, then quantise */
        size_t i;
        for (i = 0; i < o[m].n; i++) o[m].val[i] = (double)inputs[m][i];
        o[m].dirty = 1;
        fp8_commit(&o[m]);
      } else {
        oracle_convert(inputs[m], OR_F32, o[m].p, prec[m], o[m].n);
      }
    }
  }
  run_objects(a, d, sc, o);
  *pa = a;
  return 0;
}

int oracle_run_config_k(const char *kind, const int64_t *dims, int ndims, const double *sc,
                        const int *prec, const float *const *inputs, void *const *finals,
                        int *scale_exps) {
  obj_t o[8];
  const app_def_t *a;
  int64_t d[8];
  int m;
  if (run_to_objects(kind, dims, ndims, sc, prec, inputs, o, &a, d)) return 1;
  for (m = 0; m < a->nobj; m++) {
    if (finals && finals[m]) memcpy(finals[m], o[m].p, o[m].n * tsize(o[m].type));
    if (scale_exps && is_fp8(o[m].type)) scale_exps[m] = o[m].k;
  }
  free_objects(o, a->nobj);
  return 0;
}

int oracle_run_config(const char *kind, const int64_t *dims, int ndims, const double *sc,
                      const int *prec, const float *const *inputs, void *const *finals) {
  return oracle_run_config_k(kind, dims, ndims, sc, prec, inputs, finals, NULL);
}

int oracle_evaluate(const char *kind, const int64_t *dims, int ndims, const double *sc,
                    const int *prec, const float *const *inputs, const double *const *ref,
                    float *const *delivered, oracle_quality_result *res) {
  obj_t o[8];
  const app_def_t *a;
  int64_t d[8];
  int m;
  double s = 0.0, mx = 0.0;
  uint64_t nf = 0, n = 0;
  if (!ref || !res) return 1;
  if (run_to_objects(kind, dims, ndims, sc, prec, inputs, o, &a, d)) return 1;
  for (m = 0; m < a->nobj; m++) {
    float *buf;
    if (!a->outputs[m]) continue;
    /* a4: back-conversion c(o) -> orig (f32) */
    buf = (delivered && delivered[m]) ? delivered[m] : (float *)malloc(o[m].n * 4 + 4);
    if (o[m].val) {                         /* fp8: RNE_f32(q * 2^k) */
      size_t i;
      for (i = 0; i < o[m].n; i++)
        buf[i] = bits_to_float((uint32_t)oracle_convert_bits(double_to_bits(o[m].val[i]), OR_F64, OR_F32));
    } else {
      oracle_convert(o[m].p, o[m].type, buf, OR_F32, o[m].n);
    }
    /* a5: quality of the delivered output vs the fp64 run */
    oracle_quality_accumulate(buf, OR_F32, ref[m], o[m].n, &s, &mx, &nf);
    n += o[m].n;
    if (!(delivered && delivered[m])) free(buf);
  }
  free_objects(o, a->nobj);
  res->n = n;
  res->mean_rel = n ? s / (double)n : 0.0;
  res->quality = 1.0 - res->mean_rel;
  res->max_rel = mx;
  res->nonfinite = nf;
  return 0;
}

/* ===================================================================== */
/* Sampled evaluation (parity at the BASELINE sizes)                     */
/* ===================================================================== */
/* Raw final values of output object m at entries (rows[k], cols[k]) for one
 * configuration, computed with the SAME helpers, compute types and orders as
 * oracle_run_config, touching only what those entries depend on.  Input
 * objects are lazy views of the f32 inputs (a2 applied per element on load).
 * tests/test_oracle_sample.py pins it against the full run. */

static double round_to(int type, double v, int T) {
  unsigned char buf[8];
  obj_t o = {type, 1, buf, NULL, NULL, 0, 0};
  st(&o, 0, v, T);
  return ld(&o, 0);
}
static obj_t new_obj(int type, size_t n) {
  obj_t o = {type, n, calloc(n ? n : 1, tsize(type)), NULL, NULL, 0, 0};
  return o;
}

/* CORR/COVAR: column j of data after the statements that precede the SYRK
 * (mean; stddev and normalisation for CORR; centring for COVAR) into z. */
static void stats_column(int corr, obj_t *data, obj_t *mean, obj_t *sd, size_t N, size_t M,
                         size_t j, double eps_lit, obj_t *z) {
  int T1 = W2(data->type, mean->type);
  size_t i;
  st(mean, j, t_div(T1, colsum(T1, data, N, M, j, NULL, 1), t_lit(T1, (double)N)), T1);
  if (corr) {
    int T2 = W3(data->type, mean->type, sd->type);
    double s = t_sqrt(T2, t_div(T2, colsum(T2, data, N, M, j, mean, 2), t_lit(T2, (double)N)));
    double sqn = t_lit(T2, sqrt((double)N));
    st(sd, j, s <= t_lit(T2, eps_lit) ? 1.0 : s, T2);
    for (i = 0; i < N; i++) {
      double dd = t_sub(T2, ld(data, i * M + j), ld(mean, j));
      st(z, i, t_div(T2, dd, t_mul(T2, sqn, ld(sd, j))), T2);
    }
  } else {
    int T2 = W2(data->type, mean->type);
    for (i = 0; i < N; i++) st(z, i, t_sub(T2, ld(data, i * M + j), ld(mean, j)), T2);
  }
}

/* Sampling speed only (no arithmetic change): the exact values of o[0..n), as ld
 * returns them, cached in o->val so repeated loads skip the software widening.
 * The object must not be stored to while cached (ld prefers val). */
static double *cache_values(obj_t *o) {
  size_t i;
  double *buf = (double *)malloc(sizeof(double) * (o->n ? o->n : 1));
  o->val = NULL;
  for (i = 0; i < o->n; i++) buf[i] = ld(o, i);
  o->val = buf;
  return buf;
}

/* sorted distinct values of v[0..n): out[0] = count, out[1..] = values (malloc) */
static int cmp_i64(const void *x, const void *y) {
  int64_t a = *(const int64_t *)x, b = *(const int64_t *)y;
  return a < b ? -1 : (a > b ? 1 : 0);
}
static int64_t *uniq(const int64_t *v, size_t n, void *unused) {
  int64_t *o = (int64_t *)malloc(sizeof(int64_t) * (n + 1));
  size_t k, c = 0;
  (void)unused;
  if (n) memcpy(o + 1, v, sizeof(int64_t) * n);
  qsort(o + 1, n, sizeof(int64_t), cmp_i64);
  for (k = 0; k < n; k++)
    if (c == 0 || o[1 + k] != o[c]) o[1 + c++] = o[1 + k];
  o[0] = (int64_t)c;
  return o;
}
static size_t uniq_index(const int64_t *u, int64_t x) {
  size_t lo = 0, hi = (size_t)u[0];
  while (lo + 1 < hi) {
    size_t mid = (lo + hi) / 2;
    if (u[1 + mid] <= x) lo = mid; else hi = mid;
  }
  return lo;
}

int oracle_sample(const char *kind, const int64_t *dims, int ndims, const double *sc,
                  const int *prec, const float *const *inputs, int m, const int64_t *rows,
                  const int64_t *cols, size_t n, double *vals) {
  const app_def_t *a = find_app(kind);
  int64_t d[8], R[8], C[8];
  obj_t in[8];
  size_t k;
  int t;
  if (!a || full_dims(a, dims, ndims, d) || !prec || m < 0 || m >= a->nobj || !a->outputs[m] ||
      (n && (!rows || !cols || !vals)))
    return 1;
  shapes(a, d, R, C);
  memset(in, 0, sizeof(in));
  for (t = 0; t < a->nobj; t++) {
    if (prec[t] < 0 || prec[t] > 3) return 1;   /* fp8 (per-tensor scale): not sampleable */
    in[t].type = prec[t];
    in[t].n = (size_t)(R[t] * C[t]);
    if (a->roles[t] == 0 || a->roles[t] == 2) {
      if (!inputs || !inputs[t]) return 1;
      in[t].src = inputs[t];
    }
  }
  for (k = 0; k < n; k++)
    if (rows[k] < 0 || rows[k] >= R[m] || cols[k] < 0 || cols[k] >= C[m]) return 1;
  if (strcmp(kind, "fdtd2d"))
    for (t = 0; t < a->nobj; t++)
      if (in[t].src) cache_values(&in[t]);

  if (!strcmp(kind, "gemm")) {
    size_t NJ = d[1], NK = d[2];
    int T = W3(prec[0], prec[1], prec[2]);
    double al = t_lit(T, scalar_or(sc, 0, 32412.0)), be = t_lit(T, scalar_or(sc, 1, 2123.0));
    for (k = 0; k < n; k++) {
      size_t i = rows[k], j = cols[k];
      double acc = dot_chain(T, &in[0], i * NK, 1, &in[1], j, NJ, NK);
      double bc = t_mul(T, be, ld(&in[2], i * NJ + j));
      vals[k] = round_to(prec[2], t_fma(T, al, acc, bc), T);
    }
  } else if (!strcmp(kind, "2mm")) {
    size_t NJ = d[1], NK = d[2], NL = d[3], j;
    int T1 = W3(prec[0], prec[1], prec[2]), T2 = W3(prec[2], prec[3], prec[4]);
    obj_t crow = new_obj(prec[2], NJ);
    int64_t cached = -1;
    for (k = 0; k < n; k++) {
      size_t i = rows[k], l = cols[k];
      if ((int64_t)i != cached) {           /* row i of C <- A . B */
        free(crow.val);
        crow.val = NULL;
        for (j = 0; j < NJ; j++) st(&crow, j, dot_chain(T1, &in[0], i * NK, 1, &in[1], j, NJ, NK), T1);
        cache_values(&crow);
        cached = (int64_t)i;
      }
      vals[k] = round_to(prec[4], dot_chain(T2, &crow, 0, 1, &in[3], l, NL, NJ), T2);
    }
    free(crow.p);
    free(crow.val);
  } else if (!strcmp(kind, "3mm")) {
    /* every distinct row i of E <- A . B and column l of F <- C . D is computed
     * once (no arithmetic difference: each is the same R3 chain) */
    size_t NJ = d[1], NK = d[2], NL = d[3], NM = d[4], j, u;
    int T1 = W3(prec[0], prec[1], prec[4]), T2 = W3(prec[2], prec[3], prec[5]);
    int T3 = W3(prec[4], prec[5], prec[6]);
    int64_t *ur = uniq(rows, n, NULL), *uc = uniq(cols, n, NULL);
    size_t nr = (size_t)ur[0], nc = (size_t)uc[0];
    obj_t erows = new_obj(prec[4], nr * NJ), fcols = new_obj(prec[5], nc * NJ);
    for (u = 0; u < nr; u++)
      for (j = 0; j < NJ; j++)
        st(&erows, u * NJ + j, dot_chain(T1, &in[0], (size_t)ur[1 + u] * NK, 1, &in[1], j, NJ, NK), T1);
    for (u = 0; u < nc; u++)
      for (j = 0; j < NJ; j++)
        st(&fcols, u * NJ + j, dot_chain(T2, &in[2], j * NM, 1, &in[3], (size_t)uc[1 + u], NL, NM), T2);
    cache_values(&erows);
    cache_values(&fcols);
    for (k = 0; k < n; k++) {
      size_t ri = uniq_index(ur, rows[k]), li = uniq_index(uc, cols[k]);
      vals[k] = round_to(prec[6], dot_chain(T3, &erows, ri * NJ, 1, &fcols, li * NJ, 1, NJ), T3);
    }
    free(erows.p);
    free(fcols.p);
    free(erows.val);
    free(fcols.val);
    free(ur);
    free(uc);
  } else if (!strcmp(kind, "atax")) {
    size_t NX = d[0], NY = d[1], i;
    int T1 = W3(prec[0], prec[1], prec[3]), T2 = W3(prec[0], prec[3], prec[2]);
    obj_t tmp = new_obj(prec[3], NX);      /* y depends on every row-dot */
    for (i = 0; i < NX; i++) st(&tmp, i, rowdot(T1, &in[0], i * NY, NY, &in[1]), T1);
    for (k = 0; k < n; k++)
      vals[k] = round_to(prec[2], colsum(T2, &in[0], NX, NY, (size_t)cols[k], &tmp, 0), T2);
    free(tmp.p);
  } else if (!strcmp(kind, "bicg")) {
    size_t NX = d[0], NY = d[1];
    int T1 = W3(prec[0], prec[1], prec[2]), T2 = W3(prec[0], prec[3], prec[4]);
    for (k = 0; k < n; k++) {
      if (m == 2) vals[k] = round_to(prec[2], colsum(T1, &in[0], NX, NY, (size_t)cols[k], &in[1], 0), T1);
      else vals[k] = round_to(prec[4], rowdot(T2, &in[0], (size_t)cols[k] * NY, NY, &in[3]), T2);
    }
  } else if (!strcmp(kind, "gesummv")) {
    size_t N = d[0];
    int T1 = W3(prec[0], prec[2], prec[4]), T2 = W3(prec[1], prec[2], prec[3]);
    int T3 = W2(prec[4], prec[3]);
    double al = t_lit(T3, scalar_or(sc, 0, 43532.0)), be = t_lit(T3, scalar_or(sc, 1, 12313.0));
    for (k = 0; k < n; k++) {
      size_t i = cols[k];
      double tv = round_to(prec[4], rowdot(T1, &in[0], i * N, N, &in[2]), T1);
      double yv = round_to(prec[3], rowdot(T2, &in[1], i * N, N, &in[2]), T2);
      vals[k] = round_to(prec[3], t_fma(T3, al, tv, t_mul(T3, be, yv)), T3);
    }
  } else if (!strcmp(kind, "mvt")) {
    size_t N = d[0];
    int T1 = W3(prec[0], prec[1], prec[3]), T2 = W3(prec[0], prec[2], prec[4]);
    for (k = 0; k < n; k++) {
      size_t i = cols[k];
      if (m == 1)
        vals[k] = round_to(prec[1], t_add(T1, ld(&in[1], i), rowdot(T1, &in[0], i * N, N, &in[3])), T1);
      else
        vals[k] = round_to(prec[2], t_add(T2, ld(&in[2], i), colsum(T2, &in[0], N, N, i, &in[4], 0)), T2);
    }
  } else if (!strcmp(kind, "syrk")) {
    size_t N = d[0], M = d[1];
    int T = W2(prec[0], prec[1]);
    double al = t_lit(T, scalar_or(sc, 0, 32412.0)), be = t_lit(T, scalar_or(sc, 1, 2123.0));
    for (k = 0; k < n; k++) {
      size_t j1 = rows[k], j2 = cols[k];
      if (j1 > j2) { size_t s = j1; j1 = j2; j2 = s; }   /* mirrored lower triangle */
      double acc = dot_chain(T, &in[0], j1, M, &in[0], j2, M, N);
      vals[k] = round_to(prec[1], t_fma(T, al, acc, t_mul(T, be, ld(&in[1], j1 * M + j2))), T);
    }
  } else if (!strcmp(kind, "conv2d")) {
    size_t NI = d[0], NJ = d[1];
    int T = W2(prec[0], prec[1]);
    for (k = 0; k < n; k++) {
      size_t i = rows[k], j = cols[k];
      int border = (i == 0 || j == 0 || i + 1 >= NI || j + 1 >= NJ);
      vals[k] = round_to(prec[1], border ? 0.0 : conv2d_at(T, &in[0], NJ, i, j), T);
    }
  } else if (!strcmp(kind, "syr2k")) {
    size_t M = d[1], N = d[0];
    int T = W3(prec[0], prec[1], prec[2]);
    double al = t_lit(T, scalar_or(sc, 0, 32412.0)), be = t_lit(T, scalar_or(sc, 1, 2123.0));
    for (k = 0; k < n; k++) {
      size_t i = rows[k], j = cols[k];
      double s1 = dot_chain(T, &in[0], i, M, &in[1], j, M, N);
      double c1 = round_to(prec[2], t_fma(T, al, s1, t_mul(T, be, ld(&in[2], i * M + j))), T);
      double s2 = dot_chain(T, &in[1], i, M, &in[0], j, M, N);
      vals[k] = round_to(prec[2], t_fma(T, al, s2, c1), T);
    }
  } else if (!strcmp(kind, "conv3d")) {
    size_t NI = d[0], NJ = d[1], NK = d[2];
    int T = W2(prec[0], prec[1]);
    for (k = 0; k < n; k++) {
      size_t i = rows[k], j = cols[k] / NK, kk = cols[k] % NK;
      int border = i == 0 || j == 0 || kk == 0 || i + 1 >= NI || j + 1 >= NJ || kk + 1 >= NK;
      vals[k] = round_to(prec[1], border ? 0.0 : conv3d_at(T, &in[0], NJ, NK, i, j, kk), T);
    }
  } else if (!strcmp(kind, "fdtd2d")) {     /* time-stepped: every entry depends on all */
    obj_t o[8];
    const app_def_t *ap;
    int64_t dd[8];
    if (run_to_objects(kind, dims, ndims, sc, prec, inputs, o, &ap, dd)) return 1;
    for (k = 0; k < n; k++) vals[k] = ld(&o[m], (size_t)(rows[k] * C[m] + cols[k]));
    free_objects(o, ap->nobj);
  } else {                                  /* corr / covar: symmat entries */
    /* column j of the normalised (CORR) / centred (COVAR) data is computed once
     * per distinct j (no arithmetic difference: stats_column is per column) */
    int corr = !strcmp(kind, "corr");
    size_t N = d[0], M = d[1], u;
    int so = corr ? 3 : 2;
    obj_t mean = new_obj(prec[1], M), sd = new_obj(corr ? prec[2] : OR_F64, M);
    obj_t z = new_obj(prec[0], N);
    int T = W2(prec[0], prec[so]);
    double eps = scalar_or(sc, 0, 0.005);
    int64_t *lo = (int64_t *)malloc(sizeof(int64_t) * (n ? n : 1));
    int64_t *hi = (int64_t *)malloc(sizeof(int64_t) * (n ? n : 1));
    int64_t *both = (int64_t *)malloc(sizeof(int64_t) * (2 * n + 1));
    int64_t *uz;
    obj_t zc;
    for (k = 0; k < n; k++) {
      lo[k] = rows[k] < cols[k] ? rows[k] : cols[k];   /* mirrored lower triangle */
      hi[k] = rows[k] < cols[k] ? cols[k] : rows[k];
      both[k] = lo[k];
      both[n + k] = hi[k];
    }
    uz = uniq(both, 2 * n, NULL);
    zc = new_obj(prec[0], (size_t)uz[0] * N);
    for (u = 0; u < (size_t)uz[0]; u++) {
      size_t i;
      stats_column(corr, &in[0], &mean, &sd, N, M, (size_t)uz[1 + u], eps, &z);
      for (i = 0; i < N; i++) st(&zc, u * N + i, ld(&z, i), prec[0] == OR_F64 ? OR_F64 : OR_F32);
    }
    cache_values(&zc);
    for (k = 0; k < n; k++) {
      size_t j1 = (size_t)lo[k], j2 = (size_t)hi[k];
      if (corr && j1 == j2) { vals[k] = round_to(prec[so], 1.0, T); continue; }
      {
        size_t a1 = uniq_index(uz, (int64_t)j1), a2 = uniq_index(uz, (int64_t)j2);
        double acc = dot_chain(T, &zc, a1 * N, 1, &zc, a2 * N, 1, N);
        if (!corr) acc = t_div(T, acc, t_lit(T, (double)N - 1.0));
        vals[k] = round_to(prec[so], acc, T);
      }
    }
    free(mean.p); free(sd.p); free(z.p); free(zc.p); free(zc.val);
    free(lo); free(hi); free(both); free(uz);
  }
  for (t = 0; t < a->nobj; t++) free(in[t].val);
  return 0;
}
