/*
 * oracle.h -- PreScaler CPU ORACLE (TEST INFRASTRUCTURE ONLY).
 *
 * This is the plain, slow, obviously-correct CPU definition of what one PreScaler
 * configuration evaluation computes.  Only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg may load it.  It shares NO code with the CUDA path
 * (paper_conf_cgo_kangcp20_b200/csrc) and neither side includes the other.
 *
 * Citations: "P:<n>" = line n of the paper text; R1-R6 = DESIGN.md
 * readings.
 *
 * Precision codes follow the paper's descending-precision order:
 *   0 = f64, 1 = f32, 2 = f16; and, for the Blackwell extension of SURVEY §8(f)
 *   NEXT #4 (B200 tensor-core formats beyond the paper's fp16), 3 = bf16
 *   (IEEE-style binary16 with 8 exponent / 7 fraction bits).  The extended
 *   configuration space is 4^M (radix 4, same digit order).
 */
#ifndef PRESCALER_ORACLE_H
#define PRESCALER_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { OR_F64 = 0, OR_F32 = 1, OR_F16 = 2, OR_BF16 = 3, OR_E4M3 = 4, OR_E5M2 = 5 };

/* ---- fp8 object types (reading #29) ---------------
 * E4M3 (OCP "fn": bias 7, no inf, NaN 0x7F, max 448) and E5M2 (IEEE-like: bias
 * 15, inf, max 57344), 1-byte codes.  An fp8 OBJECT carries one per-tensor
 * power-of-two scale 2^k: element i holds code q_i with value q_i * 2^k.  Every
 * time the object is written (input conversion a2, or the end of a statement
 * that writes it) the whole object is re-quantised:
 *   amax = max |v_i| over its finite values (0 if none);
 *   k    = the smallest integer in [-126, 126] with amax <= FMAX * 2^k (k = 0
 *          when amax == 0; 126 when no such k exists);
 *   q_i  = RNE_fp8(v_i * 2^-k)   (one rounding of the exact product).
 * The config alphabet {f64, f32, f16, bf16, e4m3, e5m2} gives 6^M ids (radix 6). */
#define ORACLE_FP8_KMIN (-126)
#define ORACLE_FP8_KMAX 126
/* k for a given amax (>= 0) and fp8 type */
int oracle_fp8_scale_exp(double amax, int fp8_type);
/* Scaled conversion of n elements (c-1 plus the fp8 scale):
 *   dst fp8: k from the finite values of src (widened exactly), *k_io = k,
 *            dst[i] = RNE_fp8(src[i] * 2^-k);
 *   src fp8: dst[i] = RNE_dst(src[i] * 2^(*k_io))  (value of the code, scaled);
 *   both:    decode with *k_io, then re-quantise with a fresh k written back.
 *   Neither fp8: plain oracle_convert (k_io untouched).  Returns 0 on success. */
int oracle_convert_scaled(const void *src, int src_type, void *dst, int dst_type, size_t n,
                          int *k_io);

/* ---- c-1: software IEEE-754 conversion (bit manipulation only) ---------- */
uint64_t oracle_convert_bits(uint64_t bits, int src_type, int dst_type);
/* n elements, src/dst in their own storage formats (u16 / f32 / f64). */
int oracle_convert(const void *src, int src_type, void *dst, int dst_type, size_t n);

/* ---- c-5: quality (mean relative error; pass rule P:226) --------- */
typedef struct {
  double quality;   /* 1 - sum(e)/n */
  double mean_rel;  /* sum(e)/n */
  double max_rel;   /* max uncapped relative error (inf on overflow) */
  uint64_t n;
  uint64_t nonfinite;
} oracle_quality_result;
/* Accumulates into acc (sum of e in *sum_e, max, count) so several outputs can
 * be concatenated (reading #10).  Call oracle_quality for a single buffer. */
void oracle_quality_accumulate(const void *out, int out_type, const double *ref, size_t n,
                               double *sum_e, double *max_rel, uint64_t *nonfinite);
int oracle_quality(const void *out, int out_type, const double *ref, size_t n,
                   oracle_quality_result *res);

/* ---- c-2: configuration codec ((1+#ConvTypes)^N) ----------------- */
int oracle_config_decode(int num_objects, uint64_t id, int *prec);
int oracle_config_encode(int num_objects, const int *prec, uint64_t *id);
/* radix 3 (f64, f32, f16: the paper's space), 4 (+ bf16) or 6 (+ e4m3, e5m2) */
int oracle_config_decode_radix(int num_objects, int radix, uint64_t id, int *prec);
int oracle_config_encode_radix(int num_objects, int radix, const int *prec, uint64_t *id);

/* ---- c-4: applications ------------------------------------------------ */
/* Reduction-order parameters (R5).  They are part of the definition. */
#define ORACLE_ROWDOT_LANES 32   /* lanes per row-dot slab                   */
#define ORACLE_ROWDOT_TILE 8     /* slabs per row-dot tile                   */
#define ORACLE_COLSUM_CHUNK 256  /* rows per column-sum chunk                */

typedef struct {
  const char *name;
  int role;        /* 0 in, 1 out, 2 inout, 3 temp */
  int is_output;   /* delivered to the host and scored (a4, a5) */
  int64_t rows, cols;
} oracle_object_info;

/* kind: "gemm","2mm","3mm","atax","bicg","gesummv","corr","covar".
 * Returns number of objects (>0) or -1 on bad kind/dims. */
int oracle_app_objects(const char *kind, const int64_t *dims, int ndims,
                       oracle_object_info *info /* may be NULL; else >= 8 entries */);

/* Run the precision-scaled program for one configuration (a2 + a3).
 *   inputs[m]: orig (f32) data for objects with role in/inout, else ignored.
 *   finals[m]: if non-NULL, receives the final contents of object m in its
 *              assigned precision prec[m] (raw, before back-conversion).
 *   scalars:   app scalars (gemm/gesummv: alpha,beta; corr: eps) or NULL. */
int oracle_run_config(const char *kind, const int64_t *dims, int ndims,
                      const double *scalars, const int *prec,
                      const float *const *inputs, void *const *finals);
/* Same, also returning the final scale exponent k of every fp8 object
 * (scale_exps[m], untouched for other precisions); scale_exps may be NULL. */
int oracle_run_config_k(const char *kind, const int64_t *dims, int ndims,
                        const double *scalars, const int *prec,
                        const float *const *inputs, void *const *finals, int *scale_exps);

/* Full evaluation (a2-a5): run, back-convert every output object to f32
 * (delivered[m] if non-NULL), score against the fp64 reference outputs
 * ref[m] (for output objects), fill *res.  toq -> *pass. */
int oracle_evaluate(const char *kind, const int64_t *dims, int ndims,
                    const double *scalars, const int *prec,
                    const float *const *inputs, const double *const *ref,
                    float *const *delivered, oracle_quality_result *res);

/* Sampled evaluation for parity at full size: raw final values (widened to
 * double) of output object m at entries (rows[k], cols[k]), same semantics as
 * oracle_run_config, computing only what those entries depend on.  Not defined
 * for configurations with fp8 objects (their per-tensor scale depends on every
 * element): returns 1. */
int oracle_sample(const char *kind, const int64_t *dims, int ndims, const double *scalars,
                  const int *prec, const float *const *inputs, int m, const int64_t *rows,
                  const int64_t *cols, size_t n, double *vals);

#ifdef __cplusplus
}
#endif
#endif
