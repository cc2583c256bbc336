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

enum { OR_F64 = 0, OR_F32 = 1, OR_F16 = 2, OR_BF16 = 3 };

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
/* radix 3 (f64, f32, f16: the paper's space) or 4 (+ bf16) */
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

/* Full evaluation (a2-a5): run, back-convert every output object to f32
 * (delivered[m] if non-NULL), score against the fp64 reference outputs
 * ref[m] (for output objects), fill *res.  toq -> *pass. */
int oracle_evaluate(const char *kind, const int64_t *dims, int ndims,
                    const double *scalars, const int *prec,
                    const float *const *inputs, const double *const *ref,
                    float *const *delivered, oracle_quality_result *res);

/* Sampled evaluation for parity at full size: raw final values (widened to
 * double) of output object m at entries (rows[k], cols[k]), same semantics as
 * oracle_run_config, computing only what those entries depend on. */
int oracle_sample(const char *kind, const int64_t *dims, int ndims, const double *scalars,
                  const int *prec, const float *const *inputs, int m, const int64_t *rows,
                  const int64_t *cols, size_t n, double *vals);

#ifdef __cplusplus
}
#endif
#endif
