/*
 * prescaler.h -- C ABI of libprescaler.so: the B200 (sm_100a) hot path of
 * PreScaler (Kang, Choi, Park, CGO '20), i.e. the evaluation of ONE
 * memory-object-level mixed-precision configuration:
 *
 *   RunApp(config) -> KernelTime, TransferTime, Accuracy   (Alg. 1 line 8)
 *   if Accuracy < TOQ then fail                            (Alg. 1 line 10)
 *
 * ("P:<n>" = line n of the paper text.)  Every floating-point rule not fixed by
 * the paper is a reading listed in DESIGN.md §3 (R1-R6).
 *
 * Conventions
 *  - Device pointers are CALLER-OWNED (e.g. torch tensors); the library never
 *    frees them.  Host pointers are read/written only during the call (or until
 *    the stream is synchronised, where stated).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *  - Every call returns ps_status.  No C++ exception crosses the ABI.  Errors of
 *    asynchronous work surface at the next synchronising call as PS_ERR_CUDA.
 *    ps_last_error() returns a thread-local message for the last failure.
 *  - Buffers of a dtype hold IEEE binary64 / binary32 / binary16 values, or
 *    bfloat16 bit patterns (PS_BF16).
 *  - One ps_app per host thread / stream (not thread-safe per handle).
 */
#ifndef PRESCALER_H
#define PRESCALER_H
#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define PS_API __attribute__((visibility("default")))
#else
#define PS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

/* precision codes in the paper's descending-precision order; PS_BF16
 * is the Blackwell extension (reading #28): raw
 * uint16 bit patterns (1 sign, 8 exponent, 7 fraction bits), RNE narrowing with
 * subnormals, overflow to inf, canonical NaN 0x7FFF.  PS_E4M3 / PS_E5M2 are the
 * fp8 extensions (reading #29): raw uint8 codes, OCP E4M3 "fn" (bias 7, no inf,
 * NaN 0x7F, max 448; overflow -> NaN) and E5M2 (bias 15, max 57344, overflow ->
 * inf), canonical NaN 0x7F; an fp8 memory object carries a per-tensor power-of-
 * two scale (ps_fp8_scale). */
typedef enum { PS_F64 = 0, PS_F32 = 1, PS_F16 = 2, PS_BF16 = 3, PS_E4M3 = 4, PS_E5M2 = 5 } ps_dtype;

typedef enum {
  PS_OK = 0,
  PS_ERR_INVALID = 1,      /* null pointer, bad dtype, id >= radix^M, wrong ndims      */
  PS_ERR_UNSUPPORTED = 2,  /* unknown app kind / dims out of range                    */
  PS_ERR_CUDA = 3,         /* CUDA runtime error (message in ps_last_error())          */
  PS_ERR_WORKSPACE = 4     /* workspace missing or smaller than ps_app_workspace_bytes */
} ps_status;

typedef enum {
  PS_METRIC_MRE = 0,       /* quality = 1 - mean capped relative error        */
  PS_METRIC_MAX_REL = 1    /* quality = 1 - min(1, max uncapped relative error)       */
} ps_metric;

PS_API const char *ps_status_string(int status);
PS_API const char *ps_last_error(void);
PS_API const char *ps_version(void);
/* Number of CUDA kernels this library has launched in this process (all threads).
 * Used by bench.py to report how many of the library's kernels ran. */
PS_API uint64_t ps_kernel_launches(void);
/* 1 when f64 contractions on the current device run on the fp64 tensor-core MMA
 * (DMMA), 0 when they run on the DFMA kernel.  The DMMA chain is R3's fma chain
 * bit for bit only if the hardware accumulates one mma.m8n8k4.f64 as a
 * sequential fma chain (measured on B200, not specified by PTX); the library
 * checks this on adversarial operands before the first f64 contraction on each
 * device and falls back to DFMA when it does not hold.  May
 * synchronise a private stream on first use. */
PS_API int ps_f64_uses_dmma(void);

/* ------------------------------------------------------------------------- */
/* (1) Device-side type conversion of one memory object (Fig. 3c). */
/*   dst[i] = RNE_{dst_type}(src[i]) for i < n; widening is exact; subnormals   */
/*   kept; overflow -> +-inf; NaN -> canonical NaN (f16 / bf16 0x7FFF, f32      */
/*   0x7FFFFFFF, f64 0x7FFFFFFFFFFFFFFF).  f64 -> f16 and f64 -> bf16 are single */
/*   roundings; every pair of the four types is supported.  src, dst: device    */
/*   pointers, any alignment (16-byte aligned pointers take the vector path);    */
/*   overlapping ranges -> PS_ERR_INVALID; n == 0 is a no-op; src_type ==        */
/*   dst_type is a device-to-device copy.  Asynchronous on `stream`.             */
/*   fp8 types are converted UNSCALED here (scale 2^0); see ps_convert_scaled. */
PS_API ps_status ps_convert(const void *src, int src_type, void *dst, int dst_type, size_t n,
                     void *stream);

/* Per-tensor power-of-two scale of an fp8 memory object (reading #29).  A
 * 16-byte record in DEVICE memory, caller-owned: element i of the object holds
 * code q_i with value q_i * 2^k. */
typedef struct {
  uint64_t amax_bits;  /* scratch: IEEE f64 bits of the last amax (library-written) */
  int32_t k;           /* scale exponent, in [-126, 126]                             */
  int32_t reserved;
} ps_fp8_scale;
/* Scaled conversion of an fp8 memory object (reading #29):
 *   dst_type fp8, src_type f64/f32/f16/bf16: amax = max |src| over the finite
 *     elements; k = the smallest integer in [-126, 126] with amax <= FMAX * 2^k
 *     (FMAX 448 / 57344; k = 0 if amax == 0; 126 if none); dst[i] =
 *     RNE_fp8(src[i] * 2^-k) in one rounding; writes scale->k (and amax_bits);
 *   src_type fp8, dst_type f64/f32/f16/bf16: dst[i] = RNE_dst(q_i * 2^scale->k);
 *   fp8 -> fp8 and non-fp8 pairs: PS_ERR_UNSUPPORTED / use ps_convert.
 *   scale: device pointer (16-byte record); src, dst as in ps_convert.
 *   Asynchronous on `stream` (two kernels: amax, then encode). */
PS_API ps_status ps_convert_scaled(const void *src, int src_type, void *dst, int dst_type, size_t n,
                            ps_fp8_scale *scale, void *stream);

/* ------------------------------------------------------------------------- */
/* (2) Output quality of one buffer against the fp64 run (reading #7):   */
/*   e_i = 0 if o == r; 1 if o or r non-finite or r == 0; else                  */
/*   min(1, |o - r| / |r|), with o = out[i] widened exactly to fp64.           */
/*   res: mean_rel = sum(e)/n, max_rel = max uncapped relative error (inf on    */
/*   overflow), nonfinite = #non-finite o, quality per `metric`.  out (out_type)*/
/*   and ref (fp64): device pointers of n elements.  Synchronises `stream` and  */
/*   writes the host struct *res.  Uses a small library-owned device scratch.   */
typedef struct {
  double quality, mean_rel, max_rel;
  uint64_t n, nonfinite;
} ps_quality_result;
PS_API ps_status ps_quality(const void *out, int out_type, const double *ref, size_t n, int metric,
                     void *stream, ps_quality_result *res);

/* ------------------------------------------------------------------------- */
/* (3) Applications: memory objects + statements (SURVEY c-4).   */
/*   kind:  "gemm" dims {NI,NJ,NK}    scalars {alpha,beta} (default 32412,2123) */
/*          "2mm"  dims {NI,NJ,NK,NL}                                          */
/*          "3mm"  dims {NI,NJ,NK,NL,NM}                                       */
/*          "atax" dims {NX,NY}   "bicg" dims {NX,NY}                          */
/*          "gesummv" dims {N}    scalars {alpha,beta} (default 43532,12313)    */
/*          "corr" dims {N,M} scalars {eps} (default 0.005)  "covar" dims {N,M} */
/*          "mvt" dims {N}     "syrk" dims {N,M} scalars {alpha,beta}           */
/*          "conv2d" dims {NI,NJ}   "syr2k" dims {N,M} scalars {alpha,beta}     */
/*          "conv3d" dims {NI,NJ,NK}   "fdtd2d" dims {TMAX,NX,NY}              */
/*          (SYRK/SYR2K defaults 32412, 2123; readings #23-#27)                  */
/*   ndims == 1 sets every dimension to dims[0].  scalars may be NULL.          */
/*   Every object's original precision is f32 (BASELINE).  Object order is the  */
/*   configuration-id digit order.                                              */
typedef struct ps_app ps_app;
typedef struct {
  const char *name;   /* static string owned by the library */
  uint64_t n;         /* elements = rows * cols */
  int64_t rows, cols; /* row-major */
  int32_t orig;       /* ps_dtype of the original program (PS_F32) */
  int32_t role;       /* 0 in, 1 out, 2 inout, 3 temp */
  int32_t is_output;  /* delivered to the host and scored (a4/a5) */
  int32_t reserved;
} ps_object_info;

PS_API ps_status ps_app_create(const char *kind, const int64_t *dims, int ndims, const double *scalars,
                        ps_app **out);
PS_API ps_status ps_app_destroy(ps_app *app);
PS_API int ps_app_num_objects(const ps_app *app);            /* -1 if app == NULL */
PS_API ps_status ps_app_object_info(const ps_app *app, int m, ps_object_info *out);
/* flags: PS_FLAG_NO_TENSOR_CORES forces the SIMT contraction path for fp16   */
/* operands (bit-exact with R3) instead of tcgen05 (tolerance R6).  It does   */
/* not concern f64 statements: they run on the fp64 MMA (mma.sync.f64) when   */
/* the per-device self-check shows its chained result is R3's fma chain bit   */
/* for bit (ps_f64_uses_dmma), else on DFMA chains -- bit-exact either way.   */
/* PS_FLAG_BF16 extends the configuration alphabet to {f64, f32, f16, bf16}:  */
/* precision vectors may hold PS_BF16 and ids run over 4^M (radix 4, object 0 */
/* least significant); without it the space is the paper's 3^M.               */
#define PS_FLAG_NO_TENSOR_CORES 1u
#define PS_FLAG_BF16 2u
/* PS_FLAG_FP8 extends the alphabet to {f64, f32, f16, bf16, e4m3, e5m2}: ids run */
/* over 6^M (radix 6).  fp8 objects carry a per-tensor scale (reading #29); the   */
/* workspace then also holds one n*8-byte staging region per object, so set the   */
/* flags BEFORE ps_app_workspace_bytes / ps_app_bind.                             */
#define PS_FLAG_FP8 4u
PS_API ps_status ps_app_set_flags(ps_app *app, uint32_t flags);
/* Device workspace the caller must allocate (>= 256-byte aligned). */
PS_API size_t ps_app_workspace_bytes(const ps_app *app);
/* Bind the workspace and the caller's device buffers:
 *   orig_inputs[m]:  f32 device buffer (n elements) for role in/inout, else NULL;
 *                    never modified (inout objects are copied into the workspace);
 *   orig_outputs[m]: f32 device buffer receiving the back-converted output of every
 *                    is_output object (a4), else NULL. */
PS_API ps_status ps_app_bind(ps_app *app, void *workspace, size_t bytes, void *const *orig_inputs,
                      void *const *orig_outputs);
/* Copy host (preferably pinned) f32 inputs into the bound orig_inputs (H2D). */
PS_API ps_status ps_app_load_host(ps_app *app, const void *const *host_inputs, void *stream);
/* a0: run the all-f64 configuration (id 0) and copy the raw fp64 contents of each
 * output object into ref_outputs[m] (caller-owned device, n elements; NULL for
 * non-outputs).  These buffers become the quality reference of later calls. */
PS_API ps_status ps_app_reference(ps_app *app, double *const *ref_outputs, void *stream);
/* Use externally computed fp64 reference outputs instead (e.g. gathered). */
PS_API ps_status ps_app_set_reference(ps_app *app, const double *const *ref_outputs);

/* a0 sharded by contiguous output rows (north star item 5): the
 * contraction apps (GEMM, 2MM, 3MM, SYRK, SYR2K, CORR, COVAR) have one scored
 * output whose rows can be computed independently.
 *   ps_app_shard_rows:       that output's row count; 0 = the app is not
 *                            row-shardable (mat-vec / stencil references are one
 *                            streaming pass: every rank runs ps_app_reference).
 *   ps_app_shard_triangular: 1 when row i costs ~ (rows - i) (upper tiles + mirror:
 *                            SYRK, CORR, COVAR) so callers can balance the split.
 *   ps_app_reference_rows:   rows [row0, row1) of the all-f64 run written into
 *                            ref_outputs[m] at their full-matrix offsets
 *                            (ref_outputs[m]: caller-owned device, n elements);
 *                            every element of those rows is bit-identical to
 *                            ps_app_reference, except the strictly-lower part of
 *                            triangular outputs, which is left unspecified.
 *                            Other rows are not touched.  Synchronises `stream`.
 *   ps_app_reference_merge:  after the caller has assembled every row (e.g. an
 *                            NCCL all-gather), mirror the upper triangle (and the
 *                            unit diagonal of CORR) and adopt ref_outputs as the
 *                            quality reference -- afterwards identical, bit for
 *                            bit, to ps_app_reference.
 * Errors: PS_ERR_UNSUPPORTED for non-shardable apps; PS_ERR_INVALID for a row
 * range outside [0, rows) or a missing buffer; PS_ERR_WORKSPACE if not bound. */
PS_API int64_t ps_app_shard_rows(const ps_app *app);
PS_API int ps_app_shard_triangular(const ps_app *app);
PS_API ps_status ps_app_reference_rows(ps_app *app, int64_t row0, int64_t row1, double *const *ref_outputs,
                                void *stream);
PS_API ps_status ps_app_reference_merge(ps_app *app, double *const *ref_outputs, void *stream);

/* ------------------------------------------------------------------------- */
/* (4) Evaluate one configuration (the hot path).                              */
typedef struct {
  uint64_t config_id;
  float convert_ms;   /* a2: input conversion (incl. inout copies)            */
  float kernel_ms;    /* a3: precision-scaled kernels                          */
  float backconv_ms;  /* a4+a5 fused: back-conversion + per-element error      */
  float quality_ms;   /* a5: final deterministic reduction                     */
  float total_ms;     /* [transfer +] convert + kernel + backconv  (reading #19) */
  float transfer_ms;  /* host conversion + H2D + D2H (ps_run_config_host only)  */
  double quality;     /* 1 - mean relative error                               */
  double max_rel;     /* max uncapped relative error                           */
  uint64_t nonfinite; /* non-finite delivered output elements                  */
  int32_t pass;       /* quality >= toq                                        */
  int32_t status;     /* ps_status of this evaluation                          */
} ps_result;          /* 64 bytes */

/* id = sum_m code(prec[m]) * 3^m  (object 0 least significant) */
PS_API ps_status ps_config_encode(const ps_app *app, const int *prec, uint64_t *id);
PS_API ps_status ps_config_decode(const ps_app *app, uint64_t id, int *prec);
/* prec: num_objects ps_dtype codes.  out == NULL: enqueue only (no sync, no record).
 * Requires ps_app_bind and a reference (ps_app_reference / ps_app_set_reference). */
PS_API ps_status ps_run_config(ps_app *app, const int *prec, double toq, void *stream, ps_result *out);

/* ------------------------------------------------------------------------- */
/* (4b) ONE configuration evaluated by W ranks, each owning a contiguous range  */
/*   of the app's sharded rows ("very large memory objects        */
/*   sharded by contiguous range"; north star item 5).  The sharded dimension:  */
/*   the rows of A (and B) for ATAX / BICG / GESUMMV / MVT; the rows of the      */
/*   scored output for GEMM, 2MM, 3MM (F rows get their own split), SYR2K,     */
/*   2DCONV, 3DCONV; the upper-triangular output rows for SYRK, CORR, COVAR     */
/*   (CORR / COVAR split the data rows for the column statistics); the rows of  */
/*   ex / ey / hz for FDTD-2D (one halo row of ey and of hz exchanged per time   */
/*   step).  fp8 objects (a per-tensor scale needs the whole object) are not     */
/*   row-shardable: PS_ERR_UNSUPPORTED.                                          */
/*   Row bounds are aligned so every reduction keeps its single-GPU association */
/*   (R5 256-row column-sum chunks, whole quality segments, whole 256-row      */
/*   tcgen05 tiles): the record and the delivered outputs are bit-identical to */
/*   ps_run_config for every W.  Protocol, on every rank r of W:               */
/*     for (stage = 0; ; stage++) {                                            */
/*       ps_shard_step(app, prec, toq, r, W, stage, stream, &x);               */
/*       if (x.done) break;             // x.result is the configuration's record */
/*       for k < x.nregions: copy this rank's bytes [off, off + len) of        */
/*         x.region[k].ptr to the same offsets on every other rank (each rank's */
/*         (off, len) differ; e.g. an NCCL all-gather of padded pieces)        */
/*     }                                                                        */
/*   region.ptr is a device pointer into this rank's workspace (same layout on */
/*   every rank).  Delivered outputs: the rows the rank owns of a row-sharded  */
/*   output, every element of vector outputs.  ps_shard_step synchronises      */
/*   `stream` at the end of each stage; result times are summed over stages    */
/*   (device work only, exchanges excluded).  One configuration at a time per */
/*   app (stages keep state in the workspace).                                  */
typedef struct {
  void *ptr;      /* device buffer in the workspace                        */
  uint64_t off;   /* this rank's byte range [off, off + len) of ptr        */
  uint64_t len;
} ps_shard_region;
typedef struct {
  int32_t done;       /* 1: evaluation complete, `result` valid          */
  int32_t nregions;   /* regions to exchange before the next stage (<= 4) */
  ps_shard_region region[4];
  ps_result result;
} ps_shard_step_t;
/* rows of the sharded dimension, 0 = the app has no row-sharded evaluation */
PS_API int64_t ps_app_eval_shard_rows(const ps_app *app);
/* rank's row range [*row0, *row1) of that dimension among `world` ranks (may be empty) */
PS_API ps_status ps_shard_bounds(const ps_app *app, int rank, int world, int64_t *row0, int64_t *row1);
PS_API ps_status ps_shard_step(ps_app *app, const int *prec, double toq, int rank, int world, int stage,
                               void *stream, ps_shard_step_t *x);

/* ------------------------------------------------------------------------- */
/* (5) Evaluate a list of configuration ids (a7).  results[i] for config_ids[i] */
/* (host array).  *best_index = index of the fastest passing config (ties ->   */
/* lowest id), -1 if none passes.  One stream synchronisation at the end.      */
PS_API ps_status ps_sweep(ps_app *app, const uint64_t *config_ids, size_t n_configs, double toq,
                   void *stream, ps_result *results, int64_t *best_index);

/* ------------------------------------------------------------------------- */
/* (5b) Whole-program evaluation with host<->device transfers ("the  */
/*   input data of target kernels are translated to a lower precision before */
/*   data transfer from the host").  Per input object a type-conversion method */
/*   (Fig. 3):                                                     */
/*     PS_XFER_DEVICE      (c) H2D at orig (f32), device-side conversion      */
/*     PS_XFER_HOST_LOOP   (a) host single-loop (scalar) conversion, H2D at c(m) */
/*     PS_XFER_HOST_SIMD   (b) host multithreaded SIMD conversion, H2D at c(m) */
/*     PS_XFER_PIPELINE    (e) (b) in 16 MiB chunks overlapped with their H2D   */
/*     PS_XFER_TRANSIENT   (d) host -> fp16 (the intermediate type), H2D fp16, */
/*                             device fp16 -> c(m) (can add error)      */
typedef enum {
  PS_XFER_DEVICE = 0,
  PS_XFER_HOST_LOOP = 1,
  PS_XFER_HOST_SIMD = 2,
  PS_XFER_PIPELINE = 3,
  PS_XFER_TRANSIENT = 4
} ps_xfer_method;
/* Host-side RNE conversion of an f32 array (canonical NaN, bit-identical to   */
/* ps_convert): dst_type f64/f32/f16/bf16, `threads` workers (<= 1: the      */
/* caller's), simd != 0 uses F16C/AVX2 for f16/f64 when the CPU has them (bf16 */
/* is an integer-only rounding loop).  Host pointers.                         */
PS_API ps_status ps_host_convert(const float *src, void *dst, int dst_type, size_t n, int threads,
                                 int simd);
/* One object's {type conversion then transfer} with a method (the System     */
/* Inspector's probe): host f32 array -> dev_dst in dst_type.  Methods */
/* c and d need dev_stage (n*4 / n*2 bytes) for the device-side part.         */
/* Synchronous; *ms = wall-clock milliseconds of conversion + transfer.       */
PS_API ps_status ps_transfer(const float *host_src, void *dev_dst, int dst_type, size_t n,
                             int method, int threads, void *dev_stage, void *stream, float *ms);
/* Evaluate one configuration from HOST f32 inputs (host_inputs[m] for role   */
/* in/inout, pinned memory recommended): per-object method `methods[m]`      */
/* (NULL = all PS_XFER_DEVICE), `threads` host workers; the delivered f32     */
/* outputs are read back into host_outputs[m] when non-NULL.  Synchronous;    */
/* out->transfer_ms = host conversion + transfers (wall clock), and          */
/* out->total_ms includes it.                                                 */
PS_API ps_status ps_run_config_host(ps_app *app, const int *prec, const int *methods,
                                    const void *const *host_inputs, void *const *host_outputs,
                                    int threads, double toq, void *stream, ps_result *out);

/* ------------------------------------------------------------------------- */
/* (6) Decision-tree search (Sec. 4.4; Alg. 1 lines 1-13), with   */
/*   ps_run_config as RunApp (Alg. 1 line 8):                                 */
/*   - pre-full-precision scaling (Sec. 4.4.1): run the 3 uniform      */
/*     configurations, start from the fastest passing one;                    */
/*   - objects in descending order of their data volume (bytes x statements  */
/*     touching them; the device-only stand-in for "the sum of the execution  */
/*     times of related events");                                      */
/*   - per object, normal search: targets in descending precision,    */
/*     skipping the current type, stop at the first TOQ failure (line 10),   */
/*     keep the fastest passing (line 12).                                    */
/*   The wildcard test (lines 14-32) needs host-side transient conversions   */
/*   and is not part of this device-only path.  Each trial is timed as the   */
/*   median total_ms of `repeats` runs; a configuration is never re-run.      */
typedef struct {
  uint64_t config_id;     /* chosen configuration                               */
  float total_ms;         /* its median measured time                           */
  float pfp_ms;           /* time of the PFP starting configuration             */
  double quality;         /* its quality                                        */
  int32_t pass;           /* chosen configuration passes TOQ                    */
  int32_t trials;         /* distinct configurations executed (RunApp calls)    */
  uint64_t pfp_id;        /* PFP starting configuration                         */
  uint64_t trial_ids[64]; /* executed configurations in order (first 64)        */
  float trial_ms[64];     /* their median measured times (RunApp's time)        */
  int32_t trial_pass[64]; /* their TOQ decisions (Alg. 1 line 10)               */
} ps_search_result;
PS_API ps_status ps_search(ps_app *app, double toq, int repeats, void *stream,
                           ps_search_result *out);

#ifdef __cplusplus
}
#endif
#endif /* PRESCALER_H */
