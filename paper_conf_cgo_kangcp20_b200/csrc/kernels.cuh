// kernels.cuh -- internal launcher declarations of libprescaler (not part of the ABI).
#pragma once
#include "common.cuh"

namespace ps {

// ------------------------------------------------------------ conversion (a2)
ps_status convert_async(const void *src, int st, void *dst, int dt, size_t n, cudaStream_t stream);
// fp8 objects (reading #29, fp8.cu): encode with a fresh per-tensor scale computed
// into *sc (sc == nullptr: unscaled, k = 0), decode with sc->k (nullptr: k = 0)
constexpr int FP8_KMIN = -126, FP8_KMAX = 126;
ps_status fp8_encode_async(const void *src, int st, void *dst, int dt, size_t n, ps_fp8_scale *sc,
                           cudaStream_t stream);
ps_status fp8_decode_async(const void *src, int st, void *dst, int dt, size_t n, const ps_fp8_scale *sc,
                           cudaStream_t stream);
// host-side f32 -> dt conversion (host_convert.cpp; Fig. 3a/3b)
void host_convert_f32(const float *src, void *dst, int dt, size_t n, int threads, bool simd);

// ------------------------------------------------------- quality (a4 + a5)
constexpr int QTHREADS = 256;
constexpr int QBLOCKS_MAX = 1024;   // fixed, SM-count independent (determinism)
struct QPart {
  double sum;
  double mx;
  unsigned long long nf;
};
// segments of a rows x cols output: `per` elements each (whole rows when rows > 1)
struct QSeg {
  int64_t per;        // elements per segment
  int64_t rows_per;   // rows per segment (1 for a vector)
  int nb;             // segments (<= QBLOCKS_MAX)
};
QSeg qseg(int64_t rows, int64_t cols);
// segments [seg0, seg1) (seg1 < 0: all) of the output; partial of segment k -> parts[k];
// delivered == nullptr: score the exact widened value, no write (ps_quality)
ps_status backconv_quality_async(const void *out, int out_type, const double *ref, float *delivered,
                                 int64_t rows, int64_t cols, QPart *parts, cudaStream_t st,
                                 int seg0 = 0, int seg1 = -1);
ps_status quality_finalize_async(const QPart *parts, int nparts, QPart *res, cudaStream_t st);

// ------------------------------------------------------ contractions (a3)
// element (r, c) of a matrix operand lives at p[r * s_row + c * s_col]
struct MatDesc {
  const void *p;
  int type;
  int64_t s_row, s_col;
  const ps_fp8_scale *sc = nullptr;   // fp8 operand: its per-tensor scale record (reading #29)
};
enum Epilogue { EPI_PLAIN = 0, EPI_AXPBY = 1 /* fma(alpha, acc, beta*Cin) */, EPI_DIV = 2 };
struct GemmArgs {
  int64_t M, N, K;
  MatDesc A;            // A(i, k), M x K
  MatDesc B;            // B(k, j), K x N
  void *C;              // output, row-major, leading dimension ldc
  int c_type;
  int64_t ldc;
  const void *Cin;      // EPI_AXPBY: previous contents of C (row-major, ldc)
  int cin_type;
  int epi;
  double alpha, beta, div;   // fp64 literals (rounded to T on the device side)
  int upper_only;       // SYRK: skip tiles strictly below the diagonal
  int64_t row_off;      // upper_only: global index of row 0 of C (row-sharded reference / evaluation)
  int64_t tc_m_full;    // > 0: M of the unsharded statement (tcgen05 picks its kernel from it)
  int T;                // compute type PS_F32 / PS_F64
};
// R3-exact SIMT contraction (FFMA / DFMA fma chains, k ascending)
ps_status gemm_simt_async(const GemmArgs &g, cudaStream_t st);
// tcgen05 tensor-core contraction for fp16 x fp16 -> f32 accumulate (R6)
bool gemm_tc_supported(const GemmArgs &g);
ps_status gemm_tc_async(const GemmArgs &g, cudaStream_t st);
// S[j1][j2] := S[j2][j1] for j1 > j2; diag := 1 if diag_one (SYRK mirror)
ps_status mirror_async(void *S, int type, int64_t M, int diag_one, cudaStream_t st);

// ------------------------------------------------------------ mat-vec (a3)
constexpr int COLSUM_CHUNK = 256;    // R5: rows per column-sum chunk
// workspace for the chunk / tile partials of one statement on a rows x cols matrix
size_t tile_partial_bytes(int64_t rows, int64_t cols);
// out[i] = RNE_out(row-dot of row i), R5 hierarchical order (tiles.cu)
ps_status rowdot_async(const void *A, int ta, int64_t lda, const void *x, int tx, void *out,
                       int tout, int64_t rows, int64_t cols, void *partial, cudaStream_t st);
// BICG in ONE pass over A: s = A^T r (column sums), q = A p (row dots)
ps_status bicg_async(const void *A, int ta, int64_t lda, const void *r, int tr, void *s, int ts,
                     const void *p, int tp, void *q, int tq, int64_t rows, int64_t cols,
                     void *partial, cudaStream_t st);
// column sums over 256-row chunks:
//   mode 0: p = fma(A_ij, w_i, p)   mode 1: p = p + A_ij   mode 2: d = A_ij - w_j, p = fma(d, d, p)
// finalize: 0 plain, 1 total / n, 2 stddev (sqrt(total / n), <= eps -> 1)
enum ColMode { COL_DOT = 0, COL_SUM = 1, COL_SQDEV = 2 };
enum ColFin { FIN_PLAIN = 0, FIN_MEAN = 1, FIN_STDDEV = 2, FIN_ADD = 3 /* out = out_old + total */ };
// MVT in one pass over A: x1 <- x1 + A y1, x2 <- x2 + A^T y2 (n x n)
ps_status mvt_async(const void *A, int ta, int64_t n, void *x1, int t1, void *x2, int t2,
                    const void *y1, int ty1, const void *y2, int ty2, void *partial, cudaStream_t st);
// 2DCONV 3x3 stencil (reading #24): B_ij = sum of 9 rounded products, left to right; border +0
ps_status conv2d_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, cudaStream_t st);
ps_status conv2d_rows_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, int64_t ibeg,
                            int64_t iend, cudaStream_t st);   // output rows [ibeg, iend)
// 3DCONV 27-point stencil (reading #26) on NI x NJ x NK
ps_status conv3d_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, int64_t nk,
                       cudaStream_t st);
ps_status conv3d_rows_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, int64_t nk,
                            int64_t ibeg, int64_t iend, cudaStream_t st);   // output planes [ibeg, iend)
// one statement of FDTD-2D time step t (reading #27): FDTD_EY = ey row 0 from fict and
// the ey update in one pass; FDTD_EY0 / FDTD_EY1 = those two parts alone (reading #29)
enum FdtdPart { FDTD_EY = 0, FDTD_EY0 = 1, FDTD_EY1 = 2, FDTD_EX = 3, FDTD_HZ = 4 };
ps_status fdtd2d_part_async(int part, const void *fict, int tf, void *ex, int tex, void *ey, int tey,
                            void *hz, int thz, int64_t t, int64_t nx, int64_t ny, cudaStream_t st,
                            int64_t r0 = 0, int64_t r1 = -1);   // rows [r0, r1) (row-sharded)
ps_status colsum_async(const void *A, int ta, int64_t lda, const void *w, int tw, void *out,
                       int tout, int64_t rows, int64_t cols, int T, int mode, int fin, double n,
                       double eps, void *partial, cudaStream_t st);
// row-sharded pieces (tiles.cu): one rank's tile pass over its rows (column-chunk
// partials into the full array at `spart`, row dots finished locally), and the
// in-order finalize over every chunk; mode COL_* or -1 (row dots only)
ps_status tile_rows_async(int mode, const void *A, int ta, int64_t lda, const void *w, int tw,
                          const void *x, int tx, void *rd_out, int t_rd, int rd_add, int64_t rows,
                          int64_t cols, int TC, void *spart, void *qpart, cudaStream_t st);
ps_status colsum_finalize_async(const void *spart, int TC, int64_t rows, int64_t cols, void *out, int tout,
                                int fin, double n, double eps, cudaStream_t st);
size_t tile_spart_bytes(int64_t rows, int64_t cols);   // the full chunk-partial array (8-byte entries)
// y_i = RNE_y(fma(alpha, tmp_i, beta * y_i)) in T = W(tmp, y)
ps_status axpby_async(const void *tmp, int ttmp, void *y, int ty, int64_t n, double alpha,
                      double beta, cudaStream_t st);
// CORR: data_ij = (data_ij - mean_j) / (sqrt_n * std_j)   COVAR: data_ij -= mean_j
ps_status corr_normalize_async(void *data, int td, const void *mean, int tm, const void *std,
                               int ts, int64_t rows, int64_t cols, double sqrt_n, cudaStream_t st);
ps_status covar_center_async(void *data, int td, const void *mean, int tm, int64_t rows,
                             int64_t cols, cudaStream_t st);

}  // namespace ps
