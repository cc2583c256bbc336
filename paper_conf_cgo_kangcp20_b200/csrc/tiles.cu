// tiles.cu -- the bandwidth-bound statements on an R x C row-major matrix A
// (row a3 of ATAX, BICG, GESUMMV, CORR, COVAR), in reading R5's orders:
//
//   column-sum z_j = sum_i A_ij w_i : rows in chunks of 256; per chunk an fma
//     chain from +0, i ascending; chunk partials added in ascending order.
//   row-dot y_i = sum_j A_ij x_j : lane l of a 32-lane slab owns the 16-byte
//     chunk (V = 16/sizeof(A) elements) at columns 32V*s + lV.., fma chain from
//     +0; slab value = xor butterfly 16..1 (a + partner); 8 slabs form a tile,
//     slab values added left to right; tile values added left to right.
//
// One kernel shape serves every statement: a CTA = 8 warps owns one 8-slab
// column tile and walks 256-row chunks; warp w streams slab 8t+w, one 16-byte
// load per lane per row (4 rows in flight), so each element of A is read
// ONCE for the column sums AND the row dots.  BICG (s = A^T r, q = A p) is a
// single pass over A.  Partials (chunk x columns, tile x rows) go to the
// workspace and two tiny kernels finish them in order.  HBM-bound:
// algorithmic bytes = R*C*sizeof(A) per pass + O(R + C).
#include <math.h>

#include <atomic>

#include <type_traits>

#include "common.cuh"
#include "kernels.cuh"
#include "types.cuh"

namespace ps {

constexpr int TILE_SLABS = 8;               // slabs per row-dot tile = warps per CTA
constexpr int TTHREADS = 32 * TILE_SLABS;
constexpr int CM_NONE = -1;                 // no column sum (COL_DOT/SUM/SQDEV otherwise)

struct TileArgs {
  const void *A;
  int64_t lda, rows, cols;
  const void *w;   // COL_DOT: per-row weight w_i; COL_SQDEV: per-column mean mu_j
  int tw;
  const void *x;   // row-dot vector x_j
  int tx;
  void *spart;     // [nchunks][cols] column-chunk partials (TC)
  void *qpart;     // [ntiles][rows]  row-tile partials (TR)
  int64_t nchunks, ntiles, nslabs;
  int vec_ok;
};

// Minimum CTAs per SM for __launch_bounds__: 16-bit A with f32 arithmetic and row
// dots runs 16-row groups capped at 128 registers, two CTAs per SM -- these statements
// are bound by global-load latency (ncu: long_scoreboard 57% of stalls), and twice the
// rows in flight per warp beat 50% more warps: 8-row groups at 80 registers and three
// CTAs per SM measured 4.5-7.6% slower (profiles/tile_probe_{base,gr16}_r2as.jsonl).
// 0 = not specified (ptxas keeps its default, <= 128 registers here; an explicit 1
// lets it grow to ~230 and halves the occupancy of the f64 statements)
template <class SA, class TC, class TR, bool RD>
constexpr int tile_minb() {
  return (RD && sizeof(raw_t<SA>) == 2 && sizeof(TC) == 4 && sizeof(TR) == 4) ? 2 : 0;
}

template <class SA, class TC, class TR, int CM, bool RD>
__global__ void __launch_bounds__(TTHREADS, tile_minb<SA, TC, TR, RD>()) tile_kernel(TileArgs a) {
  using RA = raw_t<SA>;
  constexpr int V = 16 / sizeof(RA);
  constexpr bool SAME = std::is_same<TC, TR>::value;
  // rows per group: 16, or 8 where 16 would take more than 128 registers (2 CTAs per
  // SM instead of 1 keeps the same bytes in flight and fills all SMs; ptxas -v):
  // 16-bit chunks (V = 8) with an f64 compute type, f32 chunks (V = 4) feeding f64
  // column sums or weighted (COL_DOT) f32 column sums without row dots
  constexpr int GR = ((V == 8 && (sizeof(TC) == 8 || sizeof(TR) == 8)) ||
                      (V == 4 && !RD && (CM == COL_DOT || sizeof(TC) == 8)))
                         ? 8
                         : 16;
  __shared__ TR part[RD ? COLSUM_CHUNK : 1][TILE_SLABS + 1];
  __shared__ TC sw[CM == COL_DOT ? COLSUM_CHUNK : 1];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t tcol = blockIdx.x;
  const int64_t j0 = (tcol * TILE_SLABS + warp) * (32 * V) + (int64_t)lane * V;
  const int64_t rem = a.cols - j0;
  const int nv = rem <= 0 ? 0 : (rem >= V ? V : (int)rem);
  const bool vec = a.vec_ok && nv == V;
  const bool wfull = __all_sync(0xffffffffu, vec);   // warp-uniform fast path

  TR xv[V];
  TC mu[V];
#pragma unroll
  for (int v = 0; v < V; v++) {
    xv[v] = (RD && v < nv) ? load_any<TR>(a.x, a.tx, j0 + v) : TR(0);
    mu[v] = (CM == COL_SQDEV && v < nv) ? load_any<TC>(a.w, a.tw, j0 + v) : TC(0);
  }

  for (int64_t rc = blockIdx.y; rc < a.nchunks; rc += gridDim.y) {
    const int64_t i0 = rc * COLSUM_CHUNK;
    const int64_t i1 = (a.rows < i0 + COLSUM_CHUNK) ? a.rows : i0 + COLSUM_CHUNK;
    if (CM == COL_DOT) {   // stage this chunk's w_i (T_c) in shared memory
      sw[threadIdx.x] = (i0 + threadIdx.x < i1) ? load_any<TC>(a.w, a.tw, i0 + threadIdx.x) : TC(0);
    }
    __syncthreads();
    TC p[V];
#pragma unroll
    for (int v = 0; v < V; v++) p[v] = TC(0);

    const RA *rowp = (const RA *)a.A + i0 * a.lda + j0;
    for (int64_t g = i0; g < i1; g += GR) {
      const int nrow = (i1 - g) < GR ? (int)(i1 - g) : GR;   // warp-uniform
      union Chunk { uint4 u; RA e[V]; } ch[GR];
      TR lp[GR];
      // FULL: every lane has a whole 16-byte chunk and the group has GR rows
      // (warp-uniform), so the GR loads are issued back to back with no
      // branch between them and no per-element guards afterwards.
      auto group = [&](auto full_tag) {
        constexpr bool FULL = decltype(full_tag)::value;
        // 1) GR rows of this lane's 16-byte chunk in flight
#pragma unroll
        for (int r = 0; r < GR; r++) {
          if (FULL) {
            ch[r].u = __ldg(reinterpret_cast<const uint4 *>(rowp + r * a.lda));
          } else if (r < nrow && vec) {
            ch[r].u = __ldg(reinterpret_cast<const uint4 *>(rowp + r * a.lda));
          } else {
#pragma unroll
            for (int v = 0; v < V; v++) ch[r].e[v] = (r < nrow && v < nv) ? rowp[r * a.lda + v] : RA(0);
          }
        }
        // 2) column-sum chains (i ascending) and lane row-dot chains (v ascending)
#pragma unroll
        for (int r = 0; r < GR; r++) {
          lp[r] = TR(0);
          if (FULL || r < nrow) {
            const TC wi = (CM == COL_DOT) ? sw[g - i0 + r] : TC(0);
#pragma unroll
            for (int v = 0; v < V; v++) {
              if (FULL || v < nv) {
                const TC av = Ld<SA, TC>::get(&ch[r].e[v], 0);
                if (CM == COL_DOT) p[v] = t_fma(av, wi, p[v]);
                else if (CM == COL_SUM) p[v] = p[v] + av;
                else if (CM == COL_SQDEV) {
                  const TC d = av - mu[v];
                  p[v] = t_fma(d, d, p[v]);
                }
                if (RD) {
                  TR ar;
                  if constexpr (SAME) ar = av;
                  else ar = Ld<SA, TR>::get(&ch[r].e[v], 0);
                  lp[r] = t_fma(ar, xv[v], lp[r]);
                }
              }
            }
          }
        }
      };
      if (wfull && nrow == GR) group(std::integral_constant<bool, true>());
      else group(std::integral_constant<bool, false>());
      rowp += GR * a.lda;
      // 3) slab values of the GR rows: xor-16 butterfly step, then a transpose
      //    reduction over offsets 8,4,2,1 (same association as the 16..1 xor
      //    butterfly, 31 shuffles for 16 rows); lane l ends with row (l & 15)
      if (RD) {
        int c = GR;
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) {
          if (o >= GR) {   // plain butterfly step on every row value
#pragma unroll
            for (int r = 0; r < GR; r++) lp[r] = lp[r] + __shfl_xor_sync(0xffffffffu, lp[r], o);
          } else {         // transpose step: keep half the rows, trade the other half
            const bool up = (lane & o) != 0;
#pragma unroll
            for (int k = 0; k < GR / 2; k++) {
              if (k < c / 2) {
                const TR send = up ? lp[k] : lp[k + c / 2];
                const TR keep = up ? lp[k + c / 2] : lp[k];
                lp[k] = keep + __shfl_xor_sync(0xffffffffu, send, o);
              }
            }
            c >>= 1;
          }
        }
        const int rr = lane & (GR - 1);
        if (lane < GR && rr < nrow) part[g - i0 + rr][warp] = lp[0];
      }
    }

    if (CM != CM_NONE) {
      TC *sp = (TC *)a.spart + rc * a.cols + j0;
#pragma unroll
      for (int v = 0; v < V; v++)
        if (v < nv) sp[v] = p[v];
    }
    if (RD) {
      __syncthreads();
      if ((int64_t)threadIdx.x < i1 - i0) {
        const int64_t left = a.nslabs - tcol * TILE_SLABS;
        const int nw = left < TILE_SLABS ? (int)left : TILE_SLABS;
        TR s = part[threadIdx.x][0];
        for (int w = 1; w < nw; w++) s = s + part[threadIdx.x][w];   // slabs left to right
        ((TR *)a.qpart)[tcol * a.rows + i0 + threadIdx.x] = s;
      }
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------- finalizers
template <class T, class SO, int FIN>
__global__ void __launch_bounds__(256) colsum_finalize_kernel(const T *__restrict__ partial,
                                                              raw_t<SO> *__restrict__ out,
                                                              int64_t cols, int64_t nchunks, T n,
                                                              T eps) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= cols) return;
  // chunks in order; loads issued 8 at a time so the in-order chain does not wait
  // on one L2 round trip per term (32 at a time, predicated, measured 0.8% slower on
  // the matvec step: profiles/bench_ab_finalize_r2r.json)
  T total = partial[j];
  int64_t c = 1;
  for (; c + 8 <= nchunks; c += 8) {
    T v[8];
#pragma unroll
    for (int u = 0; u < 8; u++) v[u] = partial[(c + u) * cols + j];
#pragma unroll
    for (int u = 0; u < 8; u++) total = total + v[u];
  }
  for (; c < nchunks; c++) total = total + partial[c * cols + j];
  if (FIN == FIN_MEAN) total = total / n;
  if (FIN == FIN_STDDEV) {
    total = sqrt(total / n);
    if (total <= eps) total = T(1);
  }
  if (FIN == FIN_ADD) total = Ld<SO, T>::get(out, (size_t)j) + total;   // MVT: x2 + A^T y2
  St<SO, T>::put(out, (size_t)j, total);
}

template <class T, class SO>
__global__ void __launch_bounds__(256) rowdot_finalize_kernel(const T *__restrict__ qpart,
                                                              raw_t<SO> *__restrict__ out,
                                                              int64_t rows, int64_t ntiles, int add) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= rows) return;
  T total = qpart[i];   // tiles in order, loads batched as in colsum_finalize_kernel
  int64_t t = 1;
  for (; t + 8 <= ntiles; t += 8) {
    T v[8];
#pragma unroll
    for (int u = 0; u < 8; u++) v[u] = qpart[(t + u) * rows + i];
#pragma unroll
    for (int u = 0; u < 8; u++) total = total + v[u];
  }
  for (; t < ntiles; t++) total = total + qpart[t * rows + i];
  if (add) total = Ld<SO, T>::get(out, (size_t)i) + total;                   // MVT: x1 + A y1
  St<SO, T>::put(out, (size_t)i, total);
}

// ------------------------------------------------------------------- host
static int64_t nchunks_of(int64_t rows) { return (rows + COLSUM_CHUNK - 1) / COLSUM_CHUNK; }
static size_t spart_bytes(int64_t rows, int64_t cols) {
  return ((size_t)nchunks_of(rows) * (size_t)cols * 8 + 255) / 256 * 256;
}

size_t tile_partial_bytes(int64_t rows, int64_t cols) {
  const int64_t ntiles_max = (cols + TILE_SLABS * 32 * 2 - 1) / (TILE_SLABS * 32 * 2);   // f64 A
  return spart_bytes(rows, cols) + (size_t)ntiles_max * (size_t)rows * 8;
}

template <class SA, class TC, class TR, int CM, bool RD>
static ps_status launch_tile(const TileArgs &a, cudaStream_t st) {
  static std::atomic<int> occ_cache{0};   // same for every B200 of the box
  int occ = occ_cache.load(std::memory_order_relaxed);
  if (!occ) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tile_kernel<SA, TC, TR, CM, RD>, TTHREADS, 0);
    if (occ < 1) occ = 1;
    occ_cache.store(occ, std::memory_order_relaxed);
  }
  const int64_t cap = (int64_t)num_sms() * occ;
  int64_t gy = cap / a.ntiles;
  if (gy < 1) gy = 1;
  if (gy > a.nchunks) gy = a.nchunks;
  const int64_t per = (a.nchunks + gy - 1) / gy;   // equal chunk counts per CTA row
  gy = (a.nchunks + per - 1) / per;
  tile_kernel<SA, TC, TR, CM, RD><<<dim3((unsigned)a.ntiles, (unsigned)gy), TTHREADS, 0, st>>>(a);
  PS_CHECK_LAUNCH("tile_kernel");
  return PS_OK;
}

template <int CM, bool RD>
static ps_status tile_dispatch(const TileArgs &a, int ta, int tc, int tr, cudaStream_t st) {
  return dispatch_store(ta, [&](auto sa) -> ps_status {
    using SA = decltype(sa);
    if constexpr (std::is_same<SA, double>::value) {
      return launch_tile<SA, double, double, CM, RD>(a, st);
    } else if constexpr (CM == CM_NONE) {        // TC unused
      return tr == PS_F64 ? launch_tile<SA, double, double, CM, RD>(a, st)
                          : launch_tile<SA, float, float, CM, RD>(a, st);
    } else if constexpr (!RD) {                  // TR unused
      return tc == PS_F64 ? launch_tile<SA, double, double, CM, RD>(a, st)
                          : launch_tile<SA, float, float, CM, RD>(a, st);
    } else {
      if (tc == PS_F64 && tr == PS_F64) return launch_tile<SA, double, double, CM, RD>(a, st);
      if (tc == PS_F64) return launch_tile<SA, double, float, CM, RD>(a, st);
      if (tr == PS_F64) return launch_tile<SA, float, double, CM, RD>(a, st);
      return launch_tile<SA, float, float, CM, RD>(a, st);
    }
  });
}

static TileArgs make_args(const void *A, int ta, int64_t lda, int64_t rows, int64_t cols,
                          void *partial) {
  TileArgs a{};
  a.A = A;
  a.lda = lda;
  a.rows = rows;
  a.cols = cols;
  const int64_t V = 16 / (int64_t)dtype_size(ta);
  a.nchunks = nchunks_of(rows);
  a.nslabs = (cols + 32 * V - 1) / (32 * V);
  a.ntiles = (a.nslabs + TILE_SLABS - 1) / TILE_SLABS;
  a.spart = partial;
  a.qpart = (char *)partial + spart_bytes(rows, cols);
  a.vec_ok = ((uintptr_t)A % 16 == 0) && ((lda * (int64_t)dtype_size(ta)) % 16 == 0);
  a.w = nullptr;
  a.x = nullptr;
  a.tw = a.tx = PS_F32;
  return a;
}

template <class T>
static ps_status colsum_finalize(const TileArgs &a, void *out, int tout, int fin, double n,
                                 double eps, cudaStream_t st) {
  const unsigned fb = (unsigned)((a.cols + 255) / 256);
  // n and eps: RNE from their fp64 literal to T (R2)
  return dispatch_store(tout, [&](auto so) -> ps_status {
    using SO = decltype(so);
    const T *sp = (const T *)a.spart;
    if (fin == FIN_PLAIN)
      colsum_finalize_kernel<T, SO, FIN_PLAIN><<<fb, 256, 0, st>>>(sp, (raw_t<SO> *)out, a.cols,
                                                                  a.nchunks, (T)n, (T)eps);
    else if (fin == FIN_ADD)
      colsum_finalize_kernel<T, SO, FIN_ADD><<<fb, 256, 0, st>>>(sp, (raw_t<SO> *)out, a.cols,
                                                                a.nchunks, (T)n, (T)eps);
    else if (fin == FIN_MEAN)
      colsum_finalize_kernel<T, SO, FIN_MEAN><<<fb, 256, 0, st>>>(sp, (raw_t<SO> *)out, a.cols,
                                                                 a.nchunks, (T)n, (T)eps);
    else
      colsum_finalize_kernel<T, SO, FIN_STDDEV><<<fb, 256, 0, st>>>(sp, (raw_t<SO> *)out, a.cols,
                                                                   a.nchunks, (T)n, (T)eps);
    PS_CHECK_LAUNCH("colsum_finalize_kernel");
    return PS_OK;
  });
}

template <class T>
static ps_status rowdot_finalize(const TileArgs &a, void *out, int tout, cudaStream_t st, int add = 0) {
  const unsigned fb = (unsigned)((a.rows + 255) / 256);
  return dispatch_store(tout, [&](auto so) -> ps_status {
    using SO = decltype(so);
    rowdot_finalize_kernel<T, SO><<<fb, 256, 0, st>>>((const T *)a.qpart, (raw_t<SO> *)out, a.rows,
                                                      a.ntiles, add);
    PS_CHECK_LAUNCH("rowdot_finalize_kernel");
    return PS_OK;
  });
}

ps_status rowdot_async(const void *A, int ta, int64_t lda, const void *x, int tx, void *out,
                       int tout, int64_t rows, int64_t cols, void *partial, cudaStream_t st) {
  if (rows <= 0) return PS_OK;
  TileArgs a = make_args(A, ta, lda, rows, cols, partial);
  a.x = x;
  a.tx = tx;
  const int T = compute_type({ta, tx, tout});
  if (cols <= 0) a.ntiles = 0;
  ps_status s = a.ntiles ? tile_dispatch<CM_NONE, true>(a, ta, T, T, st) : PS_OK;
  if (s != PS_OK) return s;
  if (!a.ntiles) {   // empty rows: y = +0 (an empty sum); write via a 1-tile zero partial
    PS_CUDA(cudaMemsetAsync(a.qpart, 0, (size_t)rows * 8, st));
    a.ntiles = 1;
  }
  return T == PS_F64 ? rowdot_finalize<double>(a, out, tout, st) : rowdot_finalize<float>(a, out, tout, st);
}

ps_status colsum_async(const void *A, int ta, int64_t lda, const void *w, int tw, void *out,
                       int tout, int64_t rows, int64_t cols, int T, int mode, int fin, double n,
                       double eps, void *partial, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return PS_OK;
  TileArgs a = make_args(A, ta, lda, rows, cols, partial);
  a.w = w;
  a.tw = w ? tw : PS_F32;
  ps_status s;
  if (mode == COL_DOT) s = tile_dispatch<COL_DOT, false>(a, ta, T, T, st);
  else if (mode == COL_SUM) s = tile_dispatch<COL_SUM, false>(a, ta, T, T, st);
  else s = tile_dispatch<COL_SQDEV, false>(a, ta, T, T, st);
  if (s != PS_OK) return s;
  return T == PS_F64 ? colsum_finalize<double>(a, out, tout, fin, n, eps, st)
                     : colsum_finalize<float>(a, out, tout, fin, n, eps, st);
}

// MVT in one pass over A: x1 <- x1 + A y1 (row dots), x2 <- x2 + A^T y2 (column sums)
ps_status mvt_async(const void *A, int ta, int64_t n, void *x1, int t1, void *x2, int t2,
                    const void *y1, int ty1, const void *y2, int ty2, void *partial, cudaStream_t st) {
  if (n <= 0) return PS_OK;
  TileArgs a = make_args(A, ta, n, n, n, partial);
  a.w = y2;
  a.tw = ty2;
  a.x = y1;
  a.tx = ty1;
  const int TC = compute_type({ta, t2, ty2}), TR = compute_type({ta, t1, ty1});
  ps_status e = tile_dispatch<COL_DOT, true>(a, ta, TC, TR, st);
  if (e != PS_OK) return e;
  e = TC == PS_F64 ? colsum_finalize<double>(a, x2, t2, FIN_ADD, 0, 0, st)
                   : colsum_finalize<float>(a, x2, t2, FIN_ADD, 0, 0, st);
  if (e != PS_OK) return e;
  return TR == PS_F64 ? rowdot_finalize<double>(a, x1, t1, st, 1) : rowdot_finalize<float>(a, x1, t1, st, 1);
}

ps_status bicg_async(const void *A, int ta, int64_t lda, const void *r, int tr, void *s, int ts,
                     const void *p, int tp, void *q, int tq, int64_t rows, int64_t cols,
                     void *partial, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return PS_OK;
  TileArgs a = make_args(A, ta, lda, rows, cols, partial);
  a.w = r;
  a.tw = tr;
  a.x = p;
  a.tx = tp;
  const int TC = compute_type({ta, tr, ts}), TR = compute_type({ta, tp, tq});
  ps_status e = tile_dispatch<COL_DOT, true>(a, ta, TC, TR, st);
  if (e != PS_OK) return e;
  e = TC == PS_F64 ? colsum_finalize<double>(a, s, ts, FIN_PLAIN, 0, 0, st)
                   : colsum_finalize<float>(a, s, ts, FIN_PLAIN, 0, 0, st);
  if (e != PS_OK) return e;
  return TR == PS_F64 ? rowdot_finalize<double>(a, q, tq, st) : rowdot_finalize<float>(a, q, tq, st);
}

// ------------------------------------------------ row-sharded pieces (ps_shard_step)
// One rank's tile pass over its rows of A: A, w (COL_DOT weights) and the row-dot
// output start at the rank's first row r0 (a multiple of COLSUM_CHUNK), `spart`
// points at chunk r0 / COLSUM_CHUNK of the FULL column-chunk partial array (typed
// TC, cols per chunk), so every rank fills its own chunks of the same array; row
// dots (rd_out != nullptr) are finished locally for the rank's rows.  After the
// chunks of all ranks are in place, colsum_finalize_async adds them in chunk order
// -- the same association as the unsharded statement (R5), so the result is
// bit-identical for any rank count.
ps_status tile_rows_async(int mode, const void *A, int ta, int64_t lda, const void *w, int tw,
                          const void *x, int tx, void *rd_out, int t_rd, int rd_add, int64_t rows,
                          int64_t cols, int TC, void *spart, void *qpart, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return PS_OK;
  TileArgs a = make_args(A, ta, lda, rows, cols, nullptr);
  a.spart = spart;
  a.qpart = qpart;
  a.w = w;
  a.tw = w ? tw : PS_F32;
  a.x = x;
  a.tx = x ? tx : PS_F32;
  const bool rd = rd_out != nullptr;
  const int TR = rd ? compute_type({ta, tx, t_rd}) : TC;
  ps_status e;
  if (rd && mode == CM_NONE) e = tile_dispatch<CM_NONE, true>(a, ta, TR, TR, st);
  else if (rd && mode == COL_DOT) e = tile_dispatch<COL_DOT, true>(a, ta, TC, TR, st);
  else if (!rd && mode == COL_DOT) e = tile_dispatch<COL_DOT, false>(a, ta, TC, TC, st);
  else if (!rd && mode == COL_SUM) e = tile_dispatch<COL_SUM, false>(a, ta, TC, TC, st);
  else if (!rd && mode == COL_SQDEV) e = tile_dispatch<COL_SQDEV, false>(a, ta, TC, TC, st);
  else {
    set_error("tile_rows_async: unsupported mode");
    return PS_ERR_UNSUPPORTED;
  }
  if (e != PS_OK || !rd) return e;
  return TR == PS_F64 ? rowdot_finalize<double>(a, rd_out, t_rd, st, rd_add)
                      : rowdot_finalize<float>(a, rd_out, t_rd, st, rd_add);
}

ps_status colsum_finalize_async(const void *spart, int TC, int64_t rows, int64_t cols, void *out, int tout,
                                int fin, double n, double eps, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return PS_OK;
  TileArgs a{};
  a.spart = const_cast<void *>(spart);
  a.rows = rows;
  a.cols = cols;
  a.nchunks = nchunks_of(rows);
  return TC == PS_F64 ? colsum_finalize<double>(a, out, tout, fin, n, eps, st)
                      : colsum_finalize<float>(a, out, tout, fin, n, eps, st);
}

size_t tile_spart_bytes(int64_t rows, int64_t cols) { return spart_bytes(rows, cols); }

}  // namespace ps
