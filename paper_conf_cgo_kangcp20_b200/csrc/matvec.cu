// matvec.cu -- bandwidth-bound statements of ATAX / BICG / GESUMMV / CORR /
// COVAR (row a3), in the canonical reduction orders of reading R5.
//
//  * rowdot: one warp per row.  Lane l owns the 16-byte chunks c = t*32 + l of
//    the row (V = 16 / sizeof(stored A) elements), runs an fma chain over them
//    (t ascending, then v ascending) and the warp combines by xor butterfly
//    16,8,4,2,1 (a + partner).  Loads are 128-bit, 4 chunks in flight per lane.
//  * colsum: a thread owns V adjacent columns of one 256-row chunk and runs an
//    fma chain down the rows (i ascending, 8 rows of loads in flight); a second
//    kernel adds the chunk partials in ascending chunk order and applies the
//    finalisation (plain / mean / stddev).
// Both are HBM-bound: algorithmic bytes = rows*cols*sizeof(stored A) + O(n).
#include <math.h>

#include "common.cuh"
#include "kernels.cuh"

namespace ps {

template <class A, class B> struct Wider { using t = float; };
template <class B> struct Wider<double, B> { using t = double; };
template <class A> struct Wider<A, double> { using t = double; };
template <> struct Wider<double, double> { using t = double; };
template <class S> struct CT { using t = typename Wider<S, float>::t; };   // storage -> min compute
template <> struct CT<F16> { using t = float; };
template <class A, class B, class C>
using T3 = typename Wider<typename Wider<typename CT<A>::t, typename CT<B>::t>::t,
                          typename CT<C>::t>::t;

template <class S, class T>
__device__ __forceinline__ T ldg_t(const raw_t<S> *p, int64_t i) {
  return Ld<S, T>::get(p, (size_t)i);
}

// ------------------------------------------------------------------ rowdot
// A warp owns RB consecutive rows and walks them together: per 16-byte chunk
// position c it loads the A chunk of every row and the matching x chunk ONCE
// (vectorised, widened to T once), then advances the RB independent lane
// chains.  Per row the order is exactly R5 (lane l: chunks c = t*32 + l,
// t ascending, v ascending; butterfly 16..1), so results are unchanged by RB.
template <class SX, int V, class T>
__device__ __forceinline__ void load_x_chunk(const raw_t<SX> *__restrict__ x, int64_t j0, T *out) {
  using RX = raw_t<SX>;
  constexpr int BYTES = V * (int)sizeof(RX);
  if constexpr (BYTES >= 16) {
    const uint4 *p = reinterpret_cast<const uint4 *>(x + j0);
    constexpr int PER = 16 / (int)sizeof(RX);
#pragma unroll
    for (int k = 0; k < BYTES / 16; k++) {
      union { uint4 u; RX e[PER]; } t;
      t.u = __ldg(p + k);
#pragma unroll
      for (int e = 0; e < PER; e++) out[k * PER + e] = Ld<SX, T>::get(&t.e[e], 0);
    }
  } else if constexpr (BYTES == 8) {
    union { uint2 u; RX e[V]; } t;
    t.u = __ldg(reinterpret_cast<const uint2 *>(x + j0));
#pragma unroll
    for (int e = 0; e < V; e++) out[e] = Ld<SX, T>::get(&t.e[e], 0);
  } else {
    union { uint32_t u; RX e[V]; } t;
    t.u = __ldg(reinterpret_cast<const unsigned int *>(x + j0));
#pragma unroll
    for (int e = 0; e < V; e++) out[e] = Ld<SX, T>::get(&t.e[e], 0);
  }
}

template <class SA, class SX, class SO, int RB>
__global__ void __launch_bounds__(256) rowdot_kernel(const raw_t<SA> *__restrict__ A, int64_t lda,
                                                     const raw_t<SX> *__restrict__ x,
                                                     raw_t<SO> *__restrict__ out, int64_t rows,
                                                     int64_t cols, int vec_ok) {
  using T = T3<SA, SX, SO>;
  using RA = raw_t<SA>;
  constexpr int V = 16 / sizeof(RA);
  constexpr int UN = 2;
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  const int64_t nchunks = (cols + V - 1) / V;
  const int64_t full = cols / V;   // chunks entirely inside the row
  const int64_t ngroups = (rows + RB - 1) / RB;
  for (int64_t g = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); g < ngroups;
       g += (int64_t)gridDim.x * wpb) {
    const int64_t r0 = g * RB;
    const int nr = (int)((rows - r0) < RB ? (rows - r0) : RB);
    T acc[RB];
#pragma unroll
    for (int r = 0; r < RB; r++) acc[r] = T(0);
    int64_t c = lane;
    if (vec_ok && nr == RB) {
      const uint4 *arow[RB];
#pragma unroll
      for (int r = 0; r < RB; r++) arow[r] = reinterpret_cast<const uint4 *>(A + (r0 + r) * lda);
      for (; c + 32 * (UN - 1) < full; c += 32 * UN) {
        union { uint4 v; RA e[V]; } ch[UN][RB];
#pragma unroll
        for (int u = 0; u < UN; u++)
#pragma unroll
          for (int r = 0; r < RB; r++) ch[u][r].v = __ldg(arow[r] + c + 32 * u);
#pragma unroll
        for (int u = 0; u < UN; u++) {
          T xv[V];
          load_x_chunk<SX, V, T>(x, (c + 32 * u) * V, xv);
#pragma unroll
          for (int r = 0; r < RB; r++)
#pragma unroll
            for (int v = 0; v < V; v++)
              acc[r] = t_fma(Ld<SA, T>::get(&ch[u][r].e[v], 0), xv[v], acc[r]);
        }
      }
      for (; c < full; c += 32) {
        union { uint4 v; RA e[V]; } ch[RB];
#pragma unroll
        for (int r = 0; r < RB; r++) ch[r].v = __ldg(arow[r] + c);
        T xv[V];
        load_x_chunk<SX, V, T>(x, c * V, xv);
#pragma unroll
        for (int r = 0; r < RB; r++)
#pragma unroll
          for (int v = 0; v < V; v++) acc[r] = t_fma(Ld<SA, T>::get(&ch[r].e[v], 0), xv[v], acc[r]);
      }
    }
    // scalar path: unaligned rows, a ragged row group, the ragged last chunk
    for (; c < nchunks; c += 32) {
      const int64_t j0 = c * V;
      for (int v = 0; v < V && j0 + v < cols; v++) {
        const T xj = ldg_t<SX, T>(x, j0 + v);
#pragma unroll
        for (int r = 0; r < RB; r++)
          if (r < nr) acc[r] = t_fma(ldg_t<SA, T>(A + (r0 + r) * lda, j0 + v), xj, acc[r]);
      }
    }
    T mine = T(0);
#pragma unroll
    for (int r = 0; r < RB; r++) {
#pragma unroll
      for (int off = 16; off >= 1; off >>= 1) acc[r] = acc[r] + __shfl_xor_sync(0xffffffffu, acc[r], off);
      if (lane == r) mine = acc[r];
    }
    if (lane < nr) St<SO, T>::put(out, (size_t)(r0 + lane), mine);
  }
}

ps_status rowdot_async(const void *A, int ta, int64_t lda, const void *x, int tx, void *out,
                       int tout, int64_t rows, int64_t cols, cudaStream_t st) {
  if (rows <= 0) return PS_OK;
  constexpr int RB = 4;
  const int vec_ok = ((uintptr_t)A % 16 == 0) && ((lda * (int64_t)dtype_size(ta)) % 16 == 0) &&
                     ((uintptr_t)x % 16 == 0);
  const int64_t wpb = 8;
  const int64_t ngroups = (rows + RB - 1) / RB;
  int64_t blocks = (ngroups + wpb - 1) / wpb;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  return dispatch_store(ta, [&](auto sa) -> ps_status {
    return dispatch_store(tx, [&](auto sx) -> ps_status {
      return dispatch_store(tout, [&](auto so) -> ps_status {
        using SA = decltype(sa);
        using SX = decltype(sx);
        using SO = decltype(so);
        rowdot_kernel<SA, SX, SO, RB><<<(unsigned)blocks, 256, 0, st>>>(
            (const raw_t<SA> *)A, lda, (const raw_t<SX> *)x, (raw_t<SO> *)out, rows, cols, vec_ok);
        PS_CHECK_LAUNCH("rowdot_kernel");
        return PS_OK;
      });
    });
  });
}

// ------------------------------------------------------------------ colsum
template <class SA, class SW, class T, int MODE>
__global__ void __launch_bounds__(256) colsum_partial_kernel(const raw_t<SA> *__restrict__ A,
                                                             int64_t lda,
                                                             const raw_t<SW> *__restrict__ w,
                                                             T *__restrict__ partial, int64_t rows,
                                                             int64_t cols, int vec_ok) {
  using RA = raw_t<SA>;
  constexpr int V = 16 / sizeof(RA);
  constexpr int UR = 8;
  const int64_t chunk = blockIdx.y;
  const int64_t i0 = chunk * COLSUM_CHUNK;
  const int64_t i1 = (i0 + COLSUM_CHUNK < rows) ? i0 + COLSUM_CHUNK : rows;
  const int64_t j0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * V;
  if (j0 >= cols) return;
  T p[V];
  T mu[V];
#pragma unroll
  for (int v = 0; v < V; v++) {
    p[v] = T(0);
    mu[v] = (MODE == COL_SQDEV && j0 + v < cols) ? ldg_t<SW, T>(w, j0 + v) : T(0);
  }
  auto term = [&](int v, T a, T wi) {
    if (MODE == COL_DOT) p[v] = t_fma(a, wi, p[v]);
    else if (MODE == COL_SUM) p[v] = p[v] + a;
    else { const T d = a - mu[v]; p[v] = t_fma(d, d, p[v]); }
  };
  if (vec_ok && j0 + V <= cols) {
    int64_t i = i0;
    for (; i + UR <= i1; i += UR) {
      union { uint4 v; RA e[V]; } ch[UR];
      T wi[UR];
#pragma unroll
      for (int r = 0; r < UR; r++) {
        ch[r].v = __ldg(reinterpret_cast<const uint4 *>(A + (i + r) * lda + j0));
        wi[r] = (MODE == COL_DOT) ? ldg_t<SW, T>(w, i + r) : T(0);
      }
#pragma unroll
      for (int r = 0; r < UR; r++)
#pragma unroll
        for (int v = 0; v < V; v++) {
          const RA e = ch[r].e[v];
          term(v, Ld<SA, T>::get(&e, 0), wi[r]);
        }
    }
    for (; i < i1; i++) {
      union { uint4 v; RA e[V]; } ch;
      ch.v = __ldg(reinterpret_cast<const uint4 *>(A + i * lda + j0));
      const T wi = (MODE == COL_DOT) ? ldg_t<SW, T>(w, i) : T(0);
#pragma unroll
      for (int v = 0; v < V; v++) {
        const RA e = ch.e[v];
        term(v, Ld<SA, T>::get(&e, 0), wi);
      }
    }
  } else {
    for (int64_t i = i0; i < i1; i++) {
      const T wi = (MODE == COL_DOT) ? ldg_t<SW, T>(w, i) : T(0);
#pragma unroll
      for (int v = 0; v < V; v++)
        if (j0 + v < cols) term(v, ldg_t<SA, T>(A, i * lda + j0 + v), wi);
    }
  }
#pragma unroll
  for (int v = 0; v < V; v++)
    if (j0 + v < cols) partial[chunk * cols + j0 + v] = p[v];
}

template <class T, class SO, int FIN>
__global__ void __launch_bounds__(256) colsum_finalize_kernel(const T *__restrict__ partial,
                                                              raw_t<SO> *__restrict__ out,
                                                              int64_t cols, int64_t nchunks, T n,
                                                              T eps) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= cols) return;
  T total = partial[j];
  for (int64_t c = 1; c < nchunks; c++) total = total + partial[c * cols + j];
  if (FIN == FIN_MEAN) total = total / n;
  if (FIN == FIN_STDDEV) {
    total = sqrt(total / n);
    if (total <= eps) total = T(1);
  }
  St<SO, T>::put(out, (size_t)j, total);
}

size_t colsum_partial_bytes(int64_t rows, int64_t cols) {
  const int64_t nchunks = (rows + COLSUM_CHUNK - 1) / COLSUM_CHUNK;
  return (size_t)nchunks * (size_t)cols * sizeof(double);
}

template <class T>
static ps_status colsum_t(const void *A, int ta, int64_t lda, const void *w, int tw, void *out,
                          int tout, int64_t rows, int64_t cols, int mode, int fin, double n,
                          double eps, void *partial, cudaStream_t st) {
  const int64_t nchunks = (rows + COLSUM_CHUNK - 1) / COLSUM_CHUNK;
  const int vec_ok = ((uintptr_t)A % 16 == 0) && ((lda * (int64_t)dtype_size(ta)) % 16 == 0);
  const int V = 16 / (int)dtype_size(ta);
  dim3 grid((unsigned)((cols / V + 1 + 255) / 256), (unsigned)nchunks);
  ps_status s = dispatch_store(ta, [&](auto sa) -> ps_status {
    return dispatch_store(tw, [&](auto sw) -> ps_status {
      using SA = decltype(sa);
      using SW = decltype(sw);
      if (mode == COL_DOT)
        colsum_partial_kernel<SA, SW, T, COL_DOT><<<grid, 256, 0, st>>>(
            (const raw_t<SA> *)A, lda, (const raw_t<SW> *)w, (T *)partial, rows, cols, vec_ok);
      else if (mode == COL_SUM)
        colsum_partial_kernel<SA, SW, T, COL_SUM><<<grid, 256, 0, st>>>(
            (const raw_t<SA> *)A, lda, (const raw_t<SW> *)w, (T *)partial, rows, cols, vec_ok);
      else
        colsum_partial_kernel<SA, SW, T, COL_SQDEV><<<grid, 256, 0, st>>>(
            (const raw_t<SA> *)A, lda, (const raw_t<SW> *)w, (T *)partial, rows, cols, vec_ok);
      PS_CHECK_LAUNCH("colsum_partial_kernel");
      return PS_OK;
    });
  });
  if (s != PS_OK) return s;
  const unsigned fb = (unsigned)((cols + 255) / 256);
  // n and eps: RNE from their fp64 literal to T (R2)
  return dispatch_store(tout, [&](auto so) -> ps_status {
    using SO = decltype(so);
    if (fin == FIN_PLAIN)
      colsum_finalize_kernel<T, SO, FIN_PLAIN><<<fb, 256, 0, st>>>(
          (const T *)partial, (raw_t<SO> *)out, cols, nchunks, (T)n, (T)eps);
    else if (fin == FIN_MEAN)
      colsum_finalize_kernel<T, SO, FIN_MEAN><<<fb, 256, 0, st>>>(
          (const T *)partial, (raw_t<SO> *)out, cols, nchunks, (T)n, (T)eps);
    else
      colsum_finalize_kernel<T, SO, FIN_STDDEV><<<fb, 256, 0, st>>>(
          (const T *)partial, (raw_t<SO> *)out, cols, nchunks, (T)n, (T)eps);
    PS_CHECK_LAUNCH("colsum_finalize_kernel");
    return PS_OK;
  });
}

ps_status colsum_async(const void *A, int ta, int64_t lda, const void *w, int tw, void *out,
                       int tout, int64_t rows, int64_t cols, int T, int mode, int fin, double n,
                       double eps, void *partial, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return PS_OK;
  if (!w) tw = PS_F32;   // unused operand (COL_SUM)
  if (T == PS_F64)
    return colsum_t<double>(A, ta, lda, w, tw, out, tout, rows, cols, mode, fin, n, eps, partial, st);
  return colsum_t<float>(A, ta, lda, w, tw, out, tout, rows, cols, mode, fin, n, eps, partial, st);
}

// --------------------------------------------------- GESUMMV statement 3
template <class STMP, class SY>
__global__ void axpby_kernel(const raw_t<STMP> *__restrict__ tmp, raw_t<SY> *__restrict__ y,
                             int64_t n, typename Wider<typename CT<STMP>::t, typename CT<SY>::t>::t al,
                             typename Wider<typename CT<STMP>::t, typename CT<SY>::t>::t be) {
  using T = typename Wider<typename CT<STMP>::t, typename CT<SY>::t>::t;
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const T r = t_fma(al, ldg_t<STMP, T>(tmp, i), be * Ld<SY, T>::get(y, (size_t)i));
  St<SY, T>::put(y, (size_t)i, r);
}

ps_status axpby_async(const void *tmp, int ttmp, void *y, int ty, int64_t n, double alpha,
                      double beta, cudaStream_t st) {
  if (n <= 0) return PS_OK;
  const unsigned nb = (unsigned)((n + 255) / 256);
  return dispatch_store(ttmp, [&](auto s1) -> ps_status {
    return dispatch_store(ty, [&](auto s2) -> ps_status {
      using S1 = decltype(s1);
      using S2 = decltype(s2);
      using T = typename Wider<typename CT<S1>::t, typename CT<S2>::t>::t;
      axpby_kernel<S1, S2><<<nb, 256, 0, st>>>((const raw_t<S1> *)tmp, (raw_t<S2> *)y, n, (T)alpha,
                                               (T)beta);
      PS_CHECK_LAUNCH("axpby_kernel");
      return PS_OK;
    });
  });
}

// ------------------------------------------------------ CORR / COVAR
template <class SD, class SM, class SS>
__global__ void __launch_bounds__(256) corr_normalize_kernel(raw_t<SD> *__restrict__ data,
                                                             const raw_t<SM> *__restrict__ mean,
                                                             const raw_t<SS> *__restrict__ sd,
                                                             int64_t rows, int64_t cols,
                                                             T3<SD, SM, SS> sqn) {
  using T = T3<SD, SM, SS>;
  const int64_t total = rows * cols;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = e % cols;
    const T d = Ld<SD, T>::get(data, (size_t)e) - ldg_t<SM, T>(mean, j);
    const T den = sqn * ldg_t<SS, T>(sd, j);
    St<SD, T>::put(data, (size_t)e, d / den);
  }
}

ps_status corr_normalize_async(void *data, int td, const void *mean, int tm, const void *sd, int ts,
                               int64_t rows, int64_t cols, double sqrt_n, cudaStream_t st) {
  const int64_t total = rows * cols;
  if (total <= 0) return PS_OK;
  int64_t blocks = (total + 255) / 256;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  return dispatch_store(td, [&](auto a) -> ps_status {
    return dispatch_store(tm, [&](auto b) -> ps_status {
      return dispatch_store(ts, [&](auto c) -> ps_status {
        using SD = decltype(a);
        using SM = decltype(b);
        using SS = decltype(c);
        using T = T3<SD, SM, SS>;
        corr_normalize_kernel<SD, SM, SS><<<(unsigned)blocks, 256, 0, st>>>(
            (raw_t<SD> *)data, (const raw_t<SM> *)mean, (const raw_t<SS> *)sd, rows, cols,
            (T)sqrt_n);
        PS_CHECK_LAUNCH("corr_normalize_kernel");
        return PS_OK;
      });
    });
  });
}

template <class SD, class SM>
__global__ void __launch_bounds__(256) covar_center_kernel(raw_t<SD> *__restrict__ data,
                                                           const raw_t<SM> *__restrict__ mean,
                                                           int64_t rows, int64_t cols) {
  using T = typename Wider<typename CT<SD>::t, typename CT<SM>::t>::t;
  const int64_t total = rows * cols;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = e % cols;
    St<SD, T>::put(data, (size_t)e, Ld<SD, T>::get(data, (size_t)e) - ldg_t<SM, T>(mean, j));
  }
}

ps_status covar_center_async(void *data, int td, const void *mean, int tm, int64_t rows,
                             int64_t cols, cudaStream_t st) {
  const int64_t total = rows * cols;
  if (total <= 0) return PS_OK;
  int64_t blocks = (total + 255) / 256;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  return dispatch_store(td, [&](auto a) -> ps_status {
    return dispatch_store(tm, [&](auto b) -> ps_status {
      using SD = decltype(a);
      using SM = decltype(b);
      covar_center_kernel<SD, SM><<<(unsigned)blocks, 256, 0, st>>>(
          (raw_t<SD> *)data, (const raw_t<SM> *)mean, rows, cols);
      PS_CHECK_LAUNCH("covar_center_kernel");
      return PS_OK;
    });
  });
}

}  // namespace ps
