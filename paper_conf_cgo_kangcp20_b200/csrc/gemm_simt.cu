// gemm_simt.cu -- R3-exact SIMT contractions for the GEMM / 2MM / 3MM / SYRK
// statements whose compute type is f32 (FFMA) or f64 (DFMA), i.e. every
// contraction that does not have two fp16 multiplicands (those go to tcgen05,
// gemm_tc.cu), and every contraction when PS_FLAG_NO_TENSOR_CORES is set.
//
// Reading R3: C_ij = sum_k A_ik B_kj is an fma chain from +0 with k ascending.
// Each thread owns TM x TN accumulators and walks k tile by tile in ascending
// order, so every output is exactly the oracle's chain (bit-exact).
// Operands are loaded in their stored precision (f16/f32/f64, runtime type,
// arbitrary row/col strides so SYRK's data^T needs no transpose), widened
// exactly to T in shared memory; the epilogue rounds RNE to the output's
// precision (R1).  Register-prefetched double-buffered smem tiles.
#include "common.cuh"
#include "kernels.cuh"

namespace ps {

template <class T>
__device__ __forceinline__ T load_elem(const void *p, int type, int64_t idx) {
  switch (type) {
    case PS_F64: return (T)((const double *)p)[idx];
    case PS_F32: return (T)((const float *)p)[idx];
    default: return widen_h<T>(((const uint16_t *)p)[idx]);
  }
}

template <class T>
__device__ __forceinline__ void store_elem(void *p, int type, int64_t idx, T v) {
  switch (type) {
    case PS_F64: ((double *)p)[idx] = (double)v; break;
    case PS_F32: St<float, T>::put((float *)p, idx, v); break;
    default: St<F16, T>::put((uint16_t *)p, idx, v); break;
  }
}

template <class T> struct SimtCfg;
template <> struct SimtCfg<float> { static constexpr int BM = 128, BN = 128, BK = 8, TM = 8, TN = 8; };
template <> struct SimtCfg<double> { static constexpr int BM = 64, BN = 64, BK = 8, TM = 4, TN = 4; };

struct GemmKParams {
  int64_t M, N, K;
  const void *A;
  int ta;
  int64_t a_sr, a_sc;
  const void *B;
  int tb;
  int64_t b_sr, b_sc;
  void *C;
  int tc;
  int64_t ldc;
  const void *Cin;
  int tcin;
  int epi;
  int upper_only;
};

template <class T>
__global__ void __launch_bounds__(256) gemm_simt_kernel(GemmKParams p, T alpha, T beta, T div) {
  constexpr int BM = SimtCfg<T>::BM, BN = SimtCfg<T>::BN, BK = SimtCfg<T>::BK;
  constexpr int TM = SimtCfg<T>::TM, TN = SimtCfg<T>::TN;
  constexpr int LA = BM * BK / 256, LB = BK * BN / 256;   // elements per thread per tile
  constexpr int GM = TM / 4, GN = TN / 4;                 // 4-wide groups per thread
  __shared__ __align__(16) T As[2][BK][BM];
  __shared__ __align__(16) T Bs[2][BK][BN];

  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int64_t m0 = (int64_t)blockIdx.y * BM, n0 = (int64_t)blockIdx.x * BN;
  if (p.upper_only && m0 >= n0 + BN) return;   // tile strictly below the diagonal

  const bool a_kcontig = (p.a_sc == 1);
  const bool b_ncontig = (p.b_sc == 1);
  T ra[LA], rb[LB];

  auto load_tiles = [&](int64_t k0) {
#pragma unroll
    for (int q = 0; q < LA; q++) {
      const int e = tid + 256 * q;
      const int m = a_kcontig ? e / BK : e % BM;
      const int k = a_kcontig ? e % BK : e / BM;
      const int64_t gm = m0 + m, gk = k0 + k;
      ra[q] = (gm < p.M && gk < p.K) ? load_elem<T>(p.A, p.ta, gm * p.a_sr + gk * p.a_sc) : T(0);
    }
#pragma unroll
    for (int q = 0; q < LB; q++) {
      const int e = tid + 256 * q;
      const int n = b_ncontig ? e % BN : e / BK;
      const int k = b_ncontig ? e / BN : e % BK;
      const int64_t gn = n0 + n, gk = k0 + k;
      rb[q] = (gn < p.N && gk < p.K) ? load_elem<T>(p.B, p.tb, gk * p.b_sr + gn * p.b_sc) : T(0);
    }
  };
  auto store_tiles = [&](int buf) {
#pragma unroll
    for (int q = 0; q < LA; q++) {
      const int e = tid + 256 * q;
      const int m = a_kcontig ? e / BK : e % BM;
      const int k = a_kcontig ? e % BK : e / BM;
      As[buf][k][m] = ra[q];
    }
#pragma unroll
    for (int q = 0; q < LB; q++) {
      const int e = tid + 256 * q;
      const int n = b_ncontig ? e % BN : e / BK;
      const int k = b_ncontig ? e / BN : e % BK;
      Bs[buf][k][n] = rb[q];
    }
  };

  T acc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; i++)
#pragma unroll
    for (int j = 0; j < TN; j++) acc[i][j] = T(0);

  const int64_t ktiles = (p.K + BK - 1) / BK;
  load_tiles(0);
  store_tiles(0);
  __syncthreads();
  int buf = 0;
  for (int64_t kt = 0; kt < ktiles; kt++) {
    const bool more = kt + 1 < ktiles;
    if (more) load_tiles((kt + 1) * BK);
#pragma unroll
    for (int k = 0; k < BK; k++) {
      T a[TM], b[TN];
#pragma unroll
      for (int g = 0; g < GM; g++)
#pragma unroll
        for (int i = 0; i < 4; i++) a[g * 4 + i] = As[buf][k][g * (BM / GM) + ty * 4 + i];
#pragma unroll
      for (int g = 0; g < GN; g++)
#pragma unroll
        for (int j = 0; j < 4; j++) b[g * 4 + j] = Bs[buf][k][g * (BN / GN) + tx * 4 + j];
#pragma unroll
      for (int i = 0; i < TM; i++)
#pragma unroll
        for (int j = 0; j < TN; j++) acc[i][j] = t_fma(a[i], b[j], acc[i][j]);   // R3
    }
    if (more) {
      store_tiles(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }

  // epilogue (R3): plain / fma(alpha, acc, beta*Cin) / acc / div, then RNE store (R1)
#pragma unroll
  for (int i = 0; i < TM; i++) {
    const int64_t gm = m0 + (i / 4) * (BM / GM) + ty * 4 + (i % 4);
    if (gm >= p.M) continue;
#pragma unroll
    for (int j = 0; j < TN; j++) {
      const int64_t gn = n0 + (j / 4) * (BN / GN) + tx * 4 + (j % 4);
      if (gn >= p.N) continue;
      T r = acc[i][j];
      const int64_t idx = gm * p.ldc + gn;
      if (p.epi == EPI_AXPBY) {
        const T bc = beta * load_elem<T>(p.Cin, p.tcin, idx);
        r = t_fma(alpha, r, bc);
      } else if (p.epi == EPI_DIV) {
        r = r / div;
      }
      store_elem<T>(p.C, p.tc, idx, r);
    }
  }
}

ps_status gemm_simt_async(const GemmArgs &g, cudaStream_t st) {
  if (g.M <= 0 || g.N <= 0) return PS_OK;
  GemmKParams p{g.M, g.N, g.K, g.A.p, g.A.type, g.A.s_row, g.A.s_col, g.B.p, g.B.type,
                g.B.s_row, g.B.s_col, g.C, g.c_type, g.ldc, g.Cin, g.cin_type, g.epi,
                g.upper_only};
  if (g.T == PS_F64) {
    using C = SimtCfg<double>;
    dim3 grid((unsigned)((g.N + C::BN - 1) / C::BN), (unsigned)((g.M + C::BM - 1) / C::BM));
    gemm_simt_kernel<double><<<grid, 256, 0, st>>>(p, g.alpha, g.beta, g.div);
  } else {
    using C = SimtCfg<float>;
    dim3 grid((unsigned)((g.N + C::BN - 1) / C::BN), (unsigned)((g.M + C::BM - 1) / C::BM));
    // scalars are RNE-rounded from their fp64 literal to T (R2); host cast is RNE
    gemm_simt_kernel<float><<<grid, 256, 0, st>>>(p, (float)g.alpha, (float)g.beta, (float)g.div);
  }
  PS_CHECK_LAUNCH("gemm_simt_kernel");
  return PS_OK;
}

// ------------------------------------------------------------ SYRK mirror
template <class S>
__global__ void __launch_bounds__(256) mirror_kernel(raw_t<S> *s, int64_t M, int diag_one) {
  __shared__ raw_t<S> tile[32][33];
  const int64_t bx = blockIdx.x, by = blockIdx.y;   // source tile (row block bx, col block by), bx <= by
  if (bx > by) return;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;   // 32 x 8
  for (int r = ty; r < 32; r += 8) {
    const int64_t gi = bx * 32 + r, gj = by * 32 + tx;
    if (gi < M && gj < M) tile[r][tx] = s[gi * M + gj];
  }
  __syncthreads();
  // destination (row block by, col block bx): element (i, j) = source (j, i), for i > j
  for (int r = ty; r < 32; r += 8) {
    const int64_t gi = by * 32 + r, gj = bx * 32 + tx;
    if (gi < M && gj < M && gi > gj) s[gi * M + gj] = tile[tx][r];
  }
  if (diag_one && bx == by) {
    __syncthreads();
    if (threadIdx.x < 32) {
      const int64_t gd = bx * 32 + threadIdx.x;
      if (gd < M) St<S, float>::put(s, gd * M + gd, 1.0f);
    }
  }
}

ps_status mirror_async(void *S, int type, int64_t M, int diag_one, cudaStream_t st) {
  if (M <= 0) return PS_OK;
  dim3 grid((unsigned)((M + 31) / 32), (unsigned)((M + 31) / 32));
  return dispatch_store(type, [&](auto s) -> ps_status {
    using ST = decltype(s);
    mirror_kernel<ST><<<grid, 256, 0, st>>>((raw_t<ST> *)S, M, diag_one);
    PS_CHECK_LAUNCH("mirror_kernel");
    return PS_OK;
  });
}

}  // namespace ps
