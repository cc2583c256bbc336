// gemm_simt.cuh -- R3-exact SIMT contraction kernel template (FFMA / DFMA).
//
// Reading R3: C_ij = sum_k A_ik B_kj is an fma chain from +0, k ascending.
// Every thread owns 8 x 8 accumulators and walks k tile by tile in ascending
// order, so each output is exactly the oracle's chain (bit-exact).  Operands
// are read in their stored precision (template SA / SB), widened exactly to T
// when staged in shared memory (R1); the epilogue rounds RNE to the output's
// precision.  A is k-contiguous (row-major) or m-contiguous (SYRK's data^T),
// B is n-contiguous.  Loads are 16-byte vector runs on a CTA-uniform in-bounds
// fast path (bounds-checked scalars only on edge tiles); register-prefetched,
// double-buffered shared-memory tiles.
#pragma once
#include <type_traits>

#include "common.cuh"
#include "kernels.cuh"

namespace ps {
namespace simt {

template <class T> struct Cfg;
// CH: consecutive columns per thread chunk (one 16-byte shared load); a thread's TN
// columns are TN/CH chunks spaced TX*CH apart, so 8 lanes of a quarter-warp read 128
// contiguous bytes of B (conflict-free for 8-byte T as well as 4-byte T).  Threads:
// TX along N x 16 along M; each owns TM = 8 rows (two runs of 4, BM/2 apart).
// (Measured at 8192^3 on B200, f64: 256 threads x 8 x 8, BK = 8 -> 22.6 TFLOP/s; BK = 16
// -> 20.9 (254 registers); 512 threads x 8 x 4, BK = 16 -> 21.1.)
template <> struct Cfg<float> {
  static constexpr int BM = 128, BN = 128, BK = 16, TM = 8, TN = 8, CH = 4, TX = 16, THREADS = 256;
};
template <> struct Cfg<double> {
  static constexpr int BM = 128, BN = 128, BK = 8, TM = 8, TN = 8, CH = 2, TX = 16, THREADS = 256;
};
template <class T> constexpr int smem_bytes() {
  return 2 * Cfg<T>::BK * (Cfg<T>::BM + Cfg<T>::BN) * (int)sizeof(T);
}

struct Params {
  int64_t M, N, K;
  const void *A;
  int64_t a_sr, a_sc;
  const void *B;
  int64_t b_sr;
  void *C;
  int tc;
  int64_t ldc;
  const void *Cin;
  int tcin;
  int epi;
  int upper_only;
  int64_t row_off;    // global row of C's row 0 (upper_only test)
  int a_vec, b_vec;   // 16-byte aligned base and leading dimension
};

template <class T>
__device__ __forceinline__ T load_elem(const void *p, int type, int64_t idx) {
  switch (type) {
    case PS_F64: return (T)((const double *)p)[idx];
    case PS_F32: return (T)((const float *)p)[idx];
    case PS_BF16: return widen_b<T>(((const uint16_t *)p)[idx]);
    default: return widen_h<T>(((const uint16_t *)p)[idx]);
  }
}
template <class T>
__device__ __forceinline__ void store_elem(void *p, int type, int64_t idx, T v) {
  switch (type) {
    case PS_F64: ((double *)p)[idx] = (double)v; break;
    case PS_F32: St<float, T>::put((float *)p, idx, v); break;
    case PS_BF16: St<BF16, T>::put((uint16_t *)p, idx, v); break;
    default: St<F16, T>::put((uint16_t *)p, idx, v); break;
  }
}

// E contiguous stored elements -> T (vector loads; the run is aligned to its size or 16 B)
template <class S, int E, class T>
__device__ __forceinline__ void load_run(const raw_t<S> *p, T (&out)[E]) {
  using R = raw_t<S>;
  constexpr int BYTES = E * (int)sizeof(R);
  if constexpr (BYTES >= 16) {
    constexpr int PER = 16 / (int)sizeof(R);
#pragma unroll
    for (int q = 0; q < BYTES / 16; q++) {
      union { uint4 u; R e[PER]; } t;
      t.u = __ldg(reinterpret_cast<const uint4 *>(p) + q);
#pragma unroll
      for (int e = 0; e < PER; e++) out[q * PER + e] = Ld<S, T>::get(&t.e[e], 0);
    }
  } else if constexpr (BYTES == 8) {
    union { uint2 u; R e[E]; } t;
    t.u = __ldg(reinterpret_cast<const uint2 *>(p));
#pragma unroll
    for (int e = 0; e < E; e++) out[e] = Ld<S, T>::get(&t.e[e], 0);
  } else {
    union { unsigned int u; R e[E]; } t;
    t.u = __ldg(reinterpret_cast<const unsigned int *>(p));
#pragma unroll
    for (int e = 0; e < E; e++) out[e] = Ld<S, T>::get(&t.e[e], 0);
  }
}

// ---- cp.async and raw-run helpers (gemm_dmma.cu, gemm_ffma.cu)
__device__ __forceinline__ void cp_async16(void *smem, const void *gmem) {
  const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(gmem));
}
// 4- / 8-byte copies, zero-filled when !valid (edge tiles and unaligned rows of f64 operands)
__device__ __forceinline__ void cp_async8z(void *smem, const void *gmem, bool valid) {
  const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(sa), "l"(gmem), "r"(valid ? 8 : 0));
}
__device__ __forceinline__ void cp_async4z(void *smem, const void *gmem, bool valid) {
  const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(sa), "l"(gmem), "r"(valid ? 4 : 0));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N> __device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;\n" ::"n"(N));
}

// E contiguous stored elements (16-byte aligned run), raw bits; widened at the
// shared-memory store so the global loads stay in flight across the tile's MMAs
template <class R, int E>
__device__ __forceinline__ void load_run_raw(const R *p, R (&out)[E]) {
  constexpr int BYTES = E * (int)sizeof(R);
  if constexpr (BYTES >= 16) {
    constexpr int PER = 16 / (int)sizeof(R);
#pragma unroll
    for (int q = 0; q < BYTES / 16; q++) {
      union { uint4 u; R e[PER]; } t;
      t.u = __ldg(reinterpret_cast<const uint4 *>(p) + q);
#pragma unroll
      for (int e = 0; e < PER; e++) out[q * PER + e] = t.e[e];
    }
  } else if constexpr (BYTES == 8) {
    union { uint2 u; R e[E]; } t;
    t.u = __ldg(reinterpret_cast<const uint2 *>(p));
#pragma unroll
    for (int e = 0; e < E; e++) out[e] = t.e[e];
  } else {
    static_assert(BYTES == 4, "4-byte run");
    union { unsigned int u; R e[E]; } t;
    t.u = __ldg(reinterpret_cast<const unsigned int *>(p));
#pragma unroll
    for (int e = 0; e < E; e++) out[e] = t.e[e];
  }
}

template <class T, class SA, class SB, bool AK>
__global__ void __launch_bounds__(Cfg<T>::THREADS, 1) gemm_kernel(Params p, T alpha, T beta, T div) {
  constexpr int BM = Cfg<T>::BM, BN = Cfg<T>::BN, BK = Cfg<T>::BK;
  constexpr int TM = Cfg<T>::TM, TN = Cfg<T>::TN, CH = Cfg<T>::CH, TX = Cfg<T>::TX;
  constexpr int THREADS = Cfg<T>::THREADS;
  static_assert(TX * TN == BN && (THREADS / TX) * TM == BM, "thread tiling");
  constexpr int EA = BM * BK / THREADS, EB = BK * BN / THREADS;   // elements per thread per tile
  extern __shared__ __align__(16) unsigned char smem_dyn[];
  T(*As)[BK][BM] = reinterpret_cast<T(*)[BK][BM]>(smem_dyn);                      // [2][BK][BM]
  T(*Bs)[BK][BN] = reinterpret_cast<T(*)[BK][BN]>(smem_dyn + 2 * BK * BM * sizeof(T));   // [2][BK][BN]

  const int tid = threadIdx.x, tx = tid % TX, ty = tid / TX;
  const int64_t m0 = (int64_t)blockIdx.y * BM, n0 = (int64_t)blockIdx.x * BN;
  if (p.upper_only && m0 + p.row_off >= n0 + BN) return;   // SYRK: tile strictly below the diagonal

  // this thread's contiguous run in the A and B tiles
  const int ea = tid * EA;
  const int a_m = AK ? ea / BK : ea % BM;      // AK: run along k at row a_m
  const int a_k = AK ? ea % BK : ea / BM;      // !AK: run along m at k-row a_k
  const int eb = tid * EB;
  const int b_k = eb / BN, b_n = eb % BN;      // run along n
  const raw_t<SA> *Ap = (const raw_t<SA> *)p.A;
  const raw_t<SB> *Bp = (const raw_t<SB> *)p.B;
  const bool m_full = m0 + BM <= p.M, n_full = n0 + BN <= p.N;

  T ra[EA], rb[EB];
  auto load_tiles = [&](int64_t k0) {
    const bool k_full = k0 + BK <= p.K;
    if (p.a_vec && m_full && k_full) {
      load_run<SA, EA, T>(Ap + (m0 + a_m) * p.a_sr + (k0 + a_k) * p.a_sc, ra);
    } else {
#pragma unroll
      for (int e = 0; e < EA; e++) {
        const int64_t gm = m0 + a_m + (AK ? 0 : e), gk = k0 + a_k + (AK ? e : 0);
        ra[e] = (gm < p.M && gk < p.K) ? Ld<SA, T>::get(Ap, (size_t)(gm * p.a_sr + gk * p.a_sc)) : T(0);
      }
    }
    if (p.b_vec && n_full && k_full) {
      load_run<SB, EB, T>(Bp + (k0 + b_k) * p.b_sr + n0 + b_n, rb);
    } else {
#pragma unroll
      for (int e = 0; e < EB; e++) {
        const int64_t gk = k0 + b_k, gn = n0 + b_n + e;
        rb[e] = (gk < p.K && gn < p.N) ? Ld<SB, T>::get(Bp, (size_t)(gk * p.b_sr + gn)) : T(0);
      }
    }
  };
  auto store_tiles = [&](int buf) {
#pragma unroll
    for (int e = 0; e < EA; e++) {
      if (AK) As[buf][a_k + e][a_m] = ra[e];
      else As[buf][a_k][a_m + e] = ra[e];
    }
#pragma unroll
    for (int e = 0; e < EB; e++) Bs[buf][b_k][b_n + e] = rb[e];
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
      for (int i = 0; i < TM; i++) a[i] = As[buf][k][(i / 4) * (BM / 2) + ty * 4 + (i % 4)];
#pragma unroll
      for (int j = 0; j < TN; j++) b[j] = Bs[buf][k][(j / CH) * (TX * CH) + tx * CH + (j % CH)];
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
    const int64_t gm = m0 + (i / 4) * (BM / 2) + ty * 4 + (i % 4);
    if (gm >= p.M) continue;
#pragma unroll
    for (int j = 0; j < TN; j++) {
      const int64_t gn = n0 + (j / CH) * (TX * CH) + tx * CH + (j % CH);
      if (gn >= p.N) continue;
      T r = acc[i][j];
      const int64_t idx = gm * p.ldc + gn;
      if (p.epi == EPI_AXPBY) r = t_fma(alpha, r, beta * load_elem<T>(p.Cin, p.tcin, idx));
      else if (p.epi == EPI_DIV) r = r / div;
      store_elem<T>(p.C, p.tc, idx, r);
    }
  }
}

template <class T, class SA, class SB>
ps_status launch(const Params &p, bool ak, double alpha, double beta, double div, cudaStream_t st) {
  using C = Cfg<T>;
  constexpr int SM = smem_bytes<T>();
  PS_TRY(set_max_smem((const void *)gemm_kernel<T, SA, SB, true>, SM));
  PS_TRY(set_max_smem((const void *)gemm_kernel<T, SA, SB, false>, SM));
  dim3 grid((unsigned)((p.N + C::BN - 1) / C::BN), (unsigned)((p.M + C::BM - 1) / C::BM));
  // scalars are RNE-rounded from their fp64 literal to T (R2); the host cast is RNE
  if (ak) gemm_kernel<T, SA, SB, true><<<grid, C::THREADS, SM, st>>>(p, (T)alpha, (T)beta, (T)div);
  else gemm_kernel<T, SA, SB, false><<<grid, C::THREADS, SM, st>>>(p, (T)alpha, (T)beta, (T)div);
  PS_CHECK_LAUNCH("gemm_simt_kernel");
  return PS_OK;
}

inline Params make_params(const GemmArgs &g) {
  Params p{};
  p.M = g.M; p.N = g.N; p.K = g.K;
  p.A = g.A.p; p.a_sr = g.A.s_row; p.a_sc = g.A.s_col;
  p.B = g.B.p; p.b_sr = g.B.s_row;
  p.C = g.C; p.tc = g.c_type; p.ldc = g.ldc;
  p.Cin = g.Cin; p.tcin = g.cin_type;
  p.epi = g.epi; p.upper_only = g.upper_only; p.row_off = g.row_off;
  const int64_t lda = g.A.s_col == 1 ? g.A.s_row : g.A.s_col;
  p.a_vec = ((uintptr_t)g.A.p % 16 == 0) && ((lda * (int64_t)dtype_size(g.A.type)) % 16 == 0);
  p.b_vec = ((uintptr_t)g.B.p % 16 == 0) && ((g.B.s_row * (int64_t)dtype_size(g.B.type)) % 16 == 0);
  return p;
}

ps_status gemm_simt_f32(const GemmArgs &g, cudaStream_t st);
ps_status gemm_simt_f64(const GemmArgs &g, cudaStream_t st);
// f64 on the fp64 tensor-core MMA, R3 order (gemm_dmma.cu)
// f32 FFMA chains, two CTAs per SM, cp.async ring (gemm_ffma.cu)
ps_status gemm_ffma_f32(const GemmArgs &g, cudaStream_t st);
ps_status gemm_dmma_f64(const GemmArgs &g, cudaStream_t st);

}  // namespace simt
}  // namespace ps
