// gemm_ffma.cu -- f32 contractions (compute type f32, reading R2) as FFMA chains in
// reading R3's order: every output is acc <- fma(a_k, b_k, acc) from +0, k
// ascending, one thread per output, so the result is bit-exact with the oracle.
//
// The FFMA pipe issues one warp instruction per SMSP per clock, so the kernel is
// issue-bound: per k each thread does 64 FFMAs against 4 LDS.128 fragment loads
// (8 x 8 outputs per thread).  Shape: 128 x 128 CTA tile, 256 threads, at most
// 128 registers so TWO CTAs share an SM (16 warps: one CTA's barrier and load
// stalls are covered by the other's FFMAs); a 3-stage ring of BK = 16 tiles in
// shared memory, both operands stored [k][m] / [k][n] with 4 floats of padding:
//  * f32 operands whose rows run along m or n (B always, A when it is m-major,
//    e.g. SYRK's data^T) travel by cp.async (16 B, 4-byte zero-fill on edges);
//  * k-major A and f16 / bf16 operands are register-staged (widened exactly to f32,
//    transposed for k-major A) and stored at the end of the iteration, S-1 tiles
//    ahead of their use.
// The previous kernel (gemm_simt.cuh, 1 CTA per SM, register double buffer) is kept
// behind PS_F32_SIMT_OLD=1 for measurement.
#include <type_traits>

#include "gemm_simt.cuh"

namespace ps {
namespace simt {

namespace {
constexpr int FBM = 128, FBN = 128, FBK = 16, FST = 3, FTHREADS = 256, FPAD = 4;
constexpr int FLA = FBM + FPAD, FLB = FBN + FPAD;   // row strides of As[k][m], Bs[k][n]
constexpr int FA_EL = FBK * FLA, FB_EL = FBK * FLB;
constexpr int FSMEM = FST * (FA_EL + FB_EL) * 4;

template <class S> __device__ __forceinline__ float widen_f(raw_t<S> v) {
  if constexpr (std::is_same<S, float>::value) return v;
  else if constexpr (std::is_same<S, BF16>::value) return bf16_to_f32(v);
  else return f16_to_f32(v);
}
}  // namespace

template <class SA, class SB, bool AK>
__global__ void __launch_bounds__(FTHREADS, 2) gemm_ffma_kernel(Params p, float alpha, float beta, float div) {
  constexpr int BM = FBM, BN = FBN, BK = FBK, S = FST, THREADS = FTHREADS, LA = FLA, LB = FLB;
  constexpr int EA = BM * BK / THREADS, EB = BK * BN / THREADS;   // 8 and 8
  constexpr bool CA = !AK && std::is_same<SA, float>::value, CB = std::is_same<SB, float>::value;
  extern __shared__ __align__(16) unsigned char smem_dyn[];
  float *As0 = reinterpret_cast<float *>(smem_dyn);
  float *Bs0 = As0 + S * FA_EL;

  const int tid = threadIdx.x, tx = tid % 16, ty = tid / 16;
  const int64_t m0 = (int64_t)blockIdx.y * BM, n0 = (int64_t)blockIdx.x * BN;
  if (p.upper_only && m0 + p.row_off >= n0 + BN) return;   // SYRK: tile strictly below the diagonal

  const int ea = tid * EA;
  const int a_m = AK ? ea / BK : ea % BM;      // AK: run along k at row a_m
  const int a_k = AK ? ea % BK : ea / BM;      // !AK: run along m at k-row a_k
  const int eb = tid * EB;
  const int b_k = eb / BN, b_n = eb % BN;      // run along n
  const raw_t<SA> *Ap = (const raw_t<SA> *)p.A;
  const raw_t<SB> *Bp = (const raw_t<SB> *)p.B;
  const bool m_full = m0 + BM <= p.M, n_full = n0 + BN <= p.N;
  const int64_t ktiles = (p.K + BK - 1) / BK;

  raw_t<SA> ra[EA];
  raw_t<SB> rb[EB];
  auto issue = [&](int64_t kt, int st) {
    const int64_t k0 = kt * BK;
    const bool k_full = k0 + BK <= p.K;
    float *As = As0 + st * FA_EL, *Bs = Bs0 + st * FB_EL;
    const bool fa = p.a_vec && m_full && k_full, fb = p.b_vec && n_full && k_full;
    if constexpr (CA) {   // m-major f32 A: 16-byte runs along m
#pragma unroll
      for (int e = 0; e < BM * BK / 4 / THREADS; e++) {
        const int c = tid + e * THREADS;
        const int kr = c / (BM / 4), mc = (c % (BM / 4)) * 4;
        float *dst = As + kr * LA + mc;
        if (fa) {
          cp_async16(dst, Ap + (m0 + mc) * p.a_sr + (k0 + kr) * p.a_sc);
        } else {
#pragma unroll
          for (int h = 0; h < 4; h++) {
            const int64_t gm = m0 + mc + h, gk = k0 + kr;
            const bool ok = gm < p.M && gk < p.K;
            cp_async4z(dst + h, ok ? Ap + gm * p.a_sr + gk * p.a_sc : Ap, ok);
          }
        }
      }
    } else if (p.a_vec && m_full && k_full) {
      load_run_raw<raw_t<SA>, EA>(Ap + (m0 + a_m) * p.a_sr + (k0 + a_k) * p.a_sc, ra);
    } else {
#pragma unroll
      for (int e = 0; e < EA; e++) {
        const int64_t gm = m0 + a_m + (AK ? 0 : e), gk = k0 + a_k + (AK ? e : 0);
        ra[e] = (gm < p.M && gk < p.K) ? Ap[gm * p.a_sr + gk * p.a_sc] : raw_t<SA>(0);
      }
    }
    if constexpr (CB) {
#pragma unroll
      for (int e = 0; e < BK * BN / 4 / THREADS; e++) {
        const int c = tid + e * THREADS;
        const int kr = c / (BN / 4), nc = (c % (BN / 4)) * 4;
        float *dst = Bs + kr * LB + nc;
        if (fb) {
          cp_async16(dst, Bp + (k0 + kr) * p.b_sr + n0 + nc);
        } else {
#pragma unroll
          for (int h = 0; h < 4; h++) {
            const int64_t gk = k0 + kr, gn = n0 + nc + h;
            const bool ok = gk < p.K && gn < p.N;
            cp_async4z(dst + h, ok ? Bp + gk * p.b_sr + gn : Bp, ok);
          }
        }
      }
    } else if (fb) {
      load_run_raw<raw_t<SB>, EB>(Bp + (k0 + b_k) * p.b_sr + n0 + b_n, rb);
    } else {
#pragma unroll
      for (int e = 0; e < EB; e++) {
        const int64_t gk = k0 + b_k, gn = n0 + b_n + e;
        rb[e] = (gk < p.K && gn < p.N) ? Bp[gk * p.b_sr + gn] : raw_t<SB>(0);
      }
    }
  };
  auto store_regs = [&](int st) {
    float *As = As0 + st * FA_EL, *Bs = Bs0 + st * FB_EL;
    if constexpr (!CA) {
#pragma unroll
      for (int e = 0; e < EA; e++) {
        if (AK) As[(a_k + e) * LA + a_m] = widen_f<SA>(ra[e]);
        else As[a_k * LA + a_m + e] = widen_f<SA>(ra[e]);
      }
    }
    if constexpr (!CB) {
#pragma unroll
      for (int e = 0; e < EB; e++) Bs[b_k * LB + b_n + e] = widen_f<SB>(rb[e]);
    }
  };

  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; i++)
#pragma unroll
    for (int j = 0; j < 8; j++) acc[i][j] = 0.0f;

#pragma unroll
  for (int s = 0; s < S - 1; s++) {
    if (s < ktiles) {
      issue(s, s);
      store_regs(s);
    }
    cp_async_commit();
  }
  for (int64_t kt = 0; kt < ktiles; kt++) {
    cp_async_wait<S - 2>();   // this thread's copies of tile kt have landed
    __syncthreads();          // everyone's have; everyone is done with tile kt-1's stage
    const int64_t nt = kt + S - 1;
    if (nt < ktiles) issue(nt, (int)(nt % S));   // into the stage tile kt-1 used
    cp_async_commit();
    const int st = (int)(kt % S);
    const float *As = As0 + st * FA_EL, *Bs = Bs0 + st * FB_EL;
#pragma unroll
    for (int k = 0; k < BK; k++) {
      const float4 a0 = *reinterpret_cast<const float4 *>(As + k * LA + ty * 4);
      const float4 a1 = *reinterpret_cast<const float4 *>(As + k * LA + 64 + ty * 4);
      const float4 b0 = *reinterpret_cast<const float4 *>(Bs + k * LB + tx * 4);
      const float4 b1 = *reinterpret_cast<const float4 *>(Bs + k * LB + 64 + tx * 4);
      const float a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      const float b[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
      for (int i = 0; i < 8; i++)
#pragma unroll
        for (int j = 0; j < 8; j++) acc[i][j] = t_fma(a[i], b[j], acc[i][j]);   // R3, k ascending
    }
    if (nt < ktiles) store_regs((int)(nt % S));
  }
  cp_async_wait<0>();

  // epilogue (R3): plain / fma(alpha, acc, beta*Cin) / acc / div, then RNE store (R1)
#pragma unroll
  for (int i = 0; i < 8; i++) {
    const int64_t gm = m0 + (i / 4) * 64 + ty * 4 + (i % 4);
    if (gm >= p.M) continue;
#pragma unroll
    for (int j = 0; j < 8; j++) {
      const int64_t gn = n0 + (j / 4) * 64 + tx * 4 + (j % 4);
      if (gn >= p.N) continue;
      float r = acc[i][j];
      const int64_t idx = gm * p.ldc + gn;
      if (p.epi == EPI_AXPBY) r = t_fma(alpha, r, beta * load_elem<float>(p.Cin, p.tcin, idx));
      else if (p.epi == EPI_DIV) r = r / div;
      store_elem<float>(p.C, p.tc, idx, r);
    }
  }
}

template <class SA, class SB>
static ps_status launch_ffma(const Params &p, bool ak, double alpha, double beta, double div, cudaStream_t st) {
  PS_TRY(set_max_smem((const void *)gemm_ffma_kernel<SA, SB, true>, FSMEM));
  PS_TRY(set_max_smem((const void *)gemm_ffma_kernel<SA, SB, false>, FSMEM));
  dim3 grid((unsigned)((p.N + FBN - 1) / FBN), (unsigned)((p.M + FBM - 1) / FBM));
  // scalars are RNE-rounded from their fp64 literal to f32 (R2); the host cast is RNE
  if (ak) gemm_ffma_kernel<SA, SB, true><<<grid, FTHREADS, FSMEM, st>>>(p, (float)alpha, (float)beta, (float)div);
  else gemm_ffma_kernel<SA, SB, false><<<grid, FTHREADS, FSMEM, st>>>(p, (float)alpha, (float)beta, (float)div);
  PS_CHECK_LAUNCH("gemm_ffma_kernel");
  return PS_OK;
}

ps_status gemm_ffma_f32(const GemmArgs &g, cudaStream_t st) {
  const Params p = make_params(g);
  const bool ak = g.A.s_col == 1;
  auto pick = [&](auto sa) -> ps_status {
    using SA = decltype(sa);
    if (g.B.type == PS_F16) return launch_ffma<SA, F16>(p, ak, g.alpha, g.beta, g.div, st);
    if (g.B.type == PS_BF16) return launch_ffma<SA, BF16>(p, ak, g.alpha, g.beta, g.div, st);
    return launch_ffma<SA, float>(p, ak, g.alpha, g.beta, g.div, st);
  };
  if (g.A.type == PS_F16) return pick(F16());
  if (g.A.type == PS_BF16) return pick(BF16());
  return pick(float());
}

}  // namespace simt
}  // namespace ps
