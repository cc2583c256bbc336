// gemm_ffma.cu -- f32 contractions (compute type f32, reading R2) as FFMA chains in
// reading R3's order: every output is acc <- fma(a_k, b_k, acc) from +0, k
// ascending, one thread per output, so the result is bit-exact with the oracle.
//
// Blackwell's fma.rn.f32x2 (SASS FFMA2: two independent round-to-nearest fmas in one
// instruction, each lane exactly fma(a, b, c)) carries two neighbouring outputs of a
// row with a_i broadcast, so the kernel issues half the FMA-pipe instructions of
// scalar FFMA: with scalar FFMA the kernel was issue-bound (76% issue, 66% FMA pipe,
// round 1); with FFMA2 the FMA pipe itself is the limit (tools/ffma_probe.cu, 27
// tile shapes measured: profiles/ffma_probe_r2*.jsonl).
//
// Shape (the probe's best): 64 x 128 CTA tile, 128 threads of 8 x 8 outputs (two
// runs of 4 rows, 32 apart; two runs of 4 columns, 64 apart: LDS.128 fragments, A
// broadcast, B conflict-free), three CTAs per SM; a ring of BK-deep tiles (FTile) in
// shared memory, both operands stored [k][m] / [k][n] with 4 floats of padding:
//  * f32 operands whose rows run along m or n (B always, A when it is m-major,
//    e.g. SYRK's data^T) travel by cp.async (16 B, 4-byte zero-fill on edges);
//  * k-major A and f16 / bf16 operands are register-staged (widened exactly to f32;
//    k-major A transposed with each warp writing 32 consecutive m, conflict-free) and
//    stored at the end of the iteration, S-1 tiles ahead of their use.
#include <type_traits>

#include "gemm_simt.cuh"

namespace ps {
namespace simt {

namespace {
constexpr int FBM = 64, FBN = 128, FTHREADS = 128, FMINB = 3, FPAD = 4;
constexpr int64_t FGROUP_M = 16;
constexpr int FTM = 8, FTN = 8, FTX = FBN / FTN, FTY = FBM / FTM;   // 16 x 8 threads
constexpr int FLA = FBM + FPAD, FLB = FBN + FPAD;   // row strides of As[k][m], Bs[k][n]
// k-tile depth and ring length per operand types (measured at 8192^3, profiles/
// kernel_rates_ffma2_r2ad.jsonl vs r2ac, ffma_tile_*_r2aw.jsonl): BK = 16 x 3 stages for
// 16-bit A with f32 B (55.3 vs 51.2 TFLOP/s at BK = 8), BK = 8 x 6 stages otherwise
// (f32 53.3, 16-bit B 53.1; x 4 stages 52.8 / 51.6; BK = 16: 51.5 / 48.2): the shallower
// tile halves the register-staged run per thread, the longer ring covers its latency
template <class SA, class SB> struct FTile {
  static constexpr bool DEEP = !std::is_same<SA, float>::value && std::is_same<SB, float>::value;
  static constexpr int BK = DEEP ? 16 : 8, S = DEEP ? 3 : 6;
  static constexpr int A_EL = BK * FLA, B_EL = BK * FLB;
  static constexpr int SMEM = S * (A_EL + B_EL) * 4;
};
static_assert(FTX * FTY == FTHREADS, "thread grid");

template <class S> __device__ __forceinline__ float widen_f(raw_t<S> v) {
  if constexpr (std::is_same<S, float>::value) return v;
  else if constexpr (std::is_same<S, BF16>::value) return bf16_to_f32(v);
  else return f16_to_f32(v);
}

// E register-staged stored elements packed in 32-bit words (two 16-bit elements per
// register: a 16-element f16 run of B takes 8 registers, not 16)
template <class S, int E> struct Run {
  using R = raw_t<S>;
  static constexpr int PER = 4 / (int)sizeof(R), W = E / PER;
  uint32_t w[W];
  __device__ __forceinline__ void load(const R *p) {   // run aligned to min(its size, 16 B)
    static_assert(W % 4 == 0 || W == 2 || W == 1, "run size");
    if constexpr (W % 4 == 0) {
#pragma unroll
      for (int q = 0; q < W / 4; q++) {
        const uint4 t = __ldg(reinterpret_cast<const uint4 *>(p) + q);
        w[4 * q] = t.x; w[4 * q + 1] = t.y; w[4 * q + 2] = t.z; w[4 * q + 3] = t.w;
      }
    } else if constexpr (W == 2) {
      const uint2 t = __ldg(reinterpret_cast<const uint2 *>(p));
      w[0] = t.x; w[1] = t.y;
    } else {
      w[0] = __ldg(reinterpret_cast<const unsigned int *>(p));
    }
  }
  __device__ __forceinline__ void set(int e, R v) {
    if constexpr (PER == 1) w[e] = __float_as_uint(v);
    else w[e / 2] = (e & 1) ? ((w[e / 2] & 0xFFFFu) | ((uint32_t)v << 16)) : (uint32_t)v;
  }
  __device__ __forceinline__ float get(int e) const {
    if constexpr (PER == 1) return __uint_as_float(w[e]);
    else return widen_f<S>((R)((e & 1) ? (w[e / 2] >> 16) : (w[e / 2] & 0xFFFFu)));
  }
};
}  // namespace

// 16-bit B is register-staged (16 raw elements per thread): those instantiations are
// allowed more than 168 registers (no spills) at two CTAs per SM
template <class SB> constexpr int ffma_minb() { return FMINB; }

template <class SA, class SB, bool AK>
__global__ void __launch_bounds__(FTHREADS, ffma_minb<SB>()) gemm_ffma_kernel(Params p, float alpha, float beta, float div) {
  using TL = FTile<SA, SB>;
  constexpr int BM = FBM, BN = FBN, BK = TL::BK, S = TL::S, THREADS = FTHREADS, LA = FLA, LB = FLB;
  constexpr int FA_EL = TL::A_EL, FB_EL = TL::B_EL;
  constexpr int TM = FTM, TN = FTN, TX = FTX, TY = FTY;
  constexpr int EA = BM * BK / THREADS, EB = BK * BN / THREADS;   // 8 and 16
  constexpr bool CA = !AK && std::is_same<SA, float>::value, CB = std::is_same<SB, float>::value;
  extern __shared__ __align__(16) unsigned char smem_dyn[];
  float *As0 = reinterpret_cast<float *>(smem_dyn);
  float *Bs0 = As0 + S * FA_EL;

  const int tid = threadIdx.x, tx = tid % TX, ty = tid / TX;
  // grouped raster: consecutive CTAs walk FGROUP_M tile-rows down a tile-column, so the
  // ~444 co-resident CTAs share ~16 A row-blocks and ~28 B column-blocks in L2
  // (row-major order: 7 row-blocks against all 64 column-blocks of an 8192^2 B)
  int64_t m0, n0;
  {
    const int64_t tiles_m = (p.M + BM - 1) / BM, tiles_n = (p.N + BN - 1) / BN;
    const int64_t t = blockIdx.x, per_group = FGROUP_M * tiles_n, first = t / per_group * FGROUP_M;
    const int64_t gm = tiles_m - first < FGROUP_M ? tiles_m - first : FGROUP_M;
    m0 = (first + (t % per_group) % gm) * BM;
    n0 = ((t % per_group) / gm) * BN;
  }
  if (p.upper_only && m0 + p.row_off >= n0 + BN) return;   // SYRK: tile strictly below the diagonal

  // A staging.  AK: thread -> (row tid % BM, k-run (tid / BM) * EA): a warp's
  // transposed stores As[k][m] hit 32 consecutive m (conflict-free).  !AK: a run along m.
  const int a_m = AK ? tid % BM : (tid * EA) % BM;
  const int a_k = AK ? (tid / BM) * EA : (tid * EA) / BM;
  const int eb = tid * EB;
  const int b_k = eb / BN, b_n = eb % BN;      // run along n
  const raw_t<SA> *Ap = (const raw_t<SA> *)p.A;
  const raw_t<SB> *Bp = (const raw_t<SB> *)p.B;
  const bool m_full = m0 + BM <= p.M, n_full = n0 + BN <= p.N;
  const int ktiles = (int)((p.K + BK - 1) / BK);

  Run<SA, EA> ra;
  Run<SB, EB> rb;
  auto issue = [&](int kt, int st) {
    const int64_t k0 = (int64_t)kt * BK;
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
    } else if (fa) {
      ra.load(Ap + (m0 + a_m) * p.a_sr + (k0 + a_k) * p.a_sc);
    } else {
#pragma unroll
      for (int e = 0; e < EA; e++) {
        const int64_t gm = m0 + a_m + (AK ? 0 : e), gk = k0 + a_k + (AK ? e : 0);
        ra.set(e, (gm < p.M && gk < p.K) ? Ap[gm * p.a_sr + gk * p.a_sc] : raw_t<SA>(0));
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
      rb.load(Bp + (k0 + b_k) * p.b_sr + n0 + b_n);
    } else {
#pragma unroll
      for (int e = 0; e < EB; e++) {
        const int64_t gk = k0 + b_k, gn = n0 + b_n + e;
        rb.set(e, (gk < p.K && gn < p.N) ? Bp[gk * p.b_sr + gn] : raw_t<SB>(0));
      }
    }
  };
  auto store_regs = [&](int st) {
    float *As = As0 + st * FA_EL, *Bs = Bs0 + st * FB_EL;
    if constexpr (!CA) {
#pragma unroll
      for (int e = 0; e < EA; e++) {
        if (AK) As[(a_k + e) * LA + a_m] = ra.get(e);
        else As[a_k * LA + a_m + e] = ra.get(e);
      }
    }
    if constexpr (!CB) {
#pragma unroll
      for (int e = 0; e < EB; e++) Bs[b_k * LB + b_n + e] = rb.get(e);
    }
  };

  // acc[i][jp] = outputs (row i, columns 2jp and 2jp+1) of this thread's 8 x 8
  float2 acc[TM][TN / 2];
#pragma unroll
  for (int i = 0; i < TM; i++)
#pragma unroll
    for (int j = 0; j < TN / 2; j++) acc[i][j] = make_float2(0.f, 0.f);

#pragma unroll
  for (int s = 0; s < S - 1; s++) {
    if (s < ktiles) {
      issue(s, s);
      store_regs(s);
    }
    cp_async_commit();
  }
  int rd = 0, wr = S - 1;   // ring slots of tiles kt and kt + S - 1
  for (int kt = 0; kt < ktiles; kt++) {
    cp_async_wait<S - 2>();   // this thread's copies of tile kt have landed
    __syncthreads();          // everyone's have; everyone is done with tile kt-1's stage
    const int nt = kt + S - 1;
    if (nt < ktiles) issue(nt, wr);   // into the stage tile kt-1 used
    cp_async_commit();
    const float *As = As0 + rd * FA_EL, *Bs = Bs0 + rd * FB_EL;
#pragma unroll
    for (int k = 0; k < BK; k++) {
      const float4 a0 = *reinterpret_cast<const float4 *>(As + k * LA + ty * 4);
      const float4 a1 = *reinterpret_cast<const float4 *>(As + k * LA + TY * 4 + ty * 4);
      const float4 b0 = *reinterpret_cast<const float4 *>(Bs + k * LB + tx * 4);
      const float4 b1 = *reinterpret_cast<const float4 *>(Bs + k * LB + TX * 4 + tx * 4);
      const float a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      const float2 b[4] = {make_float2(b0.x, b0.y), make_float2(b0.z, b0.w), make_float2(b1.x, b1.y),
                           make_float2(b1.z, b1.w)};
      // R3, k ascending: fma.rn.f32x2 (SASS FFMA2) is two independent fma.rn -- each
      // lane exactly t_fma(a_i, b_j, acc_ij) -- issued as one instruction, with a_i
      // broadcast: half the issue slots of scalar FFMAs on the same FMA pipe
#pragma unroll
      for (int i = 0; i < TM; i++)
#pragma unroll
        for (int j = 0; j < TN / 2; j++) acc[i][j] = __ffma2_rn(make_float2(a[i], a[i]), b[j], acc[i][j]);
    }
    if (nt < ktiles) store_regs(wr);
    rd = rd + 1 == S ? 0 : rd + 1;
    wr = wr + 1 == S ? 0 : wr + 1;
  }
  cp_async_wait<0>();

  // epilogue (R3): plain / fma(alpha, acc, beta*Cin) / acc / div, then RNE store (R1)
#pragma unroll
  for (int i = 0; i < TM; i++) {
    const int64_t gm = m0 + (i / 4) * TY * 4 + ty * 4 + (i % 4);
    if (gm >= p.M) continue;
#pragma unroll
    for (int j = 0; j < TN; j++) {
      const int64_t gn = n0 + (j / 4) * TX * 4 + tx * 4 + (j % 4);
      if (gn >= p.N) continue;
      float r = (j & 1) ? acc[i][j / 2].y : acc[i][j / 2].x;
      const int64_t idx = gm * p.ldc + gn;
      if (p.epi == EPI_AXPBY) r = t_fma(alpha, r, beta * load_elem<float>(p.Cin, p.tcin, idx));
      else if (p.epi == EPI_DIV) r = r / div;
      store_elem<float>(p.C, p.tc, idx, r);
    }
  }
}

template <class SA, class SB>
static ps_status launch_ffma(const Params &p, bool ak, double alpha, double beta, double div, cudaStream_t st) {
  constexpr int FSMEM = FTile<SA, SB>::SMEM;
  PS_TRY(set_max_smem((const void *)gemm_ffma_kernel<SA, SB, true>, FSMEM));
  PS_TRY(set_max_smem((const void *)gemm_ffma_kernel<SA, SB, false>, FSMEM));
  dim3 grid((unsigned)(((p.N + FBN - 1) / FBN) * ((p.M + FBM - 1) / FBM)));
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
