// gemm_dmma.cu -- f64 contractions on the fp64 tensor-core MMA (DMMA) with
// reading R3's summation order.
//
// R3: C_ij = sum_k A_ik B_kj is the fma chain acc <- fma(a_k, b_k, acc) from +0,
// k ascending.  `mma.sync.m8n8k4.f64` computes D = A(8x4) B(4x8) + C; measured
// on this B200 (tools/dmma_probe.cu, profiles/dmma_probe_r1.txt) its result is,
// bit for bit, the chain d = fma(a3,b3, fma(a2,b2, fma(a1,b1, fma(a0,b0, c))))
// -- C first, k ascending, one rounding per step -- over random, wide-exponent,
// cancellation-heavy, subnormal and inf/NaN operands.  Chaining the MMAs over
// k = 0, 4, 8, ... with the accumulator as C therefore reproduces R3 exactly
// (the GPU parity tests check every f64 statement bit-exactly against the
// oracle).  Operands are read in their stored precision and widened exactly to
// f64 when staged in shared memory (R1); the epilogue is the SIMT kernel's.
//
// Default shape: CTA tile 128 x 64, 8 warps of 32 x 32 (4 x 4 MMA tiles, 32 f64
// accumulators per lane), two CTAs per SM (one's barrier stalls are covered by the
// other's MMAs), a 3-stage ring of BK = 16 tiles: cp.async for f64 operands,
// register staging with exact integer widening for f32/f16/bf16 ones.  Shared
// rows are padded by 4 doubles so every fragment load (lane (r, q) reads element
// (r, q) of an 8 x 4 block) is bank-conflict free.
#include <cstdlib>
#include <type_traits>

#include "gemm_simt.cuh"

namespace ps {
namespace simt {

// WGM x WGN warps; warp tile (BM / WGM) x (BN / WGN) = MI x NJ MMA tiles of 8 x 8
template <int WGM, int WGN, int BK_ = 16, int STAGES_ = 4, int BN_ = 128, int MINB_ = 1>
struct DCfg {
  static constexpr int BM = 128, BN = BN_, BK = BK_, THREADS = 32 * WGM * WGN, PAD = 4, MINB = MINB_;
  static constexpr int MI = BM / (8 * WGM), NJ = BN / (8 * WGN), STAGES = STAGES_;
  static constexpr int A_ELEMS = BM * (BK + PAD) > BK * (BM + PAD) ? BM * (BK + PAD) : BK * (BM + PAD);
  static constexpr int B_ELEMS = BK * (BN + PAD);
  static constexpr int SMEM = STAGES * (A_ELEMS + B_ELEMS) * 8;
};

// Exact widening of stored f32 / f16 / bf16 bits to f64 with integer operations
// (R1): cvt.f64.f32 / cvt.f64.f16 issue on the fp64 pipe the MMAs need, and cost
// the mixed-storage statements ~20% (profiles/dmma_probe_r1.txt); the integer pipe
// is otherwise idle here.  Normal numbers rebias the exponent and shift the fraction;
// subnormals are renormalised (exact); inf keeps its sign; NaN stays NaN (quiet).
__device__ __forceinline__ double f32bits_to_f64(uint32_t u) {
  const uint32_t e = (u >> 23) & 0xffu, m = u & 0x7fffffu;
  const uint64_t sign = (uint64_t)(u >> 31) << 63;
  uint64_t r = sign | ((uint64_t)(e + 896u) << 52) | ((uint64_t)m << 29);
  if (__builtin_expect(e - 1u >= 0xfeu, 0)) {
    if (e == 0xffu) {
      r = sign | (0x7ffull << 52) | ((uint64_t)m << 29) | (m ? (1ull << 51) : 0ull);
    } else if (m == 0) {
      r = sign;
    } else {
      const int p = 31 - __clz((int)m);   // leading bit: value = 1.f x 2^(p - 149)
      r = sign | ((uint64_t)(p + 874) << 52) | (((uint64_t)m << (52 - p)) & 0xfffffffffffffull);
    }
  }
  return __longlong_as_double((long long)r);
}
__device__ __forceinline__ double f16bits_to_f64(uint32_t h) {
  const uint32_t e = (h >> 10) & 0x1fu, m = h & 0x3ffu;
  const uint64_t sign = (uint64_t)((h >> 15) & 1u) << 63;
  uint64_t r = sign | ((uint64_t)(e + 1008u) << 52) | ((uint64_t)m << 42);
  if (__builtin_expect(e - 1u >= 0x1eu, 0)) {
    if (e == 0x1fu) {
      r = sign | (0x7ffull << 52) | ((uint64_t)m << 42) | (m ? (1ull << 51) : 0ull);
    } else if (m == 0) {
      r = sign;
    } else {
      const int p = 31 - __clz((int)m);   // value = 1.f x 2^(p - 24)
      r = sign | ((uint64_t)(p + 999) << 52) | (((uint64_t)m << (52 - p)) & 0xfffffffffffffull);
    }
  }
  return __longlong_as_double((long long)r);
}
template <class S> __device__ __forceinline__ double widen_i(raw_t<S> v) {
  if constexpr (std::is_same<S, double>::value) return v;
  else if constexpr (std::is_same<S, float>::value) return f32bits_to_f64(__float_as_uint(v));
  else if constexpr (std::is_same<S, BF16>::value) return f32bits_to_f64((uint32_t)v << 16);
  else return f32bits_to_f64(__float_as_uint(f16_to_f32(v)));   // cvt.f32.f16: exact, not the fp64 pipe
}
__device__ __forceinline__ void dmma(double &d0, double &d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
               : "+d"(d0), "+d"(d1)
               : "d"(a), "d"(b));
}

template <class SA, class SB, bool AK, int WGM, int WGN, int BK_, int ST_, int BN_, int MB_>
__global__ void __launch_bounds__(DCfg<WGM, WGN, BK_, ST_, BN_, MB_>::THREADS, MB_)
    gemm_dmma_kernel(Params p, double alpha, double beta, double div) {
  using DCfg = DCfg<WGM, WGN, BK_, ST_, BN_, MB_>;
  constexpr int BM = DCfg::BM, BN = DCfg::BN, BK = DCfg::BK, PAD = DCfg::PAD, THREADS = DCfg::THREADS;
  constexpr int MI = DCfg::MI, NJ = DCfg::NJ, S = DCfg::STAGES;
  constexpr int LA = AK ? BK + PAD : BM + PAD;   // A row stride: [m][k] (AK) or [k][m]
  constexpr int LB = BN + PAD;                   // B: [k][n]
  constexpr int EA = BM * BK / THREADS, EB = BK * BN / THREADS;
  // f64-stored operands travel by cp.async (16 B = 2 doubles; 8 B zero-filled on edge
  // tiles and unaligned rows), no registers; the others by register staging with
  // exact widening at the shared-memory store
  constexpr bool CA = std::is_same<SA, double>::value, CB = std::is_same<SB, double>::value;
  extern __shared__ __align__(16) unsigned char smem_dyn[];
  double *As0 = reinterpret_cast<double *>(smem_dyn);
  double *Bs0 = As0 + S * DCfg::A_ELEMS;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int r = lane >> 2, q = lane & 3;
  const int wm = (warp / WGN) * (BM / WGM), wn = (warp % WGN) * (BN / WGN);
  const int64_t m0 = (int64_t)blockIdx.y * BM, n0 = (int64_t)blockIdx.x * BN;
  if (p.upper_only && m0 + p.row_off >= n0 + BN) return;   // SYRK: tile strictly below the diagonal

  const int a_m = AK ? tid / (BK / EA) : (tid % (BM / EA)) * EA;
  const int a_k = AK ? (tid % (BK / EA)) * EA : tid / (BM / EA);
  const int b_k = tid / (BN / EB), b_n = (tid % (BN / EB)) * EB;
  const raw_t<SA> *Ap = (const raw_t<SA> *)p.A;
  const raw_t<SB> *Bp = (const raw_t<SB> *)p.B;
  const bool m_full = m0 + BM <= p.M, n_full = n0 + BN <= p.N;
  const int64_t ktiles = (p.K + BK - 1) / BK;

  raw_t<SA> ra[EA];   // raw stored bits (zero bits = +0 for every storage type)
  raw_t<SB> rb[EB];
  // issue tile kt into stage st: cp.async for f64 operands, loads into ra / rb for the
  // others (the returned flags say which operands still need store_regs)
  auto issue = [&](int64_t kt, int st, bool &reg_a, bool &reg_b) {
    const int64_t k0 = kt * BK;
    const bool k_full = k0 + BK <= p.K;
    double *As = As0 + st * DCfg::A_ELEMS, *Bs = Bs0 + st * DCfg::B_ELEMS;
    const bool fa = p.a_vec && m_full && k_full, fb = p.b_vec && n_full && k_full;
    reg_a = !CA;
    reg_b = !CB;
    if constexpr (CA) {
#pragma unroll
      for (int e = 0; e < BM * BK / 2 / THREADS; e++) {
        const int c = tid + e * THREADS;
        const int row = AK ? c / (BK / 2) : (c % (BM / 2)) * 2;   // m of the chunk's first element
        const int kr = AK ? (c % (BK / 2)) * 2 : c / (BM / 2);     // k of the chunk's first element
        double *dst = AK ? As + row * LA + kr : As + kr * LA + row;
        if (fa) {
          cp_async16(dst, Ap + (m0 + row) * p.a_sr + (k0 + kr) * p.a_sc);
        } else {
#pragma unroll
          for (int h = 0; h < 2; h++) {
            const int64_t gm = m0 + row + (AK ? 0 : h), gk = k0 + kr + (AK ? h : 0);
            const bool ok = gm < p.M && gk < p.K;
            cp_async8z(dst + h, ok ? Ap + gm * p.a_sr + gk * p.a_sc : Ap, ok);
          }
        }
      }
    } else if (fa) {
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
      for (int e = 0; e < BK * BN / 2 / THREADS; e++) {
        const int c = tid + e * THREADS;
        const int kr = c / (BN / 2), nc = (c % (BN / 2)) * 2;
        double *dst = Bs + kr * LB + nc;
        if (fb) {
          cp_async16(dst, Bp + (k0 + kr) * p.b_sr + n0 + nc);
        } else {
#pragma unroll
          for (int h = 0; h < 2; h++) {
            const int64_t gk = k0 + kr, gn = n0 + nc + h;
            const bool ok = gk < p.K && gn < p.N;
            cp_async8z(dst + h, ok ? Bp + gk * p.b_sr + gn : Bp, ok);
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
  auto store_regs = [&](int st, bool reg_a, bool reg_b) {
    double *As = As0 + st * DCfg::A_ELEMS, *Bs = Bs0 + st * DCfg::B_ELEMS;
    if (reg_a) {
      double2 *pa = reinterpret_cast<double2 *>(AK ? As + a_m * LA + a_k : As + a_k * LA + a_m);
#pragma unroll
      for (int e = 0; e < EA / 2; e++) pa[e] = make_double2(widen_i<SA>(ra[2 * e]), widen_i<SA>(ra[2 * e + 1]));
    }
    if (reg_b) {
      double2 *pb = reinterpret_cast<double2 *>(Bs + b_k * LB + b_n);
#pragma unroll
      for (int e = 0; e < EB / 2; e++) pb[e] = make_double2(widen_i<SB>(rb[2 * e]), widen_i<SB>(rb[2 * e + 1]));
    }
  };

  double acc[MI][NJ][2];
#pragma unroll
  for (int i = 0; i < MI; i++)
#pragma unroll
    for (int j = 0; j < NJ; j++) acc[i][j][0] = acc[i][j][1] = 0.0;

  // prologue: tiles 0 .. S-2 (one cp.async group each, possibly empty)
#pragma unroll
  for (int s = 0; s < S - 1; s++) {
    if (s < ktiles) {
      bool ga, gb;
      issue(s, s, ga, gb);
      store_regs(s, ga, gb);
    }
    cp_async_commit();
  }
  for (int64_t kt = 0; kt < ktiles; kt++) {
    cp_async_wait<S - 2>();   // this thread's copies of tile kt have landed
    __syncthreads();          // everyone's have; everyone is done with tile kt-1's stage
    const int64_t nt = kt + S - 1;
    bool ga = false, gb = false;
    if (nt < ktiles) issue(nt, (int)(nt % S), ga, gb);   // into the stage tile kt-1 used
    cp_async_commit();
    const int st = (int)(kt % S);
    const double *As = As0 + st * DCfg::A_ELEMS, *Bs = Bs0 + st * DCfg::B_ELEMS;
#pragma unroll
    for (int kk = 0; kk < BK; kk += 4) {
      double af[MI], bf[NJ];
#pragma unroll
      for (int i = 0; i < MI; i++)
        af[i] = AK ? As[(wm + i * 8 + r) * LA + kk + q] : As[(kk + q) * LA + wm + i * 8 + r];
#pragma unroll
      for (int j = 0; j < NJ; j++) bf[j] = Bs[(kk + q) * LB + wn + j * 8 + r];
#pragma unroll
      for (int i = 0; i < MI; i++)
#pragma unroll
        for (int j = 0; j < NJ; j++) dmma(acc[i][j][0], acc[i][j][1], af[i], bf[j]);   // R3, k ascending
    }
    if (nt < ktiles) store_regs((int)(nt % S), ga, gb);   // register-staged operands of tile nt
  }
  cp_async_wait<0>();

  // epilogue (R3): plain / fma(alpha, acc, beta*Cin) / acc / div, then RNE store (R1)
#pragma unroll
  for (int i = 0; i < MI; i++) {
    const int64_t gm = m0 + wm + i * 8 + r;
    if (gm >= p.M) continue;
#pragma unroll
    for (int j = 0; j < NJ; j++) {
#pragma unroll
      for (int e = 0; e < 2; e++) {
        const int64_t gn = n0 + wn + j * 8 + 2 * q + e;
        if (gn >= p.N) continue;
        double v = acc[i][j][e];
        const int64_t idx = gm * p.ldc + gn;
        if (p.epi == EPI_AXPBY) v = fma(alpha, v, beta * load_elem<double>(p.Cin, p.tcin, idx));
        else if (p.epi == EPI_DIV) v = v / div;
        store_elem<double>(p.C, p.tc, idx, v);
      }
    }
  }
}

template <class SA, class SB, int WGM, int WGN, int BK, int ST, int BN = 128, int MB = 1>
static ps_status launch_dmma(const Params &p, bool ak, double alpha, double beta, double div, cudaStream_t st) {
  using C = DCfg<WGM, WGN, BK, ST, BN, MB>;
  constexpr int SM = C::SMEM;
  PS_TRY(set_max_smem((const void *)gemm_dmma_kernel<SA, SB, true, WGM, WGN, BK, ST, BN, MB>, SM));
  PS_TRY(set_max_smem((const void *)gemm_dmma_kernel<SA, SB, false, WGM, WGN, BK, ST, BN, MB>, SM));
  dim3 grid((unsigned)((p.N + C::BN - 1) / C::BN), (unsigned)((p.M + C::BM - 1) / C::BM));
  if (ak) gemm_dmma_kernel<SA, SB, true, WGM, WGN, BK, ST, BN, MB><<<grid, C::THREADS, SM, st>>>(p, alpha, beta, div);
  else gemm_dmma_kernel<SA, SB, false, WGM, WGN, BK, ST, BN, MB><<<grid, C::THREADS, SM, st>>>(p, alpha, beta, div);
  PS_CHECK_LAUNCH("gemm_dmma_kernel");
  return PS_OK;
}

// Tile shape history (f64 GEMM at 8192^3, profiles/dmma_probe_r1.txt): 128 x 128 tiles of
// 16 warps, one CTA per SM, 4 stages of BK 16: 29.9 TFLOP/s; 16 warps, 3 stages of BK 32:
// 31.5; 128 x 64 tiles, two CTAs per SM, 2 stages of BK 32: 32.3; the shape below: 34.2.
// The earlier shapes are compiled only with -DPS_LEGACY_KERNELS (PS_DMMA_VARIANT=1..4).
#ifdef PS_LEGACY_KERNELS
static int dmma_variant() {
  static const int v = [] { const char *e = getenv("PS_DMMA_VARIANT"); return e ? atoi(e) : 0; }();
  return v;
}
#endif

ps_status gemm_dmma_f64(const GemmArgs &g, cudaStream_t st) {
  const Params p = make_params(g);
  const bool ak = g.A.s_col == 1;
  return dispatch_store(g.A.type, [&](auto sa) -> ps_status {
    return dispatch_store(g.B.type, [&](auto sb) -> ps_status {
      using SA = decltype(sa);
      using SB = decltype(sb);
#ifdef PS_LEGACY_KERNELS
      switch (dmma_variant()) {
        case 1: return launch_dmma<SA, SB, 4, 4, 16, 4>(p, ak, g.alpha, g.beta, g.div, st);
        case 2: return launch_dmma<SA, SB, 2, 4, 16, 4>(p, ak, g.alpha, g.beta, g.div, st);
        case 3: return launch_dmma<SA, SB, 4, 4, 32, 3>(p, ak, g.alpha, g.beta, g.div, st);
        case 4: return launch_dmma<SA, SB, 4, 2, 32, 2, 64, 2>(p, ak, g.alpha, g.beta, g.div, st);
        default: break;
      }
#endif
      // 128 x 64 CTA tiles of 8 warps (32 x 32 warp tiles), two CTAs per SM, 3 stages of BK 16
      return launch_dmma<SA, SB, 4, 2, 16, 3, 64, 2>(p, ak, g.alpha, g.beta, g.div, st);
    });
  });
}

}  // namespace simt
}  // namespace ps
