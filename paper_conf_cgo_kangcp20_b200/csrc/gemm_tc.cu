// gemm_tc.cu -- tcgen05 tensor-core contraction for statements whose two
// multiplicands are fp16 objects and whose compute type is f32 (reading R2):
// the fp16 x fp16 -> f32-accumulate path of GEMM / 2MM / 3MM / SYRK (row a3).
// Reading R6: the tensor core's internal summation order is unspecified, so
// these results are checked against the oracle with the stated tolerance, not
// bit-exactly (every other contraction is the R3-exact SIMT kernel).
//
// Structure (one 128 x 256 output tile per CTA, cta_group::1):
//   warp 0, one lane : TMA producer  -- cp.async.bulk.tensor 2D boxes of 64
//                      fp16 (128 B, SWIZZLE_128B) into a 4-stage smem ring,
//                      mbarrier expect_tx / complete_tx
//   warp 1           : TMEM allocator (256 columns = the f32 accumulator);
//                      one lane issues tcgen05.mma.kind::f16 (M=128, N=256,
//                      K=16) and tcgen05.commit frees each stage / signals
//                      the epilogue
//   warps 2..9       : epilogue -- tcgen05.ld 32x32b (warp w reads TMEM lanes
//                      32*(w%4)..), alpha/beta or divide in f32, RNE store to
//                      the output object's precision (R1)
// A may be K-major (row-major A) or M-major (SYRK's data^T); B is N-major.
//
// fp8 x fp8 (reading #29; kind::f8f6f4, E4M3/E5M2 in any mix): the same
// kernels instantiated with 1-byte elements -- a k-block is 128 elements (still
// one 128-byte swizzled row), each MMA consumes K = 32, MN-major boxes are 128
// elements wide; the epilogue multiplies the f32 accumulator by the operands'
// per-tensor scales 2^(ka + kb) (exact) before alpha/beta.
#include <cuda.h>

#include <atomic>
#include <cudaTypedefs.h>

#include "common.cuh"
#include "kernels.cuh"

namespace ps {
namespace tc {

constexpr int BM = 128, BN = 256, STAGES = 3;
constexpr int KB_BYTES = 128;                   // one k-block = one 128-byte swizzled row
constexpr int A_BYTES = BM * KB_BYTES;          // 16 KiB
constexpr int B_BYTES = BN * KB_BYTES;          // 32 KiB
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
// epilogue staging: each of the 4 epilogue warps turns a 32 x 32 accumulator chunk
// (thread = row, from tcgen05.ld.32x32b) into coalesced row segments through smem
// 16-column chunks (round 2: from 32) halve the staging buffer, which buys the 2-CTA
// kernel a sixth pipeline stage
constexpr int EPI_COLS = 16;
constexpr int EPI_STRIDE = 20;                                // floats per staged row (conflict-free STS.128)
// 8 epilogue warps: two per TMEM lane quarter (warp w may read lanes 32 (w % 4)..),
// each draining half of the accumulator's columns -- twice the memory-level
// parallelism of one warp per quarter, which paced the fp8 tiles (ncu, round 1)
constexpr int EPI_WARPS = 8;
constexpr int EPI_SMEM = EPI_WARPS * 32 * EPI_STRIDE * 4;     // 20 KiB
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 + 256 + EPI_SMEM;
constexpr int NTHREADS = 64 + 32 * EPI_WARPS;
constexpr uint32_t TMEM_COLS = 256;
// element-size dependent geometry (ES = 2: f16/bf16, ES = 1: fp8)
template <int ES> struct Geo {
  static constexpr int BK = KB_BYTES / ES;              // elements per k-block
  static constexpr int MN_BOX = 128 / ES;               // MN-major box width (elements)
  static constexpr uint32_t BOX_BYTES = 128 * BK;       // one MN-major box {MN_BOX, BK}
  static constexpr int MMA_K = 32 / ES;                 // K per tcgen05.mma
  static constexpr uint32_t MN_STEP = MMA_K * 128;      // MN-major: bytes per MMA k-step
};

struct Params {
  int M, N, K;
  int a_mn_major;
  int b_k_major;     // B(k, j) K-contiguous (a transposed copy) instead of N-major
  void *C;
  int c_type;
  int64_t ldc;
  const void *Cin;
  int cin_type;
  int epi;
  float alpha, beta, div;
  int upper_only;
  int row_off;             // upper_only: global row of output row 0 (row-sharded evaluation)
  uint32_t a_fmt, b_fmt;   // kind::f16: 0 = f16, 1 = bf16 (reading #28); kind::f8f6f4: 0 = E4M3, 1 = E5M2
  const ps_fp8_scale *sa, *sb;   // fp8 operands: per-tensor scales (reading #29)
  int vec4;                // C / Cin rows 4-element aligned: vector epilogue stores / loads
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  while (!mbar_try_wait(bar, parity)) {
  }
}
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, uint64_t *bar, int c0,
                                            int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, "
      "%4}], [%2];" ::"r"(smem_u32(dst)),
      "l"((uint64_t)map), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
// UMMA shared-memory matrix descriptor (sm100): start >> 4 [0,14), LBO >> 4
// [16,30), SBO >> 4 [32,46), version 1 [46,48), base offset 0, SWIZZLE_128B (2) [61,64)
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
template <int ES>
__device__ __forceinline__ void umma_f16(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc,
                                         uint32_t accumulate) {
  if constexpr (ES == 2)
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(idesc), "r"(accumulate));
  else
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f8f6f4 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(idesc), "r"(accumulate));
}
// the fp8 operands' scale 2^(ka + kb); 1 for f16 / bf16
__device__ __forceinline__ int scale_exp2(const Params &p) {
  return (p.sa ? p.sa->k : 0) + (p.sb ? p.sb->k : 0);
}
__device__ __forceinline__ void umma_commit(uint64_t *bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%"
      "15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
        "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
        "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
        "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
        "=r"(v[14]), "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]),
        "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]),
        "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ float load_c(const void *p, int type, int64_t idx) {
  if (type == PS_F32) return ((const float *)p)[idx];
  const uint16_t h = ((const uint16_t *)p)[idx];
  return type == PS_BF16 ? bf16_to_f32(h) : f16_to_f32(h);
}
__device__ __forceinline__ void store_c(void *p, int type, int64_t idx, float v) {
  if (type == PS_F32) ((float *)p)[idx] = v;
  else if (type == PS_BF16) ((uint16_t *)p)[idx] = rne_bf16(v);
  else ((uint16_t *)p)[idx] = rne_f16(v);
}

__device__ __forceinline__ float epi_op(const Params &p, float r, float cin) {
  if (p.epi == EPI_AXPBY) return __fmaf_rn(p.alpha, r, p.beta * cin);
  if (p.epi == EPI_DIV) return r / p.div;
  return r;
}

// Epilogue of one 32-row x 16-column accumulator chunk held by this warp (lane =
// row row0 + lane, v = columns col0..col0+15 from tcgen05.ld.32x32b.x16): staged
// through smem, then written as row segments -- lane l handles rows 8i + l/4 and
// columns 4(l%4)..+3 (one 16-byte f32 or 8-byte 16-bit access, and the matching
// Cin load for alpha/beta), so 4 lanes cover a row's 64 contiguous bytes.  fp8
// operands: accumulator x 2^kab first.
__device__ __forceinline__ void epi_chunk(const Params &p, float *stg, int lane, int64_t row0,
                                          int64_t col0, const uint32_t (&v)[16], int kab) {
  float4 *srow = reinterpret_cast<float4 *>(stg + lane * EPI_STRIDE);
#pragma unroll
  for (int q = 0; q < 4; q++)
    srow[q] = make_float4(__uint_as_float(v[4 * q]), __uint_as_float(v[4 * q + 1]),
                          __uint_as_float(v[4 * q + 2]), __uint_as_float(v[4 * q + 3]));
  __syncwarp();
  const int cq = lane & 3;
  const int64_t col = col0 + cq * 4;
  const bool vcol = p.vec4 && col + 3 < p.N;
  // 1) the chunk's 4 Cin segments of this lane, all loads in flight at once (alpha/beta)
  float c[4][4];
#pragma unroll
  for (int i = 0; i < 4; i++) {
    c[i][0] = c[i][1] = c[i][2] = c[i][3] = 0.f;
    const int64_t row = row0 + i * 8 + (lane >> 2);
    if (p.epi != EPI_AXPBY || row >= p.M) continue;
    const int64_t idx = row * p.ldc + col;
    if (vcol) {
      if (p.cin_type == PS_F32) {
        const float4 t = __ldg(reinterpret_cast<const float4 *>((const float *)p.Cin + idx));
        c[i][0] = t.x; c[i][1] = t.y; c[i][2] = t.z; c[i][3] = t.w;
      } else {
        const uint2 t = __ldg(reinterpret_cast<const uint2 *>((const uint16_t *)p.Cin + idx));
        const uint16_t h[4] = {(uint16_t)(t.x & 0xFFFF), (uint16_t)(t.x >> 16), (uint16_t)(t.y & 0xFFFF),
                               (uint16_t)(t.y >> 16)};
#pragma unroll
        for (int e = 0; e < 4; e++) c[i][e] = p.cin_type == PS_BF16 ? bf16_to_f32(h[e]) : f16_to_f32(h[e]);
      }
    } else {
#pragma unroll
      for (int e = 0; e < 4; e++)
        if (col + e < p.N) c[i][e] = load_c(p.Cin, p.cin_type, idx + e);
    }
  }
  // 2) scale, epilogue op, RNE store (R1) as row segments
#pragma unroll
  for (int i = 0; i < 4; i++) {
    const int r = i * 8 + (lane >> 2);
    const int64_t row = row0 + r;
    const float4 a = *reinterpret_cast<const float4 *>(stg + r * EPI_STRIDE + cq * 4);
    float x[4] = {a.x, a.y, a.z, a.w};
    if (row >= p.M) continue;
    if (kab) {
#pragma unroll
      for (int e = 0; e < 4; e++) x[e] = scalbnf(x[e], kab);   // exact power-of-two scale
    }
#pragma unroll
    for (int e = 0; e < 4; e++) x[e] = epi_op(p, x[e], c[i][e]);
    const int64_t idx = row * p.ldc + col;
    if (vcol) {
      if (p.c_type == PS_F32) {
        *reinterpret_cast<float4 *>((float *)p.C + idx) = make_float4(x[0], x[1], x[2], x[3]);
      } else {
        uint16_t h[4];
#pragma unroll
        for (int e = 0; e < 4; e++) h[e] = p.c_type == PS_BF16 ? rne_bf16(x[e]) : rne_f16(x[e]);
        *reinterpret_cast<uint2 *>((uint16_t *)p.C + idx) =
            make_uint2((uint32_t)h[0] | ((uint32_t)h[1] << 16), (uint32_t)h[2] | ((uint32_t)h[3] << 16));
      }
    } else {
#pragma unroll
      for (int e = 0; e < 4; e++)
        if (col + e < p.N) store_c(p.C, p.c_type, idx + e, x[e]);
    }
  }
  __syncwarp();
}

template <int ES>
__global__ void __launch_bounds__(NTHREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b,
                   Params p) {
  using G = Geo<ES>;
  constexpr int BK = G::BK;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t *sA = smem;
  uint8_t *sB = smem + STAGES * A_BYTES;
  uint64_t *full = (uint64_t *)(smem + STAGES * STAGE_BYTES);
  uint64_t *empty = full + STAGES;
  uint64_t *tfull = empty + STAGES;
  uint32_t *tmem_slot = (uint32_t *)(tfull + 1);
  float *epi_stage = (float *)(smem + STAGES * STAGE_BYTES + 256);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
  if (p.upper_only && m0 + p.row_off >= n0 + BN) return;   // SYRK: tile strictly below the diagonal
  const int nk = (p.K + BK - 1) / BK;

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tma_a) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tma_b) : "memory");
    for (int s = 0; s < STAGES; s++) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    mbar_init(tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {   // ---------------- TMA producer
      for (int kb = 0; kb < nk; kb++) {
        const int s = kb % STAGES;
        const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
        mbar_wait(&empty[s], ph ^ 1u);
        mbar_expect_tx(&full[s], STAGE_BYTES);
        const int k0 = kb * BK;
        uint8_t *a = sA + s * A_BYTES;
        if (!p.a_mn_major) {
          tma_load_2d(a, &tma_a, &full[s], k0, m0);                 // box {BK, 128 M}
        } else {
#pragma unroll
          for (int q = 0; q < BM / G::MN_BOX; q++)                  // box {MN_BOX M, BK}
            tma_load_2d(a + q * G::BOX_BYTES, &tma_a, &full[s], m0 + G::MN_BOX * q, k0);
        }
        uint8_t *b = sB + s * B_BYTES;
        if (p.b_k_major) {
          tma_load_2d(b, &tma_b, &full[s], k0, n0);                 // box {BK, 256 N}
        } else {
#pragma unroll
          for (int q = 0; q < BN / G::MN_BOX; q++)
            tma_load_2d(b + q * G::BOX_BYTES, &tma_b, &full[s], n0 + G::MN_BOX * q, k0);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {   // ---------------- MMA issuer (single thread)
      const uint32_t idesc = (1u << 4)                          // D = f32
                             | (p.a_fmt << 7) | (p.b_fmt << 10)     // A, B format
                             | ((uint32_t)p.a_mn_major << 15)   // A major
                             | ((uint32_t)(!p.b_k_major) << 16) // B major
                             | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
      for (int kb = 0; kb < nk; kb++) {
        const int s = kb % STAGES;
        const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
        mbar_wait(&full[s], ph);
        fence_after();
        const uint32_t abase = smem_u32(sA + s * A_BYTES), bbase = smem_u32(sB + s * B_BYTES);
#pragma unroll
        for (int kk = 0; kk < BK / G::MMA_K; kk++) {
          // K-major SW128: +32 B per MMA K step inside the 128 B swizzled row;
          // MN-major SW128: +MMA_K K-rows of 128 B; LBO = one MN box between boxes.
          const uint64_t ad = p.a_mn_major ? umma_desc(abase + kk * G::MN_STEP, G::BOX_BYTES, 1024)
                                           : umma_desc(abase + kk * 32, 16, 1024);
          const uint64_t bd = p.b_k_major ? umma_desc(bbase + kk * 32, 16, 1024)
                                          : umma_desc(bbase + kk * G::MN_STEP, G::BOX_BYTES, 1024);
          umma_f16<ES>(tmem, ad, bd, idesc, (kb | kk) != 0);
        }
        umma_commit(&empty[s]);   // frees the stage when these MMAs retire
      }
      umma_commit(tfull);         // accumulator complete
    }
  } else {   // ------------------------- epilogue warps 2..9
    mbar_wait(tfull, 0);
    fence_after();
    const int kab = scale_exp2(p);
    const int q = warp & 3;                 // TMEM lane quarter this warp may access
    float *stg = epi_stage + (warp - 2) * 32 * EPI_STRIDE;
    const int half = (warp - 2) / 4;        // which half of the columns this warp drains
    for (int cc = half * (BN / EPI_COLS / 2); cc < (half + 1) * (BN / EPI_COLS / 2); cc++) {
      if ((int64_t)n0 + cc * EPI_COLS >= p.N) break;
      uint32_t v[16];
      tmem_ld16(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(cc * EPI_COLS), v);
      epi_chunk(p, stg, lane, (int64_t)m0 + q * 32, (int64_t)n0 + cc * EPI_COLS, v, kab);
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS));
  }
}

// ===================================================================
// 2-CTA persistent variant: a cluster of 2 CTAs (one TPC) computes a 256 x 256
// tile with tcgen05.mma.cta_group::2 (M=256, N=256, K=16).  Each CTA stages
// 128 rows of A and 128 columns of B per k-block (32 KiB / stage, 6 stages);
// TMA in both CTAs completes on the leader's full barrier; the leader's single
// MMA thread commits (multicast) to both CTAs' empty / tmem_full barriers.
// Two TMEM accumulators (2 x 256 columns) let the epilogue of tile i overlap
// the MMAs of tile i+1.  Tiles are walked persistently, cluster c taking tiles
// c, c + #clusters, ... (SYRK: lower tiles skipped by every role alike).
namespace tc2 {

constexpr int BM = 256, BN = 256, STAGES = 6;   // 6 x 32 KiB + 20 KiB epilogue staging
constexpr int HM = BM / 2, HN = BN / 2;          // per-CTA halves
constexpr int A_BYTES = HM * tc::KB_BYTES;      // 16 KiB
constexpr int B_BYTES = HN * tc::KB_BYTES;      // 16 KiB
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 + 512 + tc::EPI_SMEM;
constexpr int NTHREADS = tc::NTHREADS;
constexpr uint32_t TMEM_COLS = 512;             // 2 accumulators x 256 f32 columns
constexpr uint32_t PEER_MASK = 0xFEFFFFFFu;     // shared::cluster address of the leader's copy

using tc::Params;
using tc::Geo;
using tc::scale_exp2;
using tc::fence_after;
using tc::fence_before;
using tc::mbar_expect_tx;
using tc::mbar_init;
using tc::mbar_wait;
using tc::smem_u32;
using tc::tmem_ld16;
using tc::tmem_ld32;
using tc::tmem_ld16;
using tc::epi_chunk;
using tc::EPI_COLS;
using tc::EPI_STRIDE;
using tc::umma_desc;
using tc::load_c;
using tc::store_c;

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void tma_load_2sm(void *dst, const CUtensorMap *map, uint64_t *bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, "
      "%4}], [%2];" ::"r"(smem_u32(dst)),
      "l"((uint64_t)map), "r"(smem_u32(bar) & PEER_MASK), "r"(c0), "r"(c1)
      : "memory");
}
// multicast variant: the box lands at the same smem offset in every CTA of `mask`;
// each destination's bytes complete on ITS pair leader's barrier (peer bit cleared)
__device__ __forceinline__ void tma_load_2sm_mc(void *dst, const CUtensorMap *map, uint64_t *bar, int c0, int c1,
                                                uint16_t mask) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster"
      " [%0], [%1, {%4, %5}], [%2], %3;" ::"r"(smem_u32(dst)),
      "l"((uint64_t)map), "r"(smem_u32(bar) & PEER_MASK), "h"(mask), "r"(c0), "r"(c1)
      : "memory");
}
template <int ES>
__device__ __forceinline__ void umma2(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  const uint32_t z = 0;
  if constexpr (ES == 2)
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, {%5, %5, %5, %5, %5, %5, %5, %5}, p;\n\t}" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(z));
  else
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::f8f6f4 [%0], %1, %2, %3, {%5, %5, %5, %5, %5, %5, %5, %5}, p;\n\t}" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc), "r"(z));
}
// commit the leader's MMAs to the barrier at this offset in every CTA of `mask`
__device__ __forceinline__ void commit_mc(uint64_t *bar, uint16_t mask) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"(mask)
      : "memory");
}
// arrive on the pair leader's copy of a barrier (remote for odd ranks)
__device__ __forceinline__ void arrive_leader(uint64_t *bar, uint32_t leader_rank) {
  uint32_t remote;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(smem_u32(bar)), "r"(leader_rank));
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(remote) : "memory");
}

struct Sched {
  int64_t tiles_m, tiles_n, total;   // tiles_n counts cluster tiles of npairs * BN columns
  int npairs;                        // CTA pairs per cluster (1, or 2 with A multicast)
  int upper_only;
  int64_t tm_off;          // upper_only: global tile row of tile row 0 (row_off / BM)
  // i-th tile of this cluster (skipping SYRK tiles wholly below the diagonal); n0 is the
  // cluster tile's first column -- pair p computes columns n0 + p * BN ..
  // Grouped raster: consecutive t walk GROUP_M tile-rows down a tile-column before
  // moving right, so the ~74 tiles in flight share ~8 A row-blocks and ~10 B column
  // blocks (~70 MB at K = 8192 fp16) that stay in L2, instead of one tile-row
  // against all of B (round-2 ncu: 2.3 GB DRAM reads per 8192^3 GEMM, L2 hit 65%).
  static constexpr int64_t GROUP_M = 8;
  __device__ bool get(int64_t cluster, int64_t nclusters, int64_t &cursor, int &m0, int &n0) const {
    for (int64_t t = cursor; t < total; t += nclusters) {
      const int64_t per_group = GROUP_M * tiles_n, g = t / per_group, first = g * GROUP_M;
      const int64_t gm = tiles_m - first < GROUP_M ? tiles_m - first : GROUP_M;
      const int64_t tm = first + (t % per_group) % gm, tn = (t % per_group) / gm;
      if (upper_only && tm + tm_off > tn * npairs + npairs - 1) continue;
      m0 = (int)(tm * BM);
      n0 = (int)(tn * BN * npairs);
      cursor = t + nclusters;
      return true;
    }
    cursor = total;
    return false;
  }
};

// CL = 2: one CTA pair per cluster.  CL = 4: two pairs side by side along N
// (a 256 x 512 cluster tile) sharing the A rows -- each CTA loads half of its A
// block (64 rows) and multicasts it to the same-rank CTA of the other pair, so a
// CTA reads 24 KiB instead of 32 KiB from L2 per k-block; a stage is free once
// BOTH pairs' MMAs retired it (empty barrier count 2, commits multicast to all 4).
template <int ES, int CL>
__global__ void __launch_bounds__(NTHREADS, 1)
    gemm_tc2_kernel(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b,
                    Params p, Sched sch) {
  using G = Geo<ES>;
  constexpr int BK = G::BK;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t *sA = smem;
  uint8_t *sB = smem + STAGES * A_BYTES;
  uint64_t *full = (uint64_t *)(smem + STAGES * STAGE_BYTES);
  uint64_t *empty = full + STAGES;
  uint64_t *tfull = empty + STAGES;      // [2]
  uint64_t *tempty = tfull + 2;          // [2]
  uint32_t *tmem_slot = (uint32_t *)(tempty + 2);
  float *epi_stage = (float *)(smem + STAGES * STAGE_BYTES + 512);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t crank = cluster_rank();
  const uint32_t rank = crank & 1u, pair = crank >> 1;   // rank within the pair, pair in the cluster
  const bool leader = rank == 0;
  const uint16_t pair_mask = (uint16_t)(3u << (2 * pair));
  const int64_t cluster = blockIdx.x / CL, nclusters = gridDim.x / CL;
  const int nk = (p.K + BK - 1) / BK;

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tma_a) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tma_b) : "memory");
    for (int s = 0; s < STAGES; s++) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], CL / 2);   // every pair leader's commit (A is shared across pairs)
    }
    for (int a = 0; a < 2; a++) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], 2 * tc::EPI_WARPS);   // every epilogue warp of both CTAs of the pair
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {   // same warp in both CTAs (cta_group::2 allocation)
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  fence_before();
  cluster_sync_all();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {   // ---------------- TMA producer (both CTAs)
      int64_t cursor = cluster;
      int m0, n0;
      uint32_t it = 0;
      while (sch.get(cluster, nclusters, cursor, m0, n0)) {
        const int am = m0 + (int)rank * HM, bn = n0 + (int)pair * BN + (int)rank * HN;
        for (int kb = 0; kb < nk; kb++, it++) {
          const int s = it % STAGES;
          const uint32_t ph = (it / STAGES) & 1u;
          mbar_wait(&empty[s], ph ^ 1u);
          if (leader) mbar_expect_tx(&full[s], 2 * STAGE_BYTES);   // both CTAs' bytes
          const int k0 = kb * BK;
          uint8_t *a = sA + s * A_BYTES;
          if constexpr (CL == 4) {   // my half of the A block, to me and my counterpart
            const uint16_t amask = (uint16_t)((1u << rank) | (1u << (rank + 2)));
            if (!p.a_mn_major)                                              // box {BK, 64 M}
              tma_load_2sm_mc(a + pair * (HM / 2) * tc::KB_BYTES, &tma_a, &full[s], k0,
                              am + (int)pair * (HM / 2), amask);
            else                                                            // box {MN_BOX M, BK}
              tma_load_2sm_mc(a + pair * G::BOX_BYTES, &tma_a, &full[s], am + G::MN_BOX * (int)pair, k0, amask);
          } else if (!p.a_mn_major) {
            tma_load_2sm(a, &tma_a, &full[s], k0, am);                    // box {BK, 128 M}
          } else {
#pragma unroll
            for (int q = 0; q < HM / G::MN_BOX; q++)                      // box {MN_BOX M, BK}
              tma_load_2sm(a + q * G::BOX_BYTES, &tma_a, &full[s], am + G::MN_BOX * q, k0);
          }
          uint8_t *b = sB + s * B_BYTES;
          if (p.b_k_major) {
            tma_load_2sm(b, &tma_b, &full[s], k0, bn);                    // box {BK, 128 N}
          } else {
#pragma unroll
            for (int q = 0; q < HN / G::MN_BOX; q++)                      // box {MN_BOX N, BK}
              tma_load_2sm(b + q * G::BOX_BYTES, &tma_b, &full[s], bn + G::MN_BOX * q, k0);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (leader && lane == 0) {   // ---- MMA issuer (leader CTA, single thread)
      const uint32_t idesc = (1u << 4) | (p.a_fmt << 7) | (p.b_fmt << 10) |
                             ((uint32_t)p.a_mn_major << 15) | ((uint32_t)(!p.b_k_major) << 16) |
                             ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
      int64_t cursor = cluster;
      int m0, n0;
      uint32_t it = 0, j = 0;
      while (sch.get(cluster, nclusters, cursor, m0, n0)) {
        const uint32_t acc = j & 1u;
        mbar_wait(&tempty[acc], ((j >> 1) & 1u) ^ 1u);   // epilogues of both CTAs drained it
        fence_after();
        const uint32_t dcol = tmem + acc * BN;
        for (int kb = 0; kb < nk; kb++, it++) {
          const int s = it % STAGES;
          mbar_wait(&full[s], (it / STAGES) & 1u);
          fence_after();
          const uint32_t abase = smem_u32(sA + s * A_BYTES), bbase = smem_u32(sB + s * B_BYTES);
#pragma unroll
          for (int kk = 0; kk < BK / G::MMA_K; kk++) {
            const uint64_t ad = p.a_mn_major ? umma_desc(abase + kk * G::MN_STEP, G::BOX_BYTES, 1024)
                                             : umma_desc(abase + kk * 32, 16, 1024);
            const uint64_t bd = p.b_k_major ? umma_desc(bbase + kk * 32, 16, 1024)
                                            : umma_desc(bbase + kk * G::MN_STEP, G::BOX_BYTES, 1024);
            umma2<ES>(dcol, ad, bd, idesc, (kb | kk) != 0);
          }
          // stage s free once these MMAs retire: both CTAs of the pair, and with A
          // multicast the other pair too (its producers write into our stage)
          commit_mc(&empty[s], CL == 4 ? (uint16_t)0xF : pair_mask);
        }
        commit_mc(&tfull[acc], pair_mask);   // accumulator acc complete in both CTAs of the pair
        j++;
      }
    }
  } else {   // ------------------------- epilogue warps 2..9 (both CTAs)
    const int q = warp & 3;
    const int kab = scale_exp2(p);
    int64_t cursor = cluster;
    int m0, n0;
    uint32_t j = 0;
    while (sch.get(cluster, nclusters, cursor, m0, n0)) {
      const uint32_t acc = j & 1u;
      mbar_wait(&tfull[acc], (j >> 1) & 1u);
      fence_after();
      const int64_t row0 = (int64_t)m0 + rank * HM + q * 32;
      const int64_t pn0 = (int64_t)n0 + pair * BN;
      float *stg = epi_stage + (warp - 2) * 32 * EPI_STRIDE;
      const int half = (warp - 2) / 4;
      for (int cc = half * (BN / EPI_COLS / 2); cc < (half + 1) * (BN / EPI_COLS / 2); cc++) {
        if (pn0 + cc * EPI_COLS >= p.N) break;
        uint32_t v[16];
        tmem_ld16(tmem + acc * BN + ((uint32_t)(q * 32) << 16) + (uint32_t)(cc * EPI_COLS), v);
        epi_chunk(p, stg, lane, row0, pn0 + cc * EPI_COLS, v, kab);
      }
      fence_before();
      __syncwarp();
      if (lane == 0) arrive_leader(&tempty[acc], crank & ~1u);
      j++;
    }
  }
  fence_before();
  __syncthreads();
  cluster_sync_all();   // both CTAs finished with TMEM and with each other's barriers
  if (warp == 1) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS));
  }
}

}  // namespace tc2
}  // namespace tc

// ------------------------------------------------------------------ host
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void *f = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
  }
  return fn;
}

// 2-D tensor map: inner (contiguous) extent, outer extent, outer stride in bytes,
// box {128 bytes of elements, box_outer}, 128-byte swizzle, zero fill out of bounds.
static bool make_map(CUtensorMap *m, const void *base, uint64_t inner, uint64_t outer,
                     uint64_t stride_bytes, uint32_t box_outer, int type) {
  auto fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {stride_bytes};
  cuuint32_t box[2] = {(cuuint32_t)(128 / dtype_size(type)), box_outer};
  cuuint32_t es[2] = {1, 1};
  const CUtensorMapDataType dt = type == PS_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                 : type == PS_F16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16
                                                  : CU_TENSOR_MAP_DATA_TYPE_UINT8;
  return fn(m, dt, 2, const_cast<void *>(base), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool gemm_tc_supported(const GemmArgs &g) {
  // both multiplicands fp16, or both bf16 (kind::f16 takes either, not a mix), or
  // both fp8 (kind::f8f6f4: E4M3 / E5M2 in any mix)
  const bool f8 = is_fp8(g.A.type) && is_fp8(g.B.type);
  if (!((g.A.type == PS_F16 && g.B.type == PS_F16) || (g.A.type == PS_BF16 && g.B.type == PS_BF16) || f8) ||
      g.T != PS_F32)
    return false;
  if (g.c_type == PS_F64 || (g.epi == EPI_AXPBY && g.cin_type == PS_F64)) return false;
  if (is_fp8(g.c_type) || (g.epi == EPI_AXPBY && is_fp8(g.cin_type))) return false;
  if (f8 && (!g.A.sc || !g.B.sc)) return false;
  if (g.M <= 0 || g.N <= 0 || g.K <= 0 || g.M > (1 << 30) || g.N > (1 << 30) || g.K > (1 << 30))
    return false;
  if ((uintptr_t)g.A.p % 16 || (uintptr_t)g.B.p % 16) return false;
  const int64_t es = (int64_t)dtype_size(g.A.type);
  const bool a_k = g.A.s_col == 1 && (g.A.s_row * es) % 16 == 0;    // row-major A
  const bool a_m = g.A.s_row == 1 && (g.A.s_col * es) % 16 == 0;    // SYRK data^T
  const bool b_n = g.B.s_col == 1 && (g.B.s_row * es) % 16 == 0;    // row-major B
  const bool b_k = g.B.s_row == 1 && (g.B.s_col * es) % 16 == 0;    // K-contiguous B
  if (!(a_k || a_m) || !(b_n || b_k)) return false;
  return encode_fn() != nullptr;
}

template <int ES>
static ps_status gemm_tc_launch(const GemmArgs &g, cudaStream_t st) {
  using namespace tc;
  using G = Geo<ES>;
  PS_TRY(set_max_smem((const void *)gemm_tc_kernel<ES>, SMEM_BYTES));
  CUtensorMap ma, mb;
  const bool a_mn = !(g.A.s_col == 1);
  const bool b_k = !(g.B.s_col == 1);
  // the kernel choice follows the unsharded shape (tc_m_full) so that every shard of
  // a row-sharded evaluation runs the same tiles as the single-GPU statement
  const int64_t m_shape = g.tc_m_full > 0 ? g.tc_m_full : g.M;
  const bool two = (m_shape > BM || g.N > BN) && !getenv("PS_TC_1SM");
  // two CTA pairs per cluster sharing A (multicast) when a row of tiles has >= 2 pair tiles;
  // f16 / bf16 only (an fp8 M-major A box is the whole 128-row half)
  // Tried in round 2: clusters of two CTA pairs sharing A by TMA multicast (a CTA reads
  // 24 instead of 32 KiB per k-block).  Correct, but only 33 four-CTA clusters are
  // co-resident on a B200 (GPC shape; ncu launch__cluster_max_active), i.e. 132 of 148
  // SMs: 1329 vs 1363 TFLOP/s fp16 at 8192^3 (profiles/kernel_rates_r2g.jsonl).  Off.
  const bool four = false;
  bool ok;
  if (!a_mn) ok = make_map(&ma, g.A.p, (uint64_t)g.K, (uint64_t)g.M, (uint64_t)g.A.s_row * ES,
                           four ? tc2::HM / 2 : BM, g.A.type);
  else ok = make_map(&ma, g.A.p, (uint64_t)g.M, (uint64_t)g.K, (uint64_t)g.A.s_col * ES, G::BK, g.A.type);
  if (!b_k) ok = ok && make_map(&mb, g.B.p, (uint64_t)g.N, (uint64_t)g.K, (uint64_t)g.B.s_row * ES, G::BK, g.B.type);
  else ok = ok && make_map(&mb, g.B.p, (uint64_t)g.K, (uint64_t)g.N, (uint64_t)g.B.s_col * ES,
                           two ? tc2::HN : BN, g.B.type);
  if (!ok) {
    set_error("cuTensorMapEncodeTiled failed");
    return PS_ERR_CUDA;
  }
  const uint32_t af = (g.A.type == PS_BF16 || g.A.type == PS_E5M2) ? 1u : 0u;
  const uint32_t bfm = (g.B.type == PS_BF16 || g.B.type == PS_E5M2) ? 1u : 0u;
  Params p{(int)g.M, (int)g.N, (int)g.K, a_mn ? 1 : 0, b_k ? 1 : 0, g.C, g.c_type, g.ldc, g.Cin, g.cin_type, g.epi,
           (float)g.alpha, (float)g.beta, (float)g.div, g.upper_only, (int)g.row_off, af, bfm,
           ES == 1 ? g.A.sc : nullptr, ES == 1 ? g.B.sc : nullptr, 0};
  {   // vector epilogue: rows of C (and Cin) start 16-byte (f32) / 8-byte (16-bit) aligned
    const int64_t cb = (int64_t)dtype_size(g.c_type);
    bool v4 = g.ldc % 4 == 0 && (uintptr_t)g.C % (4 * cb) == 0;
    if (g.epi == EPI_AXPBY) v4 = v4 && (uintptr_t)g.Cin % (4 * dtype_size(g.cin_type)) == 0;
    p.vec4 = v4 ? 1 : 0;
  }
  if (two) {   // 2-CTA persistent path (clusters of 1 or 2 CTA pairs)
    using namespace tc2;
    const int CL = four ? 4 : 2;
    const void *kfn = four ? (const void *)gemm_tc2_kernel<ES, 4> : (const void *)gemm_tc2_kernel<ES, 2>;
    PS_TRY(set_max_smem(kfn, tc2::SMEM_BYTES));
    Sched sch;
    sch.npairs = CL / 2;
    sch.tiles_m = (g.M + tc2::BM - 1) / tc2::BM;
    sch.tiles_n = (g.N + tc2::BN * sch.npairs - 1) / (tc2::BN * sch.npairs);
    sch.total = sch.tiles_m * sch.tiles_n;
    sch.upper_only = g.upper_only;
    sch.tm_off = g.row_off / tc2::BM;
    int64_t work = 0;
    for (int64_t t = 0; t < sch.total; t++)
      if (!g.upper_only || t / sch.tiles_n + sch.tm_off <= (t % sch.tiles_n) * sch.npairs + sch.npairs - 1) work++;
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)CL;
    attr[0].val.clusterDim.y = attr[0].val.clusterDim.z = 1;
    cfg.blockDim = dim3(tc2::NTHREADS);
    cfg.dynamicSmemBytes = tc2::SMEM_BYTES;
    cfg.stream = st;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    // persistent: no more clusters than can be co-resident (4-CTA clusters must fit a GPC)
    int64_t clusters = num_sms() / CL;
    {
      static std::atomic<int> resident[2] = {0, 0};
      int r = resident[CL == 4].load(std::memory_order_relaxed);
      if (!r) {
        cfg.gridDim = dim3((unsigned)(CL * clusters));
        if (cudaOccupancyMaxActiveClusters(&r, kfn, &cfg) != cudaSuccess || r < 1) r = (int)clusters;
        resident[CL == 4].store(r, std::memory_order_relaxed);
      }
      if (clusters > r) clusters = r;
    }
    if (clusters > work) clusters = work;
    if (clusters < 1) clusters = 1;
    cfg.gridDim = dim3((unsigned)(CL * clusters));
    if (four) PS_CUDA(cudaLaunchKernelEx(&cfg, gemm_tc2_kernel<ES, 4>, ma, mb, p, sch));
    else PS_CUDA(cudaLaunchKernelEx(&cfg, gemm_tc2_kernel<ES, 2>, ma, mb, p, sch));
    PS_CHECK_LAUNCH("gemm_tc2_kernel");
    return PS_OK;
  }
  dim3 grid((unsigned)((g.N + BN - 1) / BN), (unsigned)((g.M + BM - 1) / BM));
  gemm_tc_kernel<ES><<<grid, NTHREADS, SMEM_BYTES, st>>>(ma, mb, p);
  PS_CHECK_LAUNCH("gemm_tc_kernel");
  return PS_OK;
}

ps_status gemm_tc_async(const GemmArgs &g, cudaStream_t st) {
  return is_fp8(g.A.type) ? gemm_tc_launch<1>(g, st) : gemm_tc_launch<2>(g, st);
}

}  // namespace ps
