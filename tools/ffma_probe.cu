// ffma_probe.cu -- design-space probe for the f32 contraction kernel (reading R3:
// every output an fma chain from +0, k ascending).  Standalone: C = A.B with A
// row-major M x K (k-major, the GEMM layout) and B row-major K x N, f32.
// Every variant is checked bit for bit against a one-thread-per-output chain
// kernel at 1024^3, then timed at N^3 (CUDA events, best of 5).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -fmad=false -lineinfo \
//        -o /tmp/ffma_probe tools/ffma_probe.cu && /tmp/ffma_probe 8192
//
// Template: BM x BN CTA tile, THREADS threads in a TY x TX grid; a thread owns
// TM x TN outputs as (TM/4) x (TN/4) blocks of 4 x 4, spaced TY*4 rows and TX*4
// columns apart, so its fragment loads are LDS.128; BK-deep k tiles in an
// S-stage ring: B by cp.async (16 B), A register-staged one ring slot ahead and
// stored transposed [k][m] (each thread owns whole k-runs of rows, so a warp's
// transposed stores hit consecutive m: conflict-free when BK*BM/THREADS == BK).
// DB: explicit register double buffer of the k+1 fragments.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ void cp16(void *s, const void *g) {
  unsigned sa = (unsigned)__cvta_generic_to_shared(s);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(g));
}
__device__ __forceinline__ void commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N> __device__ __forceinline__ void waitg() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

__global__ void ref_kernel(const float *A, const float *B, float *C, int M, int N, int K) {
  int n = blockIdx.x * blockDim.x + threadIdx.x, m = blockIdx.y;
  if (n >= N) return;
  float acc = 0.f;
  for (int k = 0; k < K; k++) acc = __fmaf_rn(A[(size_t)m * K + k], B[(size_t)k * N + n], acc);
  C[(size_t)m * N + n] = acc;
}

template <int BM, int BN, int BK, int TM, int TN, int THREADS, int S, int MINB, bool DB, bool F2 = false>
__global__ void __launch_bounds__(THREADS, MINB) ffma_kernel(const float *__restrict__ A, const float *__restrict__ B,
                                                             float *__restrict__ C, int M, int N, int K) {
  constexpr int TX = BN / TN, TY = BM / TM;
  static_assert(TX * TY == THREADS, "grid");
  constexpr int LA = BM + 4, LB = BN + 4;
  constexpr int AEL = BK * LA, BEL = BK * LB;
  constexpr int EA = BM * BK / THREADS;            // A elements per thread per tile
  static_assert(EA % 4 == 0 && BK % EA == 0, "A run");
  extern __shared__ __align__(16) float sm[];
  float *As0 = sm, *Bs0 = sm + S * AEL;
  const int tid = threadIdx.x, tx = tid % TX, ty = tid / TX;
  const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
  // A staging: thread -> (row, k-run); consecutive threads take consecutive rows
  const int a_m = tid % BM, a_k = (tid / BM) * EA;
  const float *Ag = A + (size_t)(m0 + a_m) * K + a_k;
  const int ktiles = K / BK;
  float4 ra[EA / 4];
  auto load_a = [&](int kt) {
#pragma unroll
    for (int e = 0; e < EA / 4; e++) ra[e] = __ldg(reinterpret_cast<const float4 *>(Ag + (size_t)kt * BK) + e);
  };
  auto store_a = [&](int st) {
    float *As = As0 + st * AEL;
#pragma unroll
    for (int e = 0; e < EA / 4; e++) {
      As[(a_k + 4 * e + 0) * LA + a_m] = ra[e].x;
      As[(a_k + 4 * e + 1) * LA + a_m] = ra[e].y;
      As[(a_k + 4 * e + 2) * LA + a_m] = ra[e].z;
      As[(a_k + 4 * e + 3) * LA + a_m] = ra[e].w;
    }
  };
  auto issue_b = [&](int kt, int st) {
    float *Bs = Bs0 + st * BEL;
    constexpr int CH = BK * BN / 4;
#pragma unroll
    for (int c = tid; c < CH; c += THREADS) {
      const int kr = c / (BN / 4), nc = (c % (BN / 4)) * 4;
      cp16(Bs + kr * LB + nc, B + (size_t)(kt * BK + kr) * N + n0 + nc);
    }
  };
  float2 acc[TM][TN / 2];
#pragma unroll
  for (int i = 0; i < TM; i++)
#pragma unroll
    for (int j = 0; j < TN / 2; j++) acc[i][j] = make_float2(0.f, 0.f);
  // one output pair (columns 2j, 2j+1): FFMA2 (fma.rn.f32x2 = two independent fma.rn,
  // bit-identical to two FFMAs) with a[i] broadcast, or two FFMAs
  auto fma_pair = [&](float a, float b0, float b1, float2 &c) {
    if constexpr (F2) c = __ffma2_rn(make_float2(a, a), make_float2(b0, b1), c);
    else { c.x = __fmaf_rn(a, b0, c.x); c.y = __fmaf_rn(a, b1, c.y); }
  };

#pragma unroll
  for (int s = 0; s < S - 1; s++) {
    if (s < ktiles) { load_a(s); store_a(s); issue_b(s, s); }
    commit();
  }
  for (int kt = 0; kt < ktiles; kt++) {
    waitg<S - 2>();
    __syncthreads();
    const int nt = kt + S - 1;
    if (nt < ktiles) { load_a(nt); issue_b(nt, nt % S); }
    commit();
    const float *As = As0 + (kt % S) * AEL, *Bs = Bs0 + (kt % S) * BEL;
    if constexpr (DB) {
      float a[2][TM], b[2][TN];
      auto frag = [&](int k, int buf) {
#pragma unroll
        for (int i4 = 0; i4 < TM / 4; i4++) {
          const float4 v = *reinterpret_cast<const float4 *>(As + k * LA + ty * 4 + i4 * TY * 4);
          a[buf][i4 * 4 + 0] = v.x; a[buf][i4 * 4 + 1] = v.y; a[buf][i4 * 4 + 2] = v.z; a[buf][i4 * 4 + 3] = v.w;
        }
#pragma unroll
        for (int j4 = 0; j4 < TN / 4; j4++) {
          const float4 v = *reinterpret_cast<const float4 *>(Bs + k * LB + tx * 4 + j4 * TX * 4);
          b[buf][j4 * 4 + 0] = v.x; b[buf][j4 * 4 + 1] = v.y; b[buf][j4 * 4 + 2] = v.z; b[buf][j4 * 4 + 3] = v.w;
        }
      };
      frag(0, 0);
#pragma unroll
      for (int k = 0; k < BK; k++) {
        if (k + 1 < BK) frag(k + 1, (k + 1) & 1);
#pragma unroll
        for (int i = 0; i < TM; i++)
#pragma unroll
          for (int j = 0; j < TN / 2; j++) fma_pair(a[k & 1][i], b[k & 1][2 * j], b[k & 1][2 * j + 1], acc[i][j]);
      }
    } else {
#pragma unroll
      for (int k = 0; k < BK; k++) {
        float a[TM], b[TN];
#pragma unroll
        for (int i4 = 0; i4 < TM / 4; i4++) {
          const float4 v = *reinterpret_cast<const float4 *>(As + k * LA + ty * 4 + i4 * TY * 4);
          a[i4 * 4 + 0] = v.x; a[i4 * 4 + 1] = v.y; a[i4 * 4 + 2] = v.z; a[i4 * 4 + 3] = v.w;
        }
#pragma unroll
        for (int j4 = 0; j4 < TN / 4; j4++) {
          const float4 v = *reinterpret_cast<const float4 *>(Bs + k * LB + tx * 4 + j4 * TX * 4);
          b[j4 * 4 + 0] = v.x; b[j4 * 4 + 1] = v.y; b[j4 * 4 + 2] = v.z; b[j4 * 4 + 3] = v.w;
        }
#pragma unroll
        for (int i = 0; i < TM; i++)
#pragma unroll
          for (int j = 0; j < TN / 2; j++) fma_pair(a[i], b[2 * j], b[2 * j + 1], acc[i][j]);
      }
    }
    if (nt < ktiles) store_a(nt % S);
  }
  waitg<0>();
#pragma unroll
  for (int i = 0; i < TM; i++) {
    const int gm = m0 + (i / 4) * TY * 4 + ty * 4 + (i % 4);
#pragma unroll
    for (int j4 = 0; j4 < TN / 4; j4++) {
      const int gn = n0 + j4 * TX * 4 + tx * 4;
      *reinterpret_cast<float4 *>(C + (size_t)gm * N + gn) =
          make_float4(acc[i][j4 * 2].x, acc[i][j4 * 2].y, acc[i][j4 * 2 + 1].x, acc[i][j4 * 2 + 1].y);
    }
  }
}

static float *dA, *dB, *dC, *dR;

template <int BM, int BN, int BK, int TM, int TN, int THREADS, int S, int MINB, bool DB, bool F2 = false>
void run(const char *name, int n) {
  auto k = ffma_kernel<BM, BN, BK, TM, TN, THREADS, S, MINB, DB, F2>;
  const int smem = S * BK * ((BM + 4) + (BN + 4)) * 4;
  CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaFuncAttributes fa;
  CK(cudaFuncGetAttributes(&fa, k));
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, THREADS, smem));
  // bit-exact check at 1024^3
  const int c = 1024;
  k<<<dim3(c / BN, c / BM), THREADS, smem>>>(dA, dB, dC, c, c, c);
  ref_kernel<<<dim3(c / 256, c), 256>>>(dA, dB, dR, c, c, c);
  CK(cudaDeviceSynchronize());
  std::vector<uint32_t> h1((size_t)c * c), h2((size_t)c * c);
  CK(cudaMemcpy(h1.data(), dC, h1.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(h2.data(), dR, h2.size() * 4, cudaMemcpyDeviceToHost));
  size_t bad = 0;
  for (size_t i = 0; i < h1.size(); i++) bad += h1[i] != h2[i];
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  dim3 g(n / BN, n / BM);
  k<<<g, THREADS, smem>>>(dA, dB, dC, n, n, n);
  float best = 1e30f;
  for (int r = 0; r < 5; r++) {
    cudaEventRecord(e0);
    k<<<g, THREADS, smem>>>(dA, dB, dC, n, n, n);
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  printf("{\"variant\": \"%s\", \"regs\": %d, \"smem\": %d, \"ctas_per_sm\": %d, \"mismatch_1024\": %zu, \"N\": %d, "
         "\"ms\": %.3f, \"tflops\": %.1f}\n",
         name, fa.numRegs, smem, occ, bad, n, best, 2.0 * n * n * (double)n / (best * 1e-3) / 1e12);
  fflush(stdout);
}


// Variant family "K": A (k-major) lands by cp.async in its natural [m][k] layout
// (row stride BK + 4 floats), no register staging and no transposed stores.  A
// thread reads, per group of 4 k, one LDS.128 per owned row (4 k values) and two
// LDS.128 of B per k; 8 x 8 outputs per thread as FFMA2 pairs along n.
template <int BM, int BN, int BK, int THREADS, int S, int MINB>
__global__ void __launch_bounds__(THREADS, MINB) ffma_kacp(const float *__restrict__ A, const float *__restrict__ B,
                                                           float *__restrict__ C, int M, int N, int K) {
  constexpr int TM = 8, TN = 8, TX = BN / TN, TY = BM / TM;
  static_assert(TX * TY == THREADS, "grid");
  constexpr int LA = BK + 4, LB = BN + 4;
  constexpr int AEL = BM * LA, BEL = BK * LB;
  extern __shared__ __align__(16) float sm[];
  float *As0 = sm, *Bs0 = sm + S * AEL;
  const int tid = threadIdx.x, tx = tid % TX, ty = tid / TX;
  const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
  const int ktiles = K / BK;
  auto issue = [&](int kt, int st) {
    float *As = As0 + st * AEL, *Bs = Bs0 + st * BEL;
#pragma unroll
    for (int c = tid; c < BM * BK / 4; c += THREADS) {
      const int r = c / (BK / 4), kc = (c % (BK / 4)) * 4;
      cp16(As + r * LA + kc, A + (size_t)(m0 + r) * K + kt * BK + kc);
    }
#pragma unroll
    for (int c = tid; c < BK * BN / 4; c += THREADS) {
      const int kr = c / (BN / 4), nc = (c % (BN / 4)) * 4;
      cp16(Bs + kr * LB + nc, B + (size_t)(kt * BK + kr) * N + n0 + nc);
    }
  };
  float2 acc[TM][TN / 2];
#pragma unroll
  for (int i = 0; i < TM; i++)
#pragma unroll
    for (int j = 0; j < TN / 2; j++) acc[i][j] = make_float2(0.f, 0.f);
#pragma unroll
  for (int s = 0; s < S - 1; s++) {
    if (s < ktiles) issue(s, s);
    commit();
  }
  for (int kt = 0; kt < ktiles; kt++) {
    waitg<S - 2>();
    __syncthreads();
    const int nt = kt + S - 1;
    if (nt < ktiles) issue(nt, nt % S);
    commit();
    const float *As = As0 + (kt % S) * AEL, *Bs = Bs0 + (kt % S) * BEL;
#pragma unroll
    for (int k4 = 0; k4 < BK; k4 += 4) {
      float4 a[TM];
#pragma unroll
      for (int i = 0; i < TM; i++)
        a[i] = *reinterpret_cast<const float4 *>(As + ((i / 4) * TY * 4 + ty * 4 + (i % 4)) * LA + k4);
#pragma unroll
      for (int kk = 0; kk < 4; kk++) {
        const float4 b0 = *reinterpret_cast<const float4 *>(Bs + (k4 + kk) * LB + tx * 4);
        const float4 b1 = *reinterpret_cast<const float4 *>(Bs + (k4 + kk) * LB + TX * 4 + tx * 4);
        const float2 b[4] = {make_float2(b0.x, b0.y), make_float2(b0.z, b0.w), make_float2(b1.x, b1.y),
                             make_float2(b1.z, b1.w)};
#pragma unroll
        for (int i = 0; i < TM; i++) {
          const float ai = kk == 0 ? a[i].x : kk == 1 ? a[i].y : kk == 2 ? a[i].z : a[i].w;
#pragma unroll
          for (int j = 0; j < TN / 2; j++) acc[i][j] = __ffma2_rn(make_float2(ai, ai), b[j], acc[i][j]);
        }
      }
    }
  }
  waitg<0>();
#pragma unroll
  for (int i = 0; i < TM; i++) {
    const int gm = m0 + (i / 4) * TY * 4 + ty * 4 + (i % 4);
#pragma unroll
    for (int j4 = 0; j4 < TN / 4; j4++) {
      const int gn = n0 + j4 * TX * 4 + tx * 4;
      *reinterpret_cast<float4 *>(C + (size_t)gm * N + gn) =
          make_float4(acc[i][j4 * 2].x, acc[i][j4 * 2].y, acc[i][j4 * 2 + 1].x, acc[i][j4 * 2 + 1].y);
    }
  }
}

template <int BM, int BN, int BK, int THREADS, int S, int MINB>
void run_kacp(const char *name, int n) {
  auto k = ffma_kacp<BM, BN, BK, THREADS, S, MINB>;
  const int smem = S * (BM * (BK + 4) + BK * (BN + 4)) * 4;
  CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaFuncAttributes fa;
  CK(cudaFuncGetAttributes(&fa, k));
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, THREADS, smem));
  const int c = 1024;
  k<<<dim3(c / BN, c / BM), THREADS, smem>>>(dA, dB, dC, c, c, c);
  ref_kernel<<<dim3(c / 256, c), 256>>>(dA, dB, dR, c, c, c);
  CK(cudaDeviceSynchronize());
  std::vector<uint32_t> h1((size_t)c * c), h2((size_t)c * c);
  CK(cudaMemcpy(h1.data(), dC, h1.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(h2.data(), dR, h2.size() * 4, cudaMemcpyDeviceToHost));
  size_t bad = 0;
  for (size_t i = 0; i < h1.size(); i++) bad += h1[i] != h2[i];
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  dim3 g(n / BN, n / BM);
  k<<<g, THREADS, smem>>>(dA, dB, dC, n, n, n);
  float best = 1e30f;
  for (int r = 0; r < 5; r++) {
    cudaEventRecord(e0);
    k<<<g, THREADS, smem>>>(dA, dB, dC, n, n, n);
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  printf("{\"variant\": \"%s\", \"regs\": %d, \"smem\": %d, \"ctas_per_sm\": %d, \"mismatch_1024\": %zu, \"N\": %d, "
         "\"ms\": %.3f, \"tflops\": %.1f}\n",
         name, fa.numRegs, smem, occ, bad, n, best, 2.0 * n * n * (double)n / (best * 1e-3) / 1e12);
  fflush(stdout);
}

__global__ void fill(float *p, size_t n, uint32_t seed) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  if (i < n) {
    uint32_t x = (uint32_t)i * 2654435761u ^ seed;
    x ^= x >> 15; x *= 2246822519u; x ^= x >> 13;
    p[i] = (float)(x & 0xFFFFFF) / 16777216.0f - 0.5f;
  }
}

int main(int argc, char **argv) {
  const int n = argc > 1 ? atoi(argv[1]) : 8192;
  const size_t el = (size_t)n * n;
  CK(cudaMalloc(&dA, el * 4)); CK(cudaMalloc(&dB, el * 4)); CK(cudaMalloc(&dC, el * 4)); CK(cudaMalloc(&dR, el * 4));
  fill<<<(el + 255) / 256, 256>>>(dA, el, 1);
  fill<<<(el + 255) / 256, 256>>>(dB, el, 2);
  CK(cudaDeviceSynchronize());
  const char *only = argc > 2 ? argv[2] : "";
#define V(name, ...) if (!*only || strstr(name, only)) run<__VA_ARGS__>(name, n)
  V("A 128x128 t256 8x8 bk16 s3 minb2", 128, 128, 16, 8, 8, 256, 3, 2, false);
  V("B 128x128 t256 8x8 bk16 s3 minb2 db", 128, 128, 16, 8, 8, 256, 3, 2, true);
  V("C 128x128 t128 16x8 bk16 s4 minb2", 128, 128, 16, 16, 8, 128, 4, 2, false);
  V("D 128x128 t128 16x8 bk16 s4 minb2 db", 128, 128, 16, 16, 8, 128, 4, 2, true);
  V("E 128x128 t128 8x16 bk16 s4 minb2", 128, 128, 16, 8, 16, 128, 4, 2, false);
  V("F 256x128 t256 16x8 bk16 s4 minb1", 256, 128, 16, 16, 8, 256, 4, 1, false);
  V("G 256x128 t256 16x8 bk16 s4 minb1 db", 256, 128, 16, 16, 8, 256, 4, 1, true);
  V("H 128x128 t128 16x8 bk8 s6 minb2", 128, 128, 8, 16, 8, 128, 6, 2, false);
  V("I 128x256 t256 8x16 bk16 s3 minb1", 128, 256, 16, 8, 16, 256, 3, 1, false);
  V("J 128x64 t128 8x8 bk16 s4 minb4", 128, 64, 16, 8, 8, 128, 4, 4, false);
  V("P A+ffma2 128x128 t256 8x8 bk16 s3 minb2", 128, 128, 16, 8, 8, 256, 3, 2, false, true);
  V("Q C+ffma2 128x128 t128 16x8 bk16 s4 minb2", 128, 128, 16, 16, 8, 128, 4, 2, false, true);
  V("R F+ffma2 256x128 t256 16x8 bk16 s4 minb1", 256, 128, 16, 16, 8, 256, 4, 1, false, true);
  V("S E+ffma2 128x128 t128 8x16 bk16 s4 minb2", 128, 128, 16, 8, 16, 128, 4, 2, false, true);
  V("T I+ffma2 128x256 t256 8x16 bk16 s3 minb1", 128, 256, 16, 8, 16, 256, 3, 1, false, true);
  V("U 128x64 t128 8x8 bk16 s4 minb3 ffma2", 128, 64, 16, 8, 8, 128, 4, 3, false, true);
  V("W 128x128 t256 8x8 bk8 s4 minb2 ffma2", 128, 128, 8, 8, 8, 256, 4, 2, false, true);
  V("X 128x128 t128 16x8 bk8 s6 minb2 ffma2", 128, 128, 8, 16, 8, 128, 6, 2, false, true);
  V("Y 128x128 t256 8x8 bk16 s3 minb2 db ffma2", 128, 128, 16, 8, 8, 256, 3, 2, true, true);
  V("Z1 128x64 t128 8x8 bk16 s3 minb2 ffma2", 128, 64, 16, 8, 8, 128, 3, 2, false, true);
  V("Z2 128x64 t128 8x8 bk16 s3 minb2 db ffma2", 128, 64, 16, 8, 8, 128, 3, 2, true, true);
  V("Z3 128x64 t128 8x8 bk8 s4 minb2 db ffma2", 128, 64, 8, 8, 8, 128, 4, 2, true, true);
  V("Z4 128x128 t128 16x8 bk8 s6 minb2 db ffma2", 128, 128, 8, 16, 8, 128, 6, 2, true, true);
  V("Z5 128x256 t256 8x16 bk16 s3 minb1 db ffma2", 128, 256, 16, 8, 16, 256, 3, 1, true, true);
  V("Z6 128x128 t128 8x16 bk8 s6 minb2 ffma2", 128, 128, 8, 8, 16, 128, 6, 2, false, true);
  V("Z7 128x256 t256 8x16 bk8 s4 minb1 ffma2", 128, 256, 8, 8, 16, 256, 4, 1, false, true);
  V("Z8 64x128 t128 8x8 bk16 s3 minb2 ffma2", 64, 128, 16, 8, 8, 128, 3, 2, false, true);
  V("Z9 128x128 t128 16x8 bk16 s3 minb2 ffma2", 128, 128, 16, 16, 8, 128, 3, 2, false, true);
  V("Y10 64x128 t128 8x8 bk8 s4 minb3 ffma2", 64, 128, 8, 8, 8, 128, 4, 3, false, true);
  V("Y11 64x128 t128 8x8 bk16 s4 minb3 ffma2", 64, 128, 16, 8, 8, 128, 4, 3, false, true);
  V("Y12 64x128 t128 8x8 bk16 s3 minb2 db ffma2", 64, 128, 16, 8, 8, 128, 3, 2, true, true);
  V("Y13 64x256 t256 8x8 bk16 s3 minb2 ffma2", 64, 256, 16, 8, 8, 256, 3, 2, false, true);
  V("Y14 128x128 t256 8x8 bk16 s3 minb1 ffma2", 128, 128, 16, 8, 8, 256, 3, 1, false, true);
  V("Y15 64x128 t128 8x8 bk32 s3 minb3 ffma2", 64, 128, 32, 8, 8, 128, 3, 3, false, true);
  V("Y16 64x64 t64 8x8 bk16 s3 minb6 ffma2", 64, 64, 16, 8, 8, 64, 3, 6, false, true);
#define VK(name, ...) if (!*only || strstr(name, only)) run_kacp<__VA_ARGS__>(name, n)
  VK("K1 acp 64x128 t128 bk16 s3 minb3", 64, 128, 16, 128, 3, 3);
  VK("K2 acp 64x128 t128 bk16 s4 minb3", 64, 128, 16, 128, 4, 3);
  VK("K3 acp 64x128 t128 bk32 s3 minb2", 64, 128, 32, 128, 3, 2);
  VK("K4 acp 128x128 t256 bk16 s3 minb2", 128, 128, 16, 256, 3, 2);
  VK("K5 acp 128x128 t256 bk16 s4 minb1", 128, 128, 16, 256, 4, 1);
  VK("K6 acp 128x64 t128 bk16 s4 minb2", 128, 64, 16, 128, 4, 2);
  VK("K7 acp 64x128 t128 bk8 s6 minb3", 64, 128, 8, 128, 6, 3);
  return 0;
}
