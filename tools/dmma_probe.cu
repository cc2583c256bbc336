// dmma_probe.cu -- does the fp64 tensor-core MMA (mma.sync ... .f64) reproduce
// reading R3's fma chain (acc <- fma(a_k, b_k, acc), k ascending) bit-exactly,
// and how fast is it on this B200 next to DFMA?  Standalone probe, not product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/dmma_probe tools/dmma_probe.cu
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  printf("CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); exit(1); } } while (0)

// ---- semantics: one m8n8k4 per warp; A row-major 8x4, B col 4x8, C/D 8x8 row-major
__global__ void mma_m8n8k4(const double *A, const double *B, const double *C, double *D, int trials) {
  int lane = threadIdx.x & 31, w = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  if (w >= trials) return;
  A += w * 32; B += w * 32; C += w * 64; D += w * 64;
  int r = lane >> 2, q = lane & 3;
  double a = A[r * 4 + q];          // A[r][k=q]
  double b = B[q * 8 + r];          // B[k=q][n=r]
  double c0 = C[r * 8 + q * 2], c1 = C[r * 8 + q * 2 + 1], d0, d1;
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%4,%5};"
               : "=d"(d0), "=d"(d1) : "d"(a), "d"(b), "d"(c0), "d"(c1));
  D[r * 8 + q * 2] = d0;
  D[r * 8 + q * 2 + 1] = d1;
}

// m16n8k4: A 16x4 row, B 4x8 col, C/D 16x8
__global__ void mma_m16n8k4(const double *A, const double *B, const double *C, double *D, int trials) {
  int lane = threadIdx.x & 31, w = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  if (w >= trials) return;
  A += w * 64; B += w * 32; C += w * 128; D += w * 128;
  int g = lane >> 2, t = lane & 3;
  double a0 = A[g * 4 + t], a1 = A[(g + 8) * 4 + t];
  double b0 = B[t * 8 + g];
  double c[4] = {C[g * 8 + 2 * t], C[g * 8 + 2 * t + 1], C[(g + 8) * 8 + 2 * t], C[(g + 8) * 8 + 2 * t + 1]};
  double d[4];
  asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%7,%8,%9,%10};"
               : "=d"(d[0]), "=d"(d[1]), "=d"(d[2]), "=d"(d[3])
               : "d"(a0), "d"(a1), "d"(b0), "d"(c[0]), "d"(c[1]), "d"(c[2]), "d"(c[3]));
  D[g * 8 + 2 * t] = d[0]; D[g * 8 + 2 * t + 1] = d[1];
  D[(g + 8) * 8 + 2 * t] = d[2]; D[(g + 8) * 8 + 2 * t + 1] = d[3];
}

// m16n8k16: A 16x16 row, B 16x8 col, C/D 16x8
__global__ void mma_m16n8k16(const double *A, const double *B, const double *C, double *D, int trials) {
  int lane = threadIdx.x & 31, w = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  if (w >= trials) return;
  A += w * 256; B += w * 128; C += w * 128; D += w * 128;
  int g = lane >> 2, t = lane & 3;
  double a[8], b[4];
  // a_i: row g + 8*(i&1), col t + 4*(i>>1)
  for (int i = 0; i < 8; i++) a[i] = A[(g + 8 * (i & 1)) * 16 + t + 4 * (i >> 1)];
  // b_i: row(k) t + 4*i, col g
  for (int i = 0; i < 4; i++) b[i] = B[(t + 4 * i) * 8 + g];
  double c[4] = {C[g * 8 + 2 * t], C[g * 8 + 2 * t + 1], C[(g + 8) * 8 + 2 * t], C[(g + 8) * 8 + 2 * t + 1]};
  double d[4];
  asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, "
               "{%12,%13,%14,%15}, {%16,%17,%18,%19};"
               : "=d"(d[0]), "=d"(d[1]), "=d"(d[2]), "=d"(d[3])
               : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                 "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]), "d"(c[0]), "d"(c[1]), "d"(c[2]), "d"(c[3]));
  D[g * 8 + 2 * t] = d[0]; D[g * 8 + 2 * t + 1] = d[1];
  D[(g + 8) * 8 + 2 * t] = d[2]; D[(g + 8) * 8 + 2 * t + 1] = d[3];
}

// ---- throughput
template <int KIND>
__global__ void __launch_bounds__(256) tput(double *out, int iters, double s) {
  double a = s + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-12;
  double acc[16];
#pragma unroll
  for (int i = 0; i < 16; i++) acc[i] = i * 1e-3;
  for (int it = 0; it < iters; it++) {
    if (KIND == 0) {   // DFMA: 16 independent chains
#pragma unroll
      for (int i = 0; i < 16; i++) acc[i] = fma(a, b, acc[i]);
    } else if (KIND == 1) {   // m8n8k4: 8 independent accumulators (2 doubles each)
#pragma unroll
      for (int i = 0; i < 8; i++)
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                     : "+d"(acc[2 * i]), "+d"(acc[2 * i + 1]) : "d"(a), "d"(b));
    } else if (KIND == 2) {   // m16n8k4: 4 accumulators (4 doubles each)
#pragma unroll
      for (int i = 0; i < 4; i++)
        asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                     : "+d"(acc[4 * i]), "+d"(acc[4 * i + 1]), "+d"(acc[4 * i + 2]), "+d"(acc[4 * i + 3])
                     : "d"(a), "d"(b), "d"(b));
    } else {   // m16n8k16
#pragma unroll
      for (int i = 0; i < 4; i++)
        asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%4,%4,%4,%5,%5,%5,%5}, "
                     "{%5,%5,%5,%5}, {%0,%1,%2,%3};"
                     : "+d"(acc[4 * i]), "+d"(acc[4 * i + 1]), "+d"(acc[4 * i + 2]), "+d"(acc[4 * i + 3])
                     : "d"(a), "d"(b));
    }
  }
  double t = 0;
#pragma unroll
  for (int i = 0; i < 16; i++) t += acc[i];
  if (t == 12345.678) out[0] = t;
}

static uint64_t sm = 0x9E3779B97F4A7C15ull;
static uint64_t nxt() {
  uint64_t z = (sm += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static double rnd(int mode) {
  double u = (nxt() >> 11) * 0x1.0p-53;
  double s = (nxt() & 1) ? -1.0 : 1.0;
  if (mode == 0) return s * u;                                   // U(-1,1)
  if (mode == 1) return s * ldexp(0.5 + u / 2, (int)(nxt() % 41) - 20);   // wide exponents
  if (mode == 2) return (nxt() % 5 == 0) ? 0.0 * s : s * ldexp(0.5 + u / 2, (int)(nxt() % 7) - 3);
  if (mode == 3) return s * ldexp(1.0 + u, (int)(nxt() % 3));    // cancellation-heavy
  // mode 4: subnormal products/sums, signed zeros, infinities, NaN
  uint64_t sel = nxt() % 16;
  if (sel == 0) return s * 0.0;
  if (sel == 1) return s * INFINITY;
  if (sel == 2) return NAN;
  if (sel < 8) return s * ldexp(0.5 + u / 2, -1000 - (int)(nxt() % 70));
  return s * ldexp(0.5 + u / 2, -30 - (int)(nxt() % 20));
}

static bool same(double x, double y) { if (x != x && y != y) return true; uint64_t a, b; memcpy(&a, &x, 8); memcpy(&b, &y, 8); return a == b; }

// host models for one output: K products (a_k, b_k) and c
static double chain_asc(const double *a, const double *b, int K, double c) {
  double r = c; for (int k = 0; k < K; k++) r = fma(a[k], b[k], r); return r;
}
static double chain_desc(const double *a, const double *b, int K, double c) {
  double r = c; for (int k = K - 1; k >= 0; k--) r = fma(a[k], b[k], r); return r;
}
static double chain_from0_then_c(const double *a, const double *b, int K, double c) {
  double r = 0; for (int k = 0; k < K; k++) r = fma(a[k], b[k], r); return r + c;
}

template <int KK>
static void run_sem(const char *name, int M, int N, int trials, int mode,
                    void (*kern)(const double *, const double *, const double *, double *, int)) {
  size_t na = (size_t)trials * M * KK, nb = (size_t)trials * KK * N, nc = (size_t)trials * M * N;
  double *hA = (double *)malloc(na * 8), *hB = (double *)malloc(nb * 8), *hC = (double *)malloc(nc * 8),
         *hD = (double *)malloc(nc * 8);
  for (size_t i = 0; i < na; i++) hA[i] = rnd(mode);
  for (size_t i = 0; i < nb; i++) hB[i] = rnd(mode);
  for (size_t i = 0; i < nc; i++) hC[i] = (mode == 2 && (i & 3) == 0) ? 0.0 : rnd(mode);
  double *dA, *dB, *dC, *dD;
  CK(cudaMalloc(&dA, na * 8)); CK(cudaMalloc(&dB, nb * 8)); CK(cudaMalloc(&dC, nc * 8)); CK(cudaMalloc(&dD, nc * 8));
  CK(cudaMemcpy(dA, hA, na * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, hB, nb * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dC, hC, nc * 8, cudaMemcpyHostToDevice));
  kern<<<(trials + 7) / 8, 256>>>(dA, dB, dC, dD, trials);
  CK(cudaGetLastError());
  CK(cudaMemcpy(hD, dD, nc * 8, cudaMemcpyDeviceToHost));
  long m_asc = 0, m_desc = 0, m_0c = 0, total = 0, differ = 0;
  for (int t = 0; t < trials; t++)
    for (int i = 0; i < M; i++)
      for (int j = 0; j < N; j++) {
        double a[KK], b[KK];
        for (int k = 0; k < KK; k++) { a[k] = hA[(size_t)t * M * KK + i * KK + k]; b[k] = hB[(size_t)t * KK * N + k * N + j]; }
        double c = hC[(size_t)t * M * N + i * N + j], d = hD[(size_t)t * M * N + i * N + j];
        double x = chain_asc(a, b, KK, c), y = chain_desc(a, b, KK, c), z = chain_from0_then_c(a, b, KK, c);
        m_asc += same(d, x); m_desc += same(d, y); m_0c += same(d, z);
        differ += !same(x, y);
        total++;
      }
  printf("%-10s mode %d: %ld outputs, R3 chain (c first, k asc) matches %ld, k desc %ld, (chain from 0)+c %ld; "
         "asc!=desc on %ld\n", name, mode, total, m_asc, m_desc, m_0c, differ);
  cudaFree(dA); cudaFree(dB); cudaFree(dC); cudaFree(dD);
  free(hA); free(hB); free(hC); free(hD);
}

int main() {
  for (int mode = 0; mode < 5; mode++) {
    run_sem<4>("m8n8k4", 8, 8, 1 << 16, mode, mma_m8n8k4);
    run_sem<4>("m16n8k4", 16, 8, 1 << 15, mode, mma_m16n8k4);
    run_sem<16>("m16n8k16", 16, 8, 1 << 15, mode, mma_m16n8k16);
  }
  int nsm; CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  double *out; CK(cudaMalloc(&out, 8));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int iters = 20000;
  const char *names[4] = {"DFMA", "DMMA m8n8k4", "DMMA m16n8k4", "DMMA m16n8k16"};
  // flops per thread per iteration: DFMA 16*2; m8n8k4: 8 mma * 2*8*8*4 / 32 lanes; m16n8k4: 4*2*16*8*4/32; k16: 4*2*16*8*16/32
  const double fl[4] = {32, 8 * 512.0 / 32, 4 * 1024.0 / 32, 4 * 4096.0 / 32};
  for (int kind = 0; kind < 4; kind++)
    for (int bps = 1; bps <= 4; bps *= 2) {
      dim3 g(nsm * bps);
      for (int rep = 0; rep < 2; rep++) {
        cudaEventRecord(e0);
        if (kind == 0) tput<0><<<g, 256>>>(out, iters, 1.0);
        if (kind == 1) tput<1><<<g, 256>>>(out, iters, 1.0);
        if (kind == 2) tput<2><<<g, 256>>>(out, iters, 1.0);
        if (kind == 3) tput<3><<<g, 256>>>(out, iters, 1.0);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep) printf("%-14s %d CTA/SM x 256 thr: %.2f TFLOP/s\n", names[kind], bps,
                        fl[kind] * iters * 256.0 * g.x / (ms * 1e-3) / 1e12);
      }
    }
  return 0;
}
