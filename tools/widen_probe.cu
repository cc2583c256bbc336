// widen_probe.cu -- f16 / f32 -> f64 widening throughput inside an HBM-bound
// mat-vec-like loop (the tile kernel's inner statement: acc = fma(widen(a), x, acc)).
// Variants: 0 cvt.f64.f16 (F2F.F64.F16), 1 cvt.f32.f16 + cvt.f64.f32, 2 HADD2.F32 +
// integer re-bias (no F2F), 3 f32 compute (reference), 4 f32 source cvt.f64.f32,
// 5 f32 source integer re-bias.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/widen_probe tools/widen_probe.cu
#include <cuda_fp16.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <vector>

__device__ __forceinline__ float h2f(uint16_t h) { float f; asm("cvt.f32.f16 %0, %1;" : "=f"(f) : "h"(h)); return f; }
__device__ __forceinline__ double f2d_int(float f) {
  const uint32_t u = __float_as_uint(f), e = (u >> 23) & 0xFFu, s = u & 0x80000000u;
  uint32_t hi = s | ((e + 896u) << 20) | ((u & 0x7FFFFFu) >> 3);
  hi = e == 0 ? s : (e == 0xFFu ? (s | 0x7FF00000u | ((u & 0x7FFFFFu) >> 3)) : hi);
  const uint32_t lo = e == 0 ? 0u : (u << 29);
  return __hiloint2double((int)hi, (int)lo);
}
template <int V>
__device__ __forceinline__ double wid(uint16_t h) {
  if (V == 0) { double d; asm("cvt.f64.f16 %0, %1;" : "=d"(d) : "h"(h)); return d; }
  if (V == 1) return (double)h2f(h);
  return f2d_int(h2f(h));
}
template <int V>
__global__ void __launch_bounds__(256) k16(const uint4 *__restrict__ a, size_t n16, double x, double *out) {
  double acc0 = 0, acc1 = 0;
  float facc0 = 0, facc1 = 0;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v = __ldg(a + i);
    const uint16_t *h = reinterpret_cast<const uint16_t *>(&v);
#pragma unroll
    for (int k = 0; k < 8; k += 2) {
      if (V == 3) {
        facc0 = __fmaf_rn(h2f(h[k]), (float)x, facc0);
        facc1 = __fmaf_rn(h2f(h[k + 1]), (float)x, facc1);
      } else {
        acc0 = __fma_rn(wid<V>(h[k]), x, acc0);
        acc1 = __fma_rn(wid<V>(h[k + 1]), x, acc1);
      }
    }
  }
  if (acc0 + acc1 + facc0 + facc1 == 12345.0) out[0] = acc0;
}
template <int V>
__global__ void __launch_bounds__(256) k32(const uint4 *__restrict__ a, size_t n16, double x, double *out) {
  double acc0 = 0, acc1 = 0;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v = __ldg(a + i);
    const float *f = reinterpret_cast<const float *>(&v);
#pragma unroll
    for (int k = 0; k < 4; k += 2) {
      if (V == 4) {
        acc0 = __fma_rn((double)f[k], x, acc0);
        acc1 = __fma_rn((double)f[k + 1], x, acc1);
      } else {
        acc0 = __fma_rn(f2d_int(f[k]), x, acc0);
        acc1 = __fma_rn(f2d_int(f[k + 1]), x, acc1);
      }
    }
  }
  if (acc0 + acc1 == 12345.0) out[0] = acc0;
}
template <class F> float tm(F f) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  std::vector<float> ts;
  for (int r = 0; r < 8; r++) {
    cudaEventRecord(a);
    f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (r > 1) ts.push_back(ms);
  }
  std::sort(ts.begin(), ts.end());
  return ts[ts.size() / 2];
}
int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t bytes = (size_t)1 << 29;   // 512 MiB (16384^2 f16)
  void *a;
  double *o;
  cudaMalloc(&a, bytes);
  cudaMalloc(&o, 8);
  cudaMemset(a, 0x3c, bytes);
  const size_t n16 = bytes / 16;
  for (int bps : {4, 8}) {
    unsigned g = sms * bps;
    printf("bps %d  f16 src 512MiB: cvt.f64.f16 %.1f us | cvt.f32+cvt.f64 %.1f us | hadd2+int %.1f us | f32 compute %.1f us\n",
           bps, 1e3 * tm([&] { k16<0><<<g, 256>>>((const uint4 *)a, n16, 1.5, o); }),
           1e3 * tm([&] { k16<1><<<g, 256>>>((const uint4 *)a, n16, 1.5, o); }),
           1e3 * tm([&] { k16<2><<<g, 256>>>((const uint4 *)a, n16, 1.5, o); }),
           1e3 * tm([&] { k16<3><<<g, 256>>>((const uint4 *)a, n16, 1.5, o); }));
    printf("bps %d  f32 src 512MiB: cvt.f64.f32 %.1f us | int %.1f us\n", bps,
           1e3 * tm([&] { k32<4><<<g, 256>>>((const uint4 *)a, n16, 1.5, o); }),
           1e3 * tm([&] { k32<5><<<g, 256>>>((const uint4 *)a, n16, 1.5, o); }));
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
