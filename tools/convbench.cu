// convbench.cu -- design-space probe for the a2 conversion kernel (not part of
// the library): f32->f16 and f16->f32 over 1 GiB of source, variants of
// unroll depth U, blocks per SM, load/store cache hints and a TMA-free
// "contiguous chunk per CTA" layout.  Prints GB/s (n * (s_src + s_dst) / t).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o convbench tools/convbench.cu
#include <cuda_fp16.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>

__device__ __forceinline__ uint4 ld_na(const uint4 *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint4 ld_pf(const uint4 *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ void st_cs(uint2 *p, uint2 v) {
  asm volatile("st.global.cs.v2.u32 [%0], {%1,%2};" :: "l"(p), "r"(v.x), "r"(v.y));
}
__device__ __forceinline__ void st_cs4(uint4 *p, uint4 v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w));
}
__device__ __forceinline__ uint32_t pack2(float a, float b) {
  uint16_t x, y;
  asm("cvt.rn.f16.f32 %0, %1;" : "=h"(x) : "f"(a));
  asm("cvt.rn.f16.f32 %0, %1;" : "=h"(y) : "f"(b));
  x = (a != a) ? 0x7FFF : x;
  y = (b != b) ? 0x7FFF : y;
  return (uint32_t)x | ((uint32_t)y << 16);
}

// grid-stride, unit = 4 floats -> 4 halves
template <int U, int HINT>
__global__ void __launch_bounds__(256) k_f32_f16(const uint4 *__restrict__ s, uint2 *__restrict__ d, size_t units) {
  size_t stride = (size_t)gridDim.x * blockDim.x, g = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; g + (U - 1) * stride < units; g += U * stride) {
    uint4 in[U];
#pragma unroll
    for (int u = 0; u < U; u++) in[u] = HINT == 1 ? ld_pf(s + g + u * stride) : ld_na(s + g + u * stride);
#pragma unroll
    for (int u = 0; u < U; u++) {
      uint2 o;
      o.x = pack2(__uint_as_float(in[u].x), __uint_as_float(in[u].y));
      o.y = pack2(__uint_as_float(in[u].z), __uint_as_float(in[u].w));
      if (HINT == 2) st_cs(d + g + u * stride, o); else d[g + u * stride] = o;
    }
  }
  for (; g < units; g += stride) {
    uint4 in = ld_na(s + g);
    uint2 o;
    o.x = pack2(__uint_as_float(in.x), __uint_as_float(in.y));
    o.y = pack2(__uint_as_float(in.z), __uint_as_float(in.w));
    d[g] = o;
  }
}

// contiguous: each block owns a contiguous range; unit = 8 floats (2 x 16B) -> 16B of halves
template <int U>
__global__ void __launch_bounds__(256) k_f32_f16_blk(const uint4 *__restrict__ s, uint4 *__restrict__ d, size_t units) {
  size_t per = (units + gridDim.x - 1) / gridDim.x;
  size_t b0 = (size_t)blockIdx.x * per, b1 = min(units, b0 + per);
  for (size_t g = b0 + threadIdx.x; g < b1; g += (size_t)U * 256) {
    uint4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      size_t q = g + (size_t)u * 256;
      if (q < b1) { a[u] = ld_na(s + 2 * q); b[u] = ld_na(s + 2 * q + 1); }
    }
#pragma unroll
    for (int u = 0; u < U; u++) {
      size_t q = g + (size_t)u * 256;
      if (q < b1) {
        uint4 o;
        o.x = pack2(__uint_as_float(a[u].x), __uint_as_float(a[u].y));
        o.y = pack2(__uint_as_float(a[u].z), __uint_as_float(a[u].w));
        o.z = pack2(__uint_as_float(b[u].x), __uint_as_float(b[u].y));
        o.w = pack2(__uint_as_float(b[u].z), __uint_as_float(b[u].w));
        d[q] = o;
      }
    }
  }
}

// f16 -> f32, unit = 8 halves (16B) -> 32B
template <int U, int HINT>
__global__ void __launch_bounds__(256) k_f16_f32(const uint4 *__restrict__ s, uint4 *__restrict__ d, size_t units) {
  size_t stride = (size_t)gridDim.x * blockDim.x, g = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; g < units; g += U * stride) {
    uint4 in[U];
#pragma unroll
    for (int u = 0; u < U; u++) if (g + u * stride < units) in[u] = ld_na(s + g + u * stride);
#pragma unroll
    for (int u = 0; u < U; u++) {
      if (g + u * stride >= units) break;
      const __half2 *h = reinterpret_cast<const __half2 *>(&in[u]);
      float2 f0 = __half22float2(h[0]), f1 = __half22float2(h[1]), f2 = __half22float2(h[2]), f3 = __half22float2(h[3]);
      uint4 o0 = make_uint4(__float_as_uint(f0.x), __float_as_uint(f0.y), __float_as_uint(f1.x), __float_as_uint(f1.y));
      uint4 o1 = make_uint4(__float_as_uint(f2.x), __float_as_uint(f2.y), __float_as_uint(f3.x), __float_as_uint(f3.y));
      if (HINT == 2) { st_cs4(d + 2 * (g + u * stride), o0); st_cs4(d + 2 * (g + u * stride) + 1, o1); }
      else { d[2 * (g + u * stride)] = o0; d[2 * (g + u * stride) + 1] = o1; }
    }
  }
}

// plain copy for reference (1 GiB read + 1 GiB write)
template <int U>
__global__ void __launch_bounds__(256) k_copy(const uint4 *__restrict__ s, uint4 *__restrict__ d, size_t units) {
  size_t stride = (size_t)gridDim.x * blockDim.x, g = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; g < units; g += U * stride) {
    uint4 in[U];
#pragma unroll
    for (int u = 0; u < U; u++) if (g + u * stride < units) in[u] = ld_na(s + g + u * stride);
#pragma unroll
    for (int u = 0; u < U; u++) if (g + u * stride < units) d[g + u * stride] = in[u];
  }
}

template <class F>
float timeit(F f) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  std::vector<float> ts;
  for (int r = 0; r < 13; r++) {
    cudaEventRecord(a);
    f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (r >= 3) ts.push_back(ms);
  }
  std::sort(ts.begin(), ts.end());
  return ts[ts.size() / 2];
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t n = (size_t)1 << 28;   // floats: 1 GiB source
  void *src, *dst;
  cudaMalloc(&src, n * 4);
  cudaMalloc(&dst, n * 4);
  cudaMemset(src, 0, n * 4);
  const double bytes16 = n * 6.0;
  auto rep = [&](const char *name, float ms, double bytes) { printf("%-40s %8.3f ms %8.1f GB/s\n", name, ms, bytes / (ms * 1e-3) / 1e9); };
  for (int bps : {4, 8, 16, 32}) {
    unsigned grid = sms * bps;
    char nm[64];
#define RUN(U, H) { snprintf(nm, 64, "f32->f16 U=%d hint=%d bps=%d", U, H, bps); \
      rep(nm, timeit([&] { k_f32_f16<U, H><<<grid, 256>>>((const uint4 *)src, (uint2 *)dst, n / 4); }), bytes16); }
    RUN(4, 0) RUN(8, 0) RUN(4, 1) RUN(4, 2) RUN(8, 2)
    snprintf(nm, 64, "f32->f16 blk U=4 bps=%d", bps);
    rep(nm, timeit([&] { k_f32_f16_blk<4><<<grid, 256>>>((const uint4 *)src, (uint4 *)dst, n / 8); }), bytes16);
    snprintf(nm, 64, "f16->f32 U=4 bps=%d", bps);
    rep(nm, timeit([&] { k_f16_f32<4, 0><<<grid, 256>>>((const uint4 *)src, (uint4 *)dst, n / 16); }), n / 2 * 6.0);
    snprintf(nm, 64, "f16->f32 U=4 cs bps=%d", bps);
    rep(nm, timeit([&] { k_f16_f32<4, 2><<<grid, 256>>>((const uint4 *)src, (uint4 *)dst, n / 16); }), n / 2 * 6.0);
    snprintf(nm, 64, "copy U=4 bps=%d (1GiB)", bps);
    rep(nm, timeit([&] { k_copy<4><<<grid, 256>>>((const uint4 *)src, (uint4 *)dst, n / 4); }), n * 8.0);
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
