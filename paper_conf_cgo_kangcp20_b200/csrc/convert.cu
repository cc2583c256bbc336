// convert.cu -- device-side type conversion of a memory object (row a2;
// Fig. 3c "parallelized type conversion on GPU side") and the
// ps_convert C entry point.
//
// HBM-bound: per element s_src + s_dst bytes, zero flops.  Design:
//  * every thread moves one "unit" of E = 16 / max(s_src, s_dst) elements:
//    one 16-byte access on the wide side, one 4/8/16-byte access on the narrow
//    side, so every warp instruction is fully coalesced on both sides;
//  * U units per thread are issued back to back (loads first) for memory-level
//    parallelism; grid = a multiple of the SM count, grid-stride loop;
//  * loads use ld.global.nc.L1::no_allocate (streamed once), stores keep L2
//    allocation so a converted object that fits in L2 feeds the next kernel;
//  * a scalar head/tail handles unaligned pointers and ragged n.
#include <cstring>

#include "common.cuh"
#include "kernels.cuh"

namespace ps {

// ---------------------------------------------------- element conversion
template <class S, class D> struct Cvt;
template <> struct Cvt<float, F16> {
  static __device__ __forceinline__ uint16_t f(float x) { return rne_f16(x); }
};
template <> struct Cvt<double, F16> {
  static __device__ __forceinline__ uint16_t f(double x) { return rne_f16(x); }
};
template <> struct Cvt<double, float> {
  static __device__ __forceinline__ float f(double x) { return rne_f32(x); }
};
template <> struct Cvt<F16, float> {
  static __device__ __forceinline__ float f(uint16_t h) { return canon_f32(f16_to_f32(h)); }
};
template <> struct Cvt<F16, double> {
  static __device__ __forceinline__ double f(uint16_t h) { return canon_f64(f16_to_f64(h)); }
};
template <> struct Cvt<float, double> {
  static __device__ __forceinline__ double f(float x) { return canon_f64((double)x); }
};
// bf16 (reading #28): one RNE rounding from any wider format; widening is exact
template <> struct Cvt<float, BF16> {
  static __device__ __forceinline__ uint16_t f(float x) { return rne_bf16(x); }
};
template <> struct Cvt<double, BF16> {
  static __device__ __forceinline__ uint16_t f(double x) { return rne_bf16(x); }
};
template <> struct Cvt<F16, BF16> {   // f16 -> f32 is exact, so one rounding
  static __device__ __forceinline__ uint16_t f(uint16_t h) { return rne_bf16(f16_to_f32(h)); }
};
template <> struct Cvt<BF16, float> {
  static __device__ __forceinline__ float f(uint16_t h) { return canon_f32(bf16_to_f32(h)); }
};
template <> struct Cvt<BF16, double> {
  static __device__ __forceinline__ double f(uint16_t h) { return canon_f64((double)bf16_to_f32(h)); }
};
template <> struct Cvt<BF16, F16> {   // bf16 -> f32 is exact, so one rounding
  static __device__ __forceinline__ uint16_t f(uint16_t h) { return rne_f16(bf16_to_f32(h)); }
};

// ------------------------------------------------------- vector helpers
template <int B> struct Vec;
template <> struct Vec<16> { using t = uint4; };
template <> struct Vec<8> { using t = uint2; };
template <> struct Vec<4> { using t = uint32_t; };

__device__ __forceinline__ uint4 ld_stream(const uint4 *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint2 ld_stream(const uint2 *p) {
  uint2 r;
  asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t ld_stream(const uint32_t *p) {
  uint32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}

template <class S, class D>
struct Unit {
  using RS = raw_t<S>;
  using RD = raw_t<D>;
  static constexpr int SS = sizeof(RS), DS = sizeof(RD);
  static constexpr int E = 16 / (SS > DS ? SS : DS);
  using VS = typename Vec<E * SS>::t;
  using VD = typename Vec<E * DS>::t;
};

template <class S, class D, int U>
__global__ void __launch_bounds__(256) convert_kernel(const raw_t<S> *__restrict__ src,
                                                     raw_t<D> *__restrict__ dst, size_t n,
                                                     size_t head, size_t nunits) {
  using UT = Unit<S, D>;
  constexpr int E = UT::E;
  using VS = typename UT::VS;
  using VD = typename UT::VD;
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  const VS *s = reinterpret_cast<const VS *>(src + head);
  VD *d = reinterpret_cast<VD *>(dst + head);

  size_t g = tid;
  for (; g + (size_t)(U - 1) * stride < nunits; g += (size_t)U * stride) {
    union { VS v; raw_t<S> e[E]; } in[U];
#pragma unroll
    for (int u = 0; u < U; u++) in[u].v = ld_stream(s + g + (size_t)u * stride);
#pragma unroll
    for (int u = 0; u < U; u++) {
      union { VD v; raw_t<D> e[E]; } out;
#pragma unroll
      for (int k = 0; k < E; k++) out.e[k] = Cvt<S, D>::f(in[u].e[k]);
      d[g + (size_t)u * stride] = out.v;
    }
  }
  for (; g < nunits; g += stride) {
    union { VS v; raw_t<S> e[E]; } in;
    union { VD v; raw_t<D> e[E]; } out;
    in.v = ld_stream(s + g);
#pragma unroll
    for (int k = 0; k < E; k++) out.e[k] = Cvt<S, D>::f(in.e[k]);
    d[g] = out.v;
  }
  // scalar head [0, head) and tail [head + nunits*E, n)
  const size_t tail0 = head + nunits * E;
  if (tid < head) dst[tid] = Cvt<S, D>::f(src[tid]);
  if (tid < n - tail0) dst[tail0 + tid] = Cvt<S, D>::f(src[tail0 + tid]);
}

template <class S, class D>
static ps_status launch_convert(const void *src, void *dst, size_t n, cudaStream_t st) {
  using UT = Unit<S, D>;
  constexpr int E = UT::E;
  const uintptr_t sa = (uintptr_t)src, da = (uintptr_t)dst;
  size_t head = n;   // "no vector path"
  for (size_t h = 0; h < (size_t)E && h <= n; h++) {
    if ((sa + h * UT::SS) % (E * UT::SS) == 0 && (da + h * UT::DS) % (E * UT::DS) == 0) {
      head = h;
      break;
    }
  }
  size_t nunits = 0;
  if (head < n) nunits = (n - head) / E;
  else head = 0;   // scalar only: handled as "tail" below with nunits = 0
  const size_t scalar_max = head > (n - head - nunits * E) ? head : (n - head - nunits * E);
  constexpr int U = 4;
  const size_t threads = 256;
  size_t want = (nunits + U - 1) / U;
  if (want < scalar_max) want = scalar_max;
  size_t blocks = (want + threads - 1) / threads;
  const size_t cap = (size_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  if (blocks == 0) blocks = 1;
  // scalar parts must fit in one pass of the grid
  if (blocks * threads < scalar_max) blocks = (scalar_max + threads - 1) / threads;
  convert_kernel<S, D, U><<<(unsigned)blocks, (unsigned)threads, 0, st>>>(
      (const raw_t<S> *)src, (raw_t<D> *)dst, n, head, nunits);
  PS_CHECK_LAUNCH("convert_kernel");
  return PS_OK;
}

ps_status convert_async(const void *src, int st, void *dst, int dt, size_t n, cudaStream_t stream) {
  if (n == 0) return PS_OK;
  if (st == dt) {
    PS_CUDA(cudaMemcpyAsync(dst, src, n * dtype_size(st), cudaMemcpyDeviceToDevice, stream));
    return PS_OK;
  }
  if (is_fp8(st) && is_fp8(dt)) {
    set_error("ps_convert: e4m3 <-> e5m2 is not supported");
    return PS_ERR_UNSUPPORTED;
  }
  if (is_fp8(dt)) return fp8_encode_async(src, st, dst, dt, n, nullptr, stream);   // unscaled
  if (is_fp8(st)) return fp8_decode_async(src, st, dst, dt, n, nullptr, stream);
  if (st == PS_F32 && dt == PS_F16) return launch_convert<float, F16>(src, dst, n, stream);
  if (st == PS_F64 && dt == PS_F16) return launch_convert<double, F16>(src, dst, n, stream);
  if (st == PS_F64 && dt == PS_F32) return launch_convert<double, float>(src, dst, n, stream);
  if (st == PS_F16 && dt == PS_F32) return launch_convert<F16, float>(src, dst, n, stream);
  if (st == PS_F16 && dt == PS_F64) return launch_convert<F16, double>(src, dst, n, stream);
  if (st == PS_F32 && dt == PS_F64) return launch_convert<float, double>(src, dst, n, stream);
  if (st == PS_F32 && dt == PS_BF16) return launch_convert<float, BF16>(src, dst, n, stream);
  if (st == PS_F64 && dt == PS_BF16) return launch_convert<double, BF16>(src, dst, n, stream);
  if (st == PS_F16 && dt == PS_BF16) return launch_convert<F16, BF16>(src, dst, n, stream);
  if (st == PS_BF16 && dt == PS_F32) return launch_convert<BF16, float>(src, dst, n, stream);
  if (st == PS_BF16 && dt == PS_F64) return launch_convert<BF16, double>(src, dst, n, stream);
  if (st == PS_BF16 && dt == PS_F16) return launch_convert<BF16, F16>(src, dst, n, stream);
  set_error("ps_convert: bad dtype pair %d->%d", st, dt);
  return PS_ERR_INVALID;
}

}  // namespace ps

extern "C" ps_status ps_convert(const void *src, int src_type, void *dst, int dst_type, size_t n,
                                void *stream) {
  using namespace ps;
  if (!dtype_ok(src_type) || !dtype_ok(dst_type)) {
    set_error("ps_convert: bad dtype code (%d, %d)", src_type, dst_type);
    return PS_ERR_INVALID;
  }
  if (n == 0) return PS_OK;
  if (!src || !dst) {
    set_error("ps_convert: null pointer");
    return PS_ERR_INVALID;
  }
  const uintptr_t s0 = (uintptr_t)src, s1 = s0 + n * dtype_size(src_type);
  const uintptr_t d0 = (uintptr_t)dst, d1 = d0 + n * dtype_size(dst_type);
  if (s0 < d1 && d0 < s1) {
    set_error("ps_convert: src and dst overlap");
    return PS_ERR_INVALID;
  }
  return convert_async(src, src_type, dst, dst_type, n, (cudaStream_t)stream);
}
