// fp8.cu -- fp8 memory objects with a per-tensor power-of-two scale (DESIGN.md
// reading #29; B200 tensor-core formats beyond the
// paper's fp16).  Row a2 for fp8 objects and the re-quantisation that
// ends every statement writing one:
//
//   fp8_amax_kernel    amax = max |x_i| over the finite elements (one read)
//   fp8_encode_kernel  k = smallest k in [-126, 126] with amax <= FMAX * 2^k,
//                      q_i = RNE_fp8(x_i * 2^-k)  (one read, n-byte write)
//   fp8_decode_kernel  value_i = RNE_D(q_i * 2^k)   (n-byte read, one write)
//
// All three are HBM-bound streaming kernels: 16 elements per thread-unit (one
// 16-byte access on the fp8 side, 16 * s bytes on the wide side), grid = a
// multiple of the SM count, grid-stride.  The scale multiply by 2^-k is exact
// in the source precision (the product only loses bits below 2^-126, far under
// half the smallest fp8 subnormal), so every code is ONE rounding of the exact
// product, as in the oracle.
#include <math.h>

#include "common.cuh"
#include "kernels.cuh"

namespace ps {

// value type a source element is widened to (exactly)
template <class S> struct Wide { using t = float; };
template <> struct Wide<double> { using t = double; };

template <class S, class W> __device__ __forceinline__ W wide_of(raw_t<S> r);
template <> __device__ __forceinline__ double wide_of<double, double>(double r) { return r; }
template <> __device__ __forceinline__ float wide_of<float, float>(float r) { return r; }
template <> __device__ __forceinline__ float wide_of<F16, float>(uint16_t r) { return f16_to_f32(r); }
template <> __device__ __forceinline__ float wide_of<BF16, float>(uint16_t r) { return bf16_to_f32(r); }

__device__ __forceinline__ float absw(float v) { return fabsf(v); }
__device__ __forceinline__ double absw(double v) { return fabs(v); }
__device__ __forceinline__ double pow2(int k) { return __longlong_as_double((long long)(k + 1023) << 52); }

// reading #29: the smallest k in [-126, 126] with amax <= FMAX * 2^k
__device__ __forceinline__ int fp8_scale_exp(double amax, bool e4m3) {
  const double fmax = e4m3 ? 448.0 : 57344.0;
  if (!(amax > 0.0)) return 0;
  int k = ilogb(amax) - ilogb(fmax);
  k = k < FP8_KMIN ? FP8_KMIN : (k > FP8_KMAX ? FP8_KMAX : k);
  while (k > FP8_KMIN && amax <= fmax * pow2(k - 1)) k--;
  while (k < FP8_KMAX && amax > fmax * pow2(k)) k++;
  return k;
}

constexpr int F8_THREADS = 256;
constexpr int F8_E = 16;   // elements per thread-unit

template <class S>
__global__ void __launch_bounds__(F8_THREADS) fp8_amax_kernel(const raw_t<S> *__restrict__ src, size_t n,
                                                             unsigned long long *__restrict__ amax_bits) {
  using W = typename Wide<S>::t;
  W m = (W)0;
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  const size_t nunits = ((uintptr_t)src % 16 == 0) ? n / F8_E : 0;
  constexpr int NV = F8_E * (int)sizeof(raw_t<S>) / 16;
  for (size_t g = tid; g < nunits; g += stride) {
    union { uint4 v[NV]; raw_t<S> e[F8_E]; } in;
    const uint4 *p = reinterpret_cast<const uint4 *>(src) + g * NV;
#pragma unroll
    for (int j = 0; j < NV; j++) in.v[j] = __ldg(p + j);
#pragma unroll
    for (int e = 0; e < F8_E; e++) {
      const W a = absw(wide_of<S, W>(in.e[e]));
      if (a > m && isfinite(a)) m = a;   // NaN compares false
    }
  }
  for (size_t i = nunits * F8_E + tid; i < n; i += stride) {
    const W a = absw(wide_of<S, W>(src[i]));
    if (a > m && isfinite(a)) m = a;
  }
  double md = (double)m;
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) {
    const double o = __shfl_xor_sync(0xffffffffu, md, off);
    md = o > md ? o : md;
  }
  __shared__ double s_m[F8_THREADS / 32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) s_m[warp] = md;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < F8_THREADS / 32; w++) md = s_m[w] > md ? s_m[w] : md;
    if (md > 0.0) atomicMax(amax_bits, (unsigned long long)__double_as_longlong(md));   // >= 0: bit order = value order
  }
}

template <class S, bool E4>
__global__ void __launch_bounds__(F8_THREADS) fp8_encode_kernel(const raw_t<S> *__restrict__ src,
                                                               uint8_t *__restrict__ dst, size_t n,
                                                               ps_fp8_scale *sc) {
  using W = typename Wide<S>::t;
  const int k = sc ? fp8_scale_exp(__longlong_as_double((long long)sc->amax_bits), E4) : 0;
  const W inv = (W)pow2(-k);   // exact power of two in W (|k| <= 126)
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  if (sc && tid == 0) sc->k = k;
  const bool vec = ((uintptr_t)src % 16 == 0) && ((uintptr_t)dst % 16 == 0);
  const size_t nunits = vec ? n / F8_E : 0;
  constexpr int NV = F8_E * (int)sizeof(raw_t<S>) / 16;
  for (size_t g = tid; g < nunits; g += stride) {
    union { uint4 v[NV]; raw_t<S> e[F8_E]; } in;
    union { uint4 v; uint8_t b[F8_E]; } out;
    const uint4 *p = reinterpret_cast<const uint4 *>(src) + g * NV;
#pragma unroll
    for (int j = 0; j < NV; j++) in.v[j] = __ldg(p + j);
#pragma unroll
    for (int e = 0; e < F8_E; e++) {
      const W y = wide_of<S, W>(in.e[e]) * inv;
      if constexpr (sizeof(W) == 8) out.b[e] = f64_to_fp8(y, E4);
      else out.b[e] = f32_to_fp8(y, E4);
    }
    reinterpret_cast<uint4 *>(dst)[g] = out.v;
  }
  for (size_t i = nunits * F8_E + tid; i < n; i += stride) {
    const W y = wide_of<S, W>(src[i]) * inv;
    if constexpr (sizeof(W) == 8) dst[i] = f64_to_fp8(y, E4);
    else dst[i] = f32_to_fp8(y, E4);
  }
}

template <class D> __device__ __forceinline__ raw_t<D> fp8_value(float v, int k);
template <> __device__ __forceinline__ double fp8_value<double>(float v, int k) {
  return canon_f64((double)v * pow2(k));                 // exact
}
template <> __device__ __forceinline__ float fp8_value<float>(float v, int k) {
  return canon_f32(v * (float)pow2(k));                  // one f32 rounding (overflow only)
}
template <> __device__ __forceinline__ uint16_t fp8_value<F16>(float v, int k) {
  return rne_f16((double)v * pow2(k));                   // exact product, one rounding
}
template <> __device__ __forceinline__ uint16_t fp8_value<BF16>(float v, int k) {
  return rne_bf16((double)v * pow2(k));
}

template <bool E4, class D>
__global__ void __launch_bounds__(F8_THREADS) fp8_decode_kernel(const uint8_t *__restrict__ src,
                                                               raw_t<D> *__restrict__ dst, size_t n,
                                                               const ps_fp8_scale *sc) {
  const int k = sc ? sc->k : 0;
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  const bool vec = ((uintptr_t)src % 16 == 0) && ((uintptr_t)dst % 16 == 0);
  const size_t nunits = vec ? n / F8_E : 0;
  constexpr int NV = F8_E * (int)sizeof(raw_t<D>) / 16;
  for (size_t g = tid; g < nunits; g += stride) {
    union { uint4 v; uint8_t b[F8_E]; } in;
    union { uint4 v[NV]; raw_t<D> e[F8_E]; } out;
    in.v = __ldg(reinterpret_cast<const uint4 *>(src) + g);
#pragma unroll
    for (int e = 0; e < F8_E; e++) out.e[e] = fp8_value<D>(fp8_to_f32(in.b[e], E4), k);
    uint4 *p = reinterpret_cast<uint4 *>(dst) + g * NV;
#pragma unroll
    for (int j = 0; j < NV; j++) p[j] = out.v[j];
  }
  for (size_t i = nunits * F8_E + tid; i < n; i += stride)
    dst[i] = fp8_value<D>(fp8_to_f32(src[i], E4), k);
}

static unsigned f8_blocks(size_t n) {
  size_t b = (n / F8_E + F8_THREADS - 1) / F8_THREADS;
  const size_t cap = (size_t)num_sms() * 8;
  if (b > cap) b = cap;
  if (b == 0) b = 1;
  return (unsigned)b;
}

ps_status fp8_encode_async(const void *src, int st, void *dst, int dt, size_t n, ps_fp8_scale *sc,
                           cudaStream_t stream) {
  if (n == 0) {
    if (sc) PS_CUDA(cudaMemsetAsync(sc, 0, sizeof(ps_fp8_scale), stream));
    return PS_OK;
  }
  const unsigned blocks = f8_blocks(n);
  if (sc) PS_CUDA(cudaMemsetAsync(&sc->amax_bits, 0, sizeof(uint64_t), stream));
  return dispatch_store(st, [&](auto s) -> ps_status {
    using S = decltype(s);
    if constexpr (Store<S>::code >= PS_E4M3) {
      return PS_ERR_UNSUPPORTED;
    } else {
      if (sc) {
        fp8_amax_kernel<S><<<blocks, F8_THREADS, 0, stream>>>((const raw_t<S> *)src, n,
                                                             (unsigned long long *)&sc->amax_bits);
        PS_CHECK_LAUNCH("fp8_amax_kernel");
      }
      if (dt == PS_E4M3)
        fp8_encode_kernel<S, true><<<blocks, F8_THREADS, 0, stream>>>((const raw_t<S> *)src, (uint8_t *)dst, n, sc);
      else
        fp8_encode_kernel<S, false><<<blocks, F8_THREADS, 0, stream>>>((const raw_t<S> *)src, (uint8_t *)dst, n, sc);
      PS_CHECK_LAUNCH("fp8_encode_kernel");
      return PS_OK;
    }
  });
}

ps_status fp8_decode_async(const void *src, int st, void *dst, int dt, size_t n, const ps_fp8_scale *sc,
                           cudaStream_t stream) {
  if (n == 0) return PS_OK;
  const unsigned blocks = f8_blocks(n);
  return dispatch_store(dt, [&](auto d) -> ps_status {
    using D = decltype(d);
    if constexpr (Store<D>::code >= PS_E4M3) {
      return PS_ERR_UNSUPPORTED;
    } else {
      if (st == PS_E4M3)
        fp8_decode_kernel<true, D><<<blocks, F8_THREADS, 0, stream>>>((const uint8_t *)src, (raw_t<D> *)dst, n, sc);
      else
        fp8_decode_kernel<false, D><<<blocks, F8_THREADS, 0, stream>>>((const uint8_t *)src, (raw_t<D> *)dst, n, sc);
      PS_CHECK_LAUNCH("fp8_decode_kernel");
      return PS_OK;
    }
  });
}

}  // namespace ps

extern "C" ps_status ps_convert_scaled(const void *src, int src_type, void *dst, int dst_type, size_t n,
                                       ps_fp8_scale *scale, void *stream) {
  using namespace ps;
  if (!dtype_ok(src_type) || !dtype_ok(dst_type)) {
    set_error("ps_convert_scaled: bad dtype code (%d, %d)", src_type, dst_type);
    return PS_ERR_INVALID;
  }
  if (is_fp8(src_type) == is_fp8(dst_type)) {
    set_error("ps_convert_scaled: exactly one side must be fp8 (%d -> %d)", src_type, dst_type);
    return PS_ERR_UNSUPPORTED;
  }
  if (!scale) {
    set_error("ps_convert_scaled: null scale record");
    return PS_ERR_INVALID;
  }
  if (n && (!src || !dst)) {
    set_error("ps_convert_scaled: null pointer");
    return PS_ERR_INVALID;
  }
  const uintptr_t s0 = (uintptr_t)src, s1 = s0 + n * dtype_size(src_type);
  const uintptr_t d0 = (uintptr_t)dst, d1 = d0 + n * dtype_size(dst_type);
  if (n && s0 < d1 && d0 < s1) {
    set_error("ps_convert_scaled: src and dst overlap");
    return PS_ERR_INVALID;
  }
  cudaStream_t st = (cudaStream_t)stream;
  return is_fp8(dst_type) ? fp8_encode_async(src, src_type, dst, dst_type, n, scale, st)
                          : fp8_decode_async(src, src_type, dst, dst_type, n, scale, st);
}
