// common.cuh -- shared device/host helpers of libprescaler (sm_100a).
//
// Storage types: f64 = double, f32 = float, f16 / bf16 = uint16_t bit patterns.
// Compute type T is float or double (reading R2: widest touched precision,
// floored at f32).  The library is compiled with -fmad=false and without
// fast-math, so every +,-,*,/,sqrt below is one correctly rounded IEEE op in T
// (reading R4) and FMAs are written explicitly.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include <string>

#include "../../include/prescaler.h"

namespace ps {

// ----------------------------------------------------------------- errors
void set_error(const char *fmt, ...);
ps_status cuda_status(cudaError_t e, const char *what);

#define PS_CUDA(call)                                         \
  do {                                                        \
    cudaError_t _e = (call);                                  \
    if (_e != cudaSuccess) return ps::cuda_status(_e, #call); \
  } while (0)

#define PS_TRY(expr)                     \
  do {                                   \
    ps_status _s = (expr);               \
    if (_s != PS_OK) return _s;          \
  } while (0)

// Opt a kernel into `bytes` of dynamic shared memory on the CURRENT device.
// Thread-safe and per device (the attribute is per device); cheap after the
// first call for a (device, kernel) pair.
ps_status set_max_smem(const void *kernel, int bytes);

void count_launch();
#define PS_CHECK_LAUNCH(what)                                 \
  do {                                                        \
    ps::count_launch();                                       \
    cudaError_t _e = cudaGetLastError();                      \
    if (_e != cudaSuccess) return ps::cuda_status(_e, what);  \
  } while (0)

inline bool is_fp8(int t) { return t == PS_E4M3 || t == PS_E5M2; }
inline size_t dtype_size(int t) { return t == PS_F64 ? 8 : (t == PS_F32 ? 4 : (is_fp8(t) ? 1 : 2)); }
inline bool dtype_ok(int t) { return t >= PS_F64 && t <= PS_E5M2; }
// R2: compute type = widest (smallest code) floored at f32
inline int widest(int a, int b) { return a < b ? a : b; }
inline int compute_type(std::initializer_list<int> ts) {
  int w = PS_F32;
  for (int t : ts) w = widest(w, t);
  return w;
}
int num_sms();

// ------------------------------------------------------- storage traits
struct F16 { uint16_t b; };    // tag type for fp16 storage (IEEE binary16 bits)
struct BF16 { uint16_t b; };   // tag type for bf16 storage (reading #28)
struct E4M3 { uint8_t b; };    // fp8 storage tags (reading #29): raw codes, the
struct E5M2 { uint8_t b; };    // per-tensor scale lives beside the object

template <class S> struct Store;
template <> struct Store<double> { using raw = double; static constexpr int code = PS_F64; };
template <> struct Store<float> { using raw = float; static constexpr int code = PS_F32; };
template <> struct Store<F16> { using raw = uint16_t; static constexpr int code = PS_F16; };
template <> struct Store<BF16> { using raw = uint16_t; static constexpr int code = PS_BF16; };
template <> struct Store<E4M3> { using raw = uint8_t; static constexpr int code = PS_E4M3; };
template <> struct Store<E5M2> { using raw = uint8_t; static constexpr int code = PS_E5M2; };

// exact widening of a stored element to T (NaN payloads are irrelevant for
// arithmetic: any NaN propagates and is scored as non-finite)
__device__ __forceinline__ float f16_to_f32(uint16_t h) {
  float f;
  asm("cvt.f32.f16 %0, %1;" : "=f"(f) : "h"(h));
  return f;
}
__device__ __forceinline__ double f16_to_f64(uint16_t h) {
  double d;
  asm("cvt.f64.f16 %0, %1;" : "=d"(d) : "h"(h));
  return d;
}

// bf16 -> f32 is exact: the bf16 bits are the high half of the f32 bits
__device__ __forceinline__ float bf16_to_f32(uint16_t h) { return __uint_as_float((uint32_t)h << 16); }
template <class T> __device__ __forceinline__ T widen_b(uint16_t h) { return (T)bf16_to_f32(h); }

template <class T> __device__ __forceinline__ T widen(float v) { return (T)v; }
template <class T> __device__ __forceinline__ T widen(double v) { return (T)v; }
template <class T> __device__ __forceinline__ T widen_h(uint16_t h);
template <> __device__ __forceinline__ float widen_h<float>(uint16_t h) { return f16_to_f32(h); }
template <> __device__ __forceinline__ double widen_h<double>(uint16_t h) { return f16_to_f64(h); }

template <class S, class T> struct Ld;
template <class T> struct Ld<double, T> {
  static __device__ __forceinline__ T get(const double *p, size_t i) { return (T)p[i]; }
};
template <class T> struct Ld<float, T> {
  static __device__ __forceinline__ T get(const float *p, size_t i) { return (T)p[i]; }
};
template <class T> struct Ld<F16, T> {
  static __device__ __forceinline__ T get(const uint16_t *p, size_t i) { return widen_h<T>(p[i]); }
};
template <class T> struct Ld<BF16, T> {
  static __device__ __forceinline__ T get(const uint16_t *p, size_t i) { return widen_b<T>(p[i]); }
};

// ------------------------------------------- RNE narrowing (reading R1, c-1)
// canonical NaN (reading #5): every bit set except the sign
__device__ __forceinline__ uint16_t rne_f16(float x) {
  uint16_t h;
  asm("cvt.rn.f16.f32 %0, %1;" : "=h"(h) : "f"(x));
  return (x != x) ? (uint16_t)0x7FFF : h;
}
// f64 -> f16 in ONE rounding (never via f32: reading #6)
__device__ __forceinline__ uint16_t rne_f16(double x) {
  uint16_t h;
  asm("cvt.rn.f16.f64 %0, %1;" : "=h"(h) : "d"(x));
  return (x != x) ? (uint16_t)0x7FFF : h;
}
// bf16 (reading #28): one RNE rounding from f32 or from f64 (F2F.BF16.F64)
__device__ __forceinline__ uint16_t rne_bf16(float x) {
  uint16_t h;
  asm("cvt.rn.bf16.f32 %0, %1;" : "=h"(h) : "f"(x));
  return (x != x) ? (uint16_t)0x7FFF : h;
}
__device__ __forceinline__ uint16_t rne_bf16(double x) {
  uint16_t h;
  asm("cvt.rn.bf16.f64 %0, %1;" : "=h"(h) : "d"(x));
  return (x != x) ? (uint16_t)0x7FFF : h;
}
__device__ __forceinline__ float rne_f32(double x) {
  float f;
  asm("cvt.rn.f32.f64 %0, %1;" : "=f"(f) : "d"(x));
  return (x != x) ? __int_as_float(0x7FFFFFFF) : f;
}
__device__ __forceinline__ float canon_f32(float x) {
  return (x != x) ? __int_as_float(0x7FFFFFFF) : x;
}
__device__ __forceinline__ double canon_f64(double x) {
  return (x != x) ? __longlong_as_double(0x7FFFFFFFFFFFFFFFll) : x;
}

// store a T value into storage S (RNE; exact when S is at least as wide)
template <class S, class T> struct St;
template <class T> struct St<double, T> {
  static __device__ __forceinline__ void put(double *p, size_t i, T v) { p[i] = (double)v; }
};
template <> struct St<float, float> {
  static __device__ __forceinline__ void put(float *p, size_t i, float v) { p[i] = v; }
};
template <> struct St<float, double> {
  static __device__ __forceinline__ void put(float *p, size_t i, double v) { p[i] = rne_f32(v); }
};
template <class T> struct St<F16, T> {
  static __device__ __forceinline__ void put(uint16_t *p, size_t i, T v) { p[i] = rne_f16(v); }
};
template <class T> struct St<BF16, T> {
  static __device__ __forceinline__ void put(uint16_t *p, size_t i, T v) { p[i] = rne_bf16(v); }
};

// ------------------------------------------------ fp8 codes (reading #29)
// E4M3 (OCP "fn": no inf, NaN 0x7F/0xFF, max 448) and E5M2 (IEEE-like, max 57344).
// Decoding a code is exact in f16 (and therefore in f32 / f64).
__device__ __forceinline__ float fp8_to_f32(uint8_t q, bool e4m3) {
  uint32_t h2;
  const uint16_t in = q;
  if (e4m3) asm("cvt.rn.f16x2.e4m3x2 %0, %1;" : "=r"(h2) : "h"(in));
  else asm("cvt.rn.f16x2.e5m2x2 %0, %1;" : "=r"(h2) : "h"(in));
  return f16_to_f32((uint16_t)(h2 & 0xFFFFu));
}
// RNE of a finite-or-not f32 y to the fp8 code: non-finite inputs and
// magnitudes past the overflow midpoint follow the oracle (E4M3: NaN 0x7F; E5M2:
// +-inf), NaN -> canonical 0x7F; the satfinite cvt is only reached in range.
__device__ __forceinline__ uint8_t f32_to_fp8(float y, bool e4m3) {
  const uint32_t sign = (__float_as_uint(y) >> 24) & 0x80u;
  const float a = fabsf(y);
  if (y != y) return 0x7F;
  if (e4m3) {
    if (a > 464.0f) return 0x7F;                    // 464 is the 448/480 tie -> 448
  } else {
    if (a >= 61440.0f) return (uint8_t)(sign | 0x7Cu);   // 61440: 57344/65536 tie -> inf
  }
  uint16_t r;
  if (e4m3) asm("cvt.rn.satfinite.e4m3x2.f32 %0, %1, %2;" : "=h"(r) : "f"(0.0f), "f"(y));
  else asm("cvt.rn.satfinite.e5m2x2.f32 %0, %1, %2;" : "=h"(r) : "f"(0.0f), "f"(y));
  return (uint8_t)(r & 0xFFu);
}
// f64 -> fp8 in ONE rounding: round-to-odd to f32 (24 bits >= 4 + 2), then RNE
__device__ __forceinline__ uint8_t f64_to_fp8(double x, bool e4m3) {
  if (x != x) return 0x7F;
  float f;
  asm("cvt.rz.f32.f64 %0, %1;" : "=f"(f) : "d"(x));
  if ((double)f != x && !isinf(x)) f = __uint_as_float(__float_as_uint(f) | 1u);
  if (isinf(x)) f = (float)x;
  return f32_to_fp8(f, e4m3);
}

// R4 arithmetic helpers (explicit FMA; everything else is plain IEEE)
__device__ __forceinline__ float t_fma(float a, float b, float c) { return __fmaf_rn(a, b, c); }
__device__ __forceinline__ double t_fma(double a, double b, double c) { return __fma_rn(a, b, c); }

// type list helpers for runtime -> template dispatch
template <class F> inline ps_status dispatch_store(int t, F &&f) {
  switch (t) {
    case PS_F64: return f(double());
    case PS_F32: return f(float());
    case PS_F16: return f(F16());
    case PS_BF16: return f(BF16());
  }
  return PS_ERR_INVALID;
}
template <class F> inline ps_status dispatch_compute(int t, F &&f) {
  return t == PS_F64 ? f(double()) : f(float());
}

template <class S> using raw_t = typename Store<S>::raw;

}  // namespace ps
