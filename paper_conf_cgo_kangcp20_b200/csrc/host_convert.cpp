// host_convert.cpp -- host-side conversion of an orig (f32) memory object before
// its host-to-device transfer: the paper's host-side scaling methods (Fig. 3a
// single loop, Fig. 3b multithreaded/SIMD).  RNE with canonical NaN
// (reading #5), i.e. bit-identical to the device conversion kernels:
//   f32 -> f16 : F16C vcvtps2ph (imm = round to nearest even), NaN lanes -> 0x7FFF
//   f32 -> f64 : exact widening (AVX vcvtps2pd), NaN lanes -> 0x7FFF...F
// A portable bit-manipulation path is used when the CPU lacks F16C/AVX2.
#include <immintrin.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <thread>
#include <vector>

#include "../../include/prescaler.h"

namespace ps {

static inline uint16_t f32_to_f16_scalar(float f) {
  uint32_t x;
  memcpy(&x, &f, 4);
  const uint32_t sign = (x >> 16) & 0x8000u;
  const uint32_t e = (x >> 23) & 0xFFu, m = x & 0x7FFFFFu;
  if (e == 0xFF) return m ? (uint16_t)0x7FFF : (uint16_t)(sign | 0x7C00u);
  int32_t E = (int32_t)e - 127;                    // unbiased
  if (E > 15) return (uint16_t)(sign | 0x7C00u);   // >= 2^16: overflow
  uint32_t S = m | (e ? 0x800000u : 0u);           // 24-bit significand
  if (!e) E = -126;
  // target quantum 2^q with q = max(E, -14) - 10; value = S * 2^(E-23)
  const int32_t q = (E > -14 ? E : -14) - 10;
  const int32_t r = q - (E - 23);                  // right shift (>= 13 here)
  uint32_t K;
  if (r >= 32) K = 0;
  else {
    K = S >> r;
    const uint32_t rem = S & ((1u << r) - 1), half = 1u << (r - 1);
    if (rem > half || (rem == half && (K & 1u))) K++;
  }
  if (K >= 0x400u) {                               // normal
    int32_t biased = q + 10 + 15;
    if (K == 0x800u) { K >>= 1; biased++; }
    if (biased >= 31) return (uint16_t)(sign | 0x7C00u);
    return (uint16_t)(sign | ((uint32_t)biased << 10) | (K - 0x400u));
  }
  return (uint16_t)(sign | K);
}

static inline double f32_to_f64_scalar(float f) {
  if (f != f) {
    const uint64_t c = 0x7FFFFFFFFFFFFFFFull;
    double d;
    memcpy(&d, &c, 8);
    return d;
  }
  return (double)f;
}

__attribute__((target("f16c,avx2"))) static void f16_simd(const float *s, uint16_t *d, size_t n) {
  size_t i = 0;
  const __m128i canon = _mm_set1_epi16(0x7FFF);
  for (; i + 8 <= n; i += 8) {
    const __m256 x = _mm256_loadu_ps(s + i);
    __m128i h = _mm256_cvtps_ph(x, _MM_FROUND_TO_NEAREST_INT | _MM_FROUND_NO_EXC);
    const __m256i nan32 = _mm256_castps_si256(_mm256_cmp_ps(x, x, _CMP_UNORD_Q));
    const __m128i nan16 = _mm_packs_epi32(_mm256_castsi256_si128(nan32), _mm256_extracti128_si256(nan32, 1));
    h = _mm_blendv_epi8(h, canon, nan16);
    _mm_storeu_si128(reinterpret_cast<__m128i *>(d + i), h);
  }
  for (; i < n; i++) d[i] = f32_to_f16_scalar(s[i]);
}

__attribute__((target("avx2"))) static void f64_simd(const float *s, double *d, size_t n) {
  size_t i = 0;
  const __m256d canon = _mm256_castsi256_pd(_mm256_set1_epi64x(0x7FFFFFFFFFFFFFFFll));
  for (; i + 4 <= n; i += 4) {
    const __m256d x = _mm256_cvtps_pd(_mm_loadu_ps(s + i));
    const __m256d nan = _mm256_cmp_pd(x, x, _CMP_UNORD_Q);
    _mm256_storeu_pd(d + i, _mm256_blendv_pd(x, canon, nan));
  }
  for (; i < n; i++) d[i] = f32_to_f64_scalar(s[i]);
}

static bool simd_ok() {
  static int ok = -1;
  if (ok < 0) ok = (__builtin_cpu_supports("f16c") && __builtin_cpu_supports("avx2")) ? 1 : 0;
  return ok == 1;
}

// f32 -> bf16 (reading #28): RNE on the bit pattern -- the bf16 result is the high
// half of (bits + 0x7FFF + lsb) for every finite input (subnormals included; the
// carry into the exponent is the correct rounding up and reaches 0x7F80 = inf
// exactly on overflow); NaN -> canonical 0x7FFF
static inline uint16_t f32_to_bf16_scalar(float f) {
  uint32_t b;
  memcpy(&b, &f, 4);
  if ((b & 0x7F800000u) == 0x7F800000u && (b & 0x7FFFFFu)) return (uint16_t)0x7FFF;
  return (uint16_t)((b + 0x7FFFu + ((b >> 16) & 1u)) >> 16);
}

// One contiguous range, SIMD when available (Fig. 3b) or a plain scalar loop (Fig. 3a).
static void convert_range(const float *s, void *d, int dt, size_t n, bool simd) {
  if (dt == PS_F32) {
    memcpy(d, s, n * 4);
  } else if (dt == PS_F16) {
    uint16_t *o = (uint16_t *)d;
    if (simd && simd_ok()) f16_simd(s, o, n);
    else for (size_t i = 0; i < n; i++) o[i] = f32_to_f16_scalar(s[i]);
  } else if (dt == PS_BF16) {   // integer-only rounding: the compiler vectorises the loop
    uint16_t *o = (uint16_t *)d;
    for (size_t i = 0; i < n; i++) o[i] = f32_to_bf16_scalar(s[i]);
  } else {
    double *o = (double *)d;
    if (simd && simd_ok()) f64_simd(s, o, n);
    else for (size_t i = 0; i < n; i++) o[i] = f32_to_f64_scalar(s[i]);
  }
}

// f32 source -> dt, `threads` workers over contiguous slices (threads <= 1: caller's thread).
void host_convert_f32(const float *src, void *dst, int dt, size_t n, int threads, bool simd) {
  const size_t esz = dt == PS_F64 ? 8 : (dt == PS_F32 ? 4 : 2);
  if (threads <= 1 || n < (1u << 16)) {
    convert_range(src, dst, dt, n, simd);
    return;
  }
  std::vector<std::thread> pool;
  const size_t per = ((n + threads - 1) / threads + 63) / 64 * 64;
  for (int t = 0; t < threads; t++) {
    const size_t a = (size_t)t * per;
    if (a >= n) break;
    const size_t b = std::min(n, a + per);
    pool.emplace_back(convert_range, src + a, (char *)dst + a * esz, dt, b - a, simd);
  }
  for (auto &th : pool) th.join();
}

}  // namespace ps
