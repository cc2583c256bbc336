/*
 * hwcheck.c -- pins the oracle's software converter (oracle.c, c-1) to the
 * x86 HARDWARE converters, which share nothing with it:
 *   f32 -> f16 : F16C vcvtps2ph (imm = round-to-nearest-even), all 2^32 inputs
 *   f16 -> f32 : F16C vcvtph2ps, all 2^16 inputs (exact widening)
 *   f64 -> f16 : AVX512-FP16 vcvtsd2sh (direct, single rounding), targeted
 *                midpoint sets + random bit patterns
 *   f64 -> f32 : SSE2 cvtsd2ss under MXCSR RNE, FTZ/DAZ off
 *   f16 -> f64, f32 -> f64 : exact C widening
 *   f32 -> bf16: AVX512-BF16 vcvtneps2bf16 (RNE), all 2^32 inputs whose input
 *                and result are normal or zero (the instruction flushes
 *                subnormals: those are pinned in test_oracle_bf16.py instead)
 *   bf16 -> f32: the definition (bits << 16), all 2^16 inputs
 * NaN inputs compare NaN-ness only (the oracle canonicalises, reading #5).
 * Usage: hwcheck <mode> [count]; prints "mismatches=<n> checked=<m>".
 */
#include <immintrin.h>
#include <inttypes.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "../../oracle/oracle.h"

static int is_nan16(uint64_t h) { return ((h >> 10) & 0x1F) == 0x1F && (h & 0x3FF); }
static int is_nan32(uint64_t b) { return ((b >> 23) & 0xFF) == 0xFF && (b & 0x7FFFFF); }
static int is_nan64(uint64_t b) { return ((b >> 52) & 0x7FF) == 0x7FF && (b & 0xFFFFFFFFFFFFFull); }

static uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__attribute__((target("f16c"))) static uint16_t hw_f32_f16(uint32_t b) {
  float f;
  memcpy(&f, &b, 4);
  return (uint16_t)_cvtss_sh(f, _MM_FROUND_TO_NEAREST_INT | _MM_FROUND_NO_EXC);
}
__attribute__((target("f16c"))) static uint32_t hw_f16_f32(uint16_t h) {
  float f = _cvtsh_ss(h);
  uint32_t b;
  memcpy(&b, &f, 4);
  return b;
}
__attribute__((target("avx512fp16,avx512vl"))) static uint16_t hw_f64_f16(uint64_t b) {
  double d;
  memcpy(&d, &b, 8);
  __m128h r = _mm_cvtsd_sh(_mm_setzero_ph(), _mm_set_sd(d));
  return (uint16_t)_mm_extract_epi16((__m128i)r, 0);
}
static uint32_t hw_f64_f32(uint64_t b) {
  double d;
  float f;
  uint32_t o;
  memcpy(&d, &b, 8);
  f = (float)d;
  memcpy(&o, &f, 4);
  return o;
}

__attribute__((target("avx512bf16,avx512vl"))) static uint16_t hw_f32_bf16(uint32_t b) {
  float f;
  memcpy(&f, &b, 4);
  __m128bh r = _mm_cvtneps_pbh(_mm_set_ss(f));
  return (uint16_t)_mm_extract_epi16((__m128i)r, 0);
}
static int is_nan_bf16(uint64_t h) { return ((h >> 7) & 0xFF) == 0xFF && (h & 0x7F); }

static uint64_t check_f64_f16(uint64_t b, int *has_nan_ok) {
  uint64_t o = oracle_convert_bits(b, OR_F64, OR_F16), h = hw_f64_f16(b);
  *has_nan_ok = is_nan64(b) && is_nan16(o) && is_nan16(h);
  return (o != h) && !*has_nan_ok;
}

int main(int argc, char **argv) {
  const char *mode = argc > 1 ? argv[1] : "";
  uint64_t count = argc > 2 ? strtoull(argv[2], NULL, 0) : (1ull << 24);
  uint64_t bad = 0, checked = 0;
  if (!strcmp(mode, "f32f16")) {                 /* all 2^32 inputs */
    if (!__builtin_cpu_supports("f16c")) { printf("skip=nof16c\n"); return 0; }
#pragma omp parallel for reduction(+ : bad, checked) schedule(static)
    for (int64_t hi = 0; hi < 65536; hi++) {
      for (uint32_t lo = 0; lo < 65536; lo++) {
        uint32_t b = ((uint32_t)hi << 16) | lo;
        uint64_t o = oracle_convert_bits(b, OR_F32, OR_F16), h = hw_f32_f16(b);
        if (o != h && !(is_nan32(b) && is_nan16(o) && is_nan16(h))) bad++;
        checked++;
      }
    }
  } else if (!strcmp(mode, "f32bf16")) {         /* all 2^32 inputs (normal/zero) */
    if (!__builtin_cpu_supports("avx512bf16")) { printf("skip=noavx512bf16\n"); return 0; }
#pragma omp parallel for reduction(+ : bad, checked) schedule(static)
    for (int64_t hi = 0; hi < 65536; hi++) {
      for (uint32_t lo = 0; lo < 65536; lo++) {
        uint32_t b = ((uint32_t)hi << 16) | lo;
        uint64_t o = oracle_convert_bits(b, OR_F32, OR_BF16), h;
        if (((b >> 23) & 0xFF) == 0 && (b & 0x7FFFFF)) continue;     /* subnormal input */
        if (((o >> 7) & 0xFF) == 0 && (o & 0x7F)) continue;           /* subnormal result */
        h = hw_f32_bf16(b);
        if (o != h && !(is_nan32(b) && is_nan_bf16(o) && is_nan_bf16(h))) bad++;
        checked++;
      }
    }
  } else if (!strcmp(mode, "bf16wide")) {        /* all 2^16 inputs: exact widening */
    for (uint32_t h = 0; h < 65536; h++) {
      uint64_t o32 = oracle_convert_bits(h, OR_BF16, OR_F32), o64 = oracle_convert_bits(h, OR_BF16, OR_F64);
      uint32_t w = h << 16;
      float f;
      double d;
      uint64_t w64;
      memcpy(&f, &w, 4);
      d = (double)f;
      memcpy(&w64, &d, 8);
      if (is_nan_bf16(h)) bad += !(is_nan32(o32) && is_nan64(o64));
      else bad += (o32 != w) + (o64 != w64);
      checked++;
    }
  } else if (!strcmp(mode, "f16wide")) {         /* all 2^16 inputs, both widenings */
    if (!__builtin_cpu_supports("f16c")) { printf("skip=nof16c\n"); return 0; }
    for (uint32_t h = 0; h < 65536; h++) {
      uint64_t o32 = oracle_convert_bits(h, OR_F16, OR_F32), h32 = hw_f16_f32((uint16_t)h);
      uint64_t o64 = oracle_convert_bits(h, OR_F16, OR_F64), h64;
      float f;
      double d;
      memcpy(&f, &h32, 4);
      d = (double)f;
      memcpy(&h64, &d, 8);
      if (is_nan16(h)) { bad += !(is_nan32(o32) && is_nan64(o64)); }
      else { bad += (o32 != h32) + (o64 != h64); }
      checked++;
    }
  } else if (!strcmp(mode, "f64f16")) {          /* targeted + random */
    int nan_ok;
    if (!__builtin_cpu_supports("avx512fp16")) { printf("skip=noavx512fp16\n"); return 0; }
    /* every positive/negative fp16 midpoint (incl. subnormal and overflow edges)
       +- 0..4 fp64 ulps, and the fp16 values themselves */
    for (uint32_t h = 0; h < 0x7C00; h++) {
      uint64_t lo = oracle_convert_bits(h, OR_F16, OR_F64);
      uint64_t hi = oracle_convert_bits(h + 1, OR_F16, OR_F64);   /* 0x7C00 -> inf */
      double dl, dh, mid;
      uint64_t mb;
      memcpy(&dl, &lo, 8);
      memcpy(&dh, &hi, 8);
      if (h + 1 == 0x7C00) dh = 65536.0;          /* next binade boundary */
      mid = dl + (dh - dl) / 2;                   /* exact in fp64 */
      memcpy(&mb, &mid, 8);
      for (int k = -4; k <= 4; k++)
        for (int s = 0; s < 2; s++) {
          uint64_t b = (mb + (int64_t)k) | ((uint64_t)s << 63);
          bad += check_f64_f16(b, &nan_ok);
          bad += check_f64_f16(lo | ((uint64_t)s << 63), &nan_ok);
          checked += 2;
        }
    }
#pragma omp parallel for reduction(+ : bad, checked) private(nan_ok)
    for (int64_t i = 0; i < (int64_t)count; i++) {
      uint64_t b = splitmix64(0x5EED0000ull + (uint64_t)i);
      /* half the draws restricted to the fp16-relevant exponent window */
      if (i & 1) b = (b & 0x800FFFFFFFFFFFFFull) | ((uint64_t)(1023 - 30 + (b >> 52) % 48) << 52);
      bad += check_f64_f16(b, &nan_ok);
      checked++;
    }
  } else if (!strcmp(mode, "f64f32")) {
#pragma omp parallel for reduction(+ : bad, checked)
    for (int64_t i = 0; i < (int64_t)count; i++) {
      uint64_t b = splitmix64(0xF00D0000ull + (uint64_t)i);
      if (i % 3 == 1) b = (b & 0x800FFFFFFFFFFFFFull) | ((uint64_t)(1023 - 160 + (b >> 52) % 300) << 52);
      if (i % 3 == 2) {                           /* f32 midpoints +- few ulps */
        uint32_t f = (uint32_t)(b >> 33);
        uint64_t lo = oracle_convert_bits(f, OR_F32, OR_F64), hi2;
        double dl, dh, mid;
        if (is_nan32(f) || ((f >> 23) & 0xFF) == 0xFF) continue;
        hi2 = oracle_convert_bits(f + 1, OR_F32, OR_F64);
        memcpy(&dl, &lo, 8);
        memcpy(&dh, &hi2, 8);
        if (((f + 1) >> 23 & 0xFF) == 0xFF) continue;
        mid = dl + (dh - dl) / 2;
        memcpy(&b, &mid, 8);
        b += (int64_t)(i % 9) - 4;
      }
      uint64_t o = oracle_convert_bits(b, OR_F64, OR_F32), h = hw_f64_f32(b);
      if (o != h && !(is_nan64(b) && is_nan32(o) && is_nan32(h))) bad++;
      checked++;
    }
  } else if (!strcmp(mode, "f32f64")) {          /* exact widening, random patterns */
#pragma omp parallel for reduction(+ : bad, checked)
    for (int64_t i = 0; i < (int64_t)count; i++) {
      uint32_t b = (uint32_t)splitmix64(0xABCD0000ull + (uint64_t)i);
      float f;
      double d;
      uint64_t h;
      memcpy(&f, &b, 4);
      d = (double)f;
      memcpy(&h, &d, 8);
      uint64_t o = oracle_convert_bits(b, OR_F32, OR_F64);
      if (o != h && !(is_nan32(b) && is_nan64(o))) bad++;
      checked++;
    }
  } else {
    fprintf(stderr, "usage: hwcheck f32f16|f16wide|f64f16|f64f32|f32f64 [count]\n");
    return 2;
  }
  printf("mismatches=%" PRIu64 " checked=%" PRIu64 "\n", bad, checked);
  return bad ? 1 : 0;
}
