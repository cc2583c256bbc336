// convprobe.cu -- design-space probe for the a2 conversion kernel (not part of
// the library; round 2).  Six directions x variants, 1 GiB and 256 MiB of source,
// L2 flushed before every rep, median of 15 CUDA-event reps, plus a D2D copy of
// the same bytes as the in-run yardstick.  Prints algorithmic GB/s
// (n * (s_src + s_dst) / t) and the fraction of MEASURED_PEAKS hbm_gbs (6537).
//
// Variants:
//   R  register path (library design): LDG.128.nc.no_allocate, convert, STG; grid-stride
//      U units per thread; store hint 0 = default, 1 = .cs (streaming), 2 = L2::evict_first
//   T  TMA bulk path: persistent CTAs, S-stage ring of CH-element chunks,
//      cp.async.bulk global->smem (mbarrier complete_tx), convert smem->smem,
//      cp.async.bulk smem->global (bulk_group), one elected thread issues both.
//   H  hybrid: LDG into registers, convert, STS into a smem tile, bulk store.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/convprobe tools/convprobe.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d: %s\n", #x, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

// ------------------------------------------------------------ conversions
struct H16 { uint16_t b; };
template <class S, class D> struct Cv;
__device__ __forceinline__ uint16_t f2h(float x) { uint16_t h; asm("cvt.rn.f16.f32 %0, %1;" : "=h"(h) : "f"(x)); return x != x ? 0x7FFF : h; }
__device__ __forceinline__ uint16_t d2h(double x) { uint16_t h; asm("cvt.rn.f16.f64 %0, %1;" : "=h"(h) : "d"(x)); return x != x ? 0x7FFF : h; }
__device__ __forceinline__ float h2f(uint16_t h) { float f; asm("cvt.f32.f16 %0, %1;" : "=f"(f) : "h"(h)); return f != f ? __int_as_float(0x7FFFFFFF) : f; }
__device__ __forceinline__ double h2d(uint16_t h) { double d; asm("cvt.f64.f16 %0, %1;" : "=d"(d) : "h"(h)); return d != d ? __longlong_as_double(0x7FFFFFFFFFFFFFFFll) : d; }
__device__ __forceinline__ float d2f(double x) { float f; asm("cvt.rn.f32.f64 %0, %1;" : "=f"(f) : "d"(x)); return x != x ? __int_as_float(0x7FFFFFFF) : f; }
__device__ __forceinline__ double f2d(float x) { return x != x ? __longlong_as_double(0x7FFFFFFFFFFFFFFFll) : (double)x; }
template <> struct Cv<float, uint16_t> { static __device__ __forceinline__ uint16_t f(float x) { return f2h(x); } };
template <> struct Cv<double, uint16_t> { static __device__ __forceinline__ uint16_t f(double x) { return d2h(x); } };
template <> struct Cv<uint16_t, float> { static __device__ __forceinline__ float f(uint16_t x) { return h2f(x); } };
template <> struct Cv<uint16_t, double> { static __device__ __forceinline__ double f(uint16_t x) { return h2d(x); } };
template <> struct Cv<double, float> { static __device__ __forceinline__ float f(double x) { return d2f(x); } };
template <> struct Cv<float, double> { static __device__ __forceinline__ double f(float x) { return f2d(x); } };
template <> struct Cv<uint32_t, uint32_t> { static __device__ __forceinline__ uint32_t f(uint32_t x) { return x; } };

template <int B> struct V;
template <> struct V<16> { using t = uint4; };
template <> struct V<8> { using t = uint2; };
template <> struct V<4> { using t = uint32_t; };

__device__ __forceinline__ uint4 ldn(const uint4 *p) { uint4 r; asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p)); return r; }
__device__ __forceinline__ uint2 ldn(const uint2 *p) { uint2 r; asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p)); return r; }
__device__ __forceinline__ uint32_t ldn(const uint32_t *p) { uint32_t r; asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p)); return r; }

template <int HINT> __device__ __forceinline__ void stv(uint4 *p, uint4 v, uint64_t pol) {
  if (HINT == 1) asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
  else if (HINT == 2) asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol) : "memory");
  else *p = v;
}
template <int HINT> __device__ __forceinline__ void stv(uint2 *p, uint2 v, uint64_t pol) {
  if (HINT == 1) asm volatile("st.global.cs.v2.u32 [%0], {%1,%2};" :: "l"(p), "r"(v.x), "r"(v.y) : "memory");
  else if (HINT == 2) asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u32 [%0], {%1,%2}, %3;" :: "l"(p), "r"(v.x), "r"(v.y), "l"(pol) : "memory");
  else *p = v;
}
template <int HINT> __device__ __forceinline__ void stv(uint32_t *p, uint32_t v, uint64_t pol) {
  if (HINT == 1) asm volatile("st.global.cs.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
  else if (HINT == 2) asm volatile("st.global.L1::no_allocate.L2::cache_hint.u32 [%0], %1, %2;" :: "l"(p), "r"(v), "l"(pol) : "memory");
  else *p = v;
}

// ---------------------------------------------------------- register path
template <class S, class D, int U, int HINT>
__global__ void __launch_bounds__(256) k_reg(const S *__restrict__ src, D *__restrict__ dst, size_t nunits) {
  constexpr int SS = sizeof(S), DS = sizeof(D), E = 16 / (SS > DS ? SS : DS);
  using VS = typename V<E * SS>::t;
  using VD = typename V<E * DS>::t;
  uint64_t pol = 0;
  if (HINT == 2) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t g = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const VS *s = reinterpret_cast<const VS *>(src);
  VD *d = reinterpret_cast<VD *>(dst);
  for (; g + (size_t)(U - 1) * stride < nunits; g += (size_t)U * stride) {
    union { VS v; S e[E]; } in[U];
#pragma unroll
    for (int u = 0; u < U; u++) in[u].v = ldn(s + g + (size_t)u * stride);
#pragma unroll
    for (int u = 0; u < U; u++) {
      union { VD v; D e[E]; } o;
#pragma unroll
      for (int k = 0; k < E; k++) o.e[k] = Cv<S, D>::f(in[u].e[k]);
      stv<HINT>(d + g + (size_t)u * stride, o.v, pol);
    }
  }
  for (; g < nunits; g += stride) {
    union { VS v; S e[E]; } in;
    union { VD v; D e[E]; } o;
    in.v = ldn(s + g);
#pragma unroll
    for (int k = 0; k < E; k++) o.e[k] = Cv<S, D>::f(in.e[k]);
    stv<HINT>(d + g, o.v, pol);
  }
}

// ------------------------------------------------------------- TMA bulk path
__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t *b, int n) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(sa(b)), "r"(n)); }
__device__ __forceinline__ void mb_expect(uint64_t *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mb_wait(uint64_t *b, uint32_t ph) {
  asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}" :: "r"(sa(b)), "r"(ph) : "memory");
}
__device__ __forceinline__ void bulk_load(void *smem, const void *g, uint32_t bytes, uint64_t *bar, uint64_t pol) {
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               :: "r"(sa(smem)), "l"(g), "r"(bytes), "r"(sa(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_store(void *g, const void *smem, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" :: "l"(g), "r"(sa(smem)), "r"(bytes), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// nchunks full chunks of CH elements (the probe uses sizes that are multiples of CH)
template <class S, class D, int CH, int ST, int NT>
__global__ void __launch_bounds__(NT) k_tma(const S *__restrict__ src, D *__restrict__ dst, size_t nchunks, int evict) {
  extern __shared__ __align__(128) unsigned char sm[];
  constexpr int SS = sizeof(S), DS = sizeof(D);
  S *in = reinterpret_cast<S *>(sm);                                  // ST * CH
  D *out = reinterpret_cast<D *>(sm + (size_t)ST * CH * SS);          // ST * CH
  uint64_t *full = reinterpret_cast<uint64_t *>(sm + (size_t)ST * CH * (SS + DS));
  uint64_t pol_ld = 0, pol_st = 0;
  if (evict) {
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_ld));
    pol_st = pol_ld;
  } else {
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol_ld));
    pol_st = pol_ld;
  }
  const int t = threadIdx.x;
  if (t == 0) {
    for (int s = 0; s < ST; s++) mb_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const size_t first = blockIdx.x, step = gridDim.x;
  size_t mine = first < nchunks ? (nchunks - first + step - 1) / step : 0;
  if (t == 0) {
    for (int s = 0; s < ST && (size_t)s < mine; s++) {
      mb_expect(&full[s], CH * SS);
      bulk_load(in + (size_t)s * CH, src + (first + s * step) * CH, CH * SS, &full[s], pol_ld);
    }
  }
  for (size_t i = 0; i < mine; i++) {
    const int s = (int)(i % ST);
    const uint32_t ph = (uint32_t)((i / ST) & 1);
    mb_wait(&full[s], ph);
    if (t == 0) bulk_wait_read<ST - 1>();     // out[s]'s previous bulk store has read smem
    __syncthreads();
    const S *ip = in + (size_t)s * CH;
    D *op = out + (size_t)s * CH;
    constexpr int E = 16 / (SS > DS ? SS : DS);
    using VS = typename V<E * SS>::t;
    using VD = typename V<E * DS>::t;
#pragma unroll 4
    for (int u = t; u < CH / E; u += NT) {
      union { VS v; S e[E]; } a;
      union { VD v; D e[E]; } o;
      a.v = reinterpret_cast<const VS *>(ip)[u];
#pragma unroll
      for (int k = 0; k < E; k++) o.e[k] = Cv<S, D>::f(a.e[k]);
      reinterpret_cast<VD *>(op)[u] = o.v;
    }
    fence_async_smem();
    __syncthreads();
    if (t == 0) {
      const size_t c = first + i * step;
      bulk_store(dst + c * CH, op, CH * DS, pol_st);
      bulk_commit();
      if (i + ST < mine) {
        mb_expect(&full[s], CH * SS);
        bulk_load(in + (size_t)s * CH, src + (first + (i + ST) * step) * CH, CH * SS, &full[s], pol_ld);
      }
    }
  }
  if (t == 0) bulk_wait_all();
}

// hybrid: LDG (U units in flight per thread) -> convert -> STS -> bulk store of the CTA tile
template <class S, class D, int U, int NT>
__global__ void __launch_bounds__(NT) k_hyb(const S *__restrict__ src, D *__restrict__ dst, size_t nunits) {
  constexpr int SS = sizeof(S), DS = sizeof(D), E = 16 / (SS > DS ? SS : DS);
  using VS = typename V<E * SS>::t;
  using VD = typename V<E * DS>::t;
  constexpr int TILE = U * NT;                     // units per tile
  __shared__ __align__(128) VD obuf[2][TILE];
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  const VS *s = reinterpret_cast<const VS *>(src);
  VD *d = reinterpret_cast<VD *>(dst);
  const size_t ntiles = nunits / TILE;
  int b = 0;
  for (size_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, b ^= 1) {
    union { VS v; S e[E]; } in[U];
#pragma unroll
    for (int u = 0; u < U; u++) in[u].v = ldn(s + tile * TILE + u * NT + threadIdx.x);
    if (threadIdx.x == 0) bulk_wait_read<1>();
    __syncthreads();
#pragma unroll
    for (int u = 0; u < U; u++) {
      union { VD v; D e[E]; } o;
#pragma unroll
      for (int k = 0; k < E; k++) o.e[k] = Cv<S, D>::f(in[u].e[k]);
      obuf[b][u * NT + threadIdx.x] = o.v;
    }
    fence_async_smem();
    __syncthreads();
    if (threadIdx.x == 0) {
      bulk_store(d + tile * TILE, obuf[b], TILE * sizeof(VD), pol);
      bulk_commit();
    }
  }
  if (threadIdx.x == 0) bulk_wait_all();
}

// ----------------------------------------------------------------- harness
static void *g_flush;
static size_t g_flush_bytes = 512u << 20;
template <class F>
static float timeit(F f, int reps = 15) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  std::vector<float> ts;
  for (int r = 0; r < reps + 3; r++) {
    CK(cudaMemsetAsync(g_flush, r & 0xff, g_flush_bytes));
    cudaEventRecord(a);
    f();
    cudaEventRecord(b);
    CK(cudaEventSynchronize(b));
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (r >= 3) ts.push_back(ms);
  }
  CK(cudaGetLastError());
  std::sort(ts.begin(), ts.end());
  return ts[ts.size() / 2];
}

static int sms;
static const double PEAK = 6537.0;
static void rep(const char *dir, size_t srcb, const char *var, float ms, double bytes) {
  double gbs = bytes / (ms * 1e-3) / 1e9;
  printf("%-10s %5zuMiB %-34s %8.4f ms %8.1f GB/s %6.3f\n", dir, srcb >> 20, var, ms, gbs, gbs / PEAK);
}


template <class S, class D>
static void check_eq(const char *name, const char *var, void *a, void *b, size_t bytes) {
  static std::vector<unsigned char> ha, hb;
  ha.resize(bytes); hb.resize(bytes);
  CK(cudaMemcpy(ha.data(), a, bytes, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hb.data(), b, bytes, cudaMemcpyDeviceToHost));
  if (memcmp(ha.data(), hb.data(), bytes)) printf("MISMATCH %s %s\n", name, var);
}

template <class S, class D>
static void run_dir(const char *name, void *src, void *dst, void *dst2, size_t srcbytes) {
  const size_t n = srcbytes / sizeof(S);
  const double bytes = (double)n * (sizeof(S) + sizeof(D));
  constexpr int SS = sizeof(S), DS = sizeof(D), E = 16 / (SS > DS ? SS : DS);
  const size_t nunits = n / E;
  char v[64];
  for (int bps : {4, 16}) {
    snprintf(v, 64, "reg U=4 h0 bps=%d", bps);
    rep(name, srcbytes, v, timeit([&] { k_reg<S, D, 4, 0><<<sms * bps, 256>>>((const S *)src, (D *)dst2, nunits); }), bytes);
  }
  for (int bps : {3, 4, 6}) {
    snprintf(v, 64, "hyb U=4 bps=%d", bps);
    rep(name, srcbytes, v, timeit([&] { k_hyb<S, D, 4, 256><<<sms * bps, 256>>>((const S *)src, (D *)dst, nunits); }), bytes);
    check_eq<S, D>(name, v, dst, dst2, n * DS);
  }
  // TMA: chunk of CH elements, ST stages
#define TMA(CH, ST, NT, BPS, EV)                                                                          \
  {                                                                                                       \
    size_t smem = (size_t)ST * CH * (SS + DS) + ST * 8;                                                   \
    if (smem * BPS <= 227 * 1024) {                                                                       \
    auto kf = k_tma<S, D, CH, ST, NT>;                                                                    \
    CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));                \
    snprintf(v, 64, "tma CHB=%d ST=%d NT=%d bps=%d ev=%d", CH * SS, ST, NT, BPS, EV);                    \
    CK(cudaMemset(dst, 0xEE, n * DS));                                                                    \
    rep(name, srcbytes, v, timeit([&] { kf<<<sms * BPS, NT, smem>>>((const S *)src, (D *)dst, n / CH, EV); }), bytes); \
    check_eq<S, D>(name, v, dst, dst2, n * DS);                                                           \
    }                                                                                                     \
  }
  constexpr int C8 = 8192 / SS, C16 = 16384 / SS, C32 = 32768 / SS;
  TMA(C8, 4, 256, 2, 0)
  TMA(C8, 4, 512, 2, 0)
  TMA(C8, 6, 256, 2, 0)
  TMA(C8, 3, 256, 4, 0)
  TMA(C16, 2, 512, 2, 0)
  TMA(C16, 3, 512, 1, 0)
  TMA(C16, 3, 256, 2, 0)
  TMA(C16, 4, 512, 1, 0)
  TMA(C16, 4, 256, 1, 0)
  TMA(C32, 2, 512, 1, 0)
  TMA(C32, 3, 512, 1, 0)
  TMA(C16, 3, 512, 1, 1)
}

int main(int argc, char **argv) {
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("SMs %d\n", sms);
  const size_t maxb = (size_t)1 << 32;   // up to 4 GiB dst (f16->f64 of 1 GiB)
  void *src, *dst, *dst2;
  CK(cudaMalloc(&src, (size_t)1 << 30));
  CK(cudaMalloc(&dst, maxb));
  CK(cudaMalloc(&dst2, maxb));
  CK(cudaMalloc(&g_flush, g_flush_bytes));
  // random bit patterns (incl NaN/inf/subnormal): value-independent speed
  {
    std::vector<uint32_t> h(((size_t)1 << 30) / 4);
    uint64_t x = 0x9E3779B97F4A7C15ull;
    for (auto &w : h) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; w = (uint32_t)x; }
    CK(cudaMemcpy(src, h.data(), (size_t)1 << 30, cudaMemcpyHostToDevice));
  }
  for (size_t sb : {(size_t)1 << 30, (size_t)256 << 20, (size_t)32 << 20}) {
    rep("copy", sb, "cudaMemcpy D2D", timeit([&] { cudaMemcpyAsync(dst, src, sb, cudaMemcpyDeviceToDevice); }), 2.0 * sb);
    rep("copy", sb, "reg U=4 bps=8", timeit([&] { k_reg<uint32_t, uint32_t, 4, 0><<<sms * 8, 256>>>((const uint32_t *)src, (uint32_t *)dst, sb / 16); }), 2.0 * sb);
    run_dir<float, uint16_t>("f32->f16", src, dst, dst2, sb);
    run_dir<uint16_t, float>("f16->f32", src, dst, dst2, sb);
    run_dir<double, uint16_t>("f64->f16", src, dst, dst2, sb);
    run_dir<double, float>("f64->f32", src, dst, dst2, sb);
    run_dir<float, double>("f32->f64", src, dst, dst2, sb);
    run_dir<uint16_t, double>("f16->f64", src, dst, dst2, sb);
  }
  printf("done %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
