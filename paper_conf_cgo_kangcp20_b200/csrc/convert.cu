// convert.cu -- device-side type conversion of a memory object (row a2;
// Fig. 3c "parallelized type conversion on GPU side") and the
// ps_convert C entry point.
//
// HBM-bound: per element s_src + s_dst bytes, zero flops.  Two kernels:
//  * convert_bulk_kernel (objects >= one 32 KiB chunk per SM): persistent, one
//    512-thread CTA per SM, a 3-stage shared-memory ring.  One elected thread
//    moves every chunk with the TMA bulk engine -- cp.async.bulk global->smem
//    completing on the stage's mbarrier (UBLKCP.S.G), and after the CTA has
//    converted the chunk smem->smem, cp.async.bulk smem->global (bulk_group) --
//    so both HBM streams run as full-line bulk transfers with 2 chunks in flight
//    while the third is converted.  A chunk is 32 KiB on the wide side.  The
//    ragged remainder (and an unaligned head) is converted by the same grid
//    through the register path below.  Round-2 probe (tools/convprobe.cu,
//    profiles/convprobe_r2b.txt): 1.00-1.02 of the measured copy bandwidth at
//    1 GiB in every direction, vs 0.86-0.94 for the register path.
//  * convert_kernel (small objects, and pointers whose misalignment rules out a
//    16-byte-aligned bulk copy): every thread moves "units" of
//    E = 16 / max(s_src, s_dst) elements -- one 16-byte access on the wide side,
//    4/8/16 bytes on the narrow side, fully coalesced -- U units in flight,
//    ld.global.nc.L1::no_allocate loads, grid-stride over a multiple of the SMs.
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

// units [u0, u1) of E elements starting at element `head`, plus the scalar
// elements [0, head) and [tail0, n); thread `tid` of `nthr`
template <class S, class D, int U>
__device__ __forceinline__ void convert_units(const raw_t<S> *__restrict__ src, raw_t<D> *__restrict__ dst,
                                              size_t n, size_t head, size_t u0, size_t u1, size_t tail0,
                                              size_t tid, size_t nthr) {
  using UT = Unit<S, D>;
  constexpr int E = UT::E;
  using VS = typename UT::VS;
  using VD = typename UT::VD;
  const VS *s = reinterpret_cast<const VS *>(src + head);
  VD *d = reinterpret_cast<VD *>(dst + head);
  size_t g = u0 + tid;
  for (; g + (size_t)(U - 1) * nthr < u1; g += (size_t)U * nthr) {
    union { VS v; raw_t<S> e[E]; } in[U];
#pragma unroll
    for (int u = 0; u < U; u++) in[u].v = ld_stream(s + g + (size_t)u * nthr);
#pragma unroll
    for (int u = 0; u < U; u++) {
      union { VD v; raw_t<D> e[E]; } out;
#pragma unroll
      for (int k = 0; k < E; k++) out.e[k] = Cvt<S, D>::f(in[u].e[k]);
      d[g + (size_t)u * nthr] = out.v;
    }
  }
  for (; g < u1; g += nthr) {
    union { VS v; raw_t<S> e[E]; } in;
    union { VD v; raw_t<D> e[E]; } out;
    in.v = ld_stream(s + g);
#pragma unroll
    for (int k = 0; k < E; k++) out.e[k] = Cvt<S, D>::f(in.e[k]);
    d[g] = out.v;
  }
  for (size_t i = tid; i < head; i += nthr) dst[i] = Cvt<S, D>::f(src[i]);
  for (size_t i = tail0 + tid; i < n; i += nthr) dst[i] = Cvt<S, D>::f(src[i]);
}

template <class S, class D, int U>
__global__ void __launch_bounds__(256) convert_kernel(const raw_t<S> *__restrict__ src,
                                                     raw_t<D> *__restrict__ dst, size_t n,
                                                     size_t head, size_t nunits) {
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t nthr = (size_t)gridDim.x * blockDim.x;
  convert_units<S, D, U>(src, dst, n, head, 0, nunits, head + nunits * Unit<S, D>::E, tid, nthr);
}

// ------------------------------------------------------------- TMA bulk path
namespace bulk {
constexpr int WIDE_BYTES = 32768;   // chunk size on the wide side
constexpr int STAGES = 3;
constexpr int THREADS = 512;

__device__ __forceinline__ uint32_t saddr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(saddr(b)));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(saddr(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}" ::"r"(saddr(b)), "r"(parity) : "memory");
}
__device__ __forceinline__ void load(void *smem, const void *g, uint32_t bytes, uint64_t *bar) {
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(saddr(smem)), "l"(g), "r"(bytes), "r"(saddr(bar)) : "memory");
}
__device__ __forceinline__ void store(void *g, const void *smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
               ::"l"(g), "r"(saddr(smem)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

template <class S, class D> struct Cfg {
  static constexpr int SS = sizeof(raw_t<S>), DS = sizeof(raw_t<D>);
  static constexpr int CH = WIDE_BYTES / (SS > DS ? SS : DS);   // elements per chunk
  static constexpr size_t SMEM = (size_t)STAGES * CH * (SS + DS) + STAGES * sizeof(uint64_t);
};
}  // namespace bulk

// chunks [0, nchunks) of CH elements start at element `head` (16-byte aligned on
// both sides); chunk c belongs to CTA c mod grid.  Elements outside the chunks
// go through the register path.
template <class S, class D>
__global__ void __launch_bounds__(bulk::THREADS, 1)
    convert_bulk_kernel(const raw_t<S> *__restrict__ src, raw_t<D> *__restrict__ dst, size_t n,
                        size_t head, size_t nchunks) {
  using C = bulk::Cfg<S, D>;
  using UT = Unit<S, D>;
  constexpr int CH = C::CH, ST = bulk::STAGES, NT = bulk::THREADS, E = UT::E;
  using VS = typename UT::VS;
  using VD = typename UT::VD;
  extern __shared__ __align__(128) unsigned char smem[];
  raw_t<S> *in = reinterpret_cast<raw_t<S> *>(smem);
  raw_t<D> *out = reinterpret_cast<raw_t<D> *>(smem + (size_t)ST * CH * C::SS);
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)ST * CH * (C::SS + C::DS));
  const int t = threadIdx.x;
  const raw_t<S> *s0 = src + head;
  raw_t<D> *d0 = dst + head;
  if (t == 0) {
    for (int s = 0; s < ST; s++) bulk::mbar_init(&full[s]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const size_t first = blockIdx.x, step = gridDim.x;
  const size_t mine = first < nchunks ? (nchunks - first + step - 1) / step : 0;
  if (t == 0)
    for (int s = 0; s < ST && (size_t)s < mine; s++) {
      bulk::mbar_expect_tx(&full[s], CH * C::SS);
      bulk::load(in + (size_t)s * CH, s0 + (first + s * step) * CH, CH * C::SS, &full[s]);
    }
  for (size_t i = 0; i < mine; i++) {
    const int s = (int)(i % ST);
    bulk::mbar_wait(&full[s], (uint32_t)((i / ST) & 1));
    if (t == 0) bulk::wait_read<ST - 1>();   // the store that last read out[s] is done with it
    __syncthreads();
    const VS *ip = reinterpret_cast<const VS *>(in + (size_t)s * CH);
    VD *op = reinterpret_cast<VD *>(out + (size_t)s * CH);
#pragma unroll
    for (int u = t; u < CH / E; u += NT) {
      union { VS v; raw_t<S> e[E]; } a;
      union { VD v; raw_t<D> e[E]; } o;
      a.v = ip[u];
#pragma unroll
      for (int k = 0; k < E; k++) o.e[k] = Cvt<S, D>::f(a.e[k]);
      op[u] = o.v;
    }
    bulk::fence_async_smem();   // generic-proxy smem writes -> visible to the bulk store
    __syncthreads();
    if (t == 0) {
      bulk::store(d0 + (first + i * step) * CH, out + (size_t)s * CH, CH * C::DS);
      bulk::commit();
      if (i + ST < mine) {      // in[s] has been consumed by every thread
        bulk::mbar_expect_tx(&full[s], CH * C::SS);
        bulk::load(in + (size_t)s * CH, s0 + (first + (i + ST) * step) * CH, CH * C::SS, &full[s]);
      }
    }
  }
  // remainder: whole units after the chunks, then scalar head / tail
  const size_t units_done = nchunks * (CH / E);
  const size_t nunits = (n - head) / E;
  convert_units<S, D, 2>(src, dst, n, head, units_done, nunits, head + nunits * E,
                         (size_t)blockIdx.x * NT + t, (size_t)gridDim.x * NT);
  if (t == 0) bulk::wait_all();
}

template <class S, class D>
static ps_status launch_convert(const void *src, void *dst, size_t n, cudaStream_t st) {
  using UT = Unit<S, D>;
  using C = bulk::Cfg<S, D>;
  constexpr int E = UT::E;
  const uintptr_t sa = (uintptr_t)src, da = (uintptr_t)dst;
  // bulk path: a head h that puts both streams on 16-byte boundaries, and at
  // least one chunk per SM
  const int sms = num_sms();
  for (size_t h = 0; h < 16 && h < n; h++) {
    if ((sa + h * UT::SS) % 16 || (da + h * UT::DS) % 16) continue;
    const size_t nchunks = (n - h) / C::CH;
    if (nchunks < (size_t)sms) break;
    PS_TRY(set_max_smem((const void *)convert_bulk_kernel<S, D>, (int)C::SMEM));
    convert_bulk_kernel<S, D><<<(unsigned)sms, bulk::THREADS, C::SMEM, st>>>(
        (const raw_t<S> *)src, (raw_t<D> *)dst, n, h, nchunks);
    PS_CHECK_LAUNCH("convert_bulk_kernel");
    return PS_OK;
  }
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
  const size_t cap = (size_t)sms * 4;
  if (blocks > cap) blocks = cap;
  if (blocks == 0) blocks = 1;
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
