// quality.cu -- fused back-conversion + quality reduction (rows a4 + a5) and
// the ps_quality C entry point.
//
// Per output element (reading #7, mean relative error P:384):
//   delivered = RNE_f32(out_c[i])                (a4; exact for f32/f16)
//   o = (double)delivered, r = ref[i]
//   e = 0 if o == r; 1 if o or r non-finite or r == 0; else min(1, |o-r|/|r|)
// One read of out_c and ref, one write of the delivered f32 output; sum(e) in
// fp64, max of the uncapped relative error, count of non-finite o.
// Deterministic: the output (rows x cols) is cut into QSeg segments that depend
// on its shape only -- whole rows for a matrix (so a row-sharded evaluation,
// ps_shard_step, computes exactly the segments of its rows), ~equal pieces of a
// vector -- one block per segment with a fixed thread map and fixed shuffle/smem
// trees, never on the SM count; the finalize adds the segment partials in
// segment order.  So results are bit-identical across GPUs and rank counts.
#include <math.h>

#include "common.cuh"
#include "kernels.cuh"

namespace ps {

__device__ __forceinline__ void qual_elem(double o, double r, double &sum, double &mx,
                                          unsigned long long &nf) {
  const bool fo = isfinite(o), fr = isfinite(r);
  nf += fo ? 0ull : 1ull;
  double e, rel;
  if (o == r) { e = 0.0; rel = 0.0; }
  else if (!fo || !fr || r == 0.0) { e = 1.0; rel = INFINITY; }
  else { rel = fabs(o - r) / fabs(r); e = rel < 1.0 ? rel : 1.0; }
  sum = sum + e;
  mx = rel > mx ? rel : mx;
}

template <class S> struct Deliver;
template <> struct Deliver<double> {
  static __device__ __forceinline__ float f(double v) { return rne_f32(v); }
  static __device__ __forceinline__ double exact(double v) { return v; }
};
template <> struct Deliver<float> {
  static __device__ __forceinline__ float f(float v) { return canon_f32(v); }
  static __device__ __forceinline__ double exact(float v) { return (double)v; }
};
template <> struct Deliver<F16> {
  static __device__ __forceinline__ float f(uint16_t h) { return canon_f32(f16_to_f32(h)); }
  static __device__ __forceinline__ double exact(uint16_t h) { return f16_to_f64(h); }
};
template <> struct Deliver<BF16> {
  static __device__ __forceinline__ float f(uint16_t h) { return canon_f32(bf16_to_f32(h)); }
  static __device__ __forceinline__ double exact(uint16_t h) { return (double)bf16_to_f32(h); }
};

// fp8 codes without a scale (ps_quality; the app path decodes scaled objects first)
template <> struct Deliver<E4M3> {
  static __device__ __forceinline__ float f(uint8_t q) { return canon_f32(fp8_to_f32(q, true)); }
  static __device__ __forceinline__ double exact(uint8_t q) { return (double)fp8_to_f32(q, true); }
};
template <> struct Deliver<E5M2> {
  static __device__ __forceinline__ float f(uint8_t q) { return canon_f32(fp8_to_f32(q, false)); }
  static __device__ __forceinline__ double exact(uint8_t q) { return (double)fp8_to_f32(q, false); }
};

__device__ __forceinline__ void block_reduce3(double &sum, double &mx, unsigned long long &nf,
                                              double *s_sum, double *s_mx,
                                              unsigned long long *s_nf) {
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) {
    sum = sum + __shfl_xor_sync(0xffffffffu, sum, off);
    const double m2 = __shfl_xor_sync(0xffffffffu, mx, off);
    mx = m2 > mx ? m2 : mx;
    nf += __shfl_xor_sync(0xffffffffu, nf, off);
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  if (lane == 0) { s_sum[warp] = sum; s_mx[warp] = mx; s_nf[warp] = nf; }
  __syncthreads();
  if (warp == 0) {
    sum = lane < nw ? s_sum[lane] : 0.0;
    mx = lane < nw ? s_mx[lane] : 0.0;
    nf = lane < nw ? s_nf[lane] : 0ull;
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
      sum = sum + __shfl_xor_sync(0xffffffffu, sum, off);
      const double m2 = __shfl_xor_sync(0xffffffffu, mx, off);
      mx = m2 > mx ? m2 : mx;
      nf += __shfl_xor_sync(0xffffffffu, nf, off);
    }
  }
}

// DELIVER: round to the original precision f32 and write it (pipeline, a4);
// otherwise score the exact widened value (standalone ps_quality).  Block b
// handles segment seg0 + b = elements [seg * per, min(n, (seg + 1) * per)).
template <class S, bool DELIVER>
__global__ void __launch_bounds__(QTHREADS) backconv_quality_kernel(
    const raw_t<S> *__restrict__ out, const double *__restrict__ ref, float *__restrict__ delivered,
    size_t n, size_t per, int seg0, QPart *__restrict__ parts) {
  __shared__ double s_sum[QTHREADS / 32], s_mx[QTHREADS / 32];
  __shared__ unsigned long long s_nf[QTHREADS / 32];
  double sum = 0.0, mx = 0.0;
  unsigned long long nf = 0;
  const int seg = seg0 + (int)blockIdx.x;
  const size_t base = (size_t)seg * per;
  const size_t end = base + per < n ? base + per : n;
  auto one = [&](size_t i, raw_t<S> v, double r) {
    double o;
    if (DELIVER) {
      const float d = Deliver<S>::f(v);
      delivered[i] = d;
      o = (double)d;
    } else {
      o = Deliver<S>::exact(v);
    }
    qual_elem(o, r, sum, mx, nf);
  };
  // 4 consecutive elements per thread per step: 16-byte loads of ref (2 x double2)
  // and of out (f32) / 8-byte (f16) / 2 x 16-byte (f64) when everything is aligned
  const bool vec = base % 4 == 0 && ((uintptr_t)out % 16 == 0) && ((uintptr_t)ref % 16 == 0) &&
                   (!DELIVER || (uintptr_t)delivered % 16 == 0);
  size_t i = base + (size_t)threadIdx.x * 4;
  if (vec) {
    for (; i + 4 <= end; i += (size_t)QTHREADS * 4) {
      const double2 r0 = __ldg(reinterpret_cast<const double2 *>(ref + i));
      const double2 r1 = __ldg(reinterpret_cast<const double2 *>(ref + i) + 1);
      raw_t<S> v[4];
#pragma unroll
      for (int k = 0; k < 4; k++) v[k] = out[i + k];
      if (DELIVER) {
        float4 d;
        d.x = Deliver<S>::f(v[0]);
        d.y = Deliver<S>::f(v[1]);
        d.z = Deliver<S>::f(v[2]);
        d.w = Deliver<S>::f(v[3]);
        *reinterpret_cast<float4 *>(delivered + i) = d;
        qual_elem((double)d.x, r0.x, sum, mx, nf);
        qual_elem((double)d.y, r0.y, sum, mx, nf);
        qual_elem((double)d.z, r1.x, sum, mx, nf);
        qual_elem((double)d.w, r1.y, sum, mx, nf);
      } else {
        qual_elem(Deliver<S>::exact(v[0]), r0.x, sum, mx, nf);
        qual_elem(Deliver<S>::exact(v[1]), r0.y, sum, mx, nf);
        qual_elem(Deliver<S>::exact(v[2]), r1.x, sum, mx, nf);
        qual_elem(Deliver<S>::exact(v[3]), r1.y, sum, mx, nf);
      }
    }
    for (; i < end; i++) one(i, out[i], __ldg(ref + i));   // ragged tail (this thread's last group)
  } else {
    for (size_t e = base + threadIdx.x; e < end; e += QTHREADS) one(e, out[e], __ldg(ref + e));
  }
  block_reduce3(sum, mx, nf, s_sum, s_mx, s_nf);
  if (threadIdx.x == 0) parts[seg] = QPart{sum, mx, nf};
}

// Sums nparts partials in a fixed order into *res (one block).
__global__ void __launch_bounds__(QTHREADS) quality_finalize_kernel(const QPart *__restrict__ parts,
                                                                     int nparts, QPart *res) {
  __shared__ double s_sum[QTHREADS / 32], s_mx[QTHREADS / 32];
  __shared__ unsigned long long s_nf[QTHREADS / 32];
  double sum = 0.0, mx = 0.0;
  unsigned long long nf = 0;
  for (int i = threadIdx.x; i < nparts; i += QTHREADS) {
    const QPart p = parts[i];
    sum = sum + p.sum;
    mx = p.mx > mx ? p.mx : mx;
    nf += p.nf;
  }
  block_reduce3(sum, mx, nf, s_sum, s_mx, s_nf);
  if (threadIdx.x == 0) *res = QPart{sum, mx, nf};
}

QSeg qseg(int64_t rows, int64_t cols) {
  QSeg q;
  const int64_t n = rows * cols;
  if (n <= 0) return QSeg{1, 1, 1};
  if (rows > 1) {   // whole rows: >= ~1024 elements per segment, <= QBLOCKS_MAX segments
    int64_t rps = (rows + QBLOCKS_MAX - 1) / QBLOCKS_MAX;
    const int64_t want = (1024 + cols - 1) / cols;
    if (rps < want) rps = want;
    if (rps > rows) rps = rows;
    q.rows_per = rps;
    q.per = rps * cols;
  } else {          // a vector: ~equal pieces of 4 * QTHREADS-element multiples
    int64_t nb = (n + (int64_t)QTHREADS * 4 - 1) / ((int64_t)QTHREADS * 4);
    if (nb > QBLOCKS_MAX) nb = QBLOCKS_MAX;
    int64_t per = (n + nb - 1) / nb;
    per = (per + 3) / 4 * 4;
    q.rows_per = 1;
    q.per = per;
  }
  q.nb = (int)((n + q.per - 1) / q.per);
  return q;
}

ps_status backconv_quality_async(const void *out, int out_type, const double *ref, float *delivered,
                                 int64_t rows, int64_t cols, QPart *parts, cudaStream_t st, int seg0,
                                 int seg1) {
  const QSeg q = qseg(rows, cols);
  if (seg1 < 0 || seg1 > q.nb) seg1 = q.nb;
  if (seg0 >= seg1) return PS_OK;
  const size_t n = (size_t)(rows * cols);
  auto go = [&](auto s) -> ps_status {
    using S = decltype(s);
    if (delivered)
      backconv_quality_kernel<S, true><<<seg1 - seg0, QTHREADS, 0, st>>>(
          (const raw_t<S> *)out, ref, delivered, n, (size_t)q.per, seg0, parts);
    else
      backconv_quality_kernel<S, false><<<seg1 - seg0, QTHREADS, 0, st>>>(
          (const raw_t<S> *)out, ref, nullptr, n, (size_t)q.per, seg0, parts);
    PS_CHECK_LAUNCH("backconv_quality_kernel");
    return PS_OK;
  };
  if (out_type == PS_E4M3) return go(E4M3());
  if (out_type == PS_E5M2) return go(E5M2());
  return dispatch_store(out_type, go);
}

ps_status quality_finalize_async(const QPart *parts, int nparts, QPart *res, cudaStream_t st) {
  quality_finalize_kernel<<<1, QTHREADS, 0, st>>>(parts, nparts, res);
  PS_CHECK_LAUNCH("quality_finalize_kernel");
  return PS_OK;
}

// ------------------------------------------- library-owned scratch (ps_quality)
namespace {
struct Scratch {
  QPart *dev = nullptr;
  QPart *host = nullptr;
  int device = -1;
};
thread_local Scratch g_scratch;
}  // namespace

static ps_status scratch_get(QPart **dev, QPart **host) {
  int d;
  PS_CUDA(cudaGetDevice(&d));
  if (g_scratch.dev && g_scratch.device != d) {
    cudaFree(g_scratch.dev);
    cudaFreeHost(g_scratch.host);
    g_scratch = Scratch{};
  }
  if (!g_scratch.dev) {
    PS_CUDA(cudaMalloc(&g_scratch.dev, sizeof(QPart) * (QBLOCKS_MAX + 1)));
    PS_CUDA(cudaMallocHost(&g_scratch.host, sizeof(QPart)));
    g_scratch.device = d;
  }
  *dev = g_scratch.dev;
  *host = g_scratch.host;
  return PS_OK;
}

}  // namespace ps

extern "C" ps_status ps_quality(const void *out, int out_type, const double *ref, size_t n,
                                int metric, void *stream, ps_quality_result *res) {
  using namespace ps;
  if (!dtype_ok(out_type) || (metric != PS_METRIC_MRE && metric != PS_METRIC_MAX_REL)) {
    set_error("ps_quality: bad dtype or metric");
    return PS_ERR_INVALID;
  }
  if (!res || (n && (!out || !ref))) {
    set_error("ps_quality: null pointer");
    return PS_ERR_INVALID;
  }
  QPart tot{0.0, 0.0, 0ull};
  if (n) {
    QPart *dev, *host;
    ps_status s = scratch_get(&dev, &host);
    if (s != PS_OK) return s;
    cudaStream_t st = (cudaStream_t)stream;
    s = backconv_quality_async(out, out_type, ref, nullptr, 1, (int64_t)n, dev + 1, st);
    if (s != PS_OK) return s;
    s = quality_finalize_async(dev + 1, qseg(1, (int64_t)n).nb, dev, st);
    if (s != PS_OK) return s;
    PS_CUDA(cudaMemcpyAsync(host, dev, sizeof(QPart), cudaMemcpyDeviceToHost, st));
    PS_CUDA(cudaStreamSynchronize(st));
    tot = *host;
  }
  res->n = n;
  res->mean_rel = n ? tot.sum / (double)n : 0.0;
  res->max_rel = tot.mx;
  res->nonfinite = tot.nf;
  res->quality = metric == PS_METRIC_MRE ? 1.0 - res->mean_rel
                                         : 1.0 - (tot.mx < 1.0 ? tot.mx : 1.0);
  return PS_OK;
}
