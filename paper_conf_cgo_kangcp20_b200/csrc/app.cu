// app.cu -- ps_app: memory objects + statements of the PolyBench-shaped apps,
// the configuration codec (a1), one-configuration evaluation ps_run_config
// (a2-a6) and the sweep ps_sweep (a7).
//
// Evaluation of one configuration on one stream, no host synchronisation:
//   ev0 | a2: each object read before written is converted orig(f32) -> c(m)
//       |     into its workspace slot (c(m) == f32 inputs are used in place)
//   ev1 | a3: statements in order; each picks its kernel from its compute type
//       |     T = W(objects touched, f32) (R2): tcgen05 for fp16 x fp16 -> f32
//       |     contractions, SIMT FFMA/DFMA otherwise, warp-shuffle mat-vec
//   ev2 | a4+a5: per output object one fused back-convert + error kernel
//   ev3 | a5: deterministic final reduction into this config's result slot
//   ev4
// A sweep enqueues a batch of configurations back to back and synchronises
// once; the host then turns the (sum e, max, count) triples into ps_result.
#include <math.h>
#include <stdarg.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <map>
#include <numeric>
#include <mutex>
#include <set>
#include <thread>
#include <tuple>
#include <vector>

#include "common.cuh"
#include "kernels.cuh"

namespace ps {

// ------------------------------------------------------------- errors
static thread_local char g_err[512] = "";
void set_error(const char *fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}
ps_status cuda_status(cudaError_t e, const char *what) {
  set_error("CUDA error %d (%s) in %s", (int)e, cudaGetErrorString(e), what);
  return PS_ERR_CUDA;
}
static std::atomic<uint64_t> g_launches{0};
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
int num_sms() {
  static int cached[64] = {0};
  int d = 0;
  cudaGetDevice(&d);
  if (d < 0 || d >= 64) return 148;
  if (!cached[d]) {
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    cached[d] = v > 0 ? v : 148;
  }
  return cached[d];
}

ps_status set_max_smem(const void *kernel, int bytes) {
  static std::mutex mu;
  static std::set<std::tuple<int, const void *, int>> done;
  int d = 0;
  PS_CUDA(cudaGetDevice(&d));
  const auto key = std::make_tuple(d, kernel, bytes);
  std::lock_guard<std::mutex> lk(mu);
  if (done.count(key)) return PS_OK;
  PS_CUDA(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
  done.insert(key);
  return PS_OK;
}

// ----------------------------------------------------------- app tables
struct ObjDef {
  const char *name;
  int role;       // 0 in, 1 out, 2 inout, 3 temp
  int is_output;  // delivered + scored
};
struct AppDef {
  const char *kind;
  int nobj;
  int ndims;
  ObjDef o[8];
};
// object order = configuration digit order
static const AppDef kApps[] = {
    {"gemm", 3, 3, {{"A", 0, 0}, {"B", 0, 0}, {"C", 2, 1}}},
    {"2mm", 5, 4, {{"A", 0, 0}, {"B", 0, 0}, {"C", 3, 0}, {"D", 0, 0}, {"E", 1, 1}}},
    {"3mm", 7, 5,
     {{"A", 0, 0}, {"B", 0, 0}, {"C", 0, 0}, {"D", 0, 0}, {"E", 3, 0}, {"F", 3, 0}, {"G", 1, 1}}},
    {"atax", 4, 2, {{"A", 0, 0}, {"x", 0, 0}, {"y", 1, 1}, {"tmp", 3, 0}}},
    {"bicg", 5, 2, {{"A", 0, 0}, {"r", 0, 0}, {"s", 1, 1}, {"p", 0, 0}, {"q", 1, 1}}},
    {"gesummv", 5, 1, {{"A", 0, 0}, {"B", 0, 0}, {"x", 0, 0}, {"y", 1, 1}, {"tmp", 3, 0}}},
    {"corr", 4, 2, {{"data", 2, 0}, {"mean", 3, 0}, {"stddev", 3, 0}, {"symmat", 1, 1}}},
    {"covar", 3, 2, {{"data", 2, 0}, {"mean", 3, 0}, {"symmat", 1, 1}}},
    {"mvt", 5, 1, {{"A", 0, 0}, {"x1", 2, 1}, {"x2", 2, 1}, {"y1", 0, 0}, {"y2", 0, 0}}},
    {"syrk", 2, 2, {{"A", 0, 0}, {"C", 2, 1}}},
    {"conv2d", 2, 2, {{"A", 0, 0}, {"B", 1, 1}}},
    {"syr2k", 3, 2, {{"A", 0, 0}, {"B", 0, 0}, {"C", 2, 1}}},
    {"conv3d", 2, 3, {{"A", 0, 0}, {"B", 1, 1}}},
    {"fdtd2d", 4, 3, {{"fict", 0, 0}, {"ex", 2, 1}, {"ey", 2, 1}, {"hz", 2, 1}}},
};
enum AppKind { K_GEMM, K_2MM, K_3MM, K_ATAX, K_BICG, K_GESUMMV, K_CORR, K_COVAR, K_MVT, K_SYRK,
               K_CONV2D, K_SYR2K, K_CONV3D, K_FDTD2D };
// statements that read or write each object (for ps_search's object order)
static const int kTouch[14][8] = {
    {1, 1, 1},                  // gemm: C <- aAB + bC
    {1, 1, 2, 1, 1},            // 2mm
    {1, 1, 1, 1, 2, 2, 1},      // 3mm
    {2, 1, 1, 2},               // atax
    {2, 1, 1, 1, 1},            // bicg
    {1, 1, 2, 2, 2},            // gesummv
    {4, 3, 2, 1},               // corr
    {3, 2, 1},                  // covar
    {2, 1, 1, 1, 1},            // mvt
    {1, 1},                     // syrk
    {1, 1},                     // conv2d
    {2, 2, 2},                  // syr2k
    {1, 1},                     // conv3d
    {1, 2, 3, 3},               // fdtd2d (per time step)
};

}  // namespace ps

using namespace ps;

static constexpr int MAX_BATCH = 4096;
static constexpr int NEV = 5;

// Pinned host staging of the host-side conversion methods (Fig. 3a/b/d/e).
struct XferScratch {
  static constexpr size_t CH = (size_t)4 << 20;   // pipeline chunk: 4 Mi elements
  void *pinned = nullptr;
  size_t bytes = 0;
  void *ring[2] = {nullptr, nullptr};
  cudaEvent_t ev[2] = {nullptr, nullptr};
  ps_status reserve(size_t need) {
    if (need > bytes) {
      if (pinned) cudaFreeHost(pinned);
      pinned = nullptr;
      bytes = 0;
      PS_CUDA(cudaMallocHost(&pinned, need));
      bytes = need;
    }
    if (!ring[0])
      for (int k = 0; k < 2; k++) {
        PS_CUDA(cudaMallocHost(&ring[k], CH * 8));
        PS_CUDA(cudaEventCreateWithFlags(&ev[k], cudaEventDisableTiming));
      }
    return PS_OK;
  }
  ~XferScratch() {
    if (pinned) cudaFreeHost(pinned);
    for (int k = 0; k < 2; k++) {
      if (ring[k]) cudaFreeHost(ring[k]);
      if (ev[k]) cudaEventDestroy(ev[k]);
    }
  }
};

// Moves one f32 host array of n elements to the device in precision dt with a
// Fig. 3 method.  Host methods (a, b, e) write dst directly; the device method
// (c) writes f32 into stage and the transient method (d) writes fp16 into
// stage -- the device-side conversion of those two is done by the caller (a2).
// Synchronous with respect to the host staging buffers.
static ps_status xfer_object(XferScratch &xs, const float *src, size_t n, int dt, int method,
                             int threads, void *dst, void *stage, cudaStream_t st) {
  const size_t es = dtype_size(dt);
  if (method == PS_XFER_DEVICE) {
    PS_CUDA(cudaMemcpyAsync(stage, src, n * 4, cudaMemcpyHostToDevice, st));
    return PS_OK;
  }
  ps_status s = xs.reserve(method == PS_XFER_TRANSIENT ? n * 2 : (method == PS_XFER_PIPELINE ? 0 : n * es));
  if (s != PS_OK) return s;
  if (method == PS_XFER_TRANSIENT) {             // (d) host -> fp16 intermediate
    ps::host_convert_f32(src, xs.pinned, PS_F16, n, threads, true);
    PS_CUDA(cudaMemcpyAsync(stage, xs.pinned, n * 2, cudaMemcpyHostToDevice, st));
    PS_CUDA(cudaStreamSynchronize(st));
  } else if (method == PS_XFER_PIPELINE) {       // (e) chunked conversion overlapped with H2D
    for (size_t c0 = 0, k = 0; c0 < n; c0 += XferScratch::CH, k++) {
      const int b = (int)(k & 1);
      const size_t len = std::min(XferScratch::CH, n - c0);
      PS_CUDA(cudaEventSynchronize(xs.ev[b]));  // the slot's previous copy has left the buffer
      ps::host_convert_f32(src + c0, xs.ring[b], dt, len, threads, true);
      PS_CUDA(cudaMemcpyAsync((char *)dst + c0 * es, xs.ring[b], len * es, cudaMemcpyHostToDevice, st));
      PS_CUDA(cudaEventRecord(xs.ev[b], st));
    }
  } else {                                       // (a) single loop / (b) multithreaded SIMD
    const bool simd = method == PS_XFER_HOST_SIMD;
    ps::host_convert_f32(src, xs.pinned, dt, n, simd ? threads : 1, simd);
    PS_CUDA(cudaMemcpyAsync(dst, xs.pinned, n * es, cudaMemcpyHostToDevice, st));
    PS_CUDA(cudaStreamSynchronize(st));          // the staging buffer is reused next
  }
  return PS_OK;
}

struct ps_app {
  const AppDef *def = nullptr;
  int kind = 0;
  int64_t d[5] = {0, 0, 0, 0, 0};
  int64_t rows[8] = {0}, cols[8] = {0};
  double sc[2] = {0, 0};
  uint32_t flags = 0;
  // binding
  char *ws = nullptr;
  size_t ws_bytes = 0;
  const float *orig_in[8] = {nullptr};
  float *orig_out[8] = {nullptr};
  const double *ref[8] = {nullptr};
  bool bound = false, has_ref = false;
  // workspace layout
  size_t slot_off[8] = {0};
  size_t partial_off = 0, qparts_off = 0, qres_off = 0, total = 0;
  size_t trans_off[8] = {0};
  // fp8 (PS_FLAG_FP8, reading #29): per object a staging region of n*8 bytes (the
  // object decoded into a statement's compute type), its ps_fp8_scale record,
  // and a vector scratch (MVT's split row-dot)
  size_t stage_off[8] = {0};
  size_t scale_off = 0, scratch_off = 0;
  // host-transfer path (ps_run_config_host): per input object, where a2 takes
  // its data from: 0 = orig_in (device conversion), 1 = already in the slot at
  // c(m) (host conversion + H2D), 2 = fp16 intermediate in the transient region
  int pre[8] = {0};
  XferScratch xs;                  // pinned host staging for the host methods
  // timing
  std::vector<cudaEvent_t> ev;
  QPart *host_res = nullptr;   // pinned, MAX_BATCH
  int device = -1;
  float shard_ms[4] = {0, 0, 0, 0};   // ps_shard_step: a2 / a3 / a4+a5 / finalize, summed over stages
  ~ps_app() {
    for (auto e : ev) cudaEventDestroy(e);
    if (host_res) cudaFreeHost(host_res);
  }
};

namespace {

size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

void shapes(ps_app *a) {
  const int64_t *d = a->d;
  for (int m = 0; m < 8; m++) a->rows[m] = a->cols[m] = 1;
  auto set = [&](int m, int64_t r, int64_t c) { a->rows[m] = r; a->cols[m] = c; };
  switch (a->kind) {
    case K_GEMM: set(0, d[0], d[2]); set(1, d[2], d[1]); set(2, d[0], d[1]); break;
    case K_2MM:
      set(0, d[0], d[2]); set(1, d[2], d[1]); set(2, d[0], d[1]); set(3, d[1], d[3]);
      set(4, d[0], d[3]);
      break;
    case K_3MM:
      set(0, d[0], d[2]); set(1, d[2], d[1]); set(2, d[1], d[4]); set(3, d[4], d[3]);
      set(4, d[0], d[1]); set(5, d[1], d[3]); set(6, d[0], d[3]);
      break;
    case K_ATAX: set(0, d[0], d[1]); set(1, 1, d[1]); set(2, 1, d[1]); set(3, 1, d[0]); break;
    case K_BICG:
      set(0, d[0], d[1]); set(1, 1, d[0]); set(2, 1, d[1]); set(3, 1, d[1]); set(4, 1, d[0]);
      break;
    case K_GESUMMV:
      set(0, d[0], d[0]); set(1, d[0], d[0]); set(2, 1, d[0]); set(3, 1, d[0]); set(4, 1, d[0]);
      break;
    case K_CORR: set(0, d[0], d[1]); set(1, 1, d[1]); set(2, 1, d[1]); set(3, d[1], d[1]); break;
    case K_COVAR: set(0, d[0], d[1]); set(1, 1, d[1]); set(2, d[1], d[1]); break;
    case K_MVT:
      set(0, d[0], d[0]); set(1, 1, d[0]); set(2, 1, d[0]); set(3, 1, d[0]); set(4, 1, d[0]);
      break;
    case K_SYRK: set(0, d[0], d[1]); set(1, d[1], d[1]); break;
    case K_CONV2D: set(0, d[0], d[1]); set(1, d[0], d[1]); break;
    case K_SYR2K: set(0, d[0], d[1]); set(1, d[0], d[1]); set(2, d[1], d[1]); break;
    case K_CONV3D: set(0, d[0], d[1] * d[2]); set(1, d[0], d[1] * d[2]); break;
    case K_FDTD2D: set(0, 1, d[0]); set(1, d[1], d[2]); set(2, d[1], d[2]); set(3, d[1], d[2]); break;
  }
}

size_t nelem(const ps_app *a, int m) { return (size_t)(a->rows[m] * a->cols[m]); }

void layout(ps_app *a) {
  size_t off = 0;
  for (int m = 0; m < a->def->nobj; m++) {
    a->slot_off[m] = off;
    off = align_up(off + nelem(a, m) * 8, 256);
  }
  size_t pb = 0;
  if (a->kind == K_ATAX || a->kind == K_BICG || a->kind == K_CORR || a->kind == K_COVAR)
    pb = tile_partial_bytes(a->d[0], a->d[1]);
  if (a->kind == K_GESUMMV || a->kind == K_MVT) pb = tile_partial_bytes(a->d[0], a->d[0]);
  a->partial_off = off;
  off = align_up(off + pb, 256);
  int nout = 0;
  for (int m = 0; m < a->def->nobj; m++) nout += a->def->o[m].is_output;
  a->qparts_off = off;
  off = align_up(off + (size_t)nout * QBLOCKS_MAX * sizeof(QPart), 256);
  a->qres_off = off;
  off = align_up(off + (size_t)MAX_BATCH * sizeof(QPart), 256);
  if (a->flags & PS_FLAG_FP8) {
    size_t vmax = 1;
    for (int m = 0; m < a->def->nobj; m++) {
      a->stage_off[m] = off;
      off = align_up(off + nelem(a, m) * 8, 256);
      vmax = std::max(vmax, (size_t)std::max(a->rows[m], a->cols[m]));
    }
    a->scale_off = off;
    off = align_up(off + 8 * sizeof(ps_fp8_scale), 256);
    a->scratch_off = off;
    off = align_up(off + vmax * 8, 256);
  }
  for (int m = 0; m < a->def->nobj; m++) {   // transient (fp16 intermediate) region per input
    a->trans_off[m] = off;
    if (a->def->o[m].role == 0 || a->def->o[m].role == 2) off = align_up(off + nelem(a, m) * 2, 256);
  }
  a->total = off;
}

// ----------------------------------------------------------- statements
struct Ctx {
  ps_app *a;
  int prec[8];      // current storage type of each object (fp8 objects: staged type inside a statement)
  void *ptr[8];
  cudaStream_t st;
  // row-sharded reference: only rows [r0, r1) of the scored output of a
  // contraction app are computed (r1 < 0: all rows); syrk-like outputs skip the mirror
  int64_t r0 = 0, r1 = -1;
  bool sharded() const { return r1 >= 0; }
};

inline void *eoff(const void *p, int type, int64_t n) {
  return (char *)p + n * (int64_t)dtype_size(type);
}

// ------------------------------------------------ fp8 staging (reading #29)
// An fp8 object lives in its slot as codes with a per-tensor scale.  A statement
// that touches it sees it "staged": decoded into its stage region in the
// statement's compute type T (exact: RNE_T(q * 2^k)), so every kernel family
// runs unchanged on f32/f64 storage; objects the statement writes are then
// re-quantised (amax -> k -> RNE_fp8(v * 2^-k)) back into their slots.  The
// tcgen05 fp8 contraction reads both multiplicands natively (`native` mask).
inline unsigned OBJ(int m) { return 1u << m; }
inline ps_fp8_scale *scale_of(const ps_app *a, int m) {
  return (ps_fp8_scale *)(a->ws + a->scale_off) + m;
}

template <class F>
ps_status stmt(Ctx &c, unsigned reads, unsigned writes, F &&body, unsigned native = 0) {
  ps_app *a = c.a;
  const unsigned touched = reads | writes;
  unsigned f8 = 0;
  int T = PS_F32;   // R2: widest touched precision, floored at f32 (fp8 codes are narrower)
  for (int m = 0; m < a->def->nobj; m++) {
    if (!(touched & OBJ(m))) continue;
    T = widest(T, c.prec[m]);
    if (is_fp8(c.prec[m]) && !(native & OBJ(m))) f8 |= OBJ(m);
  }
  if (!f8) return body();
  int q[8];
  void *slot[8];
  ps_status s;
  for (int m = 0; m < a->def->nobj; m++) {
    if (!(f8 & OBJ(m))) continue;
    q[m] = c.prec[m];
    slot[m] = c.ptr[m];
    void *stage = a->ws + a->stage_off[m];
    if (reads & OBJ(m))
      if ((s = fp8_decode_async(slot[m], q[m], stage, T, nelem(a, m), scale_of(a, m), c.st)) != PS_OK) return s;
    c.ptr[m] = stage;
    c.prec[m] = T;
  }
  s = body();
  for (int m = 0; m < a->def->nobj && s == PS_OK; m++) {
    if (!(f8 & OBJ(m))) continue;
    if (writes & OBJ(m)) s = fp8_encode_async(c.ptr[m], T, slot[m], q[m], nelem(a, m), scale_of(a, m), c.st);
    c.ptr[m] = slot[m];
    c.prec[m] = q[m];
  }
  return s;
}

ps_status contraction(Ctx &c, GemmArgs g) {
  // tcgen05: fp16 x fp16 or bf16 x bf16 (kind::f16), or fp8 x fp8 (kind::f8f6f4,
  // E4M3/E5M2 in any mix, reading #29); f32 compute
  const bool pair = (g.A.type == g.B.type && (g.A.type == PS_F16 || g.A.type == PS_BF16)) ||
                    (is_fp8(g.A.type) && is_fp8(g.B.type));
  // a row offset (sharded SYRK-like output) must keep the tile grid of the unsharded
  // statement: both tcgen05 kernels then compute identical tiles
  const bool tc = !(c.a->flags & PS_FLAG_NO_TENSOR_CORES) && pair && g.T == PS_F32 && g.row_off % 256 == 0 &&
                  gemm_tc_supported(g);
  if (!tc && (is_fp8(g.A.type) || is_fp8(g.B.type))) {
    set_error("internal: fp8 multiplicands reached the SIMT contraction");
    return PS_ERR_UNSUPPORTED;
  }
  return tc ? gemm_tc_async(g, c.st) : gemm_simt_async(g, c.st);
}

// native mask for a contraction X(.)Y -> out: both multiplicands fp8, T = f32 and the
// tensor-core path takes the shape; otherwise they are staged (SIMT, R3-exact)
unsigned tc8_native(Ctx &c, int x, int y, std::initializer_list<int> others, GemmArgs g) {
  if (!is_fp8(c.prec[x]) || !is_fp8(c.prec[y]) || (c.a->flags & PS_FLAG_NO_TENSOR_CORES) || c.sharded())
    return 0;
  int T = PS_F32;
  for (int m : others) T = widest(T, c.prec[m]);
  if (T != PS_F32) return 0;
  g.T = PS_F32;
  g.c_type = PS_F32;                 // the output is staged in f32 when it is fp8
  if (g.epi == EPI_AXPBY) g.cin_type = PS_F32;
  return gemm_tc_supported(g) ? (OBJ(x) | OBJ(y)) : 0;
}

// out(M x N, row-major) = X(M x K, row-major) . Y(K x N, row-major), R3;
// rows: restrict to the shard's output rows (X and out row-sliced)
GemmArgs matmul_args(Ctx &c, int x, int y, int out, int64_t M, int64_t N, int64_t K, bool rows) {
  const int64_t r0 = rows && c.sharded() ? c.r0 : 0;
  GemmArgs g{};
  g.M = rows && c.sharded() ? c.r1 - c.r0 : M; g.N = N; g.K = K;
  g.tc_m_full = M;
  g.A = MatDesc{eoff(c.ptr[x], c.prec[x], r0 * K), c.prec[x], K, 1, scale_of(c.a, x)};
  g.B = MatDesc{c.ptr[y], c.prec[y], N, 1, scale_of(c.a, y)};
  g.C = eoff(c.ptr[out], c.prec[out], r0 * N); g.c_type = c.prec[out]; g.ldc = N;
  g.epi = EPI_PLAIN;
  g.T = compute_type({c.prec[x], c.prec[y], c.prec[out]});
  return g;
}
ps_status matmul(Ctx &c, int x, int y, int out, int64_t M, int64_t N, int64_t K, bool rows = false) {
  const unsigned nat = tc8_native(c, x, y, {out}, matmul_args(c, x, y, out, M, N, K, rows));
  return stmt(c, OBJ(x) | OBJ(y), OBJ(out), [&]() -> ps_status {
    GemmArgs g = matmul_args(c, x, y, out, M, N, K, rows);
    return g.M > 0 ? contraction(c, g) : PS_OK;
  }, nat);
}

// symmat(M x M) = data^T data over N rows, upper tiles + mirror (R3).  Sharded: the
// upper part of rows [r0, r1) only; the mirror runs after the gather (reference_merge)
GemmArgs syrk_args(Ctx &c, int data, int sym, int64_t N, int64_t M, int epi, double div) {
  const int64_t r0 = c.sharded() ? c.r0 : 0;
  GemmArgs g{};
  g.M = c.sharded() ? c.r1 - c.r0 : M; g.N = M; g.K = N;
  g.tc_m_full = M;
  g.A = MatDesc{eoff(c.ptr[data], c.prec[data], r0), c.prec[data], 1, M, scale_of(c.a, data)};   // A(j1, i) = data[i][j1]
  g.B = MatDesc{c.ptr[data], c.prec[data], M, 1, scale_of(c.a, data)};                          // B(i, j2) = data[i][j2]
  g.C = eoff(c.ptr[sym], c.prec[sym], r0 * M); g.c_type = c.prec[sym]; g.ldc = M;
  g.epi = epi; g.div = div;
  if (epi == EPI_AXPBY) {   // SYRK app: C <- alpha data^T data + beta C (C read in place)
    g.Cin = g.C; g.cin_type = c.prec[sym];
    g.alpha = c.a->sc[0]; g.beta = c.a->sc[1];
  }
  g.upper_only = 1;
  g.row_off = r0;
  g.T = compute_type({c.prec[data], c.prec[sym]});
  return g;
}
ps_status syrk(Ctx &c, int data, int sym, int64_t N, int64_t M, int epi, double div, int diag_one) {
  const unsigned nat = tc8_native(c, data, data, {sym}, syrk_args(c, data, sym, N, M, epi, div));
  const unsigned reads = OBJ(data) | (epi == EPI_AXPBY ? OBJ(sym) : 0u);
  return stmt(c, reads, OBJ(sym), [&]() -> ps_status {
    GemmArgs g = syrk_args(c, data, sym, N, M, epi, div);
    if (g.M <= 0) return PS_OK;
    ps_status s = contraction(c, g);
    if (s != PS_OK || c.sharded()) return s;
    return mirror_async(c.ptr[sym], c.prec[sym], M, diag_one, c.st);
  }, nat);
}

GemmArgs gemm_args(Ctx &c) {   // C <- alpha (A.B) + beta C
  const int64_t *d = c.a->d;
  const int64_t r0 = c.sharded() ? c.r0 : 0;
  GemmArgs g{};
  g.M = c.sharded() ? c.r1 - c.r0 : d[0]; g.N = d[1]; g.K = d[2];
  g.tc_m_full = d[0];
  g.A = MatDesc{eoff(c.ptr[0], c.prec[0], r0 * d[2]), c.prec[0], d[2], 1, scale_of(c.a, 0)};
  g.B = MatDesc{c.ptr[1], c.prec[1], d[1], 1, scale_of(c.a, 1)};
  g.C = eoff(c.ptr[2], c.prec[2], r0 * d[1]); g.c_type = c.prec[2]; g.ldc = d[1];
  g.Cin = g.C; g.cin_type = c.prec[2];
  g.epi = EPI_AXPBY; g.alpha = c.a->sc[0]; g.beta = c.a->sc[1];
  g.T = compute_type({c.prec[0], c.prec[1], c.prec[2]});
  return g;
}

GemmArgs syr2k_args(Ctx &c, int s2) {   // C <- alpha X^T Y + beta C (s2 = 0: X=A, Y=B; 1: X=B, Y=A, beta 1)
  const int64_t N = c.a->d[0], M = c.a->d[1], r0 = c.sharded() ? c.r0 : 0;
  const int x = s2 ? 1 : 0, y = s2 ? 0 : 1;
  GemmArgs g{};
  g.M = c.sharded() ? c.r1 - c.r0 : M; g.N = M; g.K = N;
  g.tc_m_full = M;
  g.A = MatDesc{eoff(c.ptr[x], c.prec[x], r0), c.prec[x], 1, M, scale_of(c.a, x)};   // A(i, k) = X[k][i]
  g.B = MatDesc{c.ptr[y], c.prec[y], M, 1, scale_of(c.a, y)};                       // B(k, j) = Y[k][j]
  g.C = eoff(c.ptr[2], c.prec[2], r0 * M); g.c_type = c.prec[2]; g.ldc = M;
  g.Cin = g.C; g.cin_type = c.prec[2];
  g.epi = EPI_AXPBY; g.alpha = c.a->sc[0]; g.beta = s2 ? 1.0 : c.a->sc[1];
  g.T = compute_type({c.prec[0], c.prec[1], c.prec[2]});
  return g;
}

bool any_fp8(const Ctx &c, unsigned mask) {
  for (int m = 0; m < c.a->def->nobj; m++)
    if ((mask & OBJ(m)) && is_fp8(c.prec[m])) return true;
  return false;
}

ps_status run_statements(Ctx &c) {
  ps_app *a = c.a;
  const int64_t *d = a->d;
  const int *p = c.prec;     // current storage types (staged inside stmt bodies)
  void **P = c.ptr;
  void *partial = a->ws + a->partial_off;
  ps_status s = PS_OK;
#define S_(x)                      \
  do {                             \
    if ((s = (x)) != PS_OK) return s; \
  } while (0)
  switch (a->kind) {
    case K_GEMM: {   // C <- alpha (A.B) + beta C
      const unsigned nat = tc8_native(c, 0, 1, {2}, gemm_args(c));
      S_(stmt(c, OBJ(0) | OBJ(1) | OBJ(2), OBJ(2), [&]() -> ps_status {
        GemmArgs g = gemm_args(c);
        return g.M > 0 ? contraction(c, g) : PS_OK;
      }, nat));
      break;
    }
    case K_2MM:
      S_(matmul(c, 0, 1, 2, d[0], d[1], d[2], true));   // C <- A.B   (rows of E need rows of C)
      S_(matmul(c, 2, 3, 4, d[0], d[3], d[1], true));   // E <- C.D
      break;
    case K_3MM:
      S_(matmul(c, 0, 1, 4, d[0], d[1], d[2], true));   // E <- A.B   (rows of G need rows of E)
      S_(matmul(c, 2, 3, 5, d[1], d[3], d[4]));         // F <- C.D   (every row of F)
      S_(matmul(c, 4, 5, 6, d[0], d[3], d[1], true));   // G <- E.F
      break;
    case K_ATAX:   // tmp <- A x ; y <- A^T tmp
      S_(stmt(c, OBJ(0) | OBJ(1), OBJ(3), [&] {
        return rowdot_async(P[0], p[0], d[1], P[1], p[1], P[3], p[3], d[0], d[1], partial, c.st);
      }));
      S_(stmt(c, OBJ(0) | OBJ(3), OBJ(2), [&] {
        return colsum_async(P[0], p[0], d[1], P[3], p[3], P[2], p[2], d[0], d[1],
                            compute_type({p[0], p[3], p[2]}), COL_DOT, FIN_PLAIN, 0, 0, partial, c.st);
      }));
      break;
    case K_BICG:   // s <- A^T r ; q <- A p   (one pass over A)
      if (!any_fp8(c, 0x1Fu)) {
        S_(bicg_async(P[0], p[0], d[1], P[1], p[1], P[2], p[2], P[3], p[3], P[4], p[4], d[0], d[1],
                      partial, c.st));
      } else {   // fp8 objects: the two statements separately (each stages A in its own T)
        S_(stmt(c, OBJ(0) | OBJ(1), OBJ(2), [&] {
          return colsum_async(P[0], p[0], d[1], P[1], p[1], P[2], p[2], d[0], d[1],
                              compute_type({p[0], p[1], p[2]}), COL_DOT, FIN_PLAIN, 0, 0, partial, c.st);
        }));
        S_(stmt(c, OBJ(0) | OBJ(3), OBJ(4), [&] {
          return rowdot_async(P[0], p[0], d[1], P[3], p[3], P[4], p[4], d[0], d[1], partial, c.st);
        }));
      }
      break;
    case K_GESUMMV:   // tmp <- A x ; y <- B x ; y <- alpha tmp + beta y
      S_(stmt(c, OBJ(0) | OBJ(2), OBJ(4), [&] {
        return rowdot_async(P[0], p[0], d[0], P[2], p[2], P[4], p[4], d[0], d[0], partial, c.st);
      }));
      S_(stmt(c, OBJ(1) | OBJ(2), OBJ(3), [&] {
        return rowdot_async(P[1], p[1], d[0], P[2], p[2], P[3], p[3], d[0], d[0], partial, c.st);
      }));
      S_(stmt(c, OBJ(4) | OBJ(3), OBJ(3), [&] {
        return axpby_async(P[4], p[4], P[3], p[3], d[0], a->sc[0], a->sc[1], c.st);
      }));
      break;
    case K_CORR: {
      const double n = (double)d[0];
      S_(stmt(c, OBJ(0), OBJ(1), [&] {
        return colsum_async(P[0], p[0], d[1], nullptr, PS_F32, P[1], p[1], d[0], d[1],
                            compute_type({p[0], p[1]}), COL_SUM, FIN_MEAN, n, 0, partial, c.st);
      }));
      S_(stmt(c, OBJ(0) | OBJ(1), OBJ(2), [&] {
        return colsum_async(P[0], p[0], d[1], P[1], p[1], P[2], p[2], d[0], d[1],
                            compute_type({p[0], p[1], p[2]}), COL_SQDEV, FIN_STDDEV, n, a->sc[0],
                            partial, c.st);
      }));
      S_(stmt(c, OBJ(0) | OBJ(1) | OBJ(2), OBJ(0), [&] {
        return corr_normalize_async(P[0], p[0], P[1], p[1], P[2], p[2], d[0], d[1], sqrt(n), c.st);
      }));
      S_(syrk(c, 0, 3, d[0], d[1], EPI_PLAIN, 0.0, 1));
      break;
    }
    case K_COVAR: {
      const double n = (double)d[0];
      S_(stmt(c, OBJ(0), OBJ(1), [&] {
        return colsum_async(P[0], p[0], d[1], nullptr, PS_F32, P[1], p[1], d[0], d[1],
                            compute_type({p[0], p[1]}), COL_SUM, FIN_MEAN, n, 0, partial, c.st);
      }));
      S_(stmt(c, OBJ(0) | OBJ(1), OBJ(0), [&] {
        return covar_center_async(P[0], p[0], P[1], p[1], d[0], d[1], c.st);
      }));
      S_(syrk(c, 0, 2, d[0], d[1], EPI_DIV, n - 1.0, 0));
      break;
    }
    case K_MVT:   // x1 <- x1 + A y1 ; x2 <- x2 + A^T y2   (one pass over A)
      if (!any_fp8(c, 0x1Fu)) {
        S_(mvt_async(P[0], p[0], d[0], P[1], p[1], P[2], p[2], P[3], p[3], P[4], p[4], partial, c.st));
      } else {   // fp8 objects: row-dot into a T-typed scratch, x1 = fma(1, dot, 1 * x1); colsum + add
        void *scratch = a->ws + a->scratch_off;
        S_(stmt(c, OBJ(0) | OBJ(1) | OBJ(3), OBJ(1), [&] {
          const int T1 = compute_type({p[0], p[1], p[3]});
          ps_status e = rowdot_async(P[0], p[0], d[0], P[3], p[3], scratch, T1, d[0], d[0], partial, c.st);
          return e != PS_OK ? e : axpby_async(scratch, T1, P[1], p[1], d[0], 1.0, 1.0, c.st);
        }));
        S_(stmt(c, OBJ(0) | OBJ(2) | OBJ(4), OBJ(2), [&] {
          return colsum_async(P[0], p[0], d[0], P[4], p[4], P[2], p[2], d[0], d[0],
                              compute_type({p[0], p[2], p[4]}), COL_DOT, FIN_ADD, 0, 0, partial, c.st);
        }));
      }
      break;
    case K_SYRK:  // C <- alpha A^T A + beta C (upper tiles, mirrored)
      S_(syrk(c, 0, 1, d[0], d[1], EPI_AXPBY, 0.0, 0));
      break;
    case K_CONV2D:   // sharded: output rows [r0, r1) (ps_shard_step)
      S_(stmt(c, OBJ(0), OBJ(1), [&] {
        return c.sharded() ? conv2d_rows_async(P[0], p[0], P[1], p[1], d[0], d[1], c.r0, c.r1, c.st)
                           : conv2d_async(P[0], p[0], P[1], p[1], d[0], d[1], c.st);
      }));
      break;
    case K_SYR2K: {   // C <- alpha A^T B + beta C ; C <- alpha B^T A + C
      for (int s2 = 0; s2 < 2; s2++) {
        const unsigned nat = tc8_native(c, 0, 1, {2}, syr2k_args(c, s2));
        S_(stmt(c, OBJ(0) | OBJ(1) | OBJ(2), OBJ(2), [&]() -> ps_status {
          GemmArgs g = syr2k_args(c, s2);
          return g.M > 0 ? contraction(c, g) : PS_OK;
        }, nat));
      }
      break;
    }
    case K_CONV3D:   // sharded: output planes [r0, r1)
      S_(stmt(c, OBJ(0), OBJ(1), [&] {
        return c.sharded() ? conv3d_rows_async(P[0], p[0], P[1], p[1], d[0], d[1], d[2], c.r0, c.r1, c.st)
                           : conv3d_async(P[0], p[0], P[1], p[1], d[0], d[1], d[2], c.st);
      }));
      break;
    case K_FDTD2D: {
      // statements per step (reading #27); with fp8 objects the ey row-0 assignment and
      // the ey update are separate statements (reading #29), otherwise one fused pass
      const bool f8 = any_fp8(c, 0xFu);
      for (int64_t t = 0; t < d[0]; t++) {
        if (!f8) {
          S_(fdtd2d_part_async(FDTD_EY, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], d[2], c.st));
        } else {
          S_(stmt(c, OBJ(0) | OBJ(2), OBJ(2), [&] {
            return fdtd2d_part_async(FDTD_EY0, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], d[2], c.st);
          }));
          S_(stmt(c, OBJ(2) | OBJ(3), OBJ(2), [&] {
            return fdtd2d_part_async(FDTD_EY1, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], d[2], c.st);
          }));
        }
        S_(stmt(c, OBJ(1) | OBJ(3), OBJ(1), [&] {
          return fdtd2d_part_async(FDTD_EX, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], d[2], c.st);
        }));
        S_(stmt(c, OBJ(1) | OBJ(2) | OBJ(3), OBJ(3), [&] {
          return fdtd2d_part_async(FDTD_HZ, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], d[2], c.st);
        }));
      }
      break;
    }
  }
#undef S_
  return PS_OK;
}

// configuration alphabet: the paper's {f64, f32, f16}, + bf16 (PS_FLAG_BF16, reading #28),
// + bf16, e4m3, e5m2 (PS_FLAG_FP8, reading #29)
int radix(const ps_app *a) { return (a->flags & PS_FLAG_FP8) ? 6 : ((a->flags & PS_FLAG_BF16) ? 4 : 3); }

ps_status check_prec(const ps_app *a, const int *prec) {
  if (!prec) { set_error("null precision vector"); return PS_ERR_INVALID; }
  for (int m = 0; m < a->def->nobj; m++)
    if (!dtype_ok(prec[m]) || prec[m] >= radix(a)) {
      set_error("bad precision code %d for object %d (alphabet of %d)", prec[m], m, radix(a));
      return PS_ERR_INVALID;
    }
  return PS_OK;
}

ps_status ensure_events(ps_app *a, size_t n) {
  int dev;
  PS_CUDA(cudaGetDevice(&dev));
  if (a->device != dev) {
    for (auto e : a->ev) cudaEventDestroy(e);
    a->ev.clear();
    a->device = dev;
  }
  while (a->ev.size() < n) {
    cudaEvent_t e;
    PS_CUDA(cudaEventCreate(&e));
    a->ev.push_back(e);
  }
  if (!a->host_res) PS_CUDA(cudaMallocHost(&a->host_res, sizeof(QPart) * MAX_BATCH));
  return PS_OK;
}

// a2 .. a5 for one configuration; events ev[0..4] (nullptr = untimed); r1 >= 0: only
// rows [r0, r1) of the scored output (row-sharded reference, no quality)
ps_status enqueue_config(ps_app *a, const int *prec, cudaStream_t st, QPart *res,
                         cudaEvent_t *ev, bool quality, int64_t r0 = 0, int64_t r1 = -1) {
  Ctx c{a, {0}, {nullptr}, st};
  for (int m = 0; m < a->def->nobj; m++) c.prec[m] = prec[m];
  c.r0 = r0;
  c.r1 = r1;
  if (ev) PS_CUDA(cudaEventRecord(ev[0], st));
  for (int m = 0; m < a->def->nobj; m++) {
    c.ptr[m] = a->ws + a->slot_off[m];
    const int role = a->def->o[m].role;
    if (role == 0 || role == 2) {
      if (a->pre[m] == 1) {
        // host-converted and transferred at c(m) already (ps_run_config_host)
      } else if (a->pre[m] == 2) {   // transient: fp16 intermediate -> c(m) on the device
        ps_status s = convert_async(a->ws + a->trans_off[m], PS_F16, c.ptr[m], prec[m], nelem(a, m), st);
        if (s != PS_OK) return s;
      } else if (role == 0 && prec[m] == PS_F32) {
        c.ptr[m] = (void *)a->orig_in[m];   // original precision: used in place
      } else if (is_fp8(prec[m])) {         // reading #29: amax -> k -> codes
        ps_status s = fp8_encode_async(a->orig_in[m], PS_F32, c.ptr[m], prec[m], nelem(a, m), scale_of(a, m), st);
        if (s != PS_OK) return s;
      } else {
        ps_status s = convert_async(a->orig_in[m], PS_F32, c.ptr[m], prec[m], nelem(a, m), st);
        if (s != PS_OK) return s;
      }
    }
  }
  if (ev) PS_CUDA(cudaEventRecord(ev[1], st));
  ps_status s = run_statements(c);
  if (s != PS_OK) return s;
  if (ev) PS_CUDA(cudaEventRecord(ev[2], st));
  if (!quality) return PS_OK;
  QPart *parts = (QPart *)(a->ws + a->qparts_off);
  int np = 0;
  for (int m = 0; m < a->def->nobj; m++) {
    if (!a->def->o[m].is_output) continue;
    const void *out = c.ptr[m];
    int ot = prec[m];
    if (is_fp8(ot)) {   // reading #29: the exact values q * 2^k, then as an f64 object
      void *stage = a->ws + a->stage_off[m];
      s = fp8_decode_async(out, ot, stage, PS_F64, nelem(a, m), scale_of(a, m), st);
      if (s != PS_OK) return s;
      out = stage;
      ot = PS_F64;
    }
    s = backconv_quality_async(out, ot, a->ref[m], a->orig_out[m], a->rows[m], a->cols[m], parts + np, st);
    if (s != PS_OK) return s;
    np += qseg(a->rows[m], a->cols[m]).nb;
  }
  if (ev) PS_CUDA(cudaEventRecord(ev[3], st));
  s = quality_finalize_async(parts, np, res, st);
  if (s != PS_OK) return s;
  if (ev) PS_CUDA(cudaEventRecord(ev[4], st));
  return PS_OK;
}

uint64_t space(const ps_app *a) {
  uint64_t s = 1;
  for (int m = 0; m < a->def->nobj; m++) s *= (uint64_t)radix(a);
  return s;
}

void decode(const ps_app *a, uint64_t id, int *prec) {
  const uint64_t r = (uint64_t)radix(a);
  for (int m = 0; m < a->def->nobj; m++) { prec[m] = (int)(id % r); id /= r; }
}

uint64_t n_outputs(const ps_app *a) {
  uint64_t n = 0;
  for (int m = 0; m < a->def->nobj; m++)
    if (a->def->o[m].is_output) n += nelem(a, m);
  return n;
}

float ms_between(cudaEvent_t x, cudaEvent_t y) {
  float t = 0.f;
  if (cudaEventElapsedTime(&t, x, y) != cudaSuccess) return NAN;
  return t;
}

// the scored output whose rows a reference shard computes (-1: not shardable; the
// mat-vec and stencil references are single streaming passes, cheaper than a gather)
int shard_object(const ps_app *a) {
  switch (a->kind) {
    case K_GEMM: return 2;
    case K_2MM: return 4;
    case K_3MM: return 6;
    case K_SYRK: return 1;
    case K_SYR2K: return 2;
    case K_CORR: return 3;
    case K_COVAR: return 2;
    default: return -1;
  }
}
bool shard_triangular(const ps_app *a) {   // upper tiles + mirror: row i costs ~ (rows - i)
  return a->kind == K_SYRK || a->kind == K_CORR || a->kind == K_COVAR;
}

ps_status ready(const ps_app *a) {
  if (!a) { set_error("null app"); return PS_ERR_INVALID; }
  if (!a->bound) { set_error("app not bound (ps_app_bind)"); return PS_ERR_WORKSPACE; }
  if (!a->has_ref) { set_error("no reference (ps_app_reference)"); return PS_ERR_INVALID; }
  return PS_OK;
}

// ================================================ row-sharded evaluation (4b)
// SURVEY §8(e) "very large objects: contiguous row-range shards".  One
// configuration is evaluated by W ranks, each owning a contiguous range of the
// app's sharded rows; the stages below exchange exactly what the statements need
// (column-chunk partials, row blocks, quality segment partials) and every
// reduction keeps its single-GPU association, so the record and the delivered
// outputs are bit-identical to ps_run_config for every W.
enum ShardProg { SP_NONE, SP_ATAX, SP_BICG, SP_GESUMMV, SP_MVT, SP_ROWS, SP_3MM, SP_SYRK, SP_CORR, SP_COVAR,
                 SP_FDTD };

struct ShardGeo {
  int prog = SP_NONE;
  int64_t rows = 0;    // the sharded dimension
  int64_t align = 1;   // row bounds are multiples of this (except the last)
  bool tri = false;    // balance on the cost of upper-triangular rows
  int out = -1;        // the row-sharded scored output (-1: vector outputs, gathered)
};

ShardGeo shard_geo(const ps_app *a) {
  ShardGeo g;
  switch (a->kind) {
    case K_ATAX: g.prog = SP_ATAX; break;
    case K_BICG: g.prog = SP_BICG; break;
    case K_GESUMMV: g.prog = SP_GESUMMV; break;
    case K_MVT: g.prog = SP_MVT; break;
    case K_GEMM: case K_2MM: case K_SYR2K: case K_CONV2D: case K_CONV3D: g.prog = SP_ROWS; break;
    case K_3MM: g.prog = SP_3MM; break;
    case K_SYRK: g.prog = SP_SYRK; break;
    case K_CORR: g.prog = SP_CORR; break;
    case K_COVAR: g.prog = SP_COVAR; break;
    case K_FDTD2D:   // rows of ex / ey / hz; one-row halos exchanged twice per time step
      g.prog = SP_FDTD;
      g.rows = a->d[1];
      g.align = 1;
      return g;
    default: return g;
  }
  if (g.prog == SP_ATAX || g.prog == SP_BICG || g.prog == SP_GESUMMV || g.prog == SP_MVT) {
    g.rows = a->d[0];    // rows of A (and B)
    g.align = g.prog == SP_GESUMMV ? 1 : COLSUM_CHUNK;
    return g;
  }
  g.out = (a->kind == K_CONV2D || a->kind == K_CONV3D) ? 1 : shard_object(a);
  g.rows = a->rows[g.out];
  g.align = qseg(a->rows[g.out], a->cols[g.out]).rows_per;
  if (a->kind != K_CONV2D && a->kind != K_CONV3D)   // contractions: whole 256-row tcgen05 tiles
    g.align = std::lcm(g.align, (int64_t)256);
  g.tri = a->kind == K_SYRK || a->kind == K_CORR || a->kind == K_COVAR;
  return g;
}

// [r0, r1) of rank `rank` among `world`: contiguous, rounded to multiples of
// `align`; tri balances sum_{i in range} (rows - i)
void split_rows(int64_t rows, int world, int rank, int64_t align, bool tri, int64_t *r0, int64_t *r1) {
  auto cut = [&](int r) -> int64_t {
    if (r <= 0) return 0;
    if (r >= world) return rows;
    double b;
    if (!tri) {
      b = (double)rows * r / world;
    } else {   // b rows cost b*rows - b(b-1)/2 = target
      const double R = (double)rows, T = R * (R + 1) / 2.0 * r / world, q = 2 * R + 1;
      b = (q - sqrt(q * q - 8 * T)) / 2;
    }
    int64_t v = (int64_t)llround(b / (double)align) * align;
    return v < 0 ? 0 : (v > rows ? rows : v);
  };
  *r0 = cut(rank);
  *r1 = std::max(*r0, cut(rank + 1));
}

Ctx shard_ctx(ps_app *a, const int *prec, cudaStream_t st) {
  Ctx c{a, {0}, {nullptr}, st};
  for (int m = 0; m < a->def->nobj; m++) {
    c.prec[m] = prec[m];
    c.ptr[m] = (a->def->o[m].role == 0 && prec[m] == PS_F32) ? (void *)a->orig_in[m] : a->ws + a->slot_off[m];
  }
  return c;
}

// a2 for rows [r0, r1) of an input / inout object (r1 < 0: every row)
ps_status a2_rows(ps_app *a, Ctx &c, int m, int64_t r0 = 0, int64_t r1 = -1) {
  const int role = a->def->o[m].role;
  if (role != 0 && role != 2) return PS_OK;
  if (role == 0 && c.prec[m] == PS_F32) return PS_OK;   // used in place
  if (r1 < 0) r1 = a->rows[m];
  r0 = std::max<int64_t>(r0, 0);
  r1 = std::min<int64_t>(r1, a->rows[m]);
  if (r1 <= r0) return PS_OK;
  const int64_t cols = a->cols[m];
  return convert_async(a->orig_in[m] + r0 * cols, PS_F32, eoff(c.ptr[m], c.prec[m], r0 * cols), c.prec[m],
                       (size_t)((r1 - r0) * cols), c.st);
}

ps_shard_region row_region(ps_app *a, Ctx &c, int m, int64_t r0, int64_t r1) {
  const uint64_t rb = (uint64_t)a->cols[m] * dtype_size(c.prec[m]);
  return ps_shard_region{c.ptr[m], (uint64_t)r0 * rb, (uint64_t)(r1 - r0) * rb};
}
// elements [e0, e1) of a vector object (the row-dot outputs of the mat-vec apps)
ps_shard_region vec_region(Ctx &c, int m, int64_t e0, int64_t e1) {
  const uint64_t es = dtype_size(c.prec[m]);
  return ps_shard_region{c.ptr[m], (uint64_t)e0 * es, (uint64_t)(e1 - e0) * es};
}

// column-chunk partials of a rows-of-A shard: T-typed [nchunks][cols] at the
// workspace partial area; the shard's chunks start at chunk r0 / COLSUM_CHUNK
void *spart_at(ps_app *a, int T, int64_t r0, int64_t cols) {
  return a->ws + a->partial_off + (size_t)(r0 / COLSUM_CHUNK) * (size_t)cols * dtype_size(T);
}
void *qpart_of(ps_app *a, int64_t rows, int64_t cols) {
  return a->ws + a->partial_off + tile_spart_bytes(rows, cols);
}
ps_shard_region spart_region(ps_app *a, int T, int64_t r0, int64_t r1, int64_t cols) {
  const uint64_t cb = (uint64_t)cols * dtype_size(T);
  const uint64_t c0 = (uint64_t)(r0 / COLSUM_CHUNK), c1 = (uint64_t)((r1 + COLSUM_CHUNK - 1) / COLSUM_CHUNK);
  return ps_shard_region{a->ws + a->partial_off, c0 * cb, (c1 > c0 ? c1 - c0 : 0) * cb};
}

// a4 + a5 of every output over its full extent (vector outputs, present on every rank)
ps_status quality_all(ps_app *a, Ctx &c, QPart *res) {
  QPart *parts = (QPart *)(a->ws + a->qparts_off);
  int np = 0;
  for (int m = 0; m < a->def->nobj; m++) {
    if (!a->def->o[m].is_output) continue;
    PS_TRY(backconv_quality_async(c.ptr[m], c.prec[m], a->ref[m], a->orig_out[m], a->rows[m], a->cols[m],
                                  parts + np, c.st));
    np += qseg(a->rows[m], a->cols[m]).nb;
  }
  return quality_finalize_async(parts, np, res, c.st);
}

// a4 + a5 partials of rows [r0, r1) of the row-sharded output m (whole segments)
ps_status quality_rows(ps_app *a, Ctx &c, int m, int64_t r0, int64_t r1, ps_shard_region *reg) {
  QPart *parts = (QPart *)(a->ws + a->qparts_off);
  const QSeg q = qseg(a->rows[m], a->cols[m]);
  const int s0 = (int)(r0 / q.rows_per);
  const int s1 = r1 >= a->rows[m] ? q.nb : (int)(r1 / q.rows_per);
  *reg = ps_shard_region{parts, (uint64_t)s0 * sizeof(QPart), (uint64_t)(s1 > s0 ? s1 - s0 : 0) * sizeof(QPart)};
  if (s1 <= s0) return PS_OK;
  return backconv_quality_async(c.ptr[m], c.prec[m], a->ref[m], a->orig_out[m], a->rows[m], a->cols[m], parts,
                                c.st, s0, s1);
}
ps_status quality_rows_finalize(ps_app *a, int m, QPart *res, cudaStream_t st) {
  return quality_finalize_async((QPart *)(a->ws + a->qparts_off), qseg(a->rows[m], a->cols[m]).nb, res, st);
}
// every output row-sharded alike (FDTD-2D's ex, ey, hz): segment partials of rows
// [r0, r1) of each output at that output's offset in the partial array (the layout
// of enqueue_config), one exchange region per output
ps_status quality_rows_all(ps_app *a, Ctx &c, int64_t r0, int64_t r1, ps_shard_step_t *x) {
  QPart *parts = (QPart *)(a->ws + a->qparts_off);
  int np = 0;
  for (int m = 0; m < a->def->nobj; m++) {
    if (!a->def->o[m].is_output) continue;
    const QSeg q = qseg(a->rows[m], a->cols[m]);
    const int s0 = (int)(r0 / q.rows_per);
    const int s1 = r1 >= a->rows[m] ? q.nb : (int)(r1 / q.rows_per);
    x->region[x->nregions++] = ps_shard_region{parts, (uint64_t)(np + s0) * sizeof(QPart),
                                               (uint64_t)(s1 > s0 ? s1 - s0 : 0) * sizeof(QPart)};
    if (s1 > s0)
      PS_TRY(backconv_quality_async(c.ptr[m], c.prec[m], a->ref[m], a->orig_out[m], a->rows[m], a->cols[m],
                                    parts + np, c.st, s0, s1));
    np += q.nb;
  }
  return PS_OK;
}
int quality_parts_all(const ps_app *a) {
  int np = 0;
  for (int m = 0; m < a->def->nobj; m++)
    if (a->def->o[m].is_output) np += qseg(a->rows[m], a->cols[m]).nb;
  return np;
}

// One stage of the program; events ev[0..4] bracket a2 / statements / a4+a5 partials /
// finalize (as enqueue_config); *done when res holds the final quality.
ps_status shard_stage(ps_app *a, const int *prec, int rank, int world, int stage, cudaStream_t st,
                      cudaEvent_t *ev, QPart *res, ps_shard_step_t *x) {
  const ShardGeo g = shard_geo(a);
  const int64_t *d = a->d;
  Ctx c = shard_ctx(a, prec, st);
  const int *p = c.prec;
  void **P = c.ptr;
  int64_t r0, r1;
  split_rows(g.rows, world, rank, g.align, g.tri, &r0, &r1);
  x->done = 0;
  x->nregions = 0;
  auto region = [&](ps_shard_region r) { x->region[x->nregions++] = r; };
  auto rec = [&](int k) -> ps_status {
    PS_CUDA(cudaEventRecord(ev[k], st));
    return PS_OK;
  };
  const int last_rec = 4;
  (void)last_rec;
  switch (g.prog) {
    // ------------------------------------------------------------ mat-vec apps
    case SP_ATAX: {   // tmp <- A x (rows) ; y <- A^T tmp (chunk partials -> gather -> finalize)
      const int T2 = compute_type({p[0], p[3], p[2]});
      if (stage == 0) {
        PS_TRY(rec(0));
        PS_TRY(a2_rows(a, c, 0, r0, r1));
        PS_TRY(a2_rows(a, c, 1));
        PS_TRY(rec(1));
        if (r1 > r0) {
          PS_TRY(tile_rows_async(-1, eoff(P[0], p[0], r0 * d[1]), p[0], d[1], nullptr, PS_F32, P[1], p[1],
                                 eoff(P[3], p[3], r0), p[3], 0, r1 - r0, d[1], PS_F32, nullptr,
                                 qpart_of(a, d[0], d[1]), st));
          PS_TRY(tile_rows_async(COL_DOT, eoff(P[0], p[0], r0 * d[1]), p[0], d[1], eoff(P[3], p[3], r0), p[3],
                                 nullptr, PS_F32, nullptr, PS_F32, 0, r1 - r0, d[1], T2, spart_at(a, T2, r0, d[1]),
                                 qpart_of(a, d[0], d[1]), st));
        }
        PS_TRY(rec(2));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(spart_region(a, T2, r0, r1, d[1]));
        return PS_OK;
      }
      PS_TRY(rec(0));
      PS_TRY(rec(1));
      PS_TRY(colsum_finalize_async(a->ws + a->partial_off, T2, d[0], d[1], P[2], p[2], FIN_PLAIN, 0, 0, st));
      PS_TRY(rec(2));
      PS_TRY(quality_all(a, c, res));
      PS_TRY(rec(3));
      PS_TRY(rec(4));
      x->done = 1;
      return PS_OK;
    }
    case SP_BICG: {   // s <- A^T r (chunk partials) ; q <- A p (rows) -- one pass over the rows
      const int T1 = compute_type({p[0], p[1], p[2]});
      if (stage == 0) {
        PS_TRY(rec(0));
        PS_TRY(a2_rows(a, c, 0, r0, r1));
        PS_TRY(a2_rows(a, c, 1));
        PS_TRY(a2_rows(a, c, 3));
        PS_TRY(rec(1));
        if (r1 > r0)
          PS_TRY(tile_rows_async(COL_DOT, eoff(P[0], p[0], r0 * d[1]), p[0], d[1], eoff(P[1], p[1], r0), p[1],
                                 P[3], p[3], eoff(P[4], p[4], r0), p[4], 0, r1 - r0, d[1], T1,
                                 spart_at(a, T1, r0, d[1]), qpart_of(a, d[0], d[1]), st));
        PS_TRY(rec(2));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(spart_region(a, T1, r0, r1, d[1]));
        region(vec_region(c, 4, r0, r1));       // q

        return PS_OK;
      }
      PS_TRY(rec(0));
      PS_TRY(rec(1));
      PS_TRY(colsum_finalize_async(a->ws + a->partial_off, T1, d[0], d[1], P[2], p[2], FIN_PLAIN, 0, 0, st));
      PS_TRY(rec(2));
      PS_TRY(quality_all(a, c, res));
      PS_TRY(rec(3));
      PS_TRY(rec(4));
      x->done = 1;
      return PS_OK;
    }
    case SP_GESUMMV: {   // tmp, y rows of A x, B x; y <- alpha tmp + beta y (rows); gather y
      if (stage == 0) {
        PS_TRY(rec(0));
        PS_TRY(a2_rows(a, c, 0, r0, r1));
        PS_TRY(a2_rows(a, c, 1, r0, r1));
        PS_TRY(a2_rows(a, c, 2));
        PS_TRY(rec(1));
        if (r1 > r0) {
          PS_TRY(tile_rows_async(-1, eoff(P[0], p[0], r0 * d[0]), p[0], d[0], nullptr, PS_F32, P[2], p[2],
                                 eoff(P[4], p[4], r0), p[4], 0, r1 - r0, d[0], PS_F32, nullptr,
                                 qpart_of(a, d[0], d[0]), st));
          PS_TRY(tile_rows_async(-1, eoff(P[1], p[1], r0 * d[0]), p[1], d[0], nullptr, PS_F32, P[2], p[2],
                                 eoff(P[3], p[3], r0), p[3], 0, r1 - r0, d[0], PS_F32, nullptr,
                                 qpart_of(a, d[0], d[0]), st));
          PS_TRY(axpby_async(eoff(P[4], p[4], r0), p[4], eoff(P[3], p[3], r0), p[3], r1 - r0, a->sc[0], a->sc[1],
                             st));
        }
        PS_TRY(rec(2));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(vec_region(c, 3, r0, r1));       // y
        return PS_OK;
      }
      PS_TRY(rec(0));
      PS_TRY(rec(1));
      PS_TRY(rec(2));
      PS_TRY(quality_all(a, c, res));
      PS_TRY(rec(3));
      PS_TRY(rec(4));
      x->done = 1;
      return PS_OK;
    }
    case SP_MVT: {   // x1 <- x1 + A y1 (rows) ; x2 <- x2 + A^T y2 (chunk partials)
      const int TC = compute_type({p[0], p[2], p[4]});
      if (stage == 0) {
        PS_TRY(rec(0));
        PS_TRY(a2_rows(a, c, 0, r0, r1));
        for (int m = 1; m < 5; m++) PS_TRY(a2_rows(a, c, m));
        PS_TRY(rec(1));
        if (r1 > r0)
          PS_TRY(tile_rows_async(COL_DOT, eoff(P[0], p[0], r0 * d[0]), p[0], d[0], eoff(P[4], p[4], r0), p[4],
                                 P[3], p[3], eoff(P[1], p[1], r0), p[1], 1, r1 - r0, d[0], TC,
                                 spart_at(a, TC, r0, d[0]), qpart_of(a, d[0], d[0]), st));
        PS_TRY(rec(2));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(vec_region(c, 1, r0, r1));       // x1
        region(spart_region(a, TC, r0, r1, d[0]));
        return PS_OK;
      }
      PS_TRY(rec(0));
      PS_TRY(rec(1));
      PS_TRY(colsum_finalize_async(a->ws + a->partial_off, TC, d[0], d[0], P[2], p[2], FIN_ADD, 0, 0, st));
      PS_TRY(rec(2));
      PS_TRY(quality_all(a, c, res));
      PS_TRY(rec(3));
      PS_TRY(rec(4));
      x->done = 1;
      return PS_OK;
    }
    // ------------------------------------------- row-local contractions / stencils
    case SP_ROWS: {   // GEMM, 2MM, SYR2K, 2DCONV, 3DCONV: rows of the output need no exchange
      if (stage == 0) {
        PS_TRY(rec(0));
        switch (a->kind) {
          case K_GEMM: PS_TRY(a2_rows(a, c, 0, r0, r1)); PS_TRY(a2_rows(a, c, 1)); PS_TRY(a2_rows(a, c, 2, r0, r1)); break;
          case K_2MM: PS_TRY(a2_rows(a, c, 0, r0, r1)); PS_TRY(a2_rows(a, c, 1)); PS_TRY(a2_rows(a, c, 3)); break;
          case K_SYR2K: PS_TRY(a2_rows(a, c, 0)); PS_TRY(a2_rows(a, c, 1)); PS_TRY(a2_rows(a, c, 2, r0, r1)); break;
          default: PS_TRY(a2_rows(a, c, 0, r0 - 1, r1 + 1)); break;   // stencils: + one-row halo
        }
        PS_TRY(rec(1));
        c.r0 = r0;
        c.r1 = r1;
        if (r1 > r0) PS_TRY(run_statements(c));
        PS_TRY(rec(2));
        ps_shard_region q;
        PS_TRY(quality_rows(a, c, g.out, r0, r1, &q));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(q);
        return PS_OK;
      }
      PS_TRY(rec(0));
      PS_TRY(rec(1));
      PS_TRY(rec(2));
      PS_TRY(rec(3));
      PS_TRY(quality_rows_finalize(a, g.out, res, st));
      PS_TRY(rec(4));
      x->done = 1;
      return PS_OK;
    }
    case SP_3MM: {   // E rows (A rows) and F rows (own split) ; gather F ; G rows ; quality
      int64_t f0, f1;
      split_rows(d[1], world, rank, 256, false, &f0, &f1);
      if (stage == 0) {
        PS_TRY(rec(0));
        PS_TRY(a2_rows(a, c, 0, r0, r1));
        PS_TRY(a2_rows(a, c, 1));
        PS_TRY(a2_rows(a, c, 2, f0, f1));
        PS_TRY(a2_rows(a, c, 3));
        PS_TRY(rec(1));
        c.r0 = r0;
        c.r1 = r1;
        if (r1 > r0) PS_TRY(matmul(c, 0, 1, 4, d[0], d[1], d[2], true));   // E <- A.B
        c.r0 = f0;
        c.r1 = f1;
        if (f1 > f0) PS_TRY(matmul(c, 2, 3, 5, d[1], d[3], d[4], true));   // F <- C.D (rows f0..f1)
        PS_TRY(rec(2));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(row_region(a, c, 5, f0, f1));
        return PS_OK;
      }
      if (stage == 1) {
        PS_TRY(rec(0));
        PS_TRY(rec(1));
        c.r0 = r0;
        c.r1 = r1;
        if (r1 > r0) PS_TRY(matmul(c, 4, 5, 6, d[0], d[3], d[1], true));   // G <- E.F
        PS_TRY(rec(2));
        ps_shard_region q;
        PS_TRY(quality_rows(a, c, 6, r0, r1, &q));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(q);
        return PS_OK;
      }
      PS_TRY(rec(0));
      PS_TRY(rec(1));
      PS_TRY(rec(2));
      PS_TRY(rec(3));
      PS_TRY(quality_rows_finalize(a, 6, res, st));
      PS_TRY(rec(4));
      x->done = 1;
      return PS_OK;
    }
    // ---------------------------------------------- symmetric outputs (upper + mirror)
    case SP_SYRK:
    case SP_CORR:
    case SP_COVAR: {
      const int sym = g.out;
      const int data_stages = g.prog == SP_SYRK ? 0 : (g.prog == SP_CORR ? 3 : 2);
      const int64_t N = d[0], M = d[1];
      int64_t d0, d1;   // data rows (CORR / COVAR column statistics)
      split_rows(N, world, rank, COLSUM_CHUNK, false, &d0, &d1);
      const int T1 = compute_type({p[0], p[1]});                                  // mean
      const int T2 = g.prog == SP_CORR ? compute_type({p[0], p[1], p[2]}) : T1;    // stddev / normalise
      PS_TRY(rec(0));
      if (stage == 0 && g.prog != SP_SYRK) {   // a2 of the data rows, mean partials
        PS_TRY(a2_rows(a, c, 0, d0, d1));
        PS_TRY(rec(1));
        if (d1 > d0)
          PS_TRY(tile_rows_async(COL_SUM, eoff(P[0], p[0], d0 * M), p[0], M, nullptr, PS_F32, nullptr, PS_F32,
                                 nullptr, PS_F32, 0, d1 - d0, M, T1, spart_at(a, T1, d0, M), qpart_of(a, N, M), st));
        region(spart_region(a, T1, d0, d1, M));
      } else if (stage == 1 && g.prog == SP_CORR) {   // mean; stddev partials
        PS_TRY(rec(1));
        PS_TRY(colsum_finalize_async(a->ws + a->partial_off, T1, N, M, P[1], p[1], FIN_MEAN, (double)N, 0, st));
        if (d1 > d0)
          PS_TRY(tile_rows_async(COL_SQDEV, eoff(P[0], p[0], d0 * M), p[0], M, P[1], p[1], nullptr, PS_F32,
                                 nullptr, PS_F32, 0, d1 - d0, M, T2, spart_at(a, T2, d0, M), qpart_of(a, N, M), st));
        region(spart_region(a, T2, d0, d1, M));
      } else if (stage == data_stages - 1 && g.prog != SP_SYRK) {   // finish stats, normalise rows
        PS_TRY(rec(1));
        if (g.prog == SP_CORR) {
          PS_TRY(colsum_finalize_async(a->ws + a->partial_off, T2, N, M, P[2], p[2], FIN_STDDEV, (double)N,
                                       a->sc[0], st));
          if (d1 > d0)
            PS_TRY(corr_normalize_async(eoff(P[0], p[0], d0 * M), p[0], P[1], p[1], P[2], p[2], d1 - d0, M,
                                        sqrt((double)N), st));
        } else {
          PS_TRY(colsum_finalize_async(a->ws + a->partial_off, T1, N, M, P[1], p[1], FIN_MEAN, (double)N, 0, st));
          if (d1 > d0) PS_TRY(covar_center_async(eoff(P[0], p[0], d0 * M), p[0], P[1], p[1], d1 - d0, M, st));
        }
        region(row_region(a, c, 0, d0, d1));
      } else if (stage == data_stages) {   // upper part of the output rows
        if (g.prog == SP_SYRK) {
          PS_TRY(a2_rows(a, c, 0));
          PS_TRY(a2_rows(a, c, 1, r0, r1));
        }
        PS_TRY(rec(1));
        c.r0 = r0;
        c.r1 = r1;
        if (r1 > r0) {
          if (g.prog == SP_SYRK) PS_TRY(syrk(c, 0, 1, N, M, EPI_AXPBY, 0.0, 0));
          else if (g.prog == SP_CORR) PS_TRY(syrk(c, 0, 3, N, M, EPI_PLAIN, 0.0, 1));
          else PS_TRY(syrk(c, 0, 2, N, M, EPI_DIV, (double)N - 1.0, 0));
        }
        region(row_region(a, c, sym, r0, r1));
      } else if (stage == data_stages + 1) {   // mirror, quality partials of the rows
        PS_TRY(rec(1));
        PS_TRY(mirror_async(P[sym], p[sym], M, g.prog == SP_CORR ? 1 : 0, st));
        PS_TRY(rec(2));
        ps_shard_region q;
        PS_TRY(quality_rows(a, c, sym, r0, r1, &q));
        PS_TRY(rec(3));
        PS_TRY(rec(4));
        region(q);
        return PS_OK;
      } else {
        PS_TRY(rec(1));
        PS_TRY(rec(2));
        PS_TRY(rec(3));
        PS_TRY(quality_rows_finalize(a, sym, res, st));
        PS_TRY(rec(4));
        x->done = 1;
        return PS_OK;
      }
      PS_TRY(rec(2));
      PS_TRY(rec(3));
      PS_TRY(rec(4));
      return PS_OK;
    }
  }
  if (g.prog == SP_FDTD) {   // FDTD-2D: per time step two stages, then quality
    const int64_t TM = d[0], NX = d[1], NY = d[2];
    (void)NX;
    auto row1 = [&](int m, int64_t r) {   // one row of object m (a halo row for a neighbour)
      return (r0 < r1) ? row_region(a, c, m, r, r + 1) : ps_shard_region{c.ptr[m], 0, 0};
    };
    if (stage < 2 * TM) {
      const int64_t t = stage / 2;
      PS_TRY(rec(0));
      if (stage == 0) {   // a2: fict whole, the rows of ex / ey / hz with a one-row halo
        PS_TRY(a2_rows(a, c, 0));
        for (int m = 1; m <= 3; m++) PS_TRY(a2_rows(a, c, m, r0 - 1, r1 + 1));
      }
      PS_TRY(rec(1));
      if (stage % 2 == 0) {   // ey (row 0 from fict, rows >= 1 need hz[i-1]: halo r0 - 1), ex
        PS_TRY(fdtd2d_part_async(FDTD_EY, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], NY, st, r0, r1));
        PS_TRY(fdtd2d_part_async(FDTD_EX, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], NY, st, r0, r1));
        region(row1(2, r0));          // my first ey row: the previous rank's hz needs ey[i+1]
      } else {                        // hz (needs ey[i+1]: halo r1)
        PS_TRY(fdtd2d_part_async(FDTD_HZ, P[0], p[0], P[1], p[1], P[2], p[2], P[3], p[3], t, d[1], NY, st, r0, r1));
        region(row1(3, r1 - 1));      // my last hz row: the next rank's ey needs hz[i-1]
      }
      PS_TRY(rec(2));
      PS_TRY(rec(3));
      PS_TRY(rec(4));
      return PS_OK;
    }
    if (stage == 2 * TM) {
      PS_TRY(rec(0));
      PS_TRY(rec(1));
      PS_TRY(rec(2));
      PS_TRY(quality_rows_all(a, c, r0, r1, x));
      PS_TRY(rec(3));
      PS_TRY(rec(4));
      return PS_OK;
    }
    PS_TRY(rec(0));
    PS_TRY(rec(1));
    PS_TRY(rec(2));
    PS_TRY(rec(3));
    PS_TRY(quality_finalize_async((QPart *)(a->ws + a->qparts_off), quality_parts_all(a), res, st));
    PS_TRY(rec(4));
    x->done = 1;
    return PS_OK;
  }
  set_error("ps_shard_step: %s has no row-sharded evaluation", a->def->kind);
  return PS_ERR_UNSUPPORTED;
}

}  // namespace

// ===================================================================== ABI
extern "C" {

const char *ps_status_string(int s) {
  switch (s) {
    case PS_OK: return "ok";
    case PS_ERR_INVALID: return "invalid argument";
    case PS_ERR_UNSUPPORTED: return "unsupported";
    case PS_ERR_CUDA: return "cuda error";
    case PS_ERR_WORKSPACE: return "workspace missing or too small";
  }
  return "unknown status";
}
const char *ps_last_error(void) { return g_err; }
const char *ps_version(void) { return "prescaler-b200 0.1 (sm_100a)"; }
uint64_t ps_kernel_launches(void) { return g_launches.load(); }

ps_status ps_app_create(const char *kind, const int64_t *dims, int ndims, const double *scalars,
                        ps_app **out) {
  if (!kind || !dims || !out) { set_error("ps_app_create: null pointer"); return PS_ERR_INVALID; }
  const AppDef *def = nullptr;
  int k = 0;
  for (size_t i = 0; i < sizeof(kApps) / sizeof(kApps[0]); i++)
    if (!strcmp(kApps[i].kind, kind)) { def = &kApps[i]; k = (int)i; }
  if (!def) { set_error("ps_app_create: unknown app '%s'", kind); return PS_ERR_UNSUPPORTED; }
  if (ndims != 1 && ndims != def->ndims) {
    set_error("ps_app_create: %s takes 1 or %d dims, got %d", kind, def->ndims, ndims);
    return PS_ERR_INVALID;
  }
  ps_app *a = new ps_app();
  a->def = def;
  a->kind = k;
  for (int i = 0; i < def->ndims; i++) {
    a->d[i] = ndims == 1 ? dims[0] : dims[i];
    if (a->d[i] <= 0 || a->d[i] > (int64_t)1 << 31) {
      delete a;
      set_error("ps_app_create: dimension out of range");
      return PS_ERR_UNSUPPORTED;
    }
  }
  if (k == K_GEMM) { a->sc[0] = 32412.0; a->sc[1] = 2123.0; }
  if (k == K_GESUMMV) { a->sc[0] = 43532.0; a->sc[1] = 12313.0; }
  if (k == K_CORR) { a->sc[0] = 0.005; }
  if (k == K_SYRK || k == K_SYR2K) { a->sc[0] = 32412.0; a->sc[1] = 2123.0; }
  if (scalars) {
    if (k == K_GEMM || k == K_GESUMMV || k == K_SYRK || k == K_SYR2K) {
      a->sc[0] = scalars[0];
      a->sc[1] = scalars[1];
    }
    if (k == K_CORR) a->sc[0] = scalars[0];
  }
  shapes(a);
  layout(a);
  *out = a;
  return PS_OK;
}

ps_status ps_app_destroy(ps_app *a) {
  delete a;
  return PS_OK;
}

int ps_app_num_objects(const ps_app *a) { return a ? a->def->nobj : -1; }

ps_status ps_app_object_info(const ps_app *a, int m, ps_object_info *out) {
  if (!a || !out || m < 0 || m >= a->def->nobj) { set_error("ps_app_object_info: bad argument"); return PS_ERR_INVALID; }
  out->name = a->def->o[m].name;
  out->rows = a->rows[m];
  out->cols = a->cols[m];
  out->n = (uint64_t)nelem(a, m);
  out->orig = PS_F32;
  out->role = a->def->o[m].role;
  out->is_output = a->def->o[m].is_output;
  out->reserved = 0;
  return PS_OK;
}

ps_status ps_app_set_flags(ps_app *a, uint32_t flags) {
  if (!a) { set_error("null app"); return PS_ERR_INVALID; }
  if (a->bound && ((flags ^ a->flags) & PS_FLAG_FP8)) {
    set_error("ps_app_set_flags: PS_FLAG_FP8 changes the workspace layout; set it before ps_app_bind");
    return PS_ERR_INVALID;
  }
  a->flags = flags;
  layout(a);
  return PS_OK;
}

size_t ps_app_workspace_bytes(const ps_app *a) { return a ? a->total : 0; }

ps_status ps_app_bind(ps_app *a, void *ws, size_t bytes, void *const *in, void *const *out) {
  if (!a || !in || !out) { set_error("ps_app_bind: null pointer"); return PS_ERR_INVALID; }
  if (!ws || bytes < a->total || ((uintptr_t)ws % 256)) {
    set_error("ps_app_bind: workspace needs %zu bytes, 256-aligned", a->total);
    return PS_ERR_WORKSPACE;
  }
  for (int m = 0; m < a->def->nobj; m++) {
    const int role = a->def->o[m].role;
    if ((role == 0 || role == 2) && !in[m]) { set_error("ps_app_bind: input %d missing", m); return PS_ERR_INVALID; }
    if (a->def->o[m].is_output && !out[m]) { set_error("ps_app_bind: output %d missing", m); return PS_ERR_INVALID; }
    a->orig_in[m] = (role == 0 || role == 2) ? (const float *)in[m] : nullptr;
    a->orig_out[m] = a->def->o[m].is_output ? (float *)out[m] : nullptr;
  }
  a->ws = (char *)ws;
  a->ws_bytes = bytes;
  a->bound = true;
  return PS_OK;
}

ps_status ps_app_load_host(ps_app *a, const void *const *host, void *stream) {
  if (!a || !host) { set_error("ps_app_load_host: null pointer"); return PS_ERR_INVALID; }
  if (!a->bound) { set_error("ps_app_load_host: app not bound"); return PS_ERR_WORKSPACE; }
  for (int m = 0; m < a->def->nobj; m++) {
    if (!a->orig_in[m]) continue;
    if (!host[m]) { set_error("ps_app_load_host: host input %d missing", m); return PS_ERR_INVALID; }
    PS_CUDA(cudaMemcpyAsync((void *)a->orig_in[m], host[m], nelem(a, m) * sizeof(float),
                            cudaMemcpyHostToDevice, (cudaStream_t)stream));
  }
  return PS_OK;
}

ps_status ps_app_reference(ps_app *a, double *const *ref, void *stream) {
  if (!a || !ref) { set_error("ps_app_reference: null pointer"); return PS_ERR_INVALID; }
  if (!a->bound) { set_error("ps_app_reference: app not bound"); return PS_ERR_WORKSPACE; }
  cudaStream_t st = (cudaStream_t)stream;
  int prec[8] = {0};   // all f64 = configuration id 0
  ps_status s = enqueue_config(a, prec, st, nullptr, nullptr, false);
  if (s != PS_OK) return s;
  for (int m = 0; m < a->def->nobj; m++) {
    if (!a->def->o[m].is_output) continue;
    if (!ref[m]) { set_error("ps_app_reference: ref %d missing", m); return PS_ERR_INVALID; }
    PS_CUDA(cudaMemcpyAsync(ref[m], a->ws + a->slot_off[m], nelem(a, m) * 8,
                            cudaMemcpyDeviceToDevice, st));
    a->ref[m] = ref[m];
  }
  PS_CUDA(cudaStreamSynchronize(st));
  a->has_ref = true;
  return PS_OK;
}

int64_t ps_app_shard_rows(const ps_app *a) {
  if (!a) return 0;
  const int m = shard_object(a);
  return m < 0 ? 0 : a->rows[m];
}

int ps_app_shard_triangular(const ps_app *a) { return a && shard_object(a) >= 0 && shard_triangular(a); }

ps_status ps_app_reference_rows(ps_app *a, int64_t row0, int64_t row1, double *const *ref, void *stream) {
  if (!a || !ref) { set_error("ps_app_reference_rows: null pointer"); return PS_ERR_INVALID; }
  if (!a->bound) { set_error("ps_app_reference_rows: app not bound"); return PS_ERR_WORKSPACE; }
  const int m = shard_object(a);
  if (m < 0) { set_error("ps_app_reference_rows: %s is not row-shardable", a->def->kind); return PS_ERR_UNSUPPORTED; }
  if (row0 < 0 || row1 < row0 || row1 > a->rows[m]) {
    set_error("ps_app_reference_rows: rows [%lld, %lld) outside [0, %lld)", (long long)row0,
              (long long)row1, (long long)a->rows[m]);
    return PS_ERR_INVALID;
  }
  if (!ref[m]) { set_error("ps_app_reference_rows: ref %d missing", m); return PS_ERR_INVALID; }
  cudaStream_t st = (cudaStream_t)stream;
  int prec[8] = {0};   // all f64 = configuration id 0
  ps_status s = enqueue_config(a, prec, st, nullptr, nullptr, false, row0, row1);
  if (s != PS_OK) return s;
  const int64_t cols = a->cols[m];
  if (row1 > row0)
    PS_CUDA(cudaMemcpyAsync(ref[m] + row0 * cols, (const double *)(a->ws + a->slot_off[m]) + row0 * cols,
                            (size_t)((row1 - row0) * cols) * 8, cudaMemcpyDeviceToDevice, st));
  PS_CUDA(cudaStreamSynchronize(st));
  return PS_OK;
}

ps_status ps_app_reference_merge(ps_app *a, double *const *ref, void *stream) {
  if (!a || !ref) { set_error("ps_app_reference_merge: null pointer"); return PS_ERR_INVALID; }
  const int m = shard_object(a);
  if (m < 0) { set_error("ps_app_reference_merge: %s is not row-shardable", a->def->kind); return PS_ERR_UNSUPPORTED; }
  if (!ref[m]) { set_error("ps_app_reference_merge: ref %d missing", m); return PS_ERR_INVALID; }
  cudaStream_t st = (cudaStream_t)stream;
  if (shard_triangular(a)) {
    ps_status s = mirror_async(ref[m], PS_F64, a->rows[m], a->kind == K_CORR ? 1 : 0, st);
    if (s != PS_OK) return s;
  }
  PS_CUDA(cudaStreamSynchronize(st));
  a->ref[m] = ref[m];
  a->has_ref = true;
  return PS_OK;
}

ps_status ps_app_set_reference(ps_app *a, const double *const *ref) {
  if (!a || !ref) { set_error("ps_app_set_reference: null pointer"); return PS_ERR_INVALID; }
  for (int m = 0; m < a->def->nobj; m++) {
    if (!a->def->o[m].is_output) continue;
    if (!ref[m]) { set_error("ps_app_set_reference: ref %d missing", m); return PS_ERR_INVALID; }
    a->ref[m] = ref[m];
  }
  a->has_ref = true;
  return PS_OK;
}

ps_status ps_config_encode(const ps_app *a, const int *prec, uint64_t *id) {
  if (!a || !id) { set_error("ps_config_encode: null pointer"); return PS_ERR_INVALID; }
  ps_status s = check_prec(a, prec);
  if (s != PS_OK) return s;
  uint64_t v = 0, w = 1;
  for (int m = 0; m < a->def->nobj; m++) { v += (uint64_t)prec[m] * w; w *= (uint64_t)radix(a); }
  *id = v;
  return PS_OK;
}

ps_status ps_config_decode(const ps_app *a, uint64_t id, int *prec) {
  if (!a || !prec) { set_error("ps_config_decode: null pointer"); return PS_ERR_INVALID; }
  if (id >= space(a)) {
    set_error("ps_config_decode: id %llu >= %d^%d", (unsigned long long)id, radix(a), a->def->nobj);
    return PS_ERR_INVALID;
  }
  decode(a, id, prec);
  return PS_OK;
}

static void fill_result(const ps_app *a, uint64_t id, const QPart &q, cudaEvent_t *ev, double toq,
                        ps_result *r) {
  const double n = (double)n_outputs(a);
  memset(r, 0, sizeof(*r));
  r->config_id = id;
  r->convert_ms = ms_between(ev[0], ev[1]);
  r->kernel_ms = ms_between(ev[1], ev[2]);
  r->backconv_ms = ms_between(ev[2], ev[3]);
  r->quality_ms = ms_between(ev[3], ev[4]);
  r->total_ms = r->convert_ms + r->kernel_ms + r->backconv_ms;
  r->quality = 1.0 - q.sum / n;
  r->max_rel = q.mx;
  r->nonfinite = q.nf;
  r->pass = r->quality >= toq;   // Alg. 1 l.10: fail iff Accuracy < TOQ
  r->status = PS_OK;
}

ps_status ps_run_config(ps_app *a, const int *prec, double toq, void *stream, ps_result *out) {
  ps_status s = ready(a);
  if (s != PS_OK) return s;
  if ((s = check_prec(a, prec)) != PS_OK) return s;
  if ((s = ensure_events(a, NEV)) != PS_OK) return s;
  cudaStream_t st = (cudaStream_t)stream;
  QPart *res = (QPart *)(a->ws + a->qres_off);
  s = enqueue_config(a, prec, st, res, out ? a->ev.data() : nullptr, true);
  if (s != PS_OK) return s;
  if (!out) return PS_OK;
  PS_CUDA(cudaMemcpyAsync(a->host_res, res, sizeof(QPart), cudaMemcpyDeviceToHost, st));
  PS_CUDA(cudaStreamSynchronize(st));
  uint64_t id = 0;
  ps_config_encode(a, prec, &id);
  fill_result(a, id, a->host_res[0], a->ev.data(), toq, out);
  return PS_OK;
}

ps_status ps_sweep(ps_app *a, const uint64_t *ids, size_t n, double toq, void *stream,
                   ps_result *results, int64_t *best) {
  ps_status s = ready(a);
  if (s != PS_OK) return s;
  if ((n && (!ids || !results)) || !best) { set_error("ps_sweep: null pointer"); return PS_ERR_INVALID; }
  const uint64_t sp = space(a);
  for (size_t i = 0; i < n; i++)
    if (ids[i] >= sp) { set_error("ps_sweep: config id %llu out of range", (unsigned long long)ids[i]); return PS_ERR_INVALID; }
  cudaStream_t st = (cudaStream_t)stream;
  QPart *res = (QPart *)(a->ws + a->qres_off);
  *best = -1;
  for (size_t b0 = 0; b0 < n; b0 += MAX_BATCH) {
    const size_t nb = std::min((size_t)MAX_BATCH, n - b0);
    if ((s = ensure_events(a, nb * NEV)) != PS_OK) return s;
    for (size_t i = 0; i < nb; i++) {
      int prec[8];
      decode(a, ids[b0 + i], prec);
      s = enqueue_config(a, prec, st, res + i, a->ev.data() + i * NEV, true);
      if (s != PS_OK) return s;
    }
    PS_CUDA(cudaMemcpyAsync(a->host_res, res, sizeof(QPart) * nb, cudaMemcpyDeviceToHost, st));
    PS_CUDA(cudaStreamSynchronize(st));
    for (size_t i = 0; i < nb; i++)
      fill_result(a, ids[b0 + i], a->host_res[i], a->ev.data() + i * NEV, toq, &results[b0 + i]);
  }
  for (size_t i = 0; i < n; i++) {
    if (!results[i].pass) continue;
    if (*best < 0 || results[i].total_ms < results[*best].total_ms ||
        (results[i].total_ms == results[*best].total_ms && results[i].config_id < results[*best].config_id))
      *best = (int64_t)i;
  }
  return PS_OK;
}

ps_status ps_host_convert(const float *src, void *dst, int dst_type, size_t n, int threads, int simd) {
  if (!dtype_ok(dst_type) || is_fp8(dst_type)) {   // fp8: the scale needs a device amax pass
    set_error("ps_host_convert: bad dtype (fp8 objects convert on the device)");
    return PS_ERR_INVALID;
  }
  if (n && (!src || !dst)) { set_error("ps_host_convert: null pointer"); return PS_ERR_INVALID; }
  ps::host_convert_f32(src, dst, dst_type, n, threads, simd != 0);
  return PS_OK;
}

// One object's conversion + transfer with a Fig. 3 method (System Inspector probe).
static thread_local XferScratch g_xs;
ps_status ps_transfer(const float *host_src, void *dev_dst, int dst_type, size_t n, int method,
                      int threads, void *dev_stage, void *stream, float *ms) {
  if (!dtype_ok(dst_type) || is_fp8(dst_type) || method < PS_XFER_DEVICE || method > PS_XFER_TRANSIENT) {
    set_error("ps_transfer: bad dtype or method");
    return PS_ERR_INVALID;
  }
  if (n && (!host_src || !dev_dst)) { set_error("ps_transfer: null pointer"); return PS_ERR_INVALID; }
  const bool staged = method == PS_XFER_DEVICE || method == PS_XFER_TRANSIENT;
  if (n && staged && !dev_stage) { set_error("ps_transfer: this method needs dev_stage"); return PS_ERR_INVALID; }
  if (threads <= 0) threads = (int)std::max(1u, std::thread::hardware_concurrency());
  cudaStream_t st = (cudaStream_t)stream;
  PS_CUDA(cudaStreamSynchronize(st));
  const auto t0 = std::chrono::steady_clock::now();
  if (n) {
    ps_status s = xfer_object(g_xs, host_src, n, dst_type, method, threads, dev_dst, dev_stage, st);
    if (s != PS_OK) return s;
    if (staged) {   // the device-side part: f32 (c) or fp16 (d) -> dst_type
      s = convert_async(dev_stage, method == PS_XFER_DEVICE ? PS_F32 : PS_F16, dev_dst, dst_type, n, st);
      if (s != PS_OK) return s;
    }
  }
  PS_CUDA(cudaStreamSynchronize(st));
  if (ms) *ms = (float)std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return PS_OK;
}

// Whole-program evaluation from host inputs with per-object conversion methods
// (Fig. 3 a-e); see prescaler.h.
ps_status ps_run_config_host(ps_app *a, const int *prec, const int *methods,
                             const void *const *host_inputs, void *const *host_outputs, int threads,
                             double toq, void *stream, ps_result *out) {
  ps_status s = ready(a);
  if (s != PS_OK) return s;
  if ((s = check_prec(a, prec)) != PS_OK) return s;
  if (!host_inputs || !out) { set_error("ps_run_config_host: null pointer"); return PS_ERR_INVALID; }
  if ((s = ensure_events(a, NEV)) != PS_OK) return s;
  if (threads <= 0) threads = (int)std::max(1u, std::thread::hardware_concurrency());
  cudaStream_t st = (cudaStream_t)stream;
  const int M = a->def->nobj;
  for (int m = 0; m < M; m++) {
    const int role = a->def->o[m].role;
    if (role != 0 && role != 2) continue;
    const int meth = methods ? methods[m] : PS_XFER_DEVICE;
    if (meth < PS_XFER_DEVICE || meth > PS_XFER_TRANSIENT || !host_inputs[m]) {
      set_error("ps_run_config_host: bad method or missing host input %d", m);
      return PS_ERR_INVALID;
    }
  }
  // a->pre[] tells enqueue_config which inputs arrived already converted; it must
  // be cleared on EVERY exit (a failed transfer must not leave stale markers
  // that make later ps_run_config / ps_sweep / ps_app_reference skip a2)
  struct PreReset {
    ps_app *a;
    int M;
    ~PreReset() { for (int m = 0; m < M; m++) a->pre[m] = 0; }
  } pre_reset{a, M};
  // ---- inputs: host conversion + H2D per object, in object order (wall clock)
  const auto t0 = std::chrono::steady_clock::now();
  for (int m = 0; m < M; m++) {
    const int role = a->def->o[m].role;
    a->pre[m] = 0;
    if (role != 0 && role != 2) continue;
    int meth = methods ? methods[m] : PS_XFER_DEVICE;
    // an f32 input already has its precision: H2D at orig, used in place by a2; an fp8
    // object's scale needs its amax on the device (reading #29): device method
    if (prec[m] == PS_F32 && role == 0 && meth != PS_XFER_TRANSIENT) meth = PS_XFER_DEVICE;
    if (is_fp8(prec[m])) meth = PS_XFER_DEVICE;
    void *stage = meth == PS_XFER_TRANSIENT ? (void *)(a->ws + a->trans_off[m]) : (void *)a->orig_in[m];
    s = xfer_object(a->xs, (const float *)host_inputs[m], nelem(a, m), prec[m], meth, threads,
                    a->ws + a->slot_off[m], stage, st);
    if (s != PS_OK) return s;
    a->pre[m] = meth == PS_XFER_DEVICE ? 0 : (meth == PS_XFER_TRANSIENT ? 2 : 1);
  }
  PS_CUDA(cudaStreamSynchronize(st));
  const double t_in = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  // ---- a2..a5 on the device
  QPart *res = (QPart *)(a->ws + a->qres_off);
  s = enqueue_config(a, prec, st, res, a->ev.data(), true);
  for (int m = 0; m < M; m++) a->pre[m] = 0;
  if (s != PS_OK) return s;
  PS_CUDA(cudaStreamSynchronize(st));
  // ---- outputs: D2H of the delivered (back-converted) outputs
  const auto t1 = std::chrono::steady_clock::now();
  if (host_outputs)
    for (int m = 0; m < M; m++)
      if (a->def->o[m].is_output && host_outputs[m])
        PS_CUDA(cudaMemcpyAsync(host_outputs[m], a->orig_out[m], nelem(a, m) * 4, cudaMemcpyDeviceToHost, st));
  PS_CUDA(cudaMemcpyAsync(a->host_res, res, sizeof(QPart), cudaMemcpyDeviceToHost, st));
  PS_CUDA(cudaStreamSynchronize(st));
  const double t_out = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t1).count();
  uint64_t id = 0;
  ps_config_encode(a, prec, &id);
  fill_result(a, id, a->host_res[0], a->ev.data(), toq, out);
  out->transfer_ms = (float)(t_in + t_out);
  out->total_ms += out->transfer_ms;
  return PS_OK;
}

// Decision-tree search (Sec. 4.4, Alg. 1 normal search + Sec. 4.4.1 PFP), see prescaler.h.
ps_status ps_search(ps_app *a, double toq, int repeats, void *stream, ps_search_result *out) {
  ps_status s = ready(a);
  if (s != PS_OK) return s;
  if (!out || repeats < 1) { set_error("ps_search: bad argument"); return PS_ERR_INVALID; }
  memset(out, 0, sizeof(*out));
  const int M = a->def->nobj;
  struct Trial { float ms; double q; bool pass; };
  std::map<uint64_t, Trial> seen;
  auto encode = [&](const int *prec) {
    uint64_t id = 0, w = 1;
    for (int m = 0; m < M; m++) { id += (uint64_t)prec[m] * w; w *= (uint64_t)radix(a); }
    return id;
  };
  // RunApp (Alg. 1 line 8): median total time of `repeats` runs; never re-run a config
  auto run = [&](const int *prec, Trial *t) -> ps_status {
    const uint64_t id = encode(prec);
    auto it = seen.find(id);
    if (it != seen.end()) { *t = it->second; return PS_OK; }
    std::vector<float> ms;
    ps_result r{};
    for (int k = 0; k < repeats; k++) {
      ps_status e = ps_run_config(a, prec, toq, stream, &r);
      if (e != PS_OK) return e;
      ms.push_back(r.total_ms);
    }
    std::sort(ms.begin(), ms.end());
    *t = Trial{ms[ms.size() / 2], r.quality, r.pass != 0};
    seen[id] = *t;
    if (out->trials < 64) {
      out->trial_ids[out->trials] = id;
      out->trial_ms[out->trials] = t->ms;
      out->trial_pass[out->trials] = t->pass;
    }
    out->trials++;
    return PS_OK;
  };
  auto better = [](const Trial &x, uint64_t xi, const Trial &y, uint64_t yi) {
    return x.ms < y.ms || (x.ms == y.ms && xi < yi);
  };

  // Sec. 4.4.1 pre-full-precision scaling: uniform configurations, descending precision
  int cur[8], cand[8];
  Trial tcur{0.f, 0.0, false};
  bool have = false;
  uint64_t cur_id = 0;
  for (int t = PS_F64; t < radix(a); t++) {
    for (int m = 0; m < M; m++) cand[m] = t;
    Trial tr;
    if ((s = run(cand, &tr)) != PS_OK) return s;
    const uint64_t id = encode(cand);
    if (tr.pass && (!have || better(tr, id, tcur, cur_id))) {
      memcpy(cur, cand, sizeof(cand));
      tcur = tr;
      cur_id = id;
      have = true;
    }
  }
  if (!have) {   // no uniform configuration passes: start from the full-precision one
    for (int m = 0; m < M; m++) cur[m] = PS_F64;
    cur_id = 0;
    if ((s = run(cur, &tcur)) != PS_OK) return s;
  }
  out->pfp_id = cur_id;
  out->pfp_ms = tcur.ms;

  // objects in descending order of data volume, ties -> lower index
  int order[8];
  for (int m = 0; m < M; m++) order[m] = m;
  std::stable_sort(order, order + M, [&](int x, int y) {
    const double wx = (double)nelem(a, x) * kTouch[a->kind][x];
    const double wy = (double)nelem(a, y) * kTouch[a->kind][y];
    return wx > wy;
  });
  // Alg. 1 lines 1-13 per object
  for (int oi = 0; oi < M; oi++) {
    const int m = order[oi];
    int best[8];
    memcpy(best, cur, sizeof(cur));
    Trial tbest = tcur;
    uint64_t best_id = cur_id;
    for (int t = PS_F64; t < radix(a); t++) {         // descending precision
      if (t == cur[m]) continue;                       // line 3
      memcpy(cand, cur, sizeof(cur));
      cand[m] = t;
      Trial tr;
      if ((s = run(cand, &tr)) != PS_OK) return s;     // line 8
      if (!tr.pass) break;                             // line 10: stop at the first failure
      const uint64_t id = encode(cand);
      if (better(tr, id, tbest, best_id)) {            // line 12
        memcpy(best, cand, sizeof(cand));
        tbest = tr;
        best_id = id;
      }
    }
    memcpy(cur, best, sizeof(best));
    tcur = tbest;
    cur_id = best_id;
  }
  out->config_id = cur_id;
  out->total_ms = tcur.ms;
  out->quality = tcur.q;
  out->pass = tcur.pass;
  return PS_OK;
}

int64_t ps_app_eval_shard_rows(const ps_app *a) { return a ? shard_geo(a).rows : 0; }

ps_status ps_shard_bounds(const ps_app *a, int rank, int world, int64_t *row0, int64_t *row1) {
  if (!a || !row0 || !row1 || world < 1 || rank < 0 || rank >= world) {
    set_error("ps_shard_bounds: bad argument");
    return PS_ERR_INVALID;
  }
  const ShardGeo g = shard_geo(a);
  if (!g.rows) { set_error("ps_shard_bounds: %s has no row-sharded evaluation", a->def->kind); return PS_ERR_UNSUPPORTED; }
  split_rows(g.rows, world, rank, g.align, g.tri, row0, row1);
  return PS_OK;
}

ps_status ps_shard_step(ps_app *a, const int *prec, double toq, int rank, int world, int stage, void *stream,
                        ps_shard_step_t *x) {
  ps_status s = ready(a);
  if (s != PS_OK) return s;
  if (!x || world < 1 || rank < 0 || rank >= world || stage < 0) {
    set_error("ps_shard_step: bad argument");
    return PS_ERR_INVALID;
  }
  if ((s = check_prec(a, prec)) != PS_OK) return s;
  for (int m = 0; m < a->def->nobj; m++)
    if (is_fp8(prec[m])) {   // a per-tensor scale needs the amax of the whole object
      set_error("ps_shard_step: fp8 objects are not row-shardable (per-tensor scale)");
      return PS_ERR_UNSUPPORTED;
    }
  if (!shard_geo(a).rows) { set_error("ps_shard_step: %s has no row-sharded evaluation", a->def->kind); return PS_ERR_UNSUPPORTED; }
  if ((s = ensure_events(a, NEV)) != PS_OK) return s;
  cudaStream_t st = (cudaStream_t)stream;
  if (stage == 0) memset(a->shard_ms, 0, sizeof(a->shard_ms));
  QPart *res = (QPart *)(a->ws + a->qres_off);
  memset(x, 0, sizeof(*x));
  s = shard_stage(a, prec, rank, world, stage, st, a->ev.data(), res, x);
  if (s != PS_OK) return s;
  if (x->done) PS_CUDA(cudaMemcpyAsync(a->host_res, res, sizeof(QPart), cudaMemcpyDeviceToHost, st));
  PS_CUDA(cudaStreamSynchronize(st));
  for (int k = 0; k < 4; k++) a->shard_ms[k] += ms_between(a->ev[k], a->ev[k + 1]);
  if (x->done) {
    uint64_t id = 0;
    ps_config_encode(a, prec, &id);
    fill_result(a, id, a->host_res[0], a->ev.data(), toq, &x->result);
    x->result.convert_ms = a->shard_ms[0];
    x->result.kernel_ms = a->shard_ms[1];
    x->result.backconv_ms = a->shard_ms[2];
    x->result.quality_ms = a->shard_ms[3];
    x->result.total_ms = a->shard_ms[0] + a->shard_ms[1] + a->shard_ms[2];
  }
  return PS_OK;
}

}  // extern "C"
