// gemm_simt_f64.cu -- compute type f64 contractions (operands stored in f64, f32,
// f16 or bf16), R3-exact fma chains.
//
// Fast path: gemm_dmma.cu chains mma.sync.m8n8k4.f64 (DMMA).  That is R3-exact
// only because this B200 returns, bit for bit, the sequential fma chain for one
// DMMA step (round-1 probe, profiles/dmma_probe_r1.txt) -- PTX does not specify
// the accumulation order.  So before the first f64 contraction on a device the
// library runs a self-check: a 128 x 128 x 64 product of adversarial operands
// (random signs, exponents spread over [-60, 60], cancelling pairs, subnormals)
// through both the DMMA kernel and the DFMA kernel below (gemm_simt.cuh: plain
// __fma_rn chains, R3 by construction) and compares every output bit.  Any
// difference selects the DFMA kernel for that device (correct, ~40% slower).
// PS_F64_DFMA=1 forces the DFMA kernel (the tests use it to keep it covered).
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "gemm_simt.cuh"

namespace ps {
namespace simt {

static ps_status gemm_dfma_f64(const GemmArgs &g, cudaStream_t st) {
  const Params p = make_params(g);
  const bool ak = g.A.s_col == 1;
  return dispatch_store(g.A.type, [&](auto sa) -> ps_status {
    return dispatch_store(g.B.type, [&](auto sb) -> ps_status {
      using SA = decltype(sa);
      using SB = decltype(sb);
      return launch<double, SA, SB>(p, ak, g.alpha, g.beta, g.div, st);
    });
  });
}

// deterministic adversarial operands (splitmix64)
static uint64_t mix(uint64_t &s) {
  uint64_t z = (s += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static double adversarial(uint64_t &s, int64_t i) {
  const uint64_t r = mix(s);
  const uint64_t sign = (r & 1) << 63, mant = (r >> 1) & 0xFFFFFFFFFFFFFull;
  if (i % 97 == 5) {                       // subnormal
    uint64_t b = sign | (mant >> 3);
    double d;
    memcpy(&d, &b, 8);
    return d;
  }
  const int e = (int)((r >> 53) % 121) - 60;   // exponent spread: cancellation + absorption
  uint64_t b = sign | ((uint64_t)(1023 + e) << 52) | mant;
  double d;
  memcpy(&d, &b, 8);
  return d;
}

// 1 = the DMMA chain equals the fma chain bit for bit, 0 = it does not, -1 = error
static int dmma_self_check() {
  const int64_t M = 128, N = 128, K = 64;
  std::vector<double> ha(M * K), hb(K * N);
  uint64_t s = 20200222;
  for (int64_t i = 0; i < M * K; i++) ha[i] = adversarial(s, i);
  for (int64_t i = 0; i < K * N; i++) hb[i] = adversarial(s, i + 3);
  for (int64_t k = 0; k + 1 < K; k += 2)   // exact cancellation inside rows of A
    for (int64_t m = 0; m < M; m += 3) ha[m * K + k + 1] = -ha[m * K + k];
  double *d = nullptr;
  cudaStream_t st = nullptr;
  const size_t bytes = (M * K + K * N + 2 * M * N) * sizeof(double);
  int ok = -1;
  if (cudaMalloc(&d, bytes) != cudaSuccess) return -1;
  if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) == cudaSuccess) {
    double *A = d, *B = d + M * K, *C1 = B + K * N, *C2 = C1 + M * N;
    cudaMemcpyAsync(A, ha.data(), M * K * 8, cudaMemcpyHostToDevice, st);
    cudaMemcpyAsync(B, hb.data(), K * N * 8, cudaMemcpyHostToDevice, st);
    GemmArgs g{};
    g.M = M; g.N = N; g.K = K;
    g.A = MatDesc{A, PS_F64, K, 1};
    g.B = MatDesc{B, PS_F64, N, 1};
    g.c_type = PS_F64; g.ldc = N; g.epi = EPI_PLAIN; g.T = PS_F64;
    g.alpha = 1.0; g.beta = 0.0; g.div = 1.0;
    g.C = C1;
    ps_status s1 = gemm_dmma_f64(g, st);
    g.C = C2;
    ps_status s2 = gemm_dfma_f64(g, st);
    std::vector<double> h1(M * N), h2(M * N);
    if (s1 == PS_OK && s2 == PS_OK &&
        cudaMemcpyAsync(h1.data(), C1, M * N * 8, cudaMemcpyDeviceToHost, st) == cudaSuccess &&
        cudaMemcpyAsync(h2.data(), C2, M * N * 8, cudaMemcpyDeviceToHost, st) == cudaSuccess &&
        cudaStreamSynchronize(st) == cudaSuccess)
      ok = memcmp(h1.data(), h2.data(), M * N * 8) == 0 ? 1 : 0;
    cudaStreamDestroy(st);
  }
  cudaFree(d);
  return ok;
}

bool use_dmma(cudaStream_t caller) {
  static const bool forced = [] { const char *e = getenv("PS_F64_DFMA"); return e && e[0] == '1'; }();
  if (forced) return false;
  static std::mutex mu;
  static int verdict[64];          // 0 unknown, 1 DMMA ok, 2 use DFMA
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return false;
  std::lock_guard<std::mutex> lk(mu);
  if (!verdict[dev]) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(caller, &cs);
    if (cs != cudaStreamCaptureStatusNone) return false;   // cannot synchronise now: DFMA
    const int r = dmma_self_check();
    if (r < 0) return false;                                 // transient error: retry next call
    verdict[dev] = r == 1 ? 1 : 2;
    if (r == 0) fprintf(stderr, "libprescaler: DMMA self-check failed on device %d; f64 contractions "
                                "use the DFMA kernel\n", dev);
  }
  return verdict[dev] == 1;
}

ps_status gemm_simt_f64(const GemmArgs &g, cudaStream_t st) {
  return use_dmma(st) ? gemm_dmma_f64(g, st) : gemm_dfma_f64(g, st);
}

}  // namespace simt
}  // namespace ps

extern "C" int ps_f64_uses_dmma(void) { return ps::simt::use_dmma(nullptr) ? 1 : 0; }
