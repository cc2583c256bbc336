// gemm_simt_f32.cu -- compute type f32 contractions (operands stored in f32, f16 or
// bf16; FFMA chains, R3-exact): gemm_ffma.cu's kernel.  The round-1 kernel of
// gemm_simt.cuh is compiled only with -DPS_LEGACY_KERNELS (measurement builds).
#include <cstdlib>

#include "gemm_simt.cuh"

namespace ps {
namespace simt {

ps_status gemm_simt_f32(const GemmArgs &g, cudaStream_t st) {
#ifdef PS_LEGACY_KERNELS
  static const bool old = [] { const char *e = getenv("PS_F32_SIMT_OLD"); return e && e[0] == '1'; }();
  if (old) {
    const Params p = make_params(g);
    const bool ak = g.A.s_col == 1;
    auto pick = [&](auto sa) -> ps_status {
      using SA = decltype(sa);
      if (g.B.type == PS_F16) return launch<float, SA, F16>(p, ak, g.alpha, g.beta, g.div, st);
      if (g.B.type == PS_BF16) return launch<float, SA, BF16>(p, ak, g.alpha, g.beta, g.div, st);
      return launch<float, SA, float>(p, ak, g.alpha, g.beta, g.div, st);
    };
    if (g.A.type == PS_F16) return pick(F16());
    if (g.A.type == PS_BF16) return pick(BF16());
    return pick(float());
  }
#endif
  return gemm_ffma_f32(g, st);
}

}  // namespace simt
}  // namespace ps
