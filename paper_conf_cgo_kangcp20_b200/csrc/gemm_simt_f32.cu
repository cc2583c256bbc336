// gemm_simt_f32.cu -- instantiations of the R3-exact SIMT contraction with
// compute type f32 (operands stored in f32, f16 or bf16; FFMA chains).
#include <cstdlib>

#include "gemm_simt.cuh"

namespace ps {
namespace simt {

// PS_F32_SIMT_OLD=1 selects this kernel instead of gemm_ffma.cu's (both R3-exact; the
// switch exists for measurement)
static bool use_old() {
  static const bool v = [] { const char *e = getenv("PS_F32_SIMT_OLD"); return e && e[0] == '1'; }();
  return v;
}

ps_status gemm_simt_f32(const GemmArgs &g, cudaStream_t st) {
  if (!use_old()) return gemm_ffma_f32(g, st);
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

}  // namespace simt
}  // namespace ps
