// gemm_simt_f64.cu -- instantiations of the R3-exact SIMT contraction with
// compute type f64 (operands stored in f64, f32 or f16; DFMA chains).
#include <cstdlib>

#include "gemm_simt.cuh"

namespace ps {
namespace simt {

// PS_F64_DFMA=1 selects the DFMA kernel below instead of the DMMA one (gemm_dmma.cu);
// both are R3-exact, the switch exists for measurement.
static bool use_dfma() {
  static const bool v = [] { const char *e = getenv("PS_F64_DFMA"); return e && e[0] == '1'; }();
  return v;
}

ps_status gemm_simt_f64(const GemmArgs &g, cudaStream_t st) {
  if (!use_dfma()) return gemm_dmma_f64(g, st);
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

}  // namespace simt
}  // namespace ps
