// gemm_tc.cu -- tcgen05 tensor-core contraction (fp16 x fp16 -> f32), reading R6.
#include "common.cuh"
#include "kernels.cuh"

namespace ps {
bool gemm_tc_supported(const GemmArgs &) { return false; }
ps_status gemm_tc_async(const GemmArgs &, cudaStream_t) {
  set_error("tcgen05 path not built");
  return PS_ERR_UNSUPPORTED;
}
}  // namespace ps
