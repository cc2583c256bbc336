// gemm_misc.cu -- SIMT contraction dispatch (f32 / f64 compute type, R2) and
// the SYRK mirror (lower triangle := upper triangle, optional unit diagonal).
#include "gemm_simt.cuh"

namespace ps {

ps_status gemm_simt_async(const GemmArgs &g, cudaStream_t st) {
  if (g.M <= 0 || g.N <= 0) return PS_OK;
  if (g.B.s_col != 1 || (g.A.s_col != 1 && g.A.s_row != 1)) {
    set_error("gemm_simt: unsupported operand strides");
    return PS_ERR_UNSUPPORTED;
  }
  return g.T == PS_F64 ? simt::gemm_simt_f64(g, st) : simt::gemm_simt_f32(g, st);
}

template <class S>
__global__ void __launch_bounds__(256) mirror_kernel(raw_t<S> *s, int64_t M, int diag_one) {
  __shared__ raw_t<S> tile[32][33];
  const int64_t bx = blockIdx.x, by = blockIdx.y;   // source tile (row block bx, col block by), bx <= by
  if (bx > by) return;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;   // 32 x 8
  for (int r = ty; r < 32; r += 8) {
    const int64_t gi = bx * 32 + r, gj = by * 32 + tx;
    if (gi < M && gj < M) tile[r][tx] = s[gi * M + gj];
  }
  __syncthreads();
  // destination (row block by, col block bx): element (i, j) = source (j, i), for i > j
  for (int r = ty; r < 32; r += 8) {
    const int64_t gi = by * 32 + r, gj = bx * 32 + tx;
    if (gi < M && gj < M && gi > gj) s[gi * M + gj] = tile[tx][r];
  }
  if (diag_one && bx == by) {
    __syncthreads();
    if (threadIdx.x < 32) {
      const int64_t gd = bx * 32 + threadIdx.x;
      if (gd < M) St<S, float>::put(s, gd * M + gd, 1.0f);
    }
  }
}

ps_status mirror_async(void *S, int type, int64_t M, int diag_one, cudaStream_t st) {
  if (M <= 0) return PS_OK;
  dim3 grid((unsigned)((M + 31) / 32), (unsigned)((M + 31) / 32));
  return dispatch_store(type, [&](auto s) -> ps_status {
    using ST = decltype(s);
    mirror_kernel<ST><<<grid, 256, 0, st>>>((raw_t<ST> *)S, M, diag_one);
    PS_CHECK_LAUNCH("mirror_kernel");
    return PS_OK;
  });
}

}  // namespace ps
