// stencil.cu -- 2DCONV (PolyBench-shaped 3x3 stencil, reading #24), row a3.
//
// B_ij = c11 A(i-1,j-1) + c12 A(i,j-1) + c13 A(i+1,j-1) + c21 A(i-1,j) + c22 A(i,j)
//      + c23 A(i+1,j) + c31 A(i-1,j+1) + c32 A(i,j+1) + c33 A(i+1,j+1)
// in T = W(A, B, f32): each product is one rounded multiply (no contraction,
// R4), sums left to right; border outputs are +0.  HBM-bound: the 3x3
// neighbourhood is staged once per CTA tile in shared memory (widened to T),
// so A is read ~once and B written once: algorithmic bytes NI*NJ*(s_A + s_B).
#include "common.cuh"
#include "kernels.cuh"
#include "types.cuh"

namespace ps {

constexpr int SX = 32, SY = 16;   // output tile per CTA (32 x 16 threads)

template <class T> struct Coef9 { T c[9]; };

template <class SA, class SB>
__global__ void __launch_bounds__(SX * SY) conv2d_kernel(const raw_t<SA> *__restrict__ A,
                                                         raw_t<SB> *__restrict__ B, int64_t ni,
                                                         int64_t nj, Coef9<T2<SA, SB>> cf) {
  using T = T2<SA, SB>;
  __shared__ T tile[SY + 2][SX + 2];
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int64_t i0 = (int64_t)blockIdx.y * SY, j0 = (int64_t)blockIdx.x * SX;
  // stage the (SY+2) x (SX+2) halo tile (rows i0-1.., cols j0-1..)
  for (int r = ty; r < SY + 2; r += SY)
    for (int c = tx; c < SX + 2; c += SX) {
      const int64_t gi = i0 - 1 + r, gj = j0 - 1 + c;
      tile[r][c] = (gi >= 0 && gi < ni && gj >= 0 && gj < nj) ? Ld<SA, T>::get(A, (size_t)(gi * nj + gj)) : T(0);
    }
  __syncthreads();
  const int64_t i = i0 + ty, j = j0 + tx;
  if (i >= ni || j >= nj) return;
  T acc = T(0);
  if (i > 0 && j > 0 && i + 1 < ni && j + 1 < nj) {
    // (di, dj) in the order c11, c12, c13, c21, c22, c23, c31, c32, c33
#pragma unroll
    for (int k = 0; k < 9; k++) {
      const int di = (k % 3) - 1, dj = (k / 3) - 1;
      const T p = cf.c[k] * tile[ty + 1 + di][tx + 1 + dj];
      acc = (k == 0) ? p : acc + p;
    }
  }
  St<SB, T>::put(B, (size_t)(i * nj + j), acc);
}

ps_status conv2d_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, cudaStream_t st) {
  if (ni <= 0 || nj <= 0) return PS_OK;
  static const double C[9] = {0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10};
  dim3 grid((unsigned)((nj + SX - 1) / SX), (unsigned)((ni + SY - 1) / SY));
  return dispatch_store(ta, [&](auto sa) -> ps_status {
    return dispatch_store(tb, [&](auto sb) -> ps_status {
      using SA = decltype(sa);
      using SB = decltype(sb);
      using T = T2<SA, SB>;
      Coef9<T> cf;
      for (int k = 0; k < 9; k++) cf.c[k] = (T)C[k];   // RNE from the fp64 literal (R2)
      conv2d_kernel<SA, SB><<<grid, dim3(SX, SY), 0, st>>>((const raw_t<SA> *)A, (raw_t<SB> *)B, ni, nj, cf);
      PS_CHECK_LAUNCH("conv2d_kernel");
      return PS_OK;
    });
  });
}

}  // namespace ps
