// stencil.cu -- 2DCONV (PolyBench-shaped 3x3 stencil, reading #24), row a3.
//
// B_ij = c11 A(i-1,j-1) + c12 A(i,j-1) + c13 A(i+1,j-1) + c21 A(i-1,j) + c22 A(i,j)
//      + c23 A(i+1,j) + c31 A(i-1,j+1) + c32 A(i,j+1) + c33 A(i+1,j+1)
// in T = W(A, B, f32): each product is one rounded multiply (no contraction,
// R4), sums left to right; border outputs are +0.  HBM-bound: a CTA stages a
// (TY+2) x (TX+2) halo tile of A (widened to T) in shared memory -- every
// thread issues ~17 independent loads before the barrier, enough bytes in
// flight per SM -- then computes TY/RY x 1 column strips of RY outputs per
// thread.  A is read ~1.06x (halo), B written once: algorithmic bytes
// NI*NJ*(s_A + s_B).
#include "common.cuh"
#include "kernels.cuh"
#include "types.cuh"

namespace ps {

constexpr int TX = 128, TY = 32;          // output tile per CTA
constexpr int NT = 256;                   // threads: 128 columns x 2 row halves
constexpr int RY = TY / (NT / TX);        // outputs per thread (column strip) = 16

template <class T> struct Coef9 { T c[9]; };

template <class SA, class SB>
__global__ void __launch_bounds__(NT) conv2d_kernel(const raw_t<SA> *__restrict__ A,
                                                    raw_t<SB> *__restrict__ B, int64_t ni,
                                                    int64_t nj, Coef9<T2<SA, SB>> cf, int vec_ok) {
  using T = T2<SA, SB>;
  using RA = raw_t<SA>;
  constexpr int V = 16 / (int)sizeof(RA);          // elements per 16-byte vector
  // staged window: rows i0-1 .. i0+TY, cols j0-V .. j0+TX+V-1 (16-byte aligned)
  constexpr int HW = TX + 2 * V, HH = TY + 2, NV = HW / V, HN = NV * HH;
  __shared__ T tile[HH][HW];
  const int64_t i0 = (int64_t)blockIdx.y * TY, j0 = (int64_t)blockIdx.x * TX;
  const bool inner = vec_ok && i0 >= 1 && j0 >= V && i0 + TY + 1 <= ni && j0 + TX + V <= nj;
  constexpr int PER = (HN + NT - 1) / NT;
  union Vec { uint4 u; RA e[V]; } v[PER];
#pragma unroll
  for (int q = 0; q < PER; q++) {            // all vector loads in flight before the barrier
    const int e = threadIdx.x + q * NT;
    const int r = e / NV, c = (e % NV) * V;
    const int64_t gi = i0 - 1 + r, gj = j0 - V + c;
    if (e < HN) {
      if (inner) {
        v[q].u = __ldg(reinterpret_cast<const uint4 *>(A + gi * nj + gj));
      } else {
#pragma unroll
        for (int k = 0; k < V; k++)
          v[q].e[k] = (gi >= 0 && gi < ni && gj + k >= 0 && gj + k < nj) ? A[gi * nj + gj + k] : RA(0);
      }
    }
  }
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int e = threadIdx.x + q * NT;
    if (e < HN) {
      const int r = e / NV, c = (e % NV) * V;
#pragma unroll
      for (int k = 0; k < V; k++) tile[r][c + k] = Ld<SA, T>::get(&v[q].e[k], 0);
    }
  }
  __syncthreads();
  const int tx = threadIdx.x % TX, ty0 = (threadIdx.x / TX) * RY;
  const int64_t j = j0 + tx;
  if (j >= nj) return;
#pragma unroll 4
  for (int r = 0; r < RY; r++) {
    const int64_t i = i0 + ty0 + r;
    if (i >= ni) break;
    T acc = T(0);
    if (i > 0 && j > 0 && i + 1 < ni && j + 1 < nj) {
      // (di, dj) in the order c11, c12, c13, c21, c22, c23, c31, c32, c33
#pragma unroll
      for (int k = 0; k < 9; k++) {
        const int di = (k % 3) - 1, dj = (k / 3) - 1;
        const T p = cf.c[k] * tile[ty0 + r + 1 + di][tx + V + dj];
        acc = (k == 0) ? p : acc + p;
      }
    }
    St<SB, T>::put(B, (size_t)(i * nj + j), acc);
  }
}

ps_status conv2d_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, cudaStream_t st) {
  if (ni <= 0 || nj <= 0) return PS_OK;
  static const double C[9] = {0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10};
  dim3 grid((unsigned)((nj + TX - 1) / TX), (unsigned)((ni + TY - 1) / TY));
  return dispatch_store(ta, [&](auto sa) -> ps_status {
    return dispatch_store(tb, [&](auto sb) -> ps_status {
      using SA = decltype(sa);
      using SB = decltype(sb);
      using T = T2<SA, SB>;
      Coef9<T> cf;
      for (int k = 0; k < 9; k++) cf.c[k] = (T)C[k];   // RNE from the fp64 literal (R2)
      const int vec_ok = ((uintptr_t)A % 16 == 0) && ((nj * (int64_t)sizeof(raw_t<SA>)) % 16 == 0);
      conv2d_kernel<SA, SB><<<grid, NT, 0, st>>>((const raw_t<SA> *)A, (raw_t<SB> *)B, ni, nj, cf, vec_ok);
      PS_CHECK_LAUNCH("conv2d_kernel");
      return PS_OK;
    });
  });
}

}  // namespace ps
