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

// ------------------------------------------------------------------- 3DCONV
// 27-point stencil (reading #26): weights g[di] * C9[(dk+1)*3 + (dj+1)], products
// rounded, summed left to right (di outer, then the 2DCONV order); border +0.
// One output per thread, k fastest; the 3x3x3 neighbourhood comes through L1.
template <class T> struct Coef27 { T c[27]; };

template <class SA, class SB>
__global__ void __launch_bounds__(256) conv3d_kernel(const raw_t<SA> *__restrict__ A,
                                                     raw_t<SB> *__restrict__ B, int64_t ni, int64_t nj,
                                                     int64_t nk, Coef27<T2<SA, SB>> cf) {
  using T = T2<SA, SB>;
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t j = blockIdx.y, i = blockIdx.z;
  if (k >= nk) return;
  T acc = T(0);
  if (i > 0 && j > 0 && k > 0 && i + 1 < ni && j + 1 < nj && k + 1 < nk) {
#pragma unroll
    for (int p = 0; p < 3; p++)
#pragma unroll
      for (int q = 0; q < 9; q++) {
        const int64_t di = p - 1, dj = (q % 3) - 1, dk = (q / 3) - 1;
        const T pr = cf.c[p * 9 + q] * ldg_t<SA, T>(A, ((i + di) * nj + (j + dj)) * nk + (k + dk));
        acc = (p == 0 && q == 0) ? pr : acc + pr;
      }
  }
  St<SB, T>::put(B, (size_t)((i * nj + j) * nk + k), acc);
}

ps_status conv3d_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, int64_t nk,
                       cudaStream_t st) {
  if (ni <= 0 || nj <= 0 || nk <= 0) return PS_OK;
  static const double C[9] = {0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10};
  static const double G[3] = {0.25, 0.5, 0.25};
  dim3 grid((unsigned)((nk + 255) / 256), (unsigned)nj, (unsigned)ni);
  return dispatch_store(ta, [&](auto sa) -> ps_status {
    return dispatch_store(tb, [&](auto sb) -> ps_status {
      using SA = decltype(sa);
      using SB = decltype(sb);
      using T = T2<SA, SB>;
      Coef27<T> cf;
      for (int p = 0; p < 3; p++)
        for (int q = 0; q < 9; q++) cf.c[p * 9 + q] = (T)(G[p] * C[q]);   // fp64 product, RNE to T
      conv3d_kernel<SA, SB><<<grid, 256, 0, st>>>((const raw_t<SA> *)A, (raw_t<SB> *)B, ni, nj, nk, cf);
      PS_CHECK_LAUNCH("conv3d_kernel");
      return PS_OK;
    });
  });
}

// ------------------------------------------------------------------ FDTD-2D
// One time step = three passes (reading #27), each in its statement's T.
template <class SF, class SE, class SH>
__global__ void __launch_bounds__(256) fdtd_ey_kernel(const raw_t<SF> *__restrict__ fict,
                                                      raw_t<SE> *__restrict__ ey,
                                                      const raw_t<SH> *__restrict__ hz, int64_t t,
                                                      int64_t nx, int64_t ny) {
  using TA = T2<SF, SE>;   // ey[0][j] = fict[t]
  using TB = T2<SE, SH>;   // ey[i][j] -= 0.5 (hz[i][j] - hz[i-1][j])
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= nx * ny) return;
  const int64_t i = e / ny;
  if (i == 0) {
    St<SE, TA>::put(ey, (size_t)e, ldg_t<SF, TA>(fict, t));
  } else {
    const TB dh = ldg_t<SH, TB>(hz, e) - ldg_t<SH, TB>(hz, e - ny);
    St<SE, TB>::put(ey, (size_t)e, Ld<SE, TB>::get(ey, (size_t)e) - TB(0.5) * dh);
  }
}

template <class SE, class SH>
__global__ void __launch_bounds__(256) fdtd_ex_kernel(raw_t<SE> *__restrict__ ex,
                                                      const raw_t<SH> *__restrict__ hz, int64_t nx,
                                                      int64_t ny) {
  using T = T2<SE, SH>;    // ex[i][j] -= 0.5 (hz[i][j] - hz[i][j-1]),  j >= 1
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= nx * ny || e % ny == 0) return;
  const T dh = ldg_t<SH, T>(hz, e) - ldg_t<SH, T>(hz, e - 1);
  St<SE, T>::put(ex, (size_t)e, Ld<SE, T>::get(ex, (size_t)e) - T(0.5) * dh);
}

template <class SH, class SX, class SY>
__global__ void __launch_bounds__(256) fdtd_hz_kernel(raw_t<SH> *__restrict__ hz,
                                                      const raw_t<SX> *__restrict__ ex,
                                                      const raw_t<SY> *__restrict__ ey, int64_t nx,
                                                      int64_t ny, T3<SH, SX, SY> c07) {
  using T = T3<SH, SX, SY>;   // hz -= 0.7 (ex[i][j+1] - ex[i][j] + ey[i+1][j] - ey[i][j])
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= nx * ny) return;
  const int64_t i = e / ny, j = e % ny;
  if (i + 1 >= nx || j + 1 >= ny) return;
  T s = ldg_t<SX, T>(ex, e + 1) - ldg_t<SX, T>(ex, e);
  s = s + ldg_t<SY, T>(ey, e + ny);
  s = s - ldg_t<SY, T>(ey, e);
  St<SH, T>::put(hz, (size_t)e, Ld<SH, T>::get(hz, (size_t)e) - c07 * s);
}

ps_status fdtd2d_step_async(const void *fict, int tf, void *ex, int tex, void *ey, int tey, void *hz,
                            int thz, int64_t t, int64_t nx, int64_t ny, cudaStream_t st) {
  const int64_t n = nx * ny;
  if (n <= 0) return PS_OK;
  const unsigned nb = (unsigned)((n + 255) / 256);
  ps_status s = dispatch_store(tf, [&](auto a) -> ps_status {
    return dispatch_store(tey, [&](auto b) -> ps_status {
      return dispatch_store(thz, [&](auto c) -> ps_status {
        using SF = decltype(a);
        using SE = decltype(b);
        using SH = decltype(c);
        fdtd_ey_kernel<SF, SE, SH><<<nb, 256, 0, st>>>((const raw_t<SF> *)fict, (raw_t<SE> *)ey,
                                                       (const raw_t<SH> *)hz, t, nx, ny);
        PS_CHECK_LAUNCH("fdtd_ey_kernel");
        return PS_OK;
      });
    });
  });
  if (s != PS_OK) return s;
  s = dispatch_store(tex, [&](auto a) -> ps_status {
    return dispatch_store(thz, [&](auto c) -> ps_status {
      using SE = decltype(a);
      using SH = decltype(c);
      fdtd_ex_kernel<SE, SH><<<nb, 256, 0, st>>>((raw_t<SE> *)ex, (const raw_t<SH> *)hz, nx, ny);
      PS_CHECK_LAUNCH("fdtd_ex_kernel");
      return PS_OK;
    });
  });
  if (s != PS_OK) return s;
  return dispatch_store(thz, [&](auto a) -> ps_status {
    return dispatch_store(tex, [&](auto b) -> ps_status {
      return dispatch_store(tey, [&](auto c) -> ps_status {
        using SH = decltype(a);
        using SX = decltype(b);
        using SY = decltype(c);
        using T = T3<SH, SX, SY>;
        fdtd_hz_kernel<SH, SX, SY><<<nb, 256, 0, st>>>((raw_t<SH> *)hz, (const raw_t<SX> *)ex,
                                                       (const raw_t<SY> *)ey, nx, ny, (T)0.7);
        PS_CHECK_LAUNCH("fdtd_hz_kernel");
        return PS_OK;
      });
    });
  });
}

}  // namespace ps
