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
                                                    int64_t nj, Coef9<T2<SA, SB>> cf, int vec_ok,
                                                    int64_t ibeg, int64_t iend) {
  using T = T2<SA, SB>;
  using RA = raw_t<SA>;
  constexpr int V = 16 / (int)sizeof(RA);          // elements per 16-byte vector
  // staged window: rows i0-1 .. i0+TY, cols j0-V .. j0+TX+V-1 (16-byte aligned)
  constexpr int HW = TX + 2 * V, HH = TY + 2, NV = HW / V, HN = NV * HH;
  __shared__ T tile[HH][HW];
  const int64_t i0 = ibeg + (int64_t)blockIdx.y * TY, j0 = (int64_t)blockIdx.x * TX;
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
    if (i >= iend) break;
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

// output rows [ibeg, iend) of the full NI x NJ problem (borders by the global
// indices); the rows read are [ibeg - 1, iend + 1) -- a row-sharded evaluation
ps_status conv2d_rows_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, int64_t ibeg,
                            int64_t iend, cudaStream_t st) {
  if (ni <= 0 || nj <= 0 || iend <= ibeg) return PS_OK;
  static const double C[9] = {0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10};
  dim3 grid((unsigned)((nj + TX - 1) / TX), (unsigned)((iend - ibeg + TY - 1) / TY));
  return dispatch_store(ta, [&](auto sa) -> ps_status {
    return dispatch_store(tb, [&](auto sb) -> ps_status {
      using SA = decltype(sa);
      using SB = decltype(sb);
      using T = T2<SA, SB>;
      Coef9<T> cf;
      for (int k = 0; k < 9; k++) cf.c[k] = (T)C[k];   // RNE from the fp64 literal (R2)
      const int vec_ok = ((uintptr_t)A % 16 == 0) && ((nj * (int64_t)sizeof(raw_t<SA>)) % 16 == 0);
      conv2d_kernel<SA, SB><<<grid, NT, 0, st>>>((const raw_t<SA> *)A, (raw_t<SB> *)B, ni, nj, cf, vec_ok,
                                                 ibeg, iend);
      PS_CHECK_LAUNCH("conv2d_kernel");
      return PS_OK;
    });
  });
}

ps_status conv2d_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, cudaStream_t st) {
  return conv2d_rows_async(A, ta, B, tb, ni, nj, 0, ni, st);
}

// ------------------------------------------------------------------- 3DCONV
// 27-point stencil (reading #26): weights g[di] * C9[(dk+1)*3 + (dj+1)], products
// rounded, summed left to right (di outer, then the 2DCONV order); border +0.
//
// 2.5-D blocking: a CTA owns a C3_TJ x C3_TK (j, k) column of outputs and
// marches down C3_IL planes along i.  Input slices (C3_TJ+2) x (C3_TK+2), widened
// to T, sit in a 4-slot shared-memory ring (one barrier per plane); slice i+3 is
// fetched into registers while plane i is computed.  Each thread owns one k column and slides a 3-row
// register window down its C3_RJ rows of j, so an output costs 9 shared loads,
// 27 rounded multiplies and 26 adds.  L2->SM traffic is ~1.3x the algorithmic
// read (halo), DRAM ~1x.  ALU ceiling: 53 FP32 ops per output at 128/clk/SM.
template <class T> struct Coef27 { T c[27]; };
constexpr int C3_TK = 128, C3_TJ = 18, C3_IL = 16, C3_NT = 256;
constexpr int C3_RJ = C3_TJ / (C3_NT / C3_TK);                 // rows per thread = 9
constexpr int C3_SH = C3_TJ + 2, C3_RING = 4;
template <class SA> struct C3Geo {                                // slice window geometry
  static constexpr int V = 16 / (int)sizeof(raw_t<SA>);         // elements per 16-byte vector
  static constexpr int SW = C3_TK + 2 * V;                      // cols k0-V .. k0+TK+V-1
  static constexpr int NV = SW / V, HN = NV * C3_SH, PER = (HN + C3_NT - 1) / C3_NT;
};

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem, bool valid) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem),
               "r"(valid ? 16 : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit_wait() {
  asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

template <class SA, class SB>
__global__ void __launch_bounds__(C3_NT, sizeof(T2<SA, SB>) == 8 ? 2 : 3) conv3d_kernel(
    const raw_t<SA> *__restrict__ A, raw_t<SB> *__restrict__ B, int64_t ni, int64_t nj, int64_t nk,
    Coef27<T2<SA, SB>> cf, int vec_ok, int64_t ibeg, int64_t iend) {
  using T = T2<SA, SB>;
  using RA = raw_t<SA>;
  using G = C3Geo<SA>;
  constexpr int V = G::V, SW = G::SW, NV = G::NV, HN = G::HN, PER = G::PER;
  // storage == compute type: slices go global -> T ring by cp.async.  Otherwise
  // cp.async lands them in a 2-slot raw ring and one pass widens raw -> T ring.
  constexpr bool SAME = std::is_same<RA, T>::value;
  extern __shared__ __align__(16) unsigned char c3_smem[];
  T(*sl)[C3_SH][SW] = reinterpret_cast<T(*)[C3_SH][SW]>(c3_smem);
  RA(*rw)[C3_SH][SW] = reinterpret_cast<RA(*)[C3_SH][SW]>(c3_smem + sizeof(T) * C3_RING * C3_SH * SW);
  const int64_t k0 = (int64_t)blockIdx.x * C3_TK, j0 = (int64_t)blockIdx.y * C3_TJ;
  const int64_t ib = ibeg + (int64_t)blockIdx.z * C3_IL;
  const int64_t ie = ib + C3_IL < iend ? ib + C3_IL : iend;   // output planes [ib, ie)
  const int64_t plane = nj * nk;
  int64_t off[PER];                                            // window element offsets in a slice
  bool in[PER];                                                // vector inside the (j, k) range
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int e = threadIdx.x + q * C3_NT;
    const int64_t gj = j0 - 1 + e / NV, gk = k0 - V + (e % NV) * V;
    off[q] = gj * nk + gk;
    // with vec_ok (nk % V == 0, A 16-byte aligned) a vector is entirely in or out of range
    in[q] = e < HN && gj >= 0 && gj < nj && gk >= 0 && gk < nk;
  }
  auto slot_of = [&](int64_t gi) { return (int)(gi - ib + 1) & (C3_RING - 1); };
  // cp.async slice gi (zero-filled outside the array) into the T ring (SAME) or raw ring
  auto fill_async = [&](int64_t gi) {
    const bool iok = gi >= 0 && gi < ni;
    RA *dst = SAME ? reinterpret_cast<RA *>(&sl[slot_of(gi)][0][0]) : &rw[(int)(gi - ib + 1) & 1][0][0];
#pragma unroll
    for (int q = 0; q < PER; q++) {
      const int e = threadIdx.x + q * C3_NT;
      if (e < HN) {
        const bool ok = iok && in[q];
        cp_async16(dst + (e / NV) * SW + (e % NV) * V, ok ? (const void *)(A + gi * plane + off[q]) : (const void *)A,
                   ok);
      }
    }
    cp_async_commit();
  };
  // raw ring -> T ring (non-SAME)
  auto widen = [&](int64_t gi) {
    const RA *src = &rw[(int)(gi - ib + 1) & 1][0][0];
    T *dst = &sl[slot_of(gi)][0][0];
    for (int e = threadIdx.x; e < C3_SH * SW; e += C3_NT) dst[e] = Ld<SA, T>::get(src, (size_t)e);
  };
  // unaligned shapes: synchronous fill straight into the T ring
  auto fill_sync = [&](int64_t gi) {
    const bool iok = gi >= 0 && gi < ni;
    const int slot = slot_of(gi);
    for (int e = threadIdx.x; e < C3_SH * SW; e += C3_NT) {
      const int64_t gj = j0 - 1 + e / SW, gk = k0 - V + e % SW;
      sl[slot][e / SW][e % SW] = (iok && gj >= 0 && gj < nj && gk >= 0 && gk < nk)
                                     ? Ld<SA, T>::get(A, (size_t)(gi * plane + gj * nk + gk)) : T(0);
    }
  };
  // prologue: slices ib-1 .. ib+1 in the T ring; non-SAME also has ib+2 in flight
  if (vec_ok) {
    if constexpr (SAME) {
      for (int64_t g = ib - 1; g <= ib + 1; g++) fill_async(g);
      cp_async_wait();
    } else {
      for (int64_t g = ib - 1; g <= ib + 1; g++) {
        fill_async(g);
        cp_async_wait();
        __syncthreads();
        widen(g);
        __syncthreads();
      }
      if (ib + 2 <= ie) {
        fill_async(ib + 2);
        cp_async_wait();                                       // widened in iteration ib
      }
    }
  } else {
    for (int64_t g = ib - 1; g <= ib + 1; g++) fill_sync(g);
  }
  const int kx = threadIdx.x % C3_TK, jr0 = (threadIdx.x / C3_TK) * C3_RJ;
  const int64_t k = k0 + kx, jt = j0 + jr0;                    // first output row of this thread
  const bool kin = k > 0 && k + 1 < nk;
  // rows r of this thread: stored if r < nval, computed (interior in j) if rlo <= r < rhi
  const int nval = (int)(nj - jt < C3_RJ ? (nj - jt > 0 ? nj - jt : 0) : C3_RJ);
  const int rlo = jt == 0 ? 1 : 0;
  const int rhi = (int)(nj - 1 - jt < C3_RJ ? (nj - 1 - jt > 0 ? nj - 1 - jt : 0) : C3_RJ);
  for (int64_t i = ib; i < ie; i++) {
    // slices <= i+1 are committed; everyone is done with plane i-1 (slot of i+2 free)
    __syncthreads();
    // slice i+2 -> its T slot (free: last read by plane i-1); lands during plane i
    if (i + 2 <= ie) {
      if (!vec_ok) fill_sync(i + 2);
      else if constexpr (SAME) fill_async(i + 2);
      else {
        widen(i + 2);                                          // arrived during plane i-1
        if (i + 3 <= ie) fill_async(i + 3);
      }
    }
    const bool pin = i > 0 && i + 1 < ni && kin && k < nk;
    const int sm1 = (int)(i - ib) & (C3_RING - 1);
    const T *q0 = &sl[sm1][jr0][kx + V - 1];
    const T *q1 = &sl[(sm1 + 1) & (C3_RING - 1)][jr0][kx + V - 1];
    const T *q2 = &sl[(sm1 + 2) & (C3_RING - 1)][jr0][kx + V - 1];
    raw_t<SB> *op = B + ((i * nj + jt) * nk + k);
    // next window row: the 9 values (p, dk) of this k column, then advance
    auto load_row = [&](T (&w)[9]) {
#pragma unroll
      for (int dk = 0; dk < 3; dk++) {
        w[0 + dk] = q0[dk];
        w[3 + dk] = q1[dk];
        w[6 + dk] = q2[dk];
      }
      q0 += SW; q1 += SW; q2 += SW;
    };
    // output row r from window rows r (j-1), r+1 (j), r+2 (j+1); FULL: every row of
    // this thread is stored and interior (no per-row tests)
    auto out_row = [&](auto full, const T (&a)[9], const T (&b)[9], const T (&c)[9], int r) {
      constexpr bool FULL = decltype(full)::value;
      if (FULL || (r < nval && k < nk)) {
        T acc = T(0);
        if (FULL || (pin && r >= rlo && r < rhi)) {
#pragma unroll
          for (int p = 0; p < 3; p++)
#pragma unroll
            for (int q = 0; q < 9; q++) {
              const int dj = q % 3, dk = q / 3;                  // (dj+1, dk+1)
              const T v = dj == 0 ? a[p * 3 + dk] : dj == 1 ? b[p * 3 + dk] : c[p * 3 + dk];
              const T pr = cf.c[p * 9 + q] * v;
              acc = (p == 0 && q == 0) ? pr : acc + pr;
            }
        }
        St<SB, T>::put(op, 0, acc);
      }
      op += nk;
    };
    auto rows = [&](auto full) {
      T w0[9], w1[9], w2[9];
      load_row(w0);
      load_row(w1);
#pragma unroll 1
      for (int r = 0; r < C3_RJ; r += 3) {                     // rotate names, no moves
        load_row(w2); out_row(full, w0, w1, w2, r);
        load_row(w0); out_row(full, w1, w2, w0, r + 1);
        load_row(w1); out_row(full, w2, w0, w1, r + 2);
      }
    };
    if (pin && nval == C3_RJ && rlo == 0 && rhi == C3_RJ) rows(std::true_type{});
    else rows(std::false_type{});
    if (vec_ok) cp_async_wait();
  }
}

// output planes [ibeg, iend) (planes [ibeg - 1, iend + 1) are read): row-sharded evaluation
ps_status conv3d_rows_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, int64_t nk,
                            int64_t ibeg, int64_t iend, cudaStream_t st) {
  if (ni <= 0 || nj <= 0 || nk <= 0 || iend <= ibeg) return PS_OK;
  static const double C[9] = {0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10};
  static const double G[3] = {0.25, 0.5, 0.25};
  dim3 grid((unsigned)((nk + C3_TK - 1) / C3_TK), (unsigned)((nj + C3_TJ - 1) / C3_TJ),
            (unsigned)((iend - ibeg + C3_IL - 1) / C3_IL));
  return dispatch_store(ta, [&](auto sa) -> ps_status {
    return dispatch_store(tb, [&](auto sb) -> ps_status {
      using SA = decltype(sa);
      using SB = decltype(sb);
      using T = T2<SA, SB>;
      Coef27<T> cf;
      for (int p = 0; p < 3; p++)
        for (int q = 0; q < 9; q++) cf.c[p * 9 + q] = (T)(G[p] * C[q]);   // fp64 product, RNE to T
      constexpr bool SAME = std::is_same<raw_t<SA>, T>::value;
      const size_t smem = (sizeof(T) * C3_RING + (SAME ? 0 : 2 * sizeof(raw_t<SA>))) * C3_SH * C3Geo<SA>::SW;
      const int vec_ok = ((uintptr_t)A % 16 == 0) && ((nk * (int64_t)sizeof(raw_t<SA>)) % 16 == 0);
      PS_TRY(set_max_smem((const void *)conv3d_kernel<SA, SB>, (int)smem));
      conv3d_kernel<SA, SB><<<grid, C3_NT, smem, st>>>((const raw_t<SA> *)A, (raw_t<SB> *)B, ni, nj, nk, cf,
                                                         vec_ok, ibeg, iend);
      PS_CHECK_LAUNCH("conv3d_kernel");
      return PS_OK;
    });
  });
}

ps_status conv3d_async(const void *A, int ta, void *B, int tb, int64_t ni, int64_t nj, int64_t nk,
                       cudaStream_t st) {
  return conv3d_rows_async(A, ta, B, tb, ni, nj, nk, 0, ni, st);
}

// ------------------------------------------------------------------ FDTD-2D
// One time step = three passes (reading #27), each in its statement's T.  2-D
// grid: blockIdx.y strides over rows i, each thread handles FD_U columns spaced
// 256 apart (coalesced, FD_U independent loads in flight), no integer division.
constexpr int FD_NT = 256, FD_U = 4, FD_COLS = FD_NT * FD_U;

template <class SF, class SE, class SH>
__global__ void __launch_bounds__(FD_NT) fdtd_ey_kernel(const raw_t<SF> *__restrict__ fict,
                                                        raw_t<SE> *__restrict__ ey,
                                                        const raw_t<SH> *__restrict__ hz, int64_t t,
                                                        int64_t nx, int64_t ny, int part, int64_t i0,
                                                        int64_t i1) {
  using TA = T2<SF, SE>;   // ey[0][j] = fict[t]
  using TB = T2<SE, SH>;   // ey[i][j] -= 0.5 (hz[i][j] - hz[i-1][j])
  const int64_t jb = (int64_t)blockIdx.x * FD_COLS + threadIdx.x;
  for (int64_t i = i0 + blockIdx.y; i < i1; i += gridDim.y) {
    const int64_t row = i * ny;
    if ((i == 0 && part == FDTD_EY1) || (i > 0 && part == FDTD_EY0)) continue;
    if (i == 0) {
      const TA f = ldg_t<SF, TA>(fict, t);
#pragma unroll
      for (int u = 0; u < FD_U; u++)
        if (jb + u * FD_NT < ny) St<SE, TA>::put(ey, (size_t)(jb + u * FD_NT), f);
      continue;
    }
    TB h[FD_U], g[FD_U], e[FD_U];
#pragma unroll
    for (int u = 0; u < FD_U; u++) {
      const int64_t j = jb + u * FD_NT;
      if (j < ny) {
        h[u] = ldg_t<SH, TB>(hz, row + j);
        g[u] = ldg_t<SH, TB>(hz, row - ny + j);
        e[u] = Ld<SE, TB>::get(ey, (size_t)(row + j));
      }
    }
#pragma unroll
    for (int u = 0; u < FD_U; u++) {
      const int64_t j = jb + u * FD_NT;
      if (j < ny) St<SE, TB>::put(ey, (size_t)(row + j), e[u] - TB(0.5) * (h[u] - g[u]));
    }
  }
}

template <class SE, class SH>
__global__ void __launch_bounds__(FD_NT) fdtd_ex_kernel(raw_t<SE> *__restrict__ ex,
                                                        const raw_t<SH> *__restrict__ hz, int64_t nx,
                                                        int64_t ny, int64_t i0, int64_t i1) {
  using T = T2<SE, SH>;    // ex[i][j] -= 0.5 (hz[i][j] - hz[i][j-1]),  j >= 1
  const int64_t jb = (int64_t)blockIdx.x * FD_COLS + threadIdx.x;
  for (int64_t i = i0 + blockIdx.y; i < i1; i += gridDim.y) {
    const int64_t row = i * ny;
    T h[FD_U], g[FD_U], e[FD_U];
#pragma unroll
    for (int u = 0; u < FD_U; u++) {
      const int64_t j = jb + u * FD_NT;
      if (j >= 1 && j < ny) {
        h[u] = ldg_t<SH, T>(hz, row + j);
        g[u] = ldg_t<SH, T>(hz, row + j - 1);
        e[u] = Ld<SE, T>::get(ex, (size_t)(row + j));
      }
    }
#pragma unroll
    for (int u = 0; u < FD_U; u++) {
      const int64_t j = jb + u * FD_NT;
      if (j >= 1 && j < ny) St<SE, T>::put(ex, (size_t)(row + j), e[u] - T(0.5) * (h[u] - g[u]));
    }
  }
}

template <class SH, class SX, class SY>
__global__ void __launch_bounds__(FD_NT) fdtd_hz_kernel(raw_t<SH> *__restrict__ hz,
                                                        const raw_t<SX> *__restrict__ ex,
                                                        const raw_t<SY> *__restrict__ ey, int64_t nx,
                                                        int64_t ny, T3<SH, SX, SY> c07, int64_t i0,
                                                        int64_t i1) {
  using T = T3<SH, SX, SY>;   // hz -= 0.7 (((ex[i][j+1] - ex[i][j]) + ey[i+1][j]) - ey[i][j])
  const int64_t jb = (int64_t)blockIdx.x * FD_COLS + threadIdx.x;
  for (int64_t i = i0 + blockIdx.y; i < i1 && i + 1 < nx; i += gridDim.y) {
    const int64_t row = i * ny;
    T x1[FD_U], x0[FD_U], y1[FD_U], y0[FD_U], h[FD_U];
#pragma unroll
    for (int u = 0; u < FD_U; u++) {
      const int64_t j = jb + u * FD_NT;
      if (j + 1 < ny) {
        x1[u] = ldg_t<SX, T>(ex, row + j + 1);
        x0[u] = ldg_t<SX, T>(ex, row + j);
        y1[u] = ldg_t<SY, T>(ey, row + ny + j);
        y0[u] = ldg_t<SY, T>(ey, row + j);
        h[u] = Ld<SH, T>::get(hz, (size_t)(row + j));
      }
    }
#pragma unroll
    for (int u = 0; u < FD_U; u++) {
      const int64_t j = jb + u * FD_NT;
      if (j + 1 < ny) {
        T s = x1[u] - x0[u];
        s = s + y1[u];
        s = s - y0[u];
        St<SH, T>::put(hz, (size_t)(row + j), h[u] - c07 * s);
      }
    }
  }
}

// rows [r0, r1) of the statement (r1 < 0: every row) -- a row-sharded evaluation
ps_status fdtd2d_part_async(int part, const void *fict, int tf, void *ex, int tex, void *ey, int tey,
                            void *hz, int thz, int64_t t, int64_t nx, int64_t ny, cudaStream_t st, int64_t r0,
                            int64_t r1) {
  if (nx <= 0 || ny <= 0) return PS_OK;
  if (r1 < 0) r1 = nx;
  if (r1 <= r0) return PS_OK;
  if (part == FDTD_EY0) {   // the row-0 assignment belongs to the rank owning row 0
    if (r0 > 0) return PS_OK;
    r1 = 1;
  }
  const int64_t rows = r1 - r0;
  if (part == FDTD_EY0) thz = PS_F32;   // the row-0 assignment reads fict only (hz unused)
  if (part == FDTD_EY1) tf = PS_F32;    // the update reads hz only (fict unused)
  const dim3 grid((unsigned)((ny + FD_COLS - 1) / FD_COLS), (unsigned)(rows < 65535 ? rows : 65535));
  if (part <= FDTD_EY1) return dispatch_store(tf, [&](auto a) -> ps_status {
    return dispatch_store(tey, [&](auto b) -> ps_status {
      return dispatch_store(thz, [&](auto c) -> ps_status {
        using SF = decltype(a);
        using SE = decltype(b);
        using SH = decltype(c);
        fdtd_ey_kernel<SF, SE, SH><<<grid, FD_NT, 0, st>>>((const raw_t<SF> *)fict, (raw_t<SE> *)ey,
                                                           (const raw_t<SH> *)hz, t, nx, ny, part, r0, r1);
        PS_CHECK_LAUNCH("fdtd_ey_kernel");
        return PS_OK;
      });
    });
  });
  if (part == FDTD_EX) return dispatch_store(tex, [&](auto a) -> ps_status {
    return dispatch_store(thz, [&](auto c) -> ps_status {
      using SE = decltype(a);
      using SH = decltype(c);
      fdtd_ex_kernel<SE, SH><<<grid, FD_NT, 0, st>>>((raw_t<SE> *)ex, (const raw_t<SH> *)hz, nx, ny, r0, r1);
      PS_CHECK_LAUNCH("fdtd_ex_kernel");
      return PS_OK;
    });
  });
  return dispatch_store(thz, [&](auto a) -> ps_status {
    return dispatch_store(tex, [&](auto b) -> ps_status {
      return dispatch_store(tey, [&](auto c) -> ps_status {
        using SH = decltype(a);
        using SX = decltype(b);
        using SY = decltype(c);
        using T = T3<SH, SX, SY>;
        fdtd_hz_kernel<SH, SX, SY><<<grid, FD_NT, 0, st>>>((raw_t<SH> *)hz, (const raw_t<SX> *)ex,
                                                           (const raw_t<SY> *)ey, nx, ny, (T)0.7, r0, r1);
        PS_CHECK_LAUNCH("fdtd_hz_kernel");
        return PS_OK;
      });
    });
  });
}

}  // namespace ps
