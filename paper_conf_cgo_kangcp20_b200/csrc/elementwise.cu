// elementwise.cu -- element-wise statements (row a3): GESUMMV's
// y <- alpha*tmp + beta*y, CORR's normalisation and COVAR's centring.
// Each op is one correctly rounded IEEE op in the statement's compute type T
// (readings R2/R4); stores round RNE to the object's precision (R1).
#include <math.h>

#include "common.cuh"
#include "kernels.cuh"
#include "types.cuh"

namespace ps {

// --------------------------------------------------- GESUMMV statement 3
template <class STMP, class SY>
__global__ void axpby_kernel(const raw_t<STMP> *__restrict__ tmp, raw_t<SY> *__restrict__ y,
                             int64_t n, T2<STMP, SY> al, T2<STMP, SY> be) {
  using T = T2<STMP, SY>;
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const T r = t_fma(al, ldg_t<STMP, T>(tmp, i), be * Ld<SY, T>::get(y, (size_t)i));
  St<SY, T>::put(y, (size_t)i, r);
}

ps_status axpby_async(const void *tmp, int ttmp, void *y, int ty, int64_t n, double alpha,
                      double beta, cudaStream_t st) {
  if (n <= 0) return PS_OK;
  const unsigned nb = (unsigned)((n + 255) / 256);
  return dispatch_store(ttmp, [&](auto s1) -> ps_status {
    return dispatch_store(ty, [&](auto s2) -> ps_status {
      using S1 = decltype(s1);
      using S2 = decltype(s2);
      using T = T2<S1, S2>;
      // alpha, beta: RNE from their fp64 literal to T (R2)
      axpby_kernel<S1, S2><<<nb, 256, 0, st>>>((const raw_t<S1> *)tmp, (raw_t<S2> *)y, n, (T)alpha,
                                               (T)beta);
      PS_CHECK_LAUNCH("axpby_kernel");
      return PS_OK;
    });
  });
}

// ------------------------------------------------------ CORR / COVAR
template <class SD, class SM, class SS>
__global__ void __launch_bounds__(256) corr_normalize_kernel(raw_t<SD> *__restrict__ data,
                                                             const raw_t<SM> *__restrict__ mean,
                                                             const raw_t<SS> *__restrict__ sd,
                                                             int64_t rows, int64_t cols,
                                                             T3<SD, SM, SS> sqn) {
  using T = T3<SD, SM, SS>;
  const int64_t total = rows * cols;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = e % cols;
    const T d = Ld<SD, T>::get(data, (size_t)e) - ldg_t<SM, T>(mean, j);
    const T den = sqn * ldg_t<SS, T>(sd, j);
    St<SD, T>::put(data, (size_t)e, d / den);
  }
}

ps_status corr_normalize_async(void *data, int td, const void *mean, int tm, const void *sd, int ts,
                               int64_t rows, int64_t cols, double sqrt_n, cudaStream_t st) {
  const int64_t total = rows * cols;
  if (total <= 0) return PS_OK;
  int64_t blocks = (total + 255) / 256;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  return dispatch_store(td, [&](auto a) -> ps_status {
    return dispatch_store(tm, [&](auto b) -> ps_status {
      return dispatch_store(ts, [&](auto c) -> ps_status {
        using SD = decltype(a);
        using SM = decltype(b);
        using SS = decltype(c);
        using T = T3<SD, SM, SS>;
        corr_normalize_kernel<SD, SM, SS><<<(unsigned)blocks, 256, 0, st>>>(
            (raw_t<SD> *)data, (const raw_t<SM> *)mean, (const raw_t<SS> *)sd, rows, cols,
            (T)sqrt_n);
        PS_CHECK_LAUNCH("corr_normalize_kernel");
        return PS_OK;
      });
    });
  });
}

template <class SD, class SM>
__global__ void __launch_bounds__(256) covar_center_kernel(raw_t<SD> *__restrict__ data,
                                                           const raw_t<SM> *__restrict__ mean,
                                                           int64_t rows, int64_t cols) {
  using T = T2<SD, SM>;
  const int64_t total = rows * cols;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = e % cols;
    St<SD, T>::put(data, (size_t)e, Ld<SD, T>::get(data, (size_t)e) - ldg_t<SM, T>(mean, j));
  }
}

ps_status covar_center_async(void *data, int td, const void *mean, int tm, int64_t rows,
                             int64_t cols, cudaStream_t st) {
  const int64_t total = rows * cols;
  if (total <= 0) return PS_OK;
  int64_t blocks = (total + 255) / 256;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  return dispatch_store(td, [&](auto a) -> ps_status {
    return dispatch_store(tm, [&](auto b) -> ps_status {
      using SD = decltype(a);
      using SM = decltype(b);
      covar_center_kernel<SD, SM><<<(unsigned)blocks, 256, 0, st>>>(
          (raw_t<SD> *)data, (const raw_t<SM> *)mean, rows, cols);
      PS_CHECK_LAUNCH("covar_center_kernel");
      return PS_OK;
    });
  });
}

}  // namespace ps
