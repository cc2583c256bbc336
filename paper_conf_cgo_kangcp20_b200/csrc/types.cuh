// types.cuh -- compile-time compute-type helpers (reading R2) shared by the
// bandwidth-bound kernels.
#pragma once
#include <type_traits>

#include "common.cuh"

namespace ps {

template <class A, class B> struct Wider { using t = float; };
template <class B> struct Wider<double, B> { using t = double; };
template <class A> struct Wider<A, double> { using t = double; };
template <> struct Wider<double, double> { using t = double; };
template <class S> struct CT { using t = typename Wider<S, float>::t; };   // storage -> min compute
template <> struct CT<F16> { using t = float; };
template <> struct CT<BF16> { using t = float; };
// R2: T = W(objects touched, f32)
template <class A, class B, class C>
using T3 = typename Wider<typename Wider<typename CT<A>::t, typename CT<B>::t>::t,
                          typename CT<C>::t>::t;
template <class A, class B>
using T2 = typename Wider<typename CT<A>::t, typename CT<B>::t>::t;

template <class S, class T>
__device__ __forceinline__ T ldg_t(const raw_t<S> *p, int64_t i) {
  return Ld<S, T>::get(p, (size_t)i);
}

// element i of a buffer whose storage type is only known at run time
template <class T>
__device__ __forceinline__ T load_any(const void *p, int type, int64_t i) {
  switch (type) {
    case PS_F64: return (T)__ldg((const double *)p + i);
    case PS_F32: return (T)__ldg((const float *)p + i);
    case PS_BF16: return widen_b<T>(__ldg((const unsigned short *)p + i));
    default: return widen_h<T>(__ldg((const unsigned short *)p + i));
  }
}

}  // namespace ps
