// kcommon.cuh — device helpers shared by the kernel templates.
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace mdh {

// ---------------------------------------------------------------- element access
__device__ __forceinline__ float bf16_to_f32(uint16_t b) { return __uint_as_float(((uint32_t)b) << 16); }

template <class V>
__device__ __forceinline__ V load_as(const void* p, int dt, int64_t i) {
  switch (dt) {
    case MDH_BF16: return (V)bf16_to_f32(((const uint16_t*)p)[i]);
    case MDH_F32: return (V)__ldg(((const float*)p) + i);
    case MDH_F64: return (V)__ldg(((const double*)p) + i);
    case MDH_I32: return (V)__ldg(((const int32_t*)p) + i);
    case MDH_U32: return (V)__ldg(((const uint32_t*)p) + i);
    case MDH_I64: return (V)__ldg(((const long long*)p) + i);
  }
  return (V)0;
}

template <class V>
__device__ __forceinline__ void store_as(void* p, int dt, int64_t i, V v) {
  switch (dt) {
    case MDH_BF16: ((__nv_bfloat16*)p)[i] = __float2bfloat16_rn((float)v); break;
    case MDH_F32: ((float*)p)[i] = (float)v; break;
    case MDH_F64: ((double*)p)[i] = (double)v; break;
    case MDH_I32: ((int32_t*)p)[i] = (int32_t)v; break;
    case MDH_U32: ((uint32_t*)p)[i] = (uint32_t)v; break;
    case MDH_I64: ((long long*)p)[i] = (long long)v; break;
  }
}

// ------------------------------------------------------- f and ⊕ (the catalog)
// int32 arithmetic wraps mod 2^32 (reading C-12): done in unsigned to avoid UB.
template <class V> struct Arith {
  __device__ static __forceinline__ V mul(V a, V b) { return a * b; }
  __device__ static __forceinline__ V add(V a, V b) { return a + b; }
  __device__ static __forceinline__ V mul_add(V acc, V w, V x) { return acc + w * x; }
};
template <> struct Arith<int32_t> {
  __device__ static __forceinline__ int32_t mul(int32_t a, int32_t b) { return (int32_t)((uint32_t)a * (uint32_t)b); }
  __device__ static __forceinline__ int32_t add(int32_t a, int32_t b) { return (int32_t)((uint32_t)a + (uint32_t)b); }
  __device__ static __forceinline__ int32_t mul_add(int32_t acc, int32_t w, int32_t x) { return add(acc, mul(w, x)); }
};
template <> struct Arith<long long> {
  __device__ static __forceinline__ long long mul(long long a, long long b) { return (long long)((unsigned long long)a * (unsigned long long)b); }
  __device__ static __forceinline__ long long add(long long a, long long b) { return (long long)((unsigned long long)a + (unsigned long long)b); }
  __device__ static __forceinline__ long long mul_add(long long acc, long long w, long long x) { return add(acc, mul(w, x)); }
};

template <class V>
__device__ __forceinline__ V combine_op(int op, V l, V r) {
  switch (op) {
    case MDH_PW_ADD: return Arith<V>::add(l, r);
    case MDH_PW_MAX: return r > l ? r : l;
    case MDH_PW_MIN: return r < l ? r : l;
  }
  return r;
}

template <int OP, class V>
__device__ __forceinline__ V combine_t(V l, V r) {
  if constexpr (OP == MDH_PW_ADD) return Arith<V>::add(l, r);
  else if constexpr (OP == MDH_PW_MAX) return r > l ? r : l;
  else return r < l ? r : l;
}

template <int OP, class V>
__device__ __forceinline__ V identity_t();

template <class V> struct Lim;
template <> struct Lim<float> { __device__ static float lo() { return -__int_as_float(0x7f800000); } __device__ static float hi() { return __int_as_float(0x7f800000); } };
template <> struct Lim<double> { __device__ static double lo() { return -__longlong_as_double(0x7ff0000000000000LL); } __device__ static double hi() { return __longlong_as_double(0x7ff0000000000000LL); } };
template <> struct Lim<int32_t> { __device__ static int32_t lo() { return INT32_MIN; } __device__ static int32_t hi() { return INT32_MAX; } };
template <> struct Lim<uint32_t> { __device__ static uint32_t lo() { return 0u; } __device__ static uint32_t hi() { return 0xFFFFFFFFu; } };
template <> struct Lim<long long> { __device__ static long long lo() { return INT64_MIN; } __device__ static long long hi() { return INT64_MAX; } };

// neutral elements of the built-in pw operators (reading C-11)
template <int OP, class V>
__device__ __forceinline__ V identity_t() {
  if constexpr (OP == MDH_PW_ADD) return (V)0;
  else if constexpr (OP == MDH_PW_MAX) return Lim<V>::lo();
  else return Lim<V>::hi();
}

template <int OP, class V>
__device__ __forceinline__ V warp_reduce(V v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = combine_t<OP, V>(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

}  // namespace mdh
