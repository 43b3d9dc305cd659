// cx.cuh -- amplitude types and streaming memory helpers shared by the kernels.
//
// S = double: complex128 amplitudes (double2, 16 B) -- the paper-faithful default
//     (reading R5);
// S = float:  complex64 amplitudes (float2, 8 B) -- NEXT-4 precision variant.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace lfqs {

template <class S>
struct CxT;
template <>
struct CxT<double> {
  using T = double2;
};
template <>
struct CxT<float> {
  using T = float2;
};
template <class S>
using cx = typename CxT<S>::T;

template <class S>
__host__ __device__ __forceinline__ cx<S> mk(S x, S y) {
  cx<S> r;
  r.x = x;
  r.y = y;
  return r;
}

// ---- streaming (evict-first) loads/stores: one amplitude, two adjacent ------
__device__ __forceinline__ double2 ld1(const double2* p) {
  double2 v;
  asm volatile("ld.global.cs.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}
__device__ __forceinline__ float2 ld1(const float2* p) {
  float2 v;
  asm volatile("ld.global.cs.v2.f32 {%0,%1}, [%2];" : "=f"(v.x), "=f"(v.y) : "l"(p));
  return v;
}
__device__ __forceinline__ void st1(double2* p, double2 v) {
  asm volatile("st.global.cs.v2.f64 [%0], {%1,%2};" ::"l"(p), "d"(v.x), "d"(v.y) : "memory");
}
__device__ __forceinline__ void st1(float2* p, float2 v) {
  asm volatile("st.global.cs.v2.f32 [%0], {%1,%2};" ::"l"(p), "f"(v.x), "f"(v.y) : "memory");
}
// Two adjacent amplitudes: 32 B (LDG/STG.256, sm_100a) for complex128, 16 B for complex64.
__device__ __forceinline__ void ld2(const double2* p, double2& a, double2& b) {
  asm volatile("ld.global.cs.v4.f64 {%0,%1,%2,%3}, [%4];"
               : "=d"(a.x), "=d"(a.y), "=d"(b.x), "=d"(b.y)
               : "l"(p));
}
__device__ __forceinline__ void ld2(const float2* p, float2& a, float2& b) {
  asm volatile("ld.global.cs.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(a.x), "=f"(a.y), "=f"(b.x), "=f"(b.y)
               : "l"(p));
}
__device__ __forceinline__ void st2(double2* p, double2 a, double2 b) {
  asm volatile("st.global.cs.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(p), "d"(a.x), "d"(a.y), "d"(b.x),
               "d"(b.y)
               : "memory");
}
__device__ __forceinline__ void st2(float2* p, float2 a, float2 b) {
  asm volatile("st.global.cs.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(a.x), "f"(a.y), "f"(b.x),
               "f"(b.y)
               : "memory");
}

// ---- arithmetic --------------------------------------------------------------
// Pinned complex multiply d*a = (dr ar - di ai, dr ai + di ar), RN, no FMA
// (R8): diagonal results value-exact against the oracle in complex128.
__device__ __forceinline__ double2 cmul_rn(double2 d, double2 a) {
  return make_double2(__dsub_rn(__dmul_rn(d.x, a.x), __dmul_rn(d.y, a.y)),
                      __dadd_rn(__dmul_rn(d.x, a.y), __dmul_rn(d.y, a.x)));
}
__device__ __forceinline__ float2 cmul_rn(float2 d, float2 a) {
  return make_float2(__fsub_rn(__fmul_rn(d.x, a.x), __fmul_rn(d.y, a.y)),
                     __fadd_rn(__fmul_rn(d.x, a.y), __fmul_rn(d.y, a.x)));
}
__device__ __forceinline__ double fma_(double a, double b, double c) { return __fma_rn(a, b, c); }
__device__ __forceinline__ float fma_(float a, float b, float c) { return __fmaf_rn(a, b, c); }
// Complex multiply with FMA: (fma(dr, ar, -(di ai)), fma(dr, ai, di ar)) -- 4 FP ops.
// Only for results in the rounding class (LFQS_FUSE_PHASE tables).
template <class C>
__device__ __forceinline__ C cmul_fma(C d, C a) {
  C r;
  r.x = fma_(d.x, a.x, -(d.y * a.y));
  r.y = fma_(d.x, a.y, d.y * a.x);
  return r;
}
// Accumulating multiply for dense gates (FMA allowed: tolerance class).
template <class C>
__device__ __forceinline__ void cfma(C& acc, C m, C v) {
  acc.x = fma_(m.x, v.x, acc.x);
  acc.x = fma_(-m.y, v.y, acc.x);
  acc.y = fma_(m.x, v.y, acc.y);
  acc.y = fma_(m.y, v.x, acc.y);
}

}  // namespace lfqs
