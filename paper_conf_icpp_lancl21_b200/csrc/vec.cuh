// 16-byte vector load / store helpers over the activation storage types
// (fp32 for the reference-precision path, bf16 for the bf16 path); all
// arithmetic is fp32.
#pragma once
#include <cuda_bf16.h>
#include <stdint.h>

namespace mars {

typedef __nv_bfloat16 bf16;

template <typename T>
struct Vec;

template <>
struct Vec<float> {
  static constexpr int N = 4;  // elements per 16 bytes
  __device__ __forceinline__ static void load(const float* p, float (&x)[4]) {
    cvt(ld(p), x);
  }
  // raw 16-byte form: a load kept in flight costs 4 registers whatever T is
  typedef float4 Raw;
  __device__ __forceinline__ static Raw ld(const float* p) {
    return __ldg(reinterpret_cast<const float4*>(p));
  }
  __device__ __forceinline__ static void cvt(const Raw& v, float (&x)[4]) {
    x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
  }
};

template <>
struct Vec<bf16> {
  static constexpr int N = 8;
  __device__ __forceinline__ static void load(const bf16* p, float (&x)[8]) {
    cvt(ld(p), x);
  }
  typedef uint4 Raw;
  __device__ __forceinline__ static Raw ld(const bf16* p) {
    return __ldg(reinterpret_cast<const uint4*>(p));
  }
  __device__ __forceinline__ static void cvt(const Raw& v, float (&x)[8]) {
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      x[2 * k] = __uint_as_float(w[k] << 16);
      x[2 * k + 1] = __uint_as_float(w[k] & 0xFFFF0000u);
    }
  }
};

// Store n consecutive values (n = 4 or 8) as T.
template <typename T, int n>
struct StoreN;

template <int n>
struct StoreN<float, n> {
  __device__ __forceinline__ static void store(float* p, const float* x) {
#pragma unroll
    for (int k = 0; k < n; k += 4)
      *reinterpret_cast<float4*>(p + k) = make_float4(x[k], x[k + 1], x[k + 2], x[k + 3]);
  }
};

__device__ __forceinline__ uint32_t pack_bf16x2(float lo, float hi) {
  const __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<const uint32_t*>(&v);
}

template <>
struct StoreN<bf16, 4> {
  __device__ __forceinline__ static void store(bf16* p, const float* x) {
    *reinterpret_cast<uint2*>(p) = make_uint2(pack_bf16x2(x[0], x[1]), pack_bf16x2(x[2], x[3]));
  }
};

template <>
struct StoreN<bf16, 8> {
  __device__ __forceinline__ static void store(bf16* p, const float* x) {
    *reinterpret_cast<uint4*>(p) = make_uint4(pack_bf16x2(x[0], x[1]), pack_bf16x2(x[2], x[3]),
                                              pack_bf16x2(x[4], x[5]), pack_bf16x2(x[6], x[7]));
  }
};

__device__ __forceinline__ float to_f(float x) { return x; }
__device__ __forceinline__ float to_f(bf16 x) { return __bfloat162float(x); }
__device__ __forceinline__ void from_f(float v, float* p) { *p = v; }
__device__ __forceinline__ void from_f(float v, bf16* p) { *p = __float2bfloat16_rn(v); }

}  // namespace mars
