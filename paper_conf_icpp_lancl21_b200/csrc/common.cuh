// Device helpers shared by the libmars.so kernels.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace mars {

constexpr unsigned kFull = 0xffffffffu;

// splitmix64 mixer (DESIGN.md c12, c14): z += golden; two xor-shift-multiply rounds.
__host__ __device__ __forceinline__ uint64_t sm64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
  return v;
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
  return v;
}

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// PReLU (c6): slope 1 for z > 0, a otherwise.
__device__ __forceinline__ float prelu(float z, float a) { return z > 0.f ? z : a * z; }

// 3xFP16 operand scaling (gemm_tc3h.cu): 2^(14 - e), e = floor(log2 m), so
// m·scale lies in [2^14, 2^15) (below fp16's 65504); 1 for non-finite m.
// An all-zero row gets the largest scale 2^100 (its products stay 0, and a
// min-reduction over row scales -- k_tc3h_dw -- is not pulled down by it).
// Large rows are never clamped (e <= 127 gives a normal 2^-113), so no finite
// row can scale past fp16's range; tiny rows (e < -86) are clamped at 2^100
// and keep their precision relative to 2^-86 (absolute, below ~2^-108).
__device__ __forceinline__ float pow2_scale(float m) {
  if (m == 0.f) return 0x1p100f;
  if (!(m > 0.f) || !(m < INFINITY)) return 1.f;
  const int e = ilogbf(m);
  const int sh = min(100, 14 - e);
  return ldexpf(1.f, sh);
}

// Launch counter bump used by every launcher (mars_dgi_last_launches).
__host__ inline void count_launch(int* launches, int n = 1) {
  if (launches) *launches += n;
}

inline unsigned cdiv(int64_t a, int64_t b) { return (unsigned)((a + b - 1) / b); }


// Split-K combination of the weight-gradient partials, deterministic:
// dW[c][h] = Σ_k part[k][h·CIN + c] in fp64.  Block = 32 consecutive outputs ×
// 8 k-groups (group j sums k = j, j+8, ...), the 8 group sums combined in order
// j = 0..7; grid = ceil(H·CIN / 32) blocks of 256 threads.
// kDwRedVec consecutive outputs per lane (16-byte loads: n = H * CIN is a
// multiple of 4); per output the same fixed order as one output per lane.
#ifndef MARS_DWRED_VEC
#define MARS_DWRED_VEC 4
#endif
constexpr int kDwRedVec = MARS_DWRED_VEC;
inline unsigned dw_reduce_blocks(int64_t n) { return (unsigned)((n + 32 * kDwRedVec - 1) / (32 * kDwRedVec)); }
__device__ __forceinline__ void dw_reduce_body(const float* __restrict__ part, int nchunk, int CIN,
                                               int H, float* __restrict__ dW) {
  constexpr int VV = kDwRedVec;
  __shared__ double sh[8][32 * VV];
  const int lane = threadIdx.x & 31, j = threadIdx.x >> 5;
  const int64_t n = (int64_t)H * CIN;
  const int64_t e = ((int64_t)blockIdx.x * 32 + lane) * VV;   // e = h * CIN + c, VV consecutive
  double t[VV];
#pragma unroll
  for (int v = 0; v < VV; ++v) t[v] = 0.0;
  auto ld = [&](int k, float (&a)[VV]) {
    if constexpr (VV == 4) {
      const float4 x = *reinterpret_cast<const float4*>(part + (int64_t)k * n + e);
      a[0] = x.x; a[1] = x.y; a[2] = x.z; a[3] = x.w;
    } else {
#pragma unroll
      for (int v = 0; v < VV; ++v) a[v] = part[(int64_t)k * n + e + v];
    }
  };
  if (e < n) {
    // loads issued four chunks at a time, summed in the fixed order k = j, j+8, ...
    int k = j;
    for (; k + 24 < nchunk; k += 32) {
      float a0[VV], a1[VV], a2[VV], a3[VV];
      ld(k, a0); ld(k + 8, a1); ld(k + 16, a2); ld(k + 24, a3);
#pragma unroll
      for (int v = 0; v < VV; ++v) {
        t[v] += (double)a0[v];
        t[v] += (double)a1[v];
        t[v] += (double)a2[v];
        t[v] += (double)a3[v];
      }
    }
    for (; k < nchunk; k += 8) {
      float a[VV];
      ld(k, a);
#pragma unroll
      for (int v = 0; v < VV; ++v) t[v] += (double)a[v];
    }
  }
#pragma unroll
  for (int v = 0; v < VV; ++v) sh[j][lane * VV + v] = t[v];
  __syncthreads();
  if (j == 0 && e < n) {
#pragma unroll
    for (int v = 0; v < VV; ++v) {
      double s = 0.0;
#pragma unroll
      for (int q = 0; q < 8; ++q) s += sh[q][lane * VV + v];
      const int h = (int)((e + v) / CIN), c = (int)((e + v) % CIN);
      dW[(int64_t)c * H + h] = (float)s;
    }
  }
}

}  // namespace mars
