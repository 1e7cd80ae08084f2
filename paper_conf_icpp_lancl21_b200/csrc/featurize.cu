// NEXT-1 featuriser: an op list -> the per-op feature matrix X
// the encoder consumes ("the operation type is encoded as a one-hot
// vector ... input and output shapes ... normalised"; reading c16).
//   X[i][t]           = 1 for t = min(type_i, F - 9)   (slots [0, F-8): one-hot type,
//                                                       overflow types share "other")
//   X[i][F - 8 + j]   = f32(dims[i][j] / D) for dims > 0, else 0
//                       (j < 4: first input's dims, j >= 4: the op's output dims;
//                        D = the largest dim of the whole graph)
// Two kernels: a grid-stride max over the 8N dims (atomicMax of per-warp
// maxima), then one thread per output element (coalesced row-major writes).
#include "../../include/mars.h"
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

__global__ void k_dims_max(const int64_t* __restrict__ dims, int64_t n,
                           unsigned long long* __restrict__ out) {
  long long m = 0;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
       e += (int64_t)gridDim.x * blockDim.x)
    m = max(m, (long long)dims[e]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(kFull, m, o));
  if ((threadIdx.x & 31) == 0 && m > 0) atomicMax(out, (unsigned long long)m);
}

__global__ void k_featurize(const int32_t* __restrict__ types, const int64_t* __restrict__ dims,
                            int32_t N, int32_t F, const unsigned long long* __restrict__ dmax,
                            float* __restrict__ X) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= (int64_t)N * F) return;
  const int32_t i = (int32_t)(e / F), c = (int32_t)(e % F);
  float x = 0.f;
  if (c < F - 8) {
    const int32_t t = types[i];
    x = (t < F - 8 ? t : F - 9) == c ? 1.f : 0.f;
  } else {
    const int64_t d = dims[(int64_t)i * 8 + (c - (F - 8))];
    if (d > 0) x = __double2float_rn(__ddiv_rn((double)d, (double)*dmax));
  }
  X[e] = x;
}

}  // namespace

cudaError_t launch_featurize(const int32_t* types, const int64_t* dims, int32_t N, int32_t F,
                             unsigned long long* dmax, float* X, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(dmax, 0, sizeof(unsigned long long), s);
  if (e != cudaSuccess) return e;
  const int64_t n = 8LL * N;
  k_dims_max<<<std::min<unsigned>(cdiv(n, 256), 1184), 256, 0, s>>>(dims, n, dmax);
  k_featurize<<<cdiv((int64_t)N * F, 256), 256, 0, s>>>(types, dims, N, F, dmax, X);
  return cudaGetLastError();
}

}  // namespace mars
