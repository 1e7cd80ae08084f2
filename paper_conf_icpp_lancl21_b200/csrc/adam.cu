// a14: Adam over the flat fp32 parameter vector, torch.optim.Adam semantics
// (no weight decay, no amsgrad; reading c13), with optional global-norm
// clipping (torch.nn.utils.clip_grad_norm_: coef = clip / (norm + 1e-6),
// applied when < 1).  Bias corrections come from the step's StepParams.
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

constexpr int kNormBlocks = 148;

__global__ void k_norm_part(const float* __restrict__ g, int64_t P, double* __restrict__ part) {
  __shared__ double sh[256];
  double t = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * 256 + threadIdx.x; i < P; i += (int64_t)gridDim.x * 256)
    t += (double)g[i] * (double)g[i];
  sh[threadIdx.x] = t;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) part[blockIdx.x] = sh[0];
}

__global__ void k_norm_final(double* __restrict__ part, float clip) {
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int k = 0; k < kNormBlocks; ++k) t += part[k];
    double coef = (double)clip / (sqrt(t) + 1e-6);
    part[kNormBlocks] = coef < 1.0 ? coef : 1.0;
  }
}

__global__ void k_adam(float* __restrict__ p, float* __restrict__ m, float* __restrict__ v,
                       const float* __restrict__ g, int64_t P, float b1, float omb1, float b2,
                       float omb2, float eps, const double* __restrict__ clip_coef,
                       const StepParams* __restrict__ sp) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P) return;
  float gi = g[i];
  if (clip_coef) gi = (float)((double)gi * clip_coef[kNormBlocks]);
  float mi = fmaf(b1, m[i], omb1 * gi);
  float vi = fmaf(b2, v[i], omb2 * gi * gi);
  m[i] = mi;
  v[i] = vi;
  float denom = sqrtf(vi) / sp->adam_bc2_sqrt + eps;
  p[i] -= sp->adam_step_size * (mi / denom);
}

__global__ void k_check_finite(const float* __restrict__ loss, int32_t* __restrict__ flag) {
  if (threadIdx.x == 0) *flag = isfinite(*loss) ? 0 : 1;
}

}  // namespace

cudaError_t launch_adam(float* params, float* m, float* v, const float* grads, int64_t P,
                        double beta1, double beta2, double eps, double clip_norm, double* norm_part,
                        const StepParams* sp, cudaStream_t s, int* launches) {
  const double* coef = nullptr;
  if (clip_norm > 0.0) {
    k_norm_part<<<kNormBlocks, 256, 0, s>>>(grads, P, norm_part);
    k_norm_final<<<1, 32, 0, s>>>(norm_part, clip_norm);
    count_launch(launches, 2);
    coef = norm_part;
  }
  // torch semantics: tensor.mul_(beta) multiplies by f32(beta), the
  // (1 - beta) factors are formed in double and rounded once.
  k_adam<<<cdiv(P, 256), 256, 0, s>>>(params, m, v, grads, P, (float)beta1, (float)(1.0 - beta1),
                                      (float)beta2, (float)(1.0 - beta2), (float)eps, coef, sp);
  count_launch(launches);
  return cudaGetLastError();
}

cudaError_t launch_check_finite(const float* loss, int32_t* flag, cudaStream_t s, int* launches) {
  k_check_finite<<<1, 32, 0, s>>>(loss, flag);
  count_launch(launches);
  return cudaGetLastError();
}

}  // namespace mars
