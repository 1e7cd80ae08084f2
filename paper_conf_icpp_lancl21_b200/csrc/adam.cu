// a14: Adam over the flat fp32 parameter vector, torch.optim.Adam semantics
// (no weight decay, no amsgrad; reading c13), with optional global-norm
// clipping (torch.nn.utils.clip_grad_norm_: coef = clip / (norm + 1e-6),
// applied when < 1).
//
// Guarded update: before Adam, k_guard_part / k_guard_final form Σ g_i² in
// fp64 over the (global, after the gradient exchange) gradient vector and
// check the loss.  Σ g_i² is non-finite iff some g_i is (fp32 squares cannot
// overflow fp64), so one pass serves both the clip norm and the finiteness
// check.  A non-finite loss or gradient skips the update (params, m, v and the
// step count t unchanged) and bumps AdamDev::skipped, which the runtime turns
// into MARS_ENUMERIC on the next read.  t and the bias corrections live on the
// device, so a skipped (or failed-to-launch) step never advances them.
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

constexpr int kGuardBlocks = 148;

__global__ void __launch_bounds__(256) k_guard_part(const float* __restrict__ g, int64_t P,
                                                    double* __restrict__ part) {
  __shared__ double sh[8];
  double t = 0.0;
  const int64_t n4 = P / 4;
  const float4* g4 = reinterpret_cast<const float4*>(g);
  for (int64_t i = (int64_t)blockIdx.x * 256 + threadIdx.x; i < n4; i += (int64_t)gridDim.x * 256) {
    const float4 x = g4[i];
    t += (double)x.x * x.x + (double)x.y * x.y + (double)x.z * x.z + (double)x.w * x.w;
  }
  if (blockIdx.x == 0 && threadIdx.x < (P & 3)) {
    const double x = g[n4 * 4 + threadIdx.x];
    t += x * x;
  }
  t = warp_sum(t);
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = t;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int k = 0; k < 8; ++k) s += sh[k];
    part[blockIdx.x] = s;
  }
}

// One thread: the decision and the bias corrections of this step.
__global__ void k_guard_final(const double* __restrict__ part, const float* __restrict__ loss,
                              float clip, double lr, double b1, double b2,
                              AdamDev* __restrict__ st) {
  if (threadIdx.x != 0) return;
  double t = 0.0;
  for (int k = 0; k < kGuardBlocks; ++k) t += part[k];
  const bool ok = isfinite(t) && isfinite(*loss);
  st->skip = ok ? 0 : 1;
  if (!ok) {
    st->skipped += 1;
    return;
  }
  const int64_t tn = st->t + 1;
  st->t = tn;
  const double coef = clip > 0.f ? (double)clip / (sqrt(t) + 1e-6) : 1.0;
  st->clip_coef = coef < 1.0 ? coef : 1.0;
  st->step_size = (float)(lr / (1.0 - pow(b1, (double)tn)));
  st->bc2_sqrt = (float)sqrt(1.0 - pow(b2, (double)tn));
}

__global__ void k_adam(float* __restrict__ p, float* __restrict__ m, float* __restrict__ v,
                       const float* __restrict__ g, int64_t P, float b1, float omb1, float b2,
                       float omb2, float eps, int clip, const AdamDev* __restrict__ st) {
  if (st->skip) return;
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P) return;
  float gi = g[i];
  if (clip) gi = (float)((double)gi * st->clip_coef);
  float mi = fmaf(b1, m[i], omb1 * gi);
  float vi = fmaf(b2, v[i], omb2 * gi * gi);
  m[i] = mi;
  v[i] = vi;
  float denom = sqrtf(vi) / st->bc2_sqrt + eps;
  p[i] -= st->step_size * (mi / denom);
}

}  // namespace

int adam_guard_doubles() { return kGuardBlocks; }

cudaError_t launch_adam(float* params, float* m, float* v, const float* grads, int64_t P,
                        double lr, double beta1, double beta2, double eps, double clip_norm,
                        double* guard_part, AdamDev* st, cudaStream_t s, int* launches) {
  k_guard_part<<<kGuardBlocks, 256, 0, s>>>(grads, P, guard_part);
  k_guard_final<<<1, 32, 0, s>>>(guard_part, grads + P, (float)clip_norm, lr, beta1, beta2, st);
  // torch semantics: tensor.mul_(beta) multiplies by f32(beta), the
  // (1 - beta) factors are formed in double and rounded once.
  k_adam<<<cdiv(P, 256), 256, 0, s>>>(params, m, v, grads, P, (float)beta1, (float)(1.0 - beta1),
                                      (float)beta2, (float)(1.0 - beta2), (float)eps,
                                      clip_norm > 0.0 ? 1 : 0, st);
  count_launch(launches, 3);
  return cudaGetLastError();
}

}  // namespace mars
