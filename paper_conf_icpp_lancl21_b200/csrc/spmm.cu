// a5 (+a4 gather, a7 PReLU, a12 PReLU'): the aggregation Y = Â_n · act(T) of
// Eq. 1 for the stacked [pos; neg] activations, and its backward
// dH = Â_nᵀ dY = Â_n dY (Â_n is symmetric, c1).
//
// Layout: T is R×C row-major with R = 2·Nt (rows [0,Nt) positive branch, rows
// [Nt,2Nt) corrupted branch).  Both branches share the CSR (the corrupted graph
// has the same structure), so one (colind, val) read feeds two row
// gathers.  Sub-warp per row: L = min(32, C/4) lanes own C/L consecutive
// columns each as float4, so every neighbour row is one coalesced transaction
// per branch; 32/L rows share a warp when C < 128.
//   fwd layer 1: T = X, neg rows gather X[pi[j]] (the corruption, fused)
//   fwd layer l>1: act = PReLU_{a_{l-1}} applied on load (H_{l-1} never stored)
//   bwd: epilogue dZ = dH ⊙ PReLU'(Z), dalpha partials Σ dH·min(Z,0) per block
// Accumulation is fp32 in ascending colind order (deterministic).
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

constexpr int kSpmmThreads = 256;
constexpr int kU = 4;           // neighbours whose gathers are in flight together

// C in {16, 32, 64, 128, 256} (mars.h restricts F and H to these widths).
template <int C>
struct SpmmShape {
  static constexpr int L = (C / 4) < 32 ? (C / 4) : 32;  // lanes per row
  static constexpr int RPW = 32 / L;                      // rows per warp
  static constexpr int NT = C / (4 * L);                  // float4 per lane per branch
  static constexpr int RPB = RPW * (kSpmmThreads / 32);   // rows per block
};

__device__ __forceinline__ float4 f4_prelu(float4 x, float a) {
  return make_float4(prelu(x.x, a), prelu(x.y, a), prelu(x.z, a), prelu(x.w, a));
}

__device__ __forceinline__ void f4_fma(float4& acc, float w, float4 x) {
  acc.x = fmaf(w, x.x, acc.x);
  acc.y = fmaf(w, x.y, acc.y);
  acc.z = fmaf(w, x.z, acc.z);
  acc.w = fmaf(w, x.w, acc.w);
}

// MODE 0: layer 1 (neg rows gather X[perm[j]]), MODE 1: PReLU on load.
template <int C, int MODE, bool BOTH>
__global__ void __launch_bounds__(kSpmmThreads)
k_spmm_fwd(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
           const float* __restrict__ vals, const float* __restrict__ T,
           const int32_t* __restrict__ perm, const float* __restrict__ alpha, int act_layer,
           int32_t Nt, float* __restrict__ Y) {
  using S = SpmmShape<C>;
  const int lane = threadIdx.x & 31;
  const int sub = lane / S::L, sl = lane % S::L;
  const unsigned gmask = (S::L == 32) ? kFull : (((1u << S::L) - 1u) << (sub * S::L));
  const int32_t i = (int32_t)(((int64_t)blockIdx.x * kSpmmThreads + threadIdx.x) / 32) * S::RPW + sub;
  if (i >= Nt) return;
  const float a = (MODE == 1) ? alpha[act_layer] : 1.f;
  const int32_t rb = rowptr[i], re = rowptr[i + 1];
  float4 accp[S::NT], accn[S::NT];
#pragma unroll
  for (int t = 0; t < S::NT; ++t) accp[t] = accn[t] = make_float4(0.f, 0.f, 0.f, 0.f);
  const float4* T4 = reinterpret_cast<const float4*>(T);
  for (int32_t k0 = rb; k0 < re; k0 += S::L) {
    int32_t cnt = min(S::L, re - k0);
    int32_t myj = 0, myjn = 0;
    float myv = 0.f;
    if (sl < cnt) {
      myj = colind[k0 + sl];
      myv = vals[k0 + sl];
      if (BOTH) myjn = (MODE == 0) ? perm[myj] : Nt + myj;
    }
    // groups of kU neighbours: every gather of the group is issued before the
    // first FMA (memory-level parallelism); FMAs stay in ascending colind order
    int t = 0;
    for (; t + kU <= cnt; t += kU) {
      int32_t j[kU], jn[kU];
      float w[kU];
      float4 xp[kU][S::NT], xn[kU][S::NT];
#pragma unroll
      for (int u = 0; u < kU; ++u) {
        j[u] = __shfl_sync(gmask, myj, t + u, S::L);
        w[u] = __shfl_sync(gmask, myv, t + u, S::L);
        jn[u] = BOTH ? __shfl_sync(gmask, myjn, t + u, S::L) : 0;
      }
#pragma unroll
      for (int u = 0; u < kU; ++u)
#pragma unroll
        for (int q = 0; q < S::NT; ++q) {
          const int c4 = sl + q * S::L;
          xp[u][q] = __ldg(T4 + (int64_t)j[u] * (C / 4) + c4);
          if (BOTH) xn[u][q] = __ldg(T4 + (int64_t)jn[u] * (C / 4) + c4);
        }
#pragma unroll
      for (int u = 0; u < kU; ++u)
#pragma unroll
        for (int q = 0; q < S::NT; ++q) {
          f4_fma(accp[q], w[u], MODE == 1 ? f4_prelu(xp[u][q], a) : xp[u][q]);
          if (BOTH) f4_fma(accn[q], w[u], MODE == 1 ? f4_prelu(xn[u][q], a) : xn[u][q]);
        }
    }
    for (; t < cnt; ++t) {
      int32_t j = __shfl_sync(gmask, myj, t, S::L);
      float w = __shfl_sync(gmask, myv, t, S::L);
      int32_t jn = BOTH ? __shfl_sync(gmask, myjn, t, S::L) : 0;
#pragma unroll
      for (int q = 0; q < S::NT; ++q) {
        int c4 = sl + q * S::L;
        float4 xp = __ldg(T4 + (int64_t)j * (C / 4) + c4);
        if (MODE == 1) xp = f4_prelu(xp, a);
        f4_fma(accp[q], w, xp);
        if (BOTH) {
          float4 xn = __ldg(T4 + (int64_t)jn * (C / 4) + c4);
          if (MODE == 1) xn = f4_prelu(xn, a);
          f4_fma(accn[q], w, xn);
        }
      }
    }
  }
  float4* Y4 = reinterpret_cast<float4*>(Y);
#pragma unroll
  for (int q = 0; q < S::NT; ++q) {
    int c4 = sl + q * S::L;
    Y4[(int64_t)i * (C / 4) + c4] = accp[q];
    if (BOTH) Y4[((int64_t)Nt + i) * (C / 4) + c4] = accn[q];
  }
}

template <int C>
__global__ void __launch_bounds__(kSpmmThreads)
k_spmm_bwd(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
           const float* __restrict__ vals, const float* __restrict__ dY,
           const float* __restrict__ Z, const float* __restrict__ alpha, int layer, int32_t Nt,
           float* __restrict__ dZ, double* __restrict__ slots) {
  using S = SpmmShape<C>;
  __shared__ double wpart[kSpmmThreads / 32];
  const int lane = threadIdx.x & 31;
  const int sub = lane / S::L, sl = lane % S::L;
  const unsigned gmask = (S::L == 32) ? kFull : (((1u << S::L) - 1u) << (sub * S::L));
  const int32_t i = (int32_t)(((int64_t)blockIdx.x * kSpmmThreads + threadIdx.x) / 32) * S::RPW + sub;
  float da = 0.f;
  if (i < Nt) {
    const float a = alpha[layer];
    const int32_t rb = rowptr[i], re = rowptr[i + 1];
    float4 accp[S::NT], accn[S::NT];
#pragma unroll
    for (int t = 0; t < S::NT; ++t) accp[t] = accn[t] = make_float4(0.f, 0.f, 0.f, 0.f);
    const float4* D4 = reinterpret_cast<const float4*>(dY);
    for (int32_t k0 = rb; k0 < re; k0 += S::L) {
      int32_t cnt = min(S::L, re - k0);
      int32_t myj = 0;
      float myv = 0.f;
      if (sl < cnt) {
        myj = colind[k0 + sl];
        myv = vals[k0 + sl];
      }
      int t = 0;
      for (; t + kU <= cnt; t += kU) {
        int32_t j[kU];
        float w[kU];
        float4 xp[kU][S::NT], xn[kU][S::NT];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
          j[u] = __shfl_sync(gmask, myj, t + u, S::L);
          w[u] = __shfl_sync(gmask, myv, t + u, S::L);
        }
#pragma unroll
        for (int u = 0; u < kU; ++u)
#pragma unroll
          for (int q = 0; q < S::NT; ++q) {
            const int c4 = sl + q * S::L;
            xp[u][q] = __ldg(D4 + (int64_t)j[u] * (C / 4) + c4);
            xn[u][q] = __ldg(D4 + ((int64_t)Nt + j[u]) * (C / 4) + c4);
          }
#pragma unroll
        for (int u = 0; u < kU; ++u)
#pragma unroll
          for (int q = 0; q < S::NT; ++q) {
            f4_fma(accp[q], w[u], xp[u][q]);
            f4_fma(accn[q], w[u], xn[u][q]);
          }
      }
      for (; t < cnt; ++t) {
        int32_t j = __shfl_sync(gmask, myj, t, S::L);
        float w = __shfl_sync(gmask, myv, t, S::L);
#pragma unroll
        for (int q = 0; q < S::NT; ++q) {
          int c4 = sl + q * S::L;
          f4_fma(accp[q], w, __ldg(D4 + (int64_t)j * (C / 4) + c4));
          f4_fma(accn[q], w, __ldg(D4 + ((int64_t)Nt + j) * (C / 4) + c4));
        }
      }
    }
    const float4* Z4 = reinterpret_cast<const float4*>(Z);
    float4* O4 = reinterpret_cast<float4*>(dZ);
#pragma unroll
    for (int q = 0; q < S::NT; ++q) {
      int c4 = sl + q * S::L;
#pragma unroll
      for (int br = 0; br < 2; ++br) {
        int64_t row = (int64_t)i + (br ? Nt : 0);
        float4 z = __ldg(Z4 + row * (C / 4) + c4);
        float4 h = br ? accn[q] : accp[q];
        float4 o;
        o.x = z.x > 0.f ? h.x : a * h.x;  da += z.x > 0.f ? 0.f : h.x * z.x;
        o.y = z.y > 0.f ? h.y : a * h.y;  da += z.y > 0.f ? 0.f : h.y * z.y;
        o.z = z.z > 0.f ? h.z : a * h.z;  da += z.z > 0.f ? 0.f : h.z * z.z;
        o.w = z.w > 0.f ? h.w : a * h.w;  da += z.w > 0.f ? 0.f : h.w * z.w;
        O4[row * (C / 4) + c4] = o;
      }
    }
  }
  double wd = warp_sum((double)da);
  if (lane == 0) wpart[threadIdx.x >> 5] = wd;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int k = 0; k < kSpmmThreads / 32; ++k) t += wpart[k];
    slots[blockIdx.x] = t;
  }
}

template <int C>
cudaError_t fwd_c(const GraphDev& g, const float* T, const int32_t* perm, const float* alpha,
                  int act_layer, float* Y, int both, cudaStream_t s) {
  using S = SpmmShape<C>;
  unsigned blocks = cdiv(g.Nt, S::RPB);
  if (act_layer < 0) {
    if (both)
      k_spmm_fwd<C, 0, true><<<blocks, kSpmmThreads, 0, s>>>(g.rowptr, g.colind, g.vals, T, perm,
                                                             alpha, 0, g.Nt, Y);
    else
      k_spmm_fwd<C, 0, false><<<blocks, kSpmmThreads, 0, s>>>(g.rowptr, g.colind, g.vals, T,
                                                              perm, alpha, 0, g.Nt, Y);
  } else {
    if (both)
      k_spmm_fwd<C, 1, true><<<blocks, kSpmmThreads, 0, s>>>(g.rowptr, g.colind, g.vals, T, perm,
                                                             alpha, act_layer, g.Nt, Y);
    else
      k_spmm_fwd<C, 1, false><<<blocks, kSpmmThreads, 0, s>>>(g.rowptr, g.colind, g.vals, T,
                                                              perm, alpha, act_layer, g.Nt, Y);
  }
  return cudaGetLastError();
}

template <int C>
cudaError_t bwd_c(const GraphDev& g, const float* dY, const float* Z, const float* alpha,
                  int layer, float* dZ, double* slots, int* nslots, cudaStream_t s) {
  using S = SpmmShape<C>;
  unsigned blocks = cdiv(g.Nt, S::RPB);
  k_spmm_bwd<C><<<blocks, kSpmmThreads, 0, s>>>(g.rowptr, g.colind, g.vals, dY, Z, alpha, layer,
                                                g.Nt, dZ, slots);
  *nslots = (int)blocks;
  return cudaGetLastError();
}

}  // namespace

// act_layer < 0: layer 1 (X with the fused corruption gather through perm).
cudaError_t launch_spmm_fwd(const GraphDev& g, int C, const float* T, const int32_t* perm,
                            const float* alpha_dev, int act_layer, float* Y, int both,
                            cudaStream_t s, int* launches) {
  count_launch(launches);
  switch (C) {
    case 16: return fwd_c<16>(g, T, perm, alpha_dev, act_layer, Y, both, s);
    case 32: return fwd_c<32>(g, T, perm, alpha_dev, act_layer, Y, both, s);
    case 64: return fwd_c<64>(g, T, perm, alpha_dev, act_layer, Y, both, s);
    case 128: return fwd_c<128>(g, T, perm, alpha_dev, act_layer, Y, both, s);
    case 256: return fwd_c<256>(g, T, perm, alpha_dev, act_layer, Y, both, s);
    default: return cudaErrorInvalidValue;
  }
}

int spmm_bwd_slots(const GraphDev& g) { return (int)cdiv(g.Nt, SpmmShape<256>::RPB) + 1; }

cudaError_t launch_spmm_bwd(const GraphDev& g, int C, const float* dY, const float* Z,
                            const float* alpha_dev, int layer, float* dZ, double* slots,
                            int* nslots, cudaStream_t s, int* launches) {
  count_launch(launches);
  switch (C) {
    case 32: return bwd_c<32>(g, dY, Z, alpha_dev, layer, dZ, slots, nslots, s);
    case 64: return bwd_c<64>(g, dY, Z, alpha_dev, layer, dZ, slots, nslots, s);
    case 128: return bwd_c<128>(g, dY, Z, alpha_dev, layer, dZ, slots, nslots, s);
    case 256: return bwd_c<256>(g, dY, Z, alpha_dev, layer, dZ, slots, nslots, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace mars
