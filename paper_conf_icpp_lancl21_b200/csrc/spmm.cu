// a5 (+a4 gather, a7 PReLU, a12 PReLU'): the aggregation Y = Â_n · act(T) of
// Eq. 1 for the stacked [pos; neg] activations, and its backward
// dH = Â_nᵀ dY = Â_n dY (Â_n is symmetric, c1).
//
// Layout: T is R×C row-major with R = 2·Nt (rows [0,Nt) positive branch, rows
// [Nt,2Nt) corrupted branch).  Both branches share the CSR (the corrupted graph
// has the same structure), so one (colind, val) read feeds two row
// gathers.  Sub-warp per row: L = min(32, C/V) lanes own C/L consecutive
// columns each as 16-byte vectors (V = 4 fp32 or 8 bf16), so every neighbour
// row is one coalesced transaction per branch; 32/L rows share a warp when the
// row is narrower than 512 bytes.  Storage is fp32 (reference path) or bf16
// (bf16 path); accumulation is always fp32, in ascending colind order
// (deterministic).  kU neighbours' gathers are issued before their FMAs.
//   fwd layer 1: T = X, neg rows gather X[pi[j]] (the corruption, fused)
//   fwd layer l>1: act = PReLU_{a_{l-1}} applied on load (H_{l-1} never stored)
//   bwd: epilogue dZ = dH ⊙ PReLU'(Z), dalpha partials Σ dH·min(Z,0) per block
#include "common.cuh"
#include "internal.cuh"
#include "vec.cuh"

namespace mars {
namespace {

constexpr int kSpmmThreads = 256;
constexpr int kU = 4;           // neighbours whose gathers are in flight together

// C in {16, 32, 64, 128, 256} (mars.h restricts F and H to these widths).
template <int C, typename T>
struct SpmmShape {
  static constexpr int V = Vec<T>::N;                     // elements per 16-byte load
  static constexpr int L = (C / V) < 32 ? (C / V) : 32;   // lanes per row
  static constexpr int RPW = 32 / L;                      // rows per warp
  static constexpr int NT = C / (V * L);                  // vectors per lane per branch
  static constexpr int RPB = RPW * (kSpmmThreads / 32);   // rows per block
};

template <int V>
__device__ __forceinline__ void vfma(float (&acc)[V], float w, const float (&x)[V]) {
#pragma unroll
  for (int e = 0; e < V; ++e) acc[e] = fmaf(w, x[e], acc[e]);
}

template <int V>
__device__ __forceinline__ void vprelu(float (&x)[V], float a) {
#pragma unroll
  for (int e = 0; e < V; ++e) x[e] = prelu(x[e], a);
}

// MODE 0: layer 1 (neg rows gather X[perm[j]]), MODE 1: PReLU on load.
template <int C, int MODE, bool BOTH, typename Tin, typename Tout>
__global__ void __launch_bounds__(kSpmmThreads)
k_spmm_fwd(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
           const float* __restrict__ vals, const Tin* __restrict__ T,
           const int32_t* __restrict__ perm, const float* __restrict__ alpha, int act_layer,
           int32_t Nt, Tout* __restrict__ Y) {
  using S = SpmmShape<C, Tin>;
  constexpr int V = S::V;
  const int lane = threadIdx.x & 31;
  const int sub = lane / S::L, sl = lane % S::L;
  const unsigned gmask = (S::L == 32) ? kFull : (((1u << S::L) - 1u) << (sub * S::L));
  const int32_t i = (int32_t)(((int64_t)blockIdx.x * kSpmmThreads + threadIdx.x) / 32) * S::RPW + sub;
  if (i >= Nt) return;
  const float a = (MODE == 1) ? alpha[act_layer] : 1.f;
  const int32_t rb = rowptr[i], re = rowptr[i + 1];
  float accp[S::NT][V], accn[S::NT][V];
#pragma unroll
  for (int q = 0; q < S::NT; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) accp[q][e] = accn[q][e] = 0.f;
  for (int32_t k0 = rb; k0 < re; k0 += S::L) {
    const int32_t cnt = min(S::L, re - k0);
    int32_t myj = 0, myjn = 0;
    float myv = 0.f;
    if (sl < cnt) {
      myj = colind[k0 + sl];
      myv = vals[k0 + sl];
      if (BOTH) myjn = (MODE == 0) ? perm[myj] : Nt + myj;
    }
    int t = 0;
    for (; t + kU <= cnt; t += kU) {
      int32_t j[kU], jn[kU];
      float w[kU];
#pragma unroll
      for (int u = 0; u < kU; ++u) {
        j[u] = __shfl_sync(gmask, myj, t + u, S::L);
        w[u] = __shfl_sync(gmask, myv, t + u, S::L);
        jn[u] = BOTH ? __shfl_sync(gmask, myjn, t + u, S::L) : 0;
      }
      float xp[kU][S::NT][V], xn[kU][S::NT][V];
#pragma unroll
      for (int u = 0; u < kU; ++u)
#pragma unroll
        for (int q = 0; q < S::NT; ++q) {
          const int c = (sl + q * S::L) * V;
          Vec<Tin>::load(T + (int64_t)j[u] * C + c, xp[u][q]);
          if (BOTH) Vec<Tin>::load(T + (int64_t)jn[u] * C + c, xn[u][q]);
        }
#pragma unroll
      for (int u = 0; u < kU; ++u)
#pragma unroll
        for (int q = 0; q < S::NT; ++q) {
          if (MODE == 1) vprelu<V>(xp[u][q], a);
          vfma<V>(accp[q], w[u], xp[u][q]);
          if (BOTH) {
            if (MODE == 1) vprelu<V>(xn[u][q], a);
            vfma<V>(accn[q], w[u], xn[u][q]);
          }
        }
    }
    for (; t < cnt; ++t) {
      const int32_t j = __shfl_sync(gmask, myj, t, S::L);
      const float w = __shfl_sync(gmask, myv, t, S::L);
      const int32_t jn = BOTH ? __shfl_sync(gmask, myjn, t, S::L) : 0;
#pragma unroll
      for (int q = 0; q < S::NT; ++q) {
        const int c = (sl + q * S::L) * V;
        float x[V];
        Vec<Tin>::load(T + (int64_t)j * C + c, x);
        if (MODE == 1) vprelu<V>(x, a);
        vfma<V>(accp[q], w, x);
        if (BOTH) {
          Vec<Tin>::load(T + (int64_t)jn * C + c, x);
          if (MODE == 1) vprelu<V>(x, a);
          vfma<V>(accn[q], w, x);
        }
      }
    }
  }
#pragma unroll
  for (int q = 0; q < S::NT; ++q) {
    const int c = (sl + q * S::L) * V;
    StoreN<Tout, V>::store(Y + (int64_t)i * C + c, accp[q]);
    if (BOTH) StoreN<Tout, V>::store(Y + ((int64_t)Nt + i) * C + c, accn[q]);
  }
}

template <int C, typename T>
__global__ void __launch_bounds__(kSpmmThreads)
k_spmm_bwd(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
           const float* __restrict__ vals, const T* __restrict__ dY, const T* __restrict__ Z,
           const float* __restrict__ alpha, int layer, int32_t Nt, T* __restrict__ dZ,
           double* __restrict__ slots) {
  using S = SpmmShape<C, T>;
  constexpr int V = S::V;
  __shared__ double wpart[kSpmmThreads / 32];
  const int lane = threadIdx.x & 31;
  const int sub = lane / S::L, sl = lane % S::L;
  const unsigned gmask = (S::L == 32) ? kFull : (((1u << S::L) - 1u) << (sub * S::L));
  const int32_t i = (int32_t)(((int64_t)blockIdx.x * kSpmmThreads + threadIdx.x) / 32) * S::RPW + sub;
  float da = 0.f;
  if (i < Nt) {
    const float a = alpha[layer];
    const int32_t rb = rowptr[i], re = rowptr[i + 1];
    float accp[S::NT][V], accn[S::NT][V];
#pragma unroll
    for (int q = 0; q < S::NT; ++q)
#pragma unroll
      for (int e = 0; e < V; ++e) accp[q][e] = accn[q][e] = 0.f;
    for (int32_t k0 = rb; k0 < re; k0 += S::L) {
      const int32_t cnt = min(S::L, re - k0);
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
#pragma unroll
        for (int u = 0; u < kU; ++u) {
          j[u] = __shfl_sync(gmask, myj, t + u, S::L);
          w[u] = __shfl_sync(gmask, myv, t + u, S::L);
        }
        float xp[kU][S::NT][V], xn[kU][S::NT][V];
#pragma unroll
        for (int u = 0; u < kU; ++u)
#pragma unroll
          for (int q = 0; q < S::NT; ++q) {
            const int c = (sl + q * S::L) * V;
            Vec<T>::load(dY + (int64_t)j[u] * C + c, xp[u][q]);
            Vec<T>::load(dY + ((int64_t)Nt + j[u]) * C + c, xn[u][q]);
          }
#pragma unroll
        for (int u = 0; u < kU; ++u)
#pragma unroll
          for (int q = 0; q < S::NT; ++q) {
            vfma<V>(accp[q], w[u], xp[u][q]);
            vfma<V>(accn[q], w[u], xn[u][q]);
          }
      }
      for (; t < cnt; ++t) {
        const int32_t j = __shfl_sync(gmask, myj, t, S::L);
        const float w = __shfl_sync(gmask, myv, t, S::L);
#pragma unroll
        for (int q = 0; q < S::NT; ++q) {
          const int c = (sl + q * S::L) * V;
          float x[V];
          Vec<T>::load(dY + (int64_t)j * C + c, x);
          vfma<V>(accp[q], w, x);
          Vec<T>::load(dY + ((int64_t)Nt + j) * C + c, x);
          vfma<V>(accn[q], w, x);
        }
      }
    }
#pragma unroll
    for (int q = 0; q < S::NT; ++q) {
      const int c = (sl + q * S::L) * V;
#pragma unroll
      for (int br = 0; br < 2; ++br) {
        const int64_t row = (int64_t)i + (br ? Nt : 0);
        float z[V], o[V];
        Vec<T>::load(Z + row * C + c, z);
#pragma unroll
        for (int e = 0; e < V; ++e) {
          const float h = br ? accn[q][e] : accp[q][e];
          o[e] = z[e] > 0.f ? h : a * h;
          da += z[e] > 0.f ? 0.f : h * z[e];
        }
        StoreN<T, V>::store(dZ + row * C + c, o);
      }
    }
  }
  const double wd = warp_sum((double)da);
  if (lane == 0) wpart[threadIdx.x >> 5] = wd;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int k = 0; k < kSpmmThreads / 32; ++k) t += wpart[k];
    slots[blockIdx.x] = t;
  }
}

template <int C, typename Tin, typename Tout>
cudaError_t fwd_c(const GraphDev& g, const Tin* T, const int32_t* perm, const float* alpha,
                  int act_layer, Tout* Y, int both, cudaStream_t s) {
  using S = SpmmShape<C, Tin>;
  const unsigned blocks = cdiv(g.Nt, S::RPB);
  if (act_layer < 0) {
    if (both)
      k_spmm_fwd<C, 0, true, Tin, Tout><<<blocks, kSpmmThreads, 0, s>>>(
          g.rowptr, g.colind, g.vals, T, perm, alpha, 0, g.Nt, Y);
    else
      k_spmm_fwd<C, 0, false, Tin, Tout><<<blocks, kSpmmThreads, 0, s>>>(
          g.rowptr, g.colind, g.vals, T, perm, alpha, 0, g.Nt, Y);
  } else {
    if (both)
      k_spmm_fwd<C, 1, true, Tin, Tout><<<blocks, kSpmmThreads, 0, s>>>(
          g.rowptr, g.colind, g.vals, T, perm, alpha, act_layer, g.Nt, Y);
    else
      k_spmm_fwd<C, 1, false, Tin, Tout><<<blocks, kSpmmThreads, 0, s>>>(
          g.rowptr, g.colind, g.vals, T, perm, alpha, act_layer, g.Nt, Y);
  }
  return cudaGetLastError();
}

template <typename Tin, typename Tout>
cudaError_t fwd_t(const GraphDev& g, int C, const void* T, const int32_t* perm, const float* alpha,
                  int act_layer, void* Y, int both, cudaStream_t s) {
  const Tin* t = static_cast<const Tin*>(T);
  Tout* y = static_cast<Tout*>(Y);
  switch (C) {
    case 16: return fwd_c<16, Tin, Tout>(g, t, perm, alpha, act_layer, y, both, s);
    case 32: return fwd_c<32, Tin, Tout>(g, t, perm, alpha, act_layer, y, both, s);
    case 64: return fwd_c<64, Tin, Tout>(g, t, perm, alpha, act_layer, y, both, s);
    case 128: return fwd_c<128, Tin, Tout>(g, t, perm, alpha, act_layer, y, both, s);
    case 256: return fwd_c<256, Tin, Tout>(g, t, perm, alpha, act_layer, y, both, s);
    default: return cudaErrorInvalidValue;
  }
}

template <int C, typename T>
cudaError_t bwd_c(const GraphDev& g, const T* dY, const T* Z, const float* alpha, int layer,
                  T* dZ, double* slots, int* nslots, cudaStream_t s) {
  using S = SpmmShape<C, T>;
  const unsigned blocks = cdiv(g.Nt, S::RPB);
  k_spmm_bwd<C, T><<<blocks, kSpmmThreads, 0, s>>>(g.rowptr, g.colind, g.vals, dY, Z, alpha,
                                                   layer, g.Nt, dZ, slots);
  *nslots = (int)blocks;
  return cudaGetLastError();
}

template <typename T>
cudaError_t bwd_t(const GraphDev& g, int C, const void* dY, const void* Z, const float* alpha,
                  int layer, void* dZ, double* slots, int* nslots, cudaStream_t s) {
  const T* d = static_cast<const T*>(dY);
  const T* z = static_cast<const T*>(Z);
  T* o = static_cast<T*>(dZ);
  switch (C) {
    case 32: return bwd_c<32, T>(g, d, z, alpha, layer, o, slots, nslots, s);
    case 64: return bwd_c<64, T>(g, d, z, alpha, layer, o, slots, nslots, s);
    case 128: return bwd_c<128, T>(g, d, z, alpha, layer, o, slots, nslots, s);
    case 256: return bwd_c<256, T>(g, d, z, alpha, layer, o, slots, nslots, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace

// act_layer < 0: layer 1 (X with the fused corruption gather through perm).
// in_bf16 / out_bf16 select the storage type of T and Y.
cudaError_t launch_spmm_fwd(const GraphDev& g, int C, const void* T, int in_bf16,
                            const int32_t* perm, const float* alpha_dev, int act_layer, void* Y,
                            int out_bf16, int both, cudaStream_t s, int* launches) {
  count_launch(launches);
  if (!in_bf16 && !out_bf16) return fwd_t<float, float>(g, C, T, perm, alpha_dev, act_layer, Y, both, s);
  if (!in_bf16 && out_bf16) return fwd_t<float, bf16>(g, C, T, perm, alpha_dev, act_layer, Y, both, s);
  if (in_bf16 && out_bf16) return fwd_t<bf16, bf16>(g, C, T, perm, alpha_dev, act_layer, Y, both, s);
  return cudaErrorInvalidValue;
}

// fp32 rows per block is the smallest RPB (largest block count) of any config.
int spmm_bwd_slots(const GraphDev& g) { return (int)cdiv(g.Nt, SpmmShape<256, float>::RPB) + 1; }

cudaError_t launch_spmm_bwd(const GraphDev& g, int C, const void* dY, const void* Z, int bf16_,
                            const float* alpha_dev, int layer, void* dZ, double* slots,
                            int* nslots, cudaStream_t s, int* launches) {
  count_launch(launches);
  if (bf16_) return bwd_t<bf16>(g, C, dY, Z, alpha_dev, layer, dZ, slots, nslots, s);
  return bwd_t<float>(g, C, dY, Z, alpha_dev, layer, dZ, slots, nslots, s);
}

}  // namespace mars
