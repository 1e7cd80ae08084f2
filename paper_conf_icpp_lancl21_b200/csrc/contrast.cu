// NEXT-4 contrastive variants ("there are many choices of the corruption
// function, readout function and loss function ... other contrastive learning
// methods should also work"; GraphSAGE in [33]).  Readings
// c34-c37 in DESIGN.md §3:
//   c34  K corruption samples per graph share ONE positive branch: the stacked
//        activations hold [pos; neg_1; ...; neg_K (; zero pad to an even block
//        count)], sample k of graph g draws pair index pair_base + pair_off[g] K
//        + (k - 1) -- the same permutations as K consecutive copies of the graph
//        in the batch API (c20), so both formulations give the same loss.
//   c35  feature-masking corruption: X~[i][f] = X[i][f] keep(i, f), keep iff
//        u >= rate, u = (sm64(sm64(k ^ 0x6D61736B) ^ (i F + f)) >> 40) 2^-24,
//        k the sample's key sm64(sm64(sm64(seed) ^ step) ^ pair) (c12).
//   c37  SAGE-GCN aggregation: Â = D^-1 (A v Aᵀ + I) (row mean over the
//        neighbourhood with the node itself); the backward uses Âᵀ, the same
//        pattern with 1/deg of the column.
//   c38  SAGE-mean encoder (GraphSAGE with a root weight): Z = H W_s +
//        (Â_N H) W_n, Â_N = D_N^-1 (A v Aᵀ) without self loops; computed
//        GEMM-first as Z_i = U_s[i] + Σ_j Â_N[i][j] U_n[j] (U = H [W_s | W_n])
//        by ONE aggregation whose self entry is redirected to the U_s rows.
//   c40  SAGE-pool encoder: P = ReLU(h W_p + b_p), agg = element-wise max of
//        P over the neighbours (argmax kept for the backward), h' = PReLU(h W_s
//        + agg W_n).
// The corrupted inputs are materialised (one pass over X per block) and layer
// 1 aggregates the stacked blocks like layers 2-3 (PReLU slope 1 = identity).
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

__global__ void k_pair_off_k(const int64_t* __restrict__ pair_off, int32_t G, int32_t K,
                             int64_t* __restrict__ out) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (int64_t)G * K) return;
  const int32_t k = (int32_t)(t / G), g = (int32_t)(t % G);
  out[t] = pair_off[g] * K + k;
}

// one thread per 4 consecutive features of one row of Xs
__global__ void k_corrupt(const float* __restrict__ X, const int32_t* __restrict__ node_graph,
                          const int32_t* __restrict__ node_off, int32_t Nt, int32_t G, int32_t F,
                          int32_t K, int32_t nb, int32_t corruption, double rate, uint64_t seed,
                          const StepParams* __restrict__ sp, const int64_t* __restrict__ pair_off_k,
                          const int32_t* __restrict__ perms, float* __restrict__ Xs) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int32_t Fq = F / 4;
  if (t >= (int64_t)nb * Nt * Fq) return;
  const int64_t r = t / Fq;
  const int32_t f0 = (int32_t)(t % Fq) * 4;
  const int32_t b = (int32_t)(r / Nt), i = (int32_t)(r % Nt);
  float4 o = make_float4(0.f, 0.f, 0.f, 0.f);
  if (b == 0) {
    o = *reinterpret_cast<const float4*>(X + (int64_t)i * F + f0);
  } else if (b <= K) {
    if (corruption == 0) {
      const int32_t src = perms[(int64_t)(b - 1) * Nt + i];
      o = *reinterpret_cast<const float4*>(X + (int64_t)src * F + f0);
    } else {
      const int32_t g = node_graph[i];
      const uint64_t pair = (uint64_t)(sp->pair_base + pair_off_k[(int64_t)(b - 1) * G + g]);
      const uint64_t kg = sm64(sm64(sm64(seed) ^ sp->step_index) ^ pair);
      const uint64_t km = sm64(kg ^ 0x6D61736BULL);
      const uint64_t e0 = (uint64_t)(i - node_off[g]) * (uint64_t)F + (uint64_t)f0;
      const float4 x = *reinterpret_cast<const float4*>(X + (int64_t)i * F + f0);
      const float xv[4] = {x.x, x.y, x.z, x.w};
      float ov[4];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const double u = (double)(sm64(km ^ (e0 + c)) >> 40) * (1.0 / 16777216.0);
        ov[c] = u >= rate ? xv[c] : 0.f;
      }
      o = make_float4(ov[0], ov[1], ov[2], ov[3]);
    }
  }
  *reinterpret_cast<float4*>(Xs + r * F + f0) = o;
}

__global__ void k_sage_vals(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
                            int32_t Nt, float* __restrict__ valsR, float* __restrict__ valsC) {
  // one warp per row: lanes stride the row's entries
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (wid >= Nt) return;
  const int32_t i = (int32_t)wid;
  const int32_t k0 = rowptr[i], k1 = rowptr[i + 1];
  const float ri = 1.0f / (float)(k1 - k0);
  for (int32_t k = k0 + lane; k < k1; k += 32) {
    const int32_t j = colind[k];
    valsR[k] = ri;
    valsC[k] = 1.0f / (float)(rowptr[j + 1] - rowptr[j]);
  }
}

// SAGE-mean encoder (c38): per CSR entry k of row i with column j,
//   colS[k] = j == i ? self_off + i : j         (self entry -> the root rows)
//   vf[k]   = j == i ? 1 : 1/(deg_i - 1)        Z_i = U_s[i] + mean_j U_n[j]
//   vb[k]   = j == i ? 1 : 1/(deg_j - 1)        its transpose (backward)
//   vn[k]   = j == i ? 0 : 1/(deg_j - 1)        Â_Nᵀ alone (dW_n)
// deg counts the self loop, so deg - 1 is the neighbour count (>= 1 for every
// neighbour entry).
__global__ void k_sage_csr(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
                           int32_t Nt, int64_t self_off, int32_t* __restrict__ colS,
                           float* __restrict__ vf, float* __restrict__ vb, float* __restrict__ vn) {
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (wid >= Nt) return;
  const int32_t i = (int32_t)wid;
  const int32_t k0 = rowptr[i], k1 = rowptr[i + 1];
  const float ri = k1 - k0 > 1 ? 1.0f / (float)(k1 - k0 - 1) : 0.f;
  for (int32_t k = k0 + lane; k < k1; k += 32) {
    const int32_t j = colind[k];
    if (j == i) {
      colS[k] = (int32_t)(self_off + i);
      vf[k] = 1.f;
      if (vb) vb[k] = 1.f;
      if (vn) vn[k] = 0.f;
    } else {
      const float rj = 1.0f / (float)(rowptr[j + 1] - rowptr[j] - 1);
      colS[k] = j;
      vf[k] = ri;
      if (vb) vb[k] = rj;
      if (vn) vn[k] = rj;
    }
  }
}

// One warp per row of C columns: out = PReLU_a(in) (a = *slope; out may be
// null) and the row's power-of-two scale (rs may be null) for the 3xFP16 GEMMs.
__global__ void k_rowprep(const float* __restrict__ in, int64_t rows, int C,
                          const float* __restrict__ slope, float* __restrict__ out,
                          float* __restrict__ rs) {
  const int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= rows) return;
  const float a = *slope;
  float m = 0.f;
  for (int c = lane * 4; c < C; c += 128) {
    const float4 x = *reinterpret_cast<const float4*>(in + r * C + c);
    const float4 y = make_float4(x.x > 0.f ? x.x : a * x.x, x.y > 0.f ? x.y : a * x.y,
                                 x.z > 0.f ? x.z : a * x.z, x.w > 0.f ? x.w : a * x.w);
    if (out) *reinterpret_cast<float4*>(out + r * C + c) = y;
    m = fmaxf(m, fmaxf(fmaxf(fabsf(y.x), fabsf(y.y)), fmaxf(fabsf(y.z), fabsf(y.w))));
  }
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  if (rs && lane == 0) rs[r] = pow2_scale(m);
}

// ---- SAGE-pool encoder (c40).  One warp per row of the stacked activations
// (row r = block b, node i = r - b Nt; neighbours in the same block); lanes
// stride the H columns.
// agg[r][c] = max_{j in N(i), j != i} ReLU(U[b Nt + j][c] + bp[c]) (0 without
// neighbours), idx[r][c] = the first j (ascending) attaining it (-1 without).
// Lanes own 4-column slices (16-byte loads), neighbours in the outer loop.
template <int H>
__global__ void k_maxagg(const float* __restrict__ U, const float* __restrict__ bp,
                         const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
                         int32_t Nt, int64_t R, float* __restrict__ agg,
                         int32_t* __restrict__ idx, float* __restrict__ rs) {
  constexpr int LPR = H / 4 < 32 ? H / 4 : 32, PER = H / (4 * LPR);
  const int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= R) return;
  const bool act = lane < LPR;
  const int64_t base = r / Nt * Nt;
  const int32_t i = (int32_t)(r - base);
  const int32_t k0 = rowptr[i], k1 = rowptr[i + 1];
  float b[PER][4], m[PER][4];
  int32_t a[PER][4];
#pragma unroll
  for (int q = 0; q < PER; ++q) {
    const float4 bv = act ? reinterpret_cast<const float4*>(bp)[lane + q * LPR] : float4{};
    b[q][0] = bv.x; b[q][1] = bv.y; b[q][2] = bv.z; b[q][3] = bv.w;
#pragma unroll
    for (int e = 0; e < 4; ++e) { m[q][e] = -1.f; a[q][e] = -1; }
  }
  for (int32_t k = k0; k < k1; ++k) {
    const int32_t j = colind[k];
    if (j == i || !act) continue;
    const float4* row = reinterpret_cast<const float4*>(U + (base + j) * H);
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const float4 u = row[lane + q * LPR];
      const float x[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float v = fmaxf(x[e] + b[q][e], 0.f);
        if (v > m[q][e]) { m[q][e] = v; a[q][e] = j; }
      }
    }
  }
  float amax = 0.f;
  if (act) {
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      float o[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) { o[e] = a[q][e] < 0 ? 0.f : m[q][e]; amax = fmaxf(amax, o[e]); }
      reinterpret_cast<float4*>(agg + r * H)[lane + q * LPR] = make_float4(o[0], o[1], o[2], o[3]);
      reinterpret_cast<int4*>(idx + r * H)[lane + q * LPR] = make_int4(a[q][0], a[q][1], a[q][2], a[q][3]);
    }
  }
  for (int o = 16; o > 0; o >>= 1) amax = fmaxf(amax, __shfl_xor_sync(0xffffffffu, amax, o));
  if (rs && lane == 0) rs[r] = pow2_scale(amax);
}

// dU[r][c] = [U[r][c] + bp[c] > 0] Σ_{i in N(j), i != j, idx[b Nt + i][c] == j}
// dagg[b Nt + i][c] (row r = b Nt + j; the pattern is symmetric, so the rows
// whose max j won are among j's own neighbours; ascending i: deterministic).
template <int H>
__global__ void k_maxagg_bwd(const float* __restrict__ dagg, const int32_t* __restrict__ idx,
                             const float* __restrict__ U, const float* __restrict__ bp,
                             const int32_t* __restrict__ rowptr,
                             const int32_t* __restrict__ colind, int32_t Nt, int64_t R,
                             float* __restrict__ dU, float* __restrict__ rs) {
  constexpr int LPR = H / 4 < 32 ? H / 4 : 32, PER = H / (4 * LPR);
  const int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= R) return;
  const bool act = lane < LPR;
  const int64_t base = r / Nt * Nt;
  const int32_t j = (int32_t)(r - base);
  const int32_t k0 = rowptr[j], k1 = rowptr[j + 1];
  float acc[PER][4];
#pragma unroll
  for (int q = 0; q < PER; ++q)
#pragma unroll
    for (int e = 0; e < 4; ++e) acc[q][e] = 0.f;
  for (int32_t k = k0; k < k1; ++k) {
    const int32_t i = colind[k];
    if (i == j || !act) continue;
    const int4* ix = reinterpret_cast<const int4*>(idx + (base + i) * H);
    const float4* dg = reinterpret_cast<const float4*>(dagg + (base + i) * H);
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const int4 w = ix[lane + q * LPR];
      if (w.x != j && w.y != j && w.z != j && w.w != j) continue;
      const float4 d = dg[lane + q * LPR];
      if (w.x == j) acc[q][0] += d.x;
      if (w.y == j) acc[q][1] += d.y;
      if (w.z == j) acc[q][2] += d.z;
      if (w.w == j) acc[q][3] += d.w;
    }
  }
  float amax = 0.f;
  if (act) {
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const float4 u = reinterpret_cast<const float4*>(U + r * H)[lane + q * LPR];
      const float4 bv = reinterpret_cast<const float4*>(bp)[lane + q * LPR];
      const float o[4] = {u.x + bv.x > 0.f ? acc[q][0] : 0.f, u.y + bv.y > 0.f ? acc[q][1] : 0.f,
                          u.z + bv.z > 0.f ? acc[q][2] : 0.f, u.w + bv.w > 0.f ? acc[q][3] : 0.f};
#pragma unroll
      for (int e = 0; e < 4; ++e) amax = fmaxf(amax, fabsf(o[e]));
      reinterpret_cast<float4*>(dU + r * H)[lane + q * LPR] = make_float4(o[0], o[1], o[2], o[3]);
    }
  }
  for (int o = 16; o > 0; o >>= 1) amax = fmaxf(amax, __shfl_xor_sync(0xffffffffu, amax, o));
  if (rs && lane == 0) rs[r] = pow2_scale(amax);
}

__global__ void k_add4(const float4* __restrict__ a, const float4* __restrict__ b,
                       float4* __restrict__ out, int64_t n4) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n4) return;
  const float4 x = a[t], y = b[t];
  out[t] = make_float4(x.x + y.x, x.y + y.y, x.z + y.z, x.w + y.w);
}

// dZ = (d1 + d2) ⊙ PReLU'_a(Z) row by row (8 rows per 256-thread block) with
// the row's power-of-two scale and the block's dα partial Σ_{Z<=0} (d1+d2) Z.
__global__ void __launch_bounds__(256) k_add_prelu_bwd(const float* __restrict__ d1,
                                                       const float* __restrict__ d2,
                                                       const float* __restrict__ Z,
                                                       const float* __restrict__ alpha, int layer,
                                                       int64_t R, int H, float* __restrict__ dZ,
                                                       float* __restrict__ rs,
                                                       double* __restrict__ slots) {
  __shared__ double sh[8];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t r = (int64_t)blockIdx.x * 8 + w;
  const float a = alpha[layer];
  double da = 0.0;
  float amax = 0.f;
  if (r < R) {
    for (int c = lane; c < H; c += 32) {
      const int64_t e = r * H + c;
      const float h = d1[e] + d2[e], z = Z[e];
      const float o = z > 0.f ? h : a * h;
      dZ[e] = o;
      da += z > 0.f ? 0.0 : (double)(h * z);
      amax = fmaxf(amax, fabsf(o));
    }
    for (int o = 16; o > 0; o >>= 1) amax = fmaxf(amax, __shfl_xor_sync(0xffffffffu, amax, o));
    if (rs && lane == 0) rs[r] = pow2_scale(amax);
  }
  da = warp_sum(da);
  if (lane == 0) sh[w] = da;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int k = 0; k < 8; ++k) t += sh[k];
    slots[blockIdx.x] = t;
  }
}

}  // namespace

cudaError_t launch_maxagg(const GraphDev& g, const float* U, const float* bp, int64_t R, int H,
                          float* agg, int32_t* idx, float* rs, cudaStream_t s, int* launches) {
  count_launch(launches);
  if (R <= 0) return cudaSuccess;
  const unsigned nb = cdiv(R * 32, 256);
  switch (H) {
#define MAXAGG(HH) \
  case HH: k_maxagg<HH><<<nb, 256, 0, s>>>(U, bp, g.rowptr, g.colind, g.Nt, R, agg, idx, rs); break;
    MAXAGG(32) MAXAGG(64) MAXAGG(128) MAXAGG(256)
#undef MAXAGG
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_maxagg_bwd(const GraphDev& g, const float* dagg, const int32_t* idx,
                              const float* U, const float* bp, int64_t R, int H, float* dU,
                              float* rs, cudaStream_t s, int* launches) {
  count_launch(launches);
  if (R <= 0) return cudaSuccess;
  const unsigned nb = cdiv(R * 32, 256);
  switch (H) {
#define MAXBWD(HH)                                                                             \
  case HH:                                                                                     \
    k_maxagg_bwd<HH><<<nb, 256, 0, s>>>(dagg, idx, U, bp, g.rowptr, g.colind, g.Nt, R, dU, rs); \
    break;
    MAXBWD(32) MAXBWD(64) MAXBWD(128) MAXBWD(256)
#undef MAXBWD
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_add(const float* a, const float* b, float* out, int64_t n, cudaStream_t s,
                       int* launches) {
  if (n % 4) return cudaErrorInvalidValue;
  count_launch(launches);
  if (n > 0)
    k_add4<<<cdiv(n / 4, 256), 256, 0, s>>>(reinterpret_cast<const float4*>(a),
                                            reinterpret_cast<const float4*>(b),
                                            reinterpret_cast<float4*>(out), n / 4);
  return cudaGetLastError();
}

cudaError_t launch_add_prelu_bwd(const float* d1, const float* d2, const float* Z,
                                 const float* alpha, int layer, int64_t R, int H, float* dZ,
                                 float* rs, double* slots, int* nslots, cudaStream_t s,
                                 int* launches) {
  count_launch(launches);
  *nslots = (int)cdiv(R, 8);
  if (R > 0)
    k_add_prelu_bwd<<<cdiv(R, 8), 256, 0, s>>>(d1, d2, Z, alpha, layer, R, H, dZ, rs, slots);
  return cudaGetLastError();
}

cudaError_t launch_sage_csr(const GraphDev& g, int64_t self_off, int32_t* colS, float* vf,
                            float* vb, float* vn, cudaStream_t s, int* launches) {
  count_launch(launches);
  if (g.Nt > 0)
    k_sage_csr<<<cdiv((int64_t)g.Nt * 32, 256), 256, 0, s>>>(g.rowptr, g.colind, g.Nt, self_off,
                                                              colS, vf, vb, vn);
  return cudaGetLastError();
}

cudaError_t launch_rowprep(const float* in, int64_t rows, int C, const float* slope, float* out,
                           float* rs, cudaStream_t s, int* launches) {
  if (C % 4) return cudaErrorInvalidValue;
  count_launch(launches);
  if (rows > 0)
    k_rowprep<<<cdiv(rows * 32, 256), 256, 0, s>>>(in, rows, C, slope, out, rs);
  return cudaGetLastError();
}

cudaError_t launch_pair_off_k(const int64_t* pair_off, int32_t G, int32_t K, int64_t* out,
                              cudaStream_t s, int* launches) {
  count_launch(launches);
  k_pair_off_k<<<cdiv((int64_t)G * K, 256), 256, 0, s>>>(pair_off, G, K, out);
  return cudaGetLastError();
}

cudaError_t launch_corrupt(const GraphDev& g, int32_t K, int32_t nb, int32_t corruption,
                           float mask_rate, uint64_t seed, const StepParams* sp,
                           const int64_t* pair_off_k, const int32_t* perms, float* Xs,
                           cudaStream_t s, int* launches) {
  if (g.F % 4 || K < 1 || K >= nb) return cudaErrorInvalidValue;
  count_launch(launches);
  const int64_t n = (int64_t)nb * g.Nt * (g.F / 4);
  k_corrupt<<<cdiv(n, 256), 256, 0, s>>>(g.X, g.node_graph, g.node_off, g.Nt, g.G, g.F, K, nb,
                                          corruption, (double)mask_rate, seed, sp, pair_off_k,
                                          perms, Xs);
  return cudaGetLastError();
}

cudaError_t launch_sage_vals(const GraphDev& g, float* valsR, float* valsC, cudaStream_t s,
                             int* launches) {
  count_launch(launches);
  if (g.Nt > 0)
    k_sage_vals<<<cdiv((int64_t)g.Nt * 32, 256), 256, 0, s>>>(g.rowptr, g.colind, g.Nt, valsR,
                                                               valsC);
  return cudaGetLastError();
}

}  // namespace mars
