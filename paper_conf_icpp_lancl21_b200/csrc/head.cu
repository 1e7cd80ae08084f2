// a8-a11 and the layer-3 part of a12: readout (Eq. 4), bilinear
// discriminator (Eq. 5), BCE/JSD loss (Eq. 6 as read in c8,
// P:L143-L145) and their backward, for every (graph, sample) pair of the set.
//
//   H3 = PReLU_{a3}(Z3)                     (recomputed on load, never stored)
//   m_g = (1/N_g) Σ_{i∈g, pos} H3[i]; s_g = sig(m_g); v_g = M s_g
//   l_i = H3[i]·v_g, l~_i = H3~[i]·v_g
//   L = (1/B) Σ_g (1/(2N_g)) Σ_i [softplus(-l_i) + softplus(l~_i)]
//   dl_i = (sig(l_i)-1)/(2 N_g B), dl~_i = sig(l~_i)/(2 N_g B)
//   dv_g = Σ dl_i H3[i] + Σ dl~_i H3~[i]; dM = Σ_g dv_g s_gᵀ; ds = Mᵀ dv;
//   dm = ds ⊙ s(1-s); dH3 = dl v_g + [pos] dm_g / N_g; dZ3 = dH3 ⊙ PReLU'(Z3)
// NEXT-4 variants (HeadWork nb / K / readout; readings c34-c36): the stacked
// activations hold nb blocks of Nt rows -- block 0 positive, blocks 1..K
// corrupted (each weighted 1/K in the loss), blocks > K zero padding (weight
// 0) -- and the readout is sig(mean) (default) or the plain mean.
// Every cross-row reduction is two-stage with fixed-order fp64 combination
// over row chunks (<= 256 rows, never straddling a graph): deterministic, no
// float atomics.  The per-graph second stages are small and latency-bound; they
// are spread over G x H/32 blocks.  Z3 / dZ3 are stored fp32 or bf16 (the
// storage type of the path); arithmetic is fp32 / fp64.
#include "common.cuh"
#include "internal.cuh"
#include "vec.cuh"

#include <type_traits>

namespace mars {
namespace {

constexpr int kWarps = 8;

// Row tiling shared by the three streaming kernels: lanes cover a row with
// 16-byte vectors of T (LPR lanes, PER vectors each); a warp keeps RU
// consecutive rows in flight per iteration so every SM has >= 32 KB of loads
// outstanding (Little's law at ~7 TB/s).
template <int NC, typename T>
struct RowTile {
  static constexpr int H = NC * 32;
  static constexpr int V = Vec<T>::N;
  static constexpr int LPR = (H / V) < 32 ? (H / V) : 32;
  static constexpr int PER = H / (V * LPR);
  static constexpr int RU = PER >= 8 ? 1 : 8 / PER;
};

// Stage 1 of m_g: per-chunk column sums of H3 over positive rows.  Block = 8
// warps; warp w takes RU consecutive rows per iteration, fp32 sums over the RU
// rows folded into fp64, warp partials combined in fixed order through shared
// memory.
template <int NC, typename T>
__global__ void __launch_bounds__(kWarps * 32, 3)
k_colsum(const T* __restrict__ Z3, const float* __restrict__ alpha,
         const int32_t* __restrict__ chunk_row, double* __restrict__ part) {
  using RT = RowTile<NC, T>;
  constexpr int H = RT::H, V = RT::V, LPR = RT::LPR, PER = RT::PER, RU = RT::RU;
  __shared__ double sh[kWarps][H];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ch = blockIdx.x;
  const float a = alpha[2];
  const int32_t r0 = chunk_row[ch], r1 = chunk_row[ch + 1];
  const bool act = lane < LPR;
  double d[PER][V];
#pragma unroll
  for (int q = 0; q < PER; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) d[q][e] = 0.0;
  for (int32_t r = r0 + w * RU; r < r1; r += kWarps * RU) {
    typename Vec<T>::Raw xr[RU][PER];
#pragma unroll
    for (int u = 0; u < RU; ++u)
#pragma unroll
      for (int q = 0; q < PER; ++q)
        xr[u][q] = (act && r + u < r1)
                       ? Vec<T>::ld(Z3 + (int64_t)(r + u) * H + (lane + q * LPR) * V)
                       : typename Vec<T>::Raw{};
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      float f[V];
#pragma unroll
      for (int e = 0; e < V; ++e) f[e] = 0.f;
#pragma unroll
      for (int u = 0; u < RU; ++u) {
        float x[V];
        Vec<T>::cvt(xr[u][q], x);
#pragma unroll
        for (int e = 0; e < V; ++e) f[e] += prelu(x[e], a);
      }
#pragma unroll
      for (int e = 0; e < V; ++e) d[q][e] += (double)f[e];
    }
  }
  if (act) {
#pragma unroll
    for (int q = 0; q < PER; ++q)
#pragma unroll
      for (int e = 0; e < V; ++e) sh[w][(lane + q * LPR) * V + e] = d[q][e];
  }
  __syncthreads();
  for (int c = threadIdx.x; c < H; c += kWarps * 32) {
    double t = 0.0;
#pragma unroll
    for (int k = 0; k < kWarps; ++k) t += sh[k][c];
    part[(int64_t)ch * H + c] = t;
  }
}

// Second stage of a per-graph column reduction over the graph's chunks, for 32
// columns per block: grid (G, H/32), 8 warps; warp w sums chunks w, w+8, ...
// (lanes = columns), the 8 warp sums are combined in fixed order.
//   mode 0 (readout, Eq. 4): s = sig(Σ / N_g) -> outd (fp64), outf (fp32)
//   mode 1 (dv):             Σ -> outd, outf; block (g, 0) also sums the
//                            graph's loss partials -> loss_g[g]
//   outf == nullptr (row-sharded graph): the raw shard-local Σ -> outd only
//                            (summed over shards and finished in k_head_xsum)
//   rep > 1: every chunk has rep consecutive partials (one per block pair of
//            k_score), summed like rep times as many chunks
__global__ void k_chunk_sum(const double* __restrict__ part, const int32_t* __restrict__ graph_chunk,
                            const int32_t* __restrict__ gsize, int H, int mode, int rep,
                            int readout, double* __restrict__ outd, float* __restrict__ outf,
                            const double* __restrict__ loss_part, double* __restrict__ loss_g) {
  __shared__ double sh[kWarps][32];
  const int g = blockIdx.x, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int c = blockIdx.y * 32 + lane;
  const int cb = graph_chunk[g] * rep, ce = graph_chunk[g + 1] * rep;
  double acc = 0.0;
  for (int ch = cb + w; ch < ce; ch += kWarps) acc += part[(int64_t)ch * H + c];
  sh[w][lane] = acc;
  __syncthreads();
  if (w == 0) {
    double t = 0.0;
#pragma unroll
    for (int k = 0; k < kWarps; ++k) t += sh[k][lane];
    if (mode == 0 && outf)
      t = readout ? t / (double)gsize[g] : 1.0 / (1.0 + exp(-(t / (double)gsize[g])));
    outd[(int64_t)g * H + c] = t;
    if (outf) outf[(int64_t)g * H + c] = (float)t;
  }
  if (mode == 1 && blockIdx.y == 0 && w == 1) {          // graph loss: lanes stride, fixed tree
    double t = 0.0;
    for (int ch = cb + lane; ch < ce; ch += 32) t += loss_part[ch];
    t = warp_sum(t);
    if (lane == 0) loss_g[g] = t;
  }
}

// v_g = M s_g (Eq. 5): grid (G, H/32); warp w computes rows r0 + 4w .. +3,
// lanes stride the columns (coalesced rows of M), fixed-order warp reduction.
__global__ void k_Mv(const float* __restrict__ M, const double* __restrict__ sd, int H,
                     float* __restrict__ vf) {
  const int g = blockIdx.x, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const double* s = sd + (int64_t)g * H;
  // H <= 256: at most 8 columns per lane; every load of the 4 rows issued
  // before the (fixed-order) sums
  double sv[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) sv[q] = lane + 32 * q < H ? s[lane + 32 * q] : 0.0;
  float mv[4][8];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int r = blockIdx.y * 32 + w * 4 + i;
#pragma unroll
    for (int q = 0; q < 8; ++q)
      mv[i][q] = lane + 32 * q < H ? M[(int64_t)r * H + lane + 32 * q] : 0.f;
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int r = blockIdx.y * 32 + w * 4 + i;
    double t = 0.0;
#pragma unroll
    for (int q = 0; q < 8; ++q) t += (double)mv[i][q] * sv[q];
    t = warp_sum(t);
    if (lane == 0) vf[(int64_t)g * H + r] = (float)t;
  }
}

// ds = Mᵀ dv_g and dm = ds s (1 - s) / N_g: grid (G, H/32); lanes own 32
// columns, warp w sums rows w, w+8, ... (coalesced), fixed-order combine.
__global__ void k_MTv(const float* __restrict__ M, const double* __restrict__ dvd,
                      const double* __restrict__ sd, const int32_t* __restrict__ gsize, int H,
                      int readout, float* __restrict__ dmf) {
  __shared__ double sh[kWarps][32];
  const int g = blockIdx.x, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int c = blockIdx.y * 32 + lane;
  const double* dv = dvd + (int64_t)g * H;
  double acc = 0.0;
  // H <= 256: at most 32 rows per warp, loaded 8 at a time, summed in order
  for (int r0 = w; r0 < H; r0 += 8 * kWarps) {
    float mv[8];
    double dd[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const int r = r0 + q * kWarps;
      mv[q] = r < H ? M[(int64_t)r * H + c] : 0.f;
      dd[q] = r < H ? dv[r] : 0.0;
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) acc += (double)mv[q] * dd[q];
  }
  sh[w][lane] = acc;
  __syncthreads();
  if (w == 0) {
    double ds = 0.0;
#pragma unroll
    for (int k = 0; k < kWarps; ++k) ds += sh[k][lane];
    const double s = sd[(int64_t)g * H + c];
    dmf[(int64_t)g * H + c] = (float)((readout ? ds : ds * s * (1.0 - s)) / (double)gsize[g]);
  }
}

__device__ __forceinline__ double softplus_d(double x) {
  return (x > 0.0 ? x : 0.0) + log1p(exp(-fabs(x)));
}

// Scores, loss partials, dl, and dv partials.  One block (8 warps) per (chunk,
// block pair bp); warp w takes NU consecutive nodes i per iteration, each with
// its rows in blocks 2bp and 2bp+1 (2 NU rows in flight; bp = 0: the positive row
// i and the corrupted row Nt+i); lanes own H/32 columns.
// The 2 NU logits are reduced across the warp, then lane j < 2 NU evaluates
// the sigmoid / softplus of logit j in fp64 (parallel over lanes) and the
// dl values are broadcast back.
template <int NC, typename T>
#ifndef MARS_SCORE_RS
#define MARS_SCORE_RS 1      // logit warp sums as one reduce-scatter (k_score)
#endif
#ifndef MARS_SCORE_MINB
#define MARS_SCORE_MINB 2
#endif
__global__ void __launch_bounds__(kWarps * 32, MARS_SCORE_MINB)
k_score(const T* __restrict__ Z3, const float* __restrict__ alpha,
        const int32_t* __restrict__ chunk_row, const int32_t* __restrict__ chunk_graph,
        const int32_t* __restrict__ gsize, const float* __restrict__ vf,
        const StepParams* __restrict__ sp, int32_t Nt, int32_t K, float* __restrict__ dl,
        double* __restrict__ dv_part, double* __restrict__ loss_part) {
  using RT = RowTile<NC, T>;
  constexpr int H = RT::H, V = RT::V, LPR = RT::LPR, PER = RT::PER;
#ifndef MARS_SCORE_NU
#define MARS_SCORE_NU 4     // 8 rows in flight per warp (A/B: profiles/r1s3_spmm_ab.md)
#endif
  constexpr int NU = RT::RU >= 4 ? MARS_SCORE_NU : 1;   // nodes per iteration (2 NU rows)
  __shared__ double sh_dv[kWarps][H];
  __shared__ double sh_loss[kWarps];
  const int ch = blockIdx.x, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int bp = blockIdx.y, nbp = gridDim.y;
  const bool act = lane < LPR;
  const int g = chunk_graph[ch];
  const float a = alpha[2];
  const double Ng = (double)gsize[g];
  const double coef = (double)sp->inv_batch / (2.0 * Ng);
  // block 2bp: positive (bp = 0, weight 1) or corrupted sample 2bp (1/K);
  // block 2bp+1: corrupted sample 2bp+1 (1/K) or padding (> K, weight 0)
  const int64_t rowA = 2LL * bp * Nt, rowB = rowA + Nt;
  const double wA = bp == 0 ? 1.0 : 1.0 / K, wB = 2 * bp + 1 <= K ? 1.0 / K : 0.0;
  const int32_t r0 = chunk_row[ch], r1 = chunk_row[ch + 1];
  float v[PER][V];
  double dv[PER][V];
#pragma unroll
  for (int q = 0; q < PER; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) {
      v[q][e] = act ? vf[(int64_t)g * H + (lane + q * LPR) * V + e] : 0.f;
      dv[q][e] = 0.0;
    }
  double loss = 0.0;
  for (int32_t i = r0 + w * NU; i < r1; i += kWarps * NU) {
    // rows kept as raw 16-byte vectors (4 registers each) and converted on use
    typename Vec<T>::Raw h[2 * NU][PER];
#pragma unroll
    for (int u = 0; u < NU; ++u)
#pragma unroll
      for (int q = 0; q < PER; ++q) {
        const int c = (lane + q * LPR) * V;
        if (act && i + u < r1) {
          h[2 * u][q] = Vec<T>::ld(Z3 + (rowA + i + u) * H + c);
          h[2 * u + 1][q] = Vec<T>::ld(Z3 + (rowB + i + u) * H + c);
        } else {
          h[2 * u][q] = h[2 * u + 1][q] = typename Vec<T>::Raw{};
        }
      }
    float l[2 * NU];
#pragma unroll
    for (int j = 0; j < 2 * NU; ++j) {
      float t = 0.f;
#pragma unroll
      for (int q = 0; q < PER; ++q) {
        float x[V];
        Vec<T>::cvt(h[j][q], x);
#pragma unroll
        for (int e = 0; e < V; ++e) t = fmaf(prelu(x[e], a), v[q][e], t);
      }
      l[j] = (MARS_SCORE_RS && 2 * NU == 8) ? t : warp_sum(t);
    }
    float mine = l[0];
    if constexpr (MARS_SCORE_RS && 2 * NU == 8) {
      // the 8 logits' warp sums as one reduce-scatter (9 shuffles instead of
      // 40): halving exchanges over lane bits 4, 3, 2 leave lane L with a
      // partial of logit 4 b4 + 2 b3 + b2, then bits 1, 0 finish it
      const bool b4 = lane & 16, b3 = lane & 8, b2 = lane & 4;
      float u4[4], u2[2];
#pragma unroll
      for (int k = 0; k < 4; ++k)
        u4[k] = (b4 ? l[k + 4] : l[k]) + __shfl_xor_sync(kFull, b4 ? l[k] : l[k + 4], 16);
#pragma unroll
      for (int k = 0; k < 2; ++k)
        u2[k] = (b3 ? u4[k + 2] : u4[k]) + __shfl_xor_sync(kFull, b3 ? u4[k] : u4[k + 2], 8);
      float u1 = (b2 ? u2[1] : u2[0]) + __shfl_xor_sync(kFull, b2 ? u2[0] : u2[1], 4);
      u1 += __shfl_xor_sync(kFull, u1, 2);
      u1 += __shfl_xor_sync(kFull, u1, 1);
      const int src = ((lane & 4) << 2) | ((lane & 2) << 2) | ((lane & 1) << 2);   // logit lane & 7
      mine = __shfl_sync(kFull, u1, src);
    } else {
#pragma unroll
      for (int j = 1; j < 2 * NU; ++j) mine = lane == j ? l[j] : mine;
    }
    float dmine = 0.f;
    if (lane < 2 * NU && i + (lane >> 1) < r1) {
      const double x = (double)mine;
      const double sg = 1.0 / (1.0 + exp(-x));
      const bool isB = lane & 1, neg = isB || bp > 0;
      const double wt = isB ? wB : wA;
      dmine = (float)((neg ? sg : sg - 1.0) * (coef * wt));
      dl[(isB ? rowB : rowA) + i + (lane >> 1)] = dmine;
      loss += wt * (neg ? softplus_d(x) : softplus_d(-x));
    }
    float dvp[PER][V];
#pragma unroll
    for (int q = 0; q < PER; ++q)
#pragma unroll
      for (int e = 0; e < V; ++e) dvp[q][e] = 0.f;
#pragma unroll
    for (int j = 0; j < 2 * NU; ++j) {
      const float dj = __shfl_sync(kFull, dmine, j);
#pragma unroll
      for (int q = 0; q < PER; ++q) {
        float x[V];
        Vec<T>::cvt(h[j][q], x);
#pragma unroll
        for (int e = 0; e < V; ++e) dvp[q][e] = fmaf(dj, prelu(x[e], a), dvp[q][e]);
      }
    }
#pragma unroll
    for (int q = 0; q < PER; ++q)
#pragma unroll
      for (int e = 0; e < V; ++e) dv[q][e] += (double)dvp[q][e];
  }
  if (act) {
#pragma unroll
    for (int q = 0; q < PER; ++q)
#pragma unroll
      for (int e = 0; e < V; ++e) sh_dv[w][(lane + q * LPR) * V + e] = dv[q][e];
  }
  loss = warp_sum(loss);
  if (lane == 0) sh_loss[w] = loss;
  __syncthreads();
  for (int c = threadIdx.x; c < H; c += kWarps * 32) {
    double t = 0.0;
#pragma unroll
    for (int k = 0; k < kWarps; ++k) t += sh_dv[k][c];
    dv_part[((int64_t)ch * nbp + bp) * H + c] = t;
  }
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int k = 0; k < kWarps; ++k) t += sh_loss[k];
    loss_part[(int64_t)ch * nbp + bp] = t * coef;   // (1/B) (1/(2 N_g)) Σ weighted softplus terms
  }
}

// ---- InfoNCE (c39): per node i, one positive logit l_i0 (block 0) against
// its K corrupted counterparts l_ik (blocks 1..K, same node index):
//   L = (1/B) Σ_g (1/N_g) Σ_i [log Σ_k e^{l_ik} - l_i0]
//   dl_i0 = (p_i0 - 1)/(N_g B), dl_ik = p_ik/(N_g B), p = softmax over k.
// Three passes replace k_score: logits of every real row, the per-node
// softmax (dl, loss partials), and the dv partials Σ dl h.
template <int NC, typename T>
__global__ void __launch_bounds__(kWarps * 32, 3)
k_logits(const T* __restrict__ Z3, const float* __restrict__ alpha,
         const int32_t* __restrict__ chunk_row, const int32_t* __restrict__ chunk_graph,
         const float* __restrict__ vf, int32_t Nt, float* __restrict__ lg) {
  using RT = RowTile<NC, T>;
  constexpr int H = RT::H, V = RT::V, LPR = RT::LPR, PER = RT::PER, RU = RT::RU;
  const int ch = blockIdx.x, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const bool act = lane < LPR;
  const int g = chunk_graph[ch];
  const float a = alpha[2];
  const int64_t base = (int64_t)blockIdx.y * Nt;
  const int32_t r0 = chunk_row[ch], r1 = chunk_row[ch + 1];
  float v[PER][V];
#pragma unroll
  for (int q = 0; q < PER; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) v[q][e] = act ? vf[(int64_t)g * H + (lane + q * LPR) * V + e] : 0.f;
  for (int32_t r = r0 + w * RU; r < r1; r += kWarps * RU) {
    typename Vec<T>::Raw zr[RU][PER];
#pragma unroll
    for (int u = 0; u < RU; ++u)
#pragma unroll
      for (int q = 0; q < PER; ++q)
        zr[u][q] = (act && r + u < r1) ? Vec<T>::ld(Z3 + (base + r + u) * H + (lane + q * LPR) * V)
                                       : typename Vec<T>::Raw{};
#pragma unroll
    for (int u = 0; u < RU; ++u) {
      float t = 0.f;
#pragma unroll
      for (int q = 0; q < PER; ++q) {
        float x[V];
        Vec<T>::cvt(zr[u][q], x);
#pragma unroll
        for (int e = 0; e < V; ++e) t = fmaf(prelu(x[e], a), v[q][e], t);
      }
      t = warp_sum(t);
      if (lane == 0 && r + u < r1) lg[base + r + u] = t;
    }
  }
}

// One block per chunk, one thread per node: softmax over the node's K + 1
// logits (fp64), dl in place of the logits (0 on padding blocks), and the
// chunk's loss partial at loss_part[ch * (K + 1)] (the other K slots 0, so the
// dv reduction's rep = K + 1 sums it once).
__global__ void __launch_bounds__(256)
k_nce(const int32_t* __restrict__ chunk_row, const int32_t* __restrict__ chunk_graph,
      const int32_t* __restrict__ gsize, const StepParams* __restrict__ sp, int32_t Nt, int32_t K,
      int32_t nb, float* __restrict__ dl, double* __restrict__ loss_part) {
  __shared__ double sh[256];
  const int ch = blockIdx.x;
  const int32_t r = chunk_row[ch] + threadIdx.x, r1 = chunk_row[ch + 1];
  const double coef = (double)sp->inv_batch / (double)gsize[chunk_graph[ch]];
  double loss = 0.0;
  if (r < r1) {
    double m = -INFINITY;
    for (int k = 0; k <= K; ++k) m = fmax(m, (double)dl[(int64_t)k * Nt + r]);
    double se = 0.0;
    for (int k = 0; k <= K; ++k) se += exp((double)dl[(int64_t)k * Nt + r] - m);
    const double lse = m + log(se);
    const double l0 = (double)dl[r];
    loss = lse - l0;
    for (int k = 0; k <= K; ++k) {
      const int64_t o = (int64_t)k * Nt + r;
      const double p = exp((double)dl[o] - lse);
      dl[o] = (float)(coef * (k == 0 ? p - 1.0 : p));
    }
    for (int k = K + 1; k < nb; ++k) dl[(int64_t)k * Nt + r] = 0.f;
  }
  sh[threadIdx.x] = loss;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x <= K) loss_part[(int64_t)ch * (K + 1) + threadIdx.x] = threadIdx.x ? 0.0 : sh[0] * coef;
}

// dv partials Σ_rows dl_i H3_i per (chunk, block b in 0..K) -> part[(ch (K+1) + b) H]
template <int NC, typename T>
__global__ void __launch_bounds__(kWarps * 32, 3)
k_dvp(const T* __restrict__ Z3, const float* __restrict__ alpha,
      const int32_t* __restrict__ chunk_row, const float* __restrict__ dl, int32_t Nt,
      double* __restrict__ part) {
  using RT = RowTile<NC, T>;
  constexpr int H = RT::H, V = RT::V, LPR = RT::LPR, PER = RT::PER, RU = RT::RU;
  __shared__ double sh[kWarps][H];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ch = blockIdx.x;
  const float a = alpha[2];
  const int64_t base = (int64_t)blockIdx.y * Nt;
  const int32_t r0 = chunk_row[ch], r1 = chunk_row[ch + 1];
  const bool act = lane < LPR;
  double d[PER][V];
#pragma unroll
  for (int q = 0; q < PER; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) d[q][e] = 0.0;
  for (int32_t r = r0 + w * RU; r < r1; r += kWarps * RU) {
    typename Vec<T>::Raw xr[RU][PER];
    float c[RU];
#pragma unroll
    for (int u = 0; u < RU; ++u) {
      c[u] = r + u < r1 ? dl[base + r + u] : 0.f;
#pragma unroll
      for (int q = 0; q < PER; ++q)
        xr[u][q] = (act && r + u < r1) ? Vec<T>::ld(Z3 + (base + r + u) * H + (lane + q * LPR) * V)
                                       : typename Vec<T>::Raw{};
    }
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      float f[V];
#pragma unroll
      for (int e = 0; e < V; ++e) f[e] = 0.f;
#pragma unroll
      for (int u = 0; u < RU; ++u) {
        float x[V];
        Vec<T>::cvt(xr[u][q], x);
#pragma unroll
        for (int e = 0; e < V; ++e) f[e] = fmaf(c[u], prelu(x[e], a), f[e]);
      }
#pragma unroll
      for (int e = 0; e < V; ++e) d[q][e] += (double)f[e];
    }
  }
  if (act) {
#pragma unroll
    for (int q = 0; q < PER; ++q)
#pragma unroll
      for (int e = 0; e < V; ++e) sh[w][(lane + q * LPR) * V + e] = d[q][e];
  }
  __syncthreads();
  for (int cc = threadIdx.x; cc < H; cc += kWarps * 32) {
    double t = 0.0;
#pragma unroll
    for (int k = 0; k < kWarps; ++k) t += sh[k][cc];
    part[((int64_t)ch * gridDim.y + blockIdx.y) * H + cc] = t;
  }
}

// dM[r][c] = Σ_g dv_g[r] s_g[c] (fixed order); block 0 also writes the loss.
__global__ void k_dM(const double* __restrict__ dvd, const double* __restrict__ sd, int G, int H,
                     const double* __restrict__ loss_g, float* __restrict__ gM,
                     float* __restrict__ loss_out) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < (int64_t)H * H) {
    int r = (int)(e / H), c = (int)(e % H);
    double t = 0.0;
    int g = 0;
    for (; g + 4 <= G; g += 4) {            // four graphs' loads in flight, summed in order
      const double a0 = dvd[(int64_t)g * H + r], b0 = sd[(int64_t)g * H + c];
      const double a1 = dvd[(int64_t)(g + 1) * H + r], b1 = sd[(int64_t)(g + 1) * H + c];
      const double a2 = dvd[(int64_t)(g + 2) * H + r], b2 = sd[(int64_t)(g + 2) * H + c];
      const double a3 = dvd[(int64_t)(g + 3) * H + r], b3 = sd[(int64_t)(g + 3) * H + c];
      t += a0 * b0;
      t += a1 * b1;
      t += a2 * b2;
      t += a3 * b3;
    }
    for (; g < G; ++g) t += dvd[(int64_t)g * H + r] * sd[(int64_t)g * H + c];
    gM[e] = (float)t;
  }
  if (e == 0) {
    double t = 0.0;
    for (int g = 0; g < G; ++g) t += loss_g[g];
    *loss_out = (float)t;
  }
}

// dZ3 = (dl v_g + [pos] dm_g) ⊙ PReLU'(Z3), dalpha3 partials.  Grid (chunk,
// half): block (ch, 0) covers the chunk's positive rows, (ch, 1) the matching
// corrupted rows Nt + i.  v_g and dm_g are loaded once per block into
// registers; warp w streams RU consecutive rows per iteration.  One dalpha
// slot per block, folded in fixed order.
template <int NC, typename T>
__global__ void __launch_bounds__(kWarps * 32, 3)
k_dz3(const T* __restrict__ Z3, const float* __restrict__ alpha,
      const int32_t* __restrict__ chunk_row, const int32_t* __restrict__ chunk_graph,
      const float* __restrict__ dl, const float* __restrict__ vf, const float* __restrict__ dmf,
      int32_t Nt, T* __restrict__ dZ, double* __restrict__ slots, float* __restrict__ rs) {
  using RT = RowTile<NC, T>;
  constexpr int H = RT::H, V = RT::V, LPR = RT::LPR, PER = RT::PER, RU = RT::RU;
  __shared__ double wpart[kWarps];
  const int ch = blockIdx.x, half = blockIdx.y;     // half: stacked block (0 = positive)
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const bool act = lane < LPR;
  const int g = chunk_graph[ch];
  const float a = alpha[2];
  const int32_t r0 = chunk_row[ch], r1 = chunk_row[ch + 1];
  const int64_t base = (int64_t)half * Nt;
  float vg[PER][V], mg[PER][V];
#pragma unroll
  for (int q = 0; q < PER; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) {
      const int64_t c = (int64_t)g * H + (lane + q * LPR) * V + e;
      vg[q][e] = act ? vf[c] : 0.f;
      mg[q][e] = (act && !half) ? dmf[c] : 0.f;
    }
  double da = 0.0;
  for (int32_t r = r0 + w * RU; r < r1; r += kWarps * RU) {
    typename Vec<T>::Raw zr[RU][PER];
    float d[RU];
#pragma unroll
    for (int u = 0; u < RU; ++u) {
      const bool ok = r + u < r1;
      d[u] = ok ? dl[base + r + u] : 0.f;
#pragma unroll
      for (int q = 0; q < PER; ++q)
        zr[u][q] = (act && ok) ? Vec<T>::ld(Z3 + (base + r + u) * H + (lane + q * LPR) * V)
                               : typename Vec<T>::Raw{};
    }
    float daf = 0.f;
#pragma unroll
    for (int u = 0; u < RU; ++u) {
      float mx = 0.f;
#pragma unroll
      for (int q = 0; q < PER; ++q) {
        float o[V], z[V];
        Vec<T>::cvt(zr[u][q], z);
#pragma unroll
        for (int e = 0; e < V; ++e) {
          const float dh = fmaf(d[u], vg[q][e], mg[q][e]);
          o[e] = z[e] > 0.f ? dh : a * dh;
          daf += z[e] > 0.f ? 0.f : dh * z[e];
          mx = fmaxf(mx, act ? fabsf(o[e]) : 0.f);
        }
        if (act && r + u < r1) StoreN<T, V>::store(dZ + (base + r + u) * H + (lane + q * LPR) * V, o);
      }
      if (rs) {                     // row scale of the stored dZ3 row (3xFP16 dY GEMM)
        // |values| >= 0: the unsigned max of the bit patterns is the float max
        mx = __uint_as_float(__reduce_max_sync(kFull, __float_as_uint(mx)));
        if (lane == 0 && r + u < r1) rs[base + r + u] = pow2_scale(mx);
      }
    }
    da += (double)daf;
  }
  da = warp_sum(da);
  if (lane == 0) wpart[w] = da;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int k = 0; k < kWarps; ++k) s += wpart[k];
    slots[(int64_t)ch * gridDim.y + half] = s;
  }
}

// Sum of n fp64 partials -> fp32, one block of 1024 threads: thread t keeps
// four accumulators (k = t + 4096 i + 1024 q), then a fixed-shape tree.
__global__ void __launch_bounds__(1024) k_reduce_slots(const double* __restrict__ slots, int n,
                                                       float* __restrict__ out) {
  __shared__ double sh[1024];
  double t0 = 0.0, t1 = 0.0, t2 = 0.0, t3 = 0.0;
  int k = threadIdx.x;
  for (; k + 3072 < n; k += 4096) {
    t0 += slots[k];
    t1 += slots[k + 1024];
    t2 += slots[k + 2048];
    t3 += slots[k + 3072];
  }
  for (; k < n; k += 1024) t0 += slots[k];
  sh[threadIdx.x] = (t0 + t1) + (t2 + t3);
  __syncthreads();
  for (int o = 512; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) *out = (float)sh[0];
}

// Stage 1 of a long slot reduction: block b sums the contiguous range
// [b·n/NB, (b+1)·n/NB) in a fixed order (per-thread strides, then a tree).
constexpr int kRedParts = 128;
__global__ void __launch_bounds__(256) k_reduce_part(const double* __restrict__ slots, int n,
                                                     double* __restrict__ part) {
  __shared__ double sh[256];
  const int64_t b0 = (int64_t)n * blockIdx.x / kRedParts, b1 = (int64_t)n * (blockIdx.x + 1) / kRedParts;
  double t = 0.0;
  for (int64_t k = b0 + threadIdx.x; k < b1; k += 256) t += slots[k];
  sh[threadIdx.x] = t;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) part[blockIdx.x] = sh[0];
}

template <typename T>
__global__ void k_prelu(const T* __restrict__ Z, const float* __restrict__ alpha, int layer,
                        float* __restrict__ out, int64_t n) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < n) out[e] = prelu(to_f(Z[e]), alpha[layer]);
}

__global__ void k_upcast(const bf16* __restrict__ in, float* __restrict__ out, int64_t n) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < n) out[e] = __bfloat162float(in[e]);
}

template <int NC, typename T>
cudaError_t head_nc(const GraphDev& g, const T* Z3, const float* M, const float* alpha,
                    const StepParams* sp, const HeadWork& w, T* dZ, float* gM, float* loss_out,
                    int* nslots, cudaStream_t s, const HeadShard* hs) {
  constexpr int H = NC * 32;
  const dim3 gh(g.G, H / 32);
  cudaError_t e;
  const int nb = w.nb, nbp = nb / 2;
  if (nb < 2 || (nb & 1) || w.K < 1 || w.K >= nb || (hs && (nb != 2 || w.readout || w.loss)))
    return cudaErrorInvalidValue;
  k_colsum<NC, T><<<g.nchunks, kWarps * 32, 0, s>>>(Z3, alpha, g.chunk_row, w.colsum_part);
  if (!hs) {
    k_chunk_sum<<<gh, 256, 0, s>>>(w.colsum_part, g.graph_chunk, g.gsize, H, 0, 1, w.readout,
                                   w.sd, w.s, nullptr, nullptr);
  } else {      // shard-local sums -> own exchange buffer; barrier; sum over shards
    k_chunk_sum<<<gh, 256, 0, s>>>(w.colsum_part, g.graph_chunk, g.gsize, H, 0, 1, 0,
                                   hs->x_own[0], nullptr, nullptr, nullptr);
    if ((e = launch_shard_barrier(*hs->sync, s, nullptr)) != cudaSuccess) return e;
    if ((e = launch_head_xsum(hs->x_peers[0], hs->sync->P, H, 0, g.gsize, w.sd, w.s, nullptr, s,
                              nullptr)) != cudaSuccess)
      return e;
  }
  k_Mv<<<gh, 256, 0, s>>>(M, w.sd, H, w.v);
  if (w.loss) {                   // InfoNCE (c39)
    const dim3 gk(g.nchunks, w.K + 1);
    k_logits<NC, T><<<gk, kWarps * 32, 0, s>>>(Z3, alpha, g.chunk_row, g.chunk_graph, w.v, g.Nt,
                                                w.dl);
    k_nce<<<g.nchunks, 256, 0, s>>>(g.chunk_row, g.chunk_graph, g.gsize, sp, g.Nt, w.K, nb, w.dl,
                                    w.loss_part);
    k_dvp<NC, T><<<gk, kWarps * 32, 0, s>>>(Z3, alpha, g.chunk_row, w.dl, g.Nt, w.dv_part);
    k_chunk_sum<<<gh, 256, 0, s>>>(w.dv_part, g.graph_chunk, g.gsize, H, 1, w.K + 1, 0, w.dvd,
                                   w.dv, w.loss_part, w.loss_g);
  } else if (!hs) {
    k_score<NC, T><<<dim3(g.nchunks, nbp), kWarps * 32, 0, s>>>(
        Z3, alpha, g.chunk_row, g.chunk_graph, g.gsize, w.v, sp, g.Nt, w.K, w.dl, w.dv_part,
        w.loss_part);
    k_chunk_sum<<<gh, 256, 0, s>>>(w.dv_part, g.graph_chunk, g.gsize, H, 1, nbp, 0, w.dvd, w.dv,
                                   w.loss_part, w.loss_g);
  } else {
    k_score<NC, T><<<dim3(g.nchunks, nbp), kWarps * 32, 0, s>>>(
        Z3, alpha, g.chunk_row, g.chunk_graph, g.gsize, w.v, sp, g.Nt, w.K, w.dl, w.dv_part,
        w.loss_part);
    k_chunk_sum<<<gh, 256, 0, s>>>(w.dv_part, g.graph_chunk, g.gsize, H, 1, 1, 0, hs->x_own[1],
                                   nullptr, w.loss_part, hs->x_own[1] + H);
    if ((e = launch_shard_barrier(*hs->sync, s, nullptr)) != cudaSuccess) return e;
    if ((e = launch_head_xsum(hs->x_peers[1], hs->sync->P, H, 1, g.gsize, w.dvd, w.dv, w.loss_g,
                              s, nullptr)) != cudaSuccess)
      return e;
  }
  k_MTv<<<gh, 256, 0, s>>>(M, w.dvd, w.sd, g.gsize, H, w.readout, w.dm);
  k_dM<<<cdiv((int64_t)H * H, 256), 256, 0, s>>>(w.dvd, w.sd, g.G, H, w.loss_g, gM, loss_out);
  k_dz3<NC, T><<<dim3(g.nchunks, nb), kWarps * 32, 0, s>>>(Z3, alpha, g.chunk_row, g.chunk_graph,
                                                          w.dl, w.v, w.dm, g.Nt, dZ, w.slots,
                                                          std::is_same<T, float>::value ? w.rs_dz3
                                                                                        : nullptr);
  *nslots = nb * g.nchunks;
  return cudaGetLastError();
}

template <typename T>
cudaError_t head_t(const GraphDev& g, int H, const void* Z3, const float* M, const float* alpha,
                   const StepParams* sp, const HeadWork& w, void* dZ, float* gM, float* loss,
                   int* nslots, cudaStream_t s, const HeadShard* hs) {
  const T* z = static_cast<const T*>(Z3);
  T* d = static_cast<T*>(dZ);
  switch (H) {
    case 32: return head_nc<1, T>(g, z, M, alpha, sp, w, d, gM, loss, nslots, s, hs);
    case 64: return head_nc<2, T>(g, z, M, alpha, sp, w, d, gM, loss, nslots, s, hs);
    case 128: return head_nc<4, T>(g, z, M, alpha, sp, w, d, gM, loss, nslots, s, hs);
    case 256: return head_nc<8, T>(g, z, M, alpha, sp, w, d, gM, loss, nslots, s, hs);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace

int head_slots(const GraphDev& g, int nb) {       // + reduction scratch
  return nb * g.nchunks + 1 + kRedParts;
}

cudaError_t launch_head(const GraphDev& g, int H, const void* Z3, int bf16_, const float* params_M,
                        const float* alpha_dev, const StepParams* sp, const HeadWork& w, void* dZ,
                        float* grad_M, float* loss_out, int* nslots, cudaStream_t s,
                        int* launches, const HeadShard* hs) {
  count_launch(launches, hs ? 12 : w.loss ? 10 : 8);
  if (bf16_)
    return head_t<bf16>(g, H, Z3, params_M, alpha_dev, sp, w, dZ, grad_M, loss_out, nslots, s, hs);
  return head_t<float>(g, H, Z3, params_M, alpha_dev, sp, w, dZ, grad_M, loss_out, nslots, s, hs);
}

cudaError_t launch_reduce_slots(double* slots, int n, float* grad, cudaStream_t s,
                                int* launches) {
  count_launch(launches, n > 8192 ? 2 : 1);
  if (n > 8192) {   // long slot lists (one per SpMM warp-block): two stages, scratch after them
    k_reduce_part<<<kRedParts, 256, 0, s>>>(slots, n, slots + n);
    k_reduce_slots<<<1, 1024, 0, s>>>(slots + n, kRedParts, grad);
  } else {
    k_reduce_slots<<<1, 1024, 0, s>>>(slots, n, grad);
  }
  return cudaGetLastError();
}

cudaError_t launch_prelu(const void* Z, int bf16_, const float* alpha_dev, int layer, float* out,
                         int64_t n, cudaStream_t s, int* launches) {
  count_launch(launches);
  if (bf16_)
    k_prelu<bf16><<<cdiv(n, 256), 256, 0, s>>>(static_cast<const bf16*>(Z), alpha_dev, layer, out, n);
  else
    k_prelu<float><<<cdiv(n, 256), 256, 0, s>>>(static_cast<const float*>(Z), alpha_dev, layer, out, n);
  return cudaGetLastError();
}

cudaError_t launch_upcast(const void* in, float* out, int64_t n, cudaStream_t s) {
  k_upcast<<<cdiv(n, 256), 256, 0, s>>>(static_cast<const bf16*>(in), out, n);
  return cudaGetLastError();
}

}  // namespace mars
