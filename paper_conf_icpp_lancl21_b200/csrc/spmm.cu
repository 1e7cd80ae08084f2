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
// Row-sharded graph (shard.cu): layers 2-3 and the backward
// gather neighbour rows by GLOBAL column id from the owning shard's buffer
// (PeerSrc: peer-mapped memory over NVLink, or CUDA IPC) -- the halo exchange
// is fused into the aggregation; row i of the output is local.
#include "common.cuh"
#include "internal.cuh"
#include "vec.cuh"

#include <algorithm>
#include <type_traits>

namespace mars {
namespace {

constexpr int kSpmmThreads = 32;   // one warp per block: a slow (hub) row holds no other warps
#ifndef MARS_SPMM_MINB             // resident blocks per SM: caps registers at 64
#define MARS_SPMM_MINB 32
#endif
#ifndef MARS_SPMM_KU
#define MARS_SPMM_KU 4
#endif
#ifndef MARS_SPMM_REDUX
#define MARS_SPMM_REDUX 1           // row-scale maxima by redux.sync (whole-warp rows)
#endif
constexpr int kU = MARS_SPMM_KU;   // neighbours whose gathers are in flight together
// The backward rows also stream their own Z rows (PReLU') and write dZ: with
// 2 neighbours per gather batch (fp32) they fit the 64-register budget
// without spilling, measured -8 % against 4 ((17)).
#ifndef MARS_SPMM_KU_BWD
#define MARS_SPMM_KU_BWD 2
#endif
#ifndef MARS_SPMM_KU_BWD16
#define MARS_SPMM_KU_BWD16 4
#endif
template <typename T>
constexpr int kUB = std::is_same<T, float>::value ? MARS_SPMM_KU_BWD : MARS_SPMM_KU_BWD16;

// C in {16, 32, 64, 128, 256} (mars.h restricts F and H to these widths).
#ifndef MARS_SPMM_LMAX_BF16
#define MARS_SPMM_LMAX_BF16 32     // lanes per bf16 row at most (A/B: 16 = two rows per warp)
#endif
template <int C, typename T>
struct SpmmShape {
  static constexpr int V = Vec<T>::N;                     // elements per 16-byte load
  static constexpr int LMAX = std::is_same<T, float>::value ? 32 : MARS_SPMM_LMAX_BF16;
  static constexpr int L = (C / V) < LMAX ? (C / V) : LMAX;   // lanes per row
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

// Measured and rejected on the bench step: a persistent grid
// interleaving rows i, i + NG, ... over all SMs (+10-17 % fp32), and software
// pipelining across rows (next row's first (colind, val) chunk and the row
// after's rowptr in flight during this row's gathers, +25-48 % fp32).

// Sources of the gathered rows: pos row j, neg row (j, or perm[j] for layer 1).
template <typename T, int C>
struct StackedSrc {     // [pos; neg] stacked in one 2*Nt-row buffer
  const T* base;
  int32_t Nt;
  __device__ __forceinline__ const T* pos(int32_t j) const { return base + (int64_t)j * C; }
  __device__ __forceinline__ const T* neg(int32_t j, int32_t) const {
    return base + ((int64_t)Nt + j) * C;
  }
};
template <typename T, int C>
struct PermSrc {        // layer 1: pos X[j], neg X[perm[j]]
  const T* X;
  __device__ __forceinline__ const T* pos(int32_t j) const { return X + (int64_t)j * C; }
  __device__ __forceinline__ const T* neg(int32_t, int32_t jn) const { return X + (int64_t)jn * C; }
};

template <typename T, int C>
struct PeerSrc {        // row-sharded graph: global row j lives on shard owner(j)
  const PeerRows& pr;   // a __grid_constant__ kernel parameter (constant bank)
  __device__ __forceinline__ int owner(int32_t j) const {
    int p = 0;
#pragma unroll
    for (int q = 1; q < kMaxShards; ++q) p += j >= pr.start[q] ? 1 : 0;
    return p;
  }
  __device__ __forceinline__ const T* pos(int32_t j) const {
    const int p = owner(j);
    return static_cast<const T*>(pr.base[p]) + (int64_t)(j - pr.start[p]) * C;
  }
  __device__ __forceinline__ const T* neg(int32_t j, int32_t) const {
    const int p = owner(j);
    const int32_t n = pr.start[p + 1] - pr.start[p];
    return static_cast<const T*>(pr.base[p]) + ((int64_t)n + j - pr.start[p]) * C;
  }
};

// One batch of K neighbours t .. t+K-1 of the current chunk: all 2K gathers
// are issued before the FMAs.  Slots u >= nvalid re-gather neighbour t (a
// valid row, usually an L1 hit) with weight 0, so the batch needs no branch
// and its loads stay independent.  Adding 0·x leaves the ascending-order sum
// unchanged.
template <class S, int K, bool BOTH, int ACT, bool PERM, typename T, class Src>
__device__ __forceinline__ void gather_batch(const Src& src, int t, int nvalid, int32_t cj,
                                             float cv, int32_t cjn, unsigned gmask, int sl,
                                             float a, float (&accp)[S::NT][S::V],
                                             float (&accn)[S::NT][S::V]) {
  constexpr int V = S::V;
  int32_t j[K], jn[K];
  float w[K];
#pragma unroll
  for (int u = 0; u < K; ++u) {
    const int lane_u = u < nvalid ? t + u : t;
    j[u] = __shfl_sync(gmask, cj, lane_u, S::L);
    w[u] = __shfl_sync(gmask, cv, lane_u, S::L);
    jn[u] = (PERM && BOTH) ? __shfl_sync(gmask, cjn, lane_u, S::L) : 0;
    if (u >= nvalid) w[u] = 0.f;
  }
  if constexpr (ACT == 2) {
    // PReLU on packed bf16 pairs before widening: max(x, bf16(a·x)), exact
    // for 0 <= a <= 1 up to the bf16 rounding of a·x (the kernel selects
    // this form at run time only for such a; bf16 path only)
    typename Vec<T>::Raw rp[K][S::NT], rn[K][S::NT];
#pragma unroll
    for (int u = 0; u < K; ++u)
#pragma unroll
      for (int q = 0; q < S::NT; ++q) {
        const int c = (sl + q * S::L) * V;
        rp[u][q] = Vec<T>::ld(src.pos(j[u]) + c);
        if (BOTH) rn[u][q] = Vec<T>::ld(src.neg(j[u], jn[u]) + c);
      }
    const __nv_bfloat162 a2 = __float2bfloat162_rn(a);
    auto hp = [&](uint32_t& wv) {
      __nv_bfloat162 x = *reinterpret_cast<__nv_bfloat162*>(&wv);
      x = __hmax2(x, __hmul2(x, a2));
      wv = *reinterpret_cast<uint32_t*>(&x);
    };
#pragma unroll
    for (int u = 0; u < K; ++u)
#pragma unroll
      for (int q = 0; q < S::NT; ++q) {
        float x[V];
        hp(rp[u][q].x); hp(rp[u][q].y); hp(rp[u][q].z); hp(rp[u][q].w);
        Vec<T>::cvt(rp[u][q], x);
        vfma<V>(accp[q], w[u], x);
        if (BOTH) {
          hp(rn[u][q].x); hp(rn[u][q].y); hp(rn[u][q].z); hp(rn[u][q].w);
          Vec<T>::cvt(rn[u][q], x);
          vfma<V>(accn[q], w[u], x);
        }
      }
  } else {
    float xp[K][S::NT][V], xn[K][S::NT][V];
#pragma unroll
    for (int u = 0; u < K; ++u)
#pragma unroll
      for (int q = 0; q < S::NT; ++q) {
        const int c = (sl + q * S::L) * V;
        Vec<T>::load(src.pos(j[u]) + c, xp[u][q]);
        if (BOTH) Vec<T>::load(src.neg(j[u], jn[u]) + c, xn[u][q]);
      }
#pragma unroll
    for (int u = 0; u < K; ++u)
#pragma unroll
      for (int q = 0; q < S::NT; ++q) {
        if (ACT) vprelu<V>(xp[u][q], a);
        vfma<V>(accp[q], w[u], xp[u][q]);
        if (BOTH) {
          if (ACT) vprelu<V>(xn[u][q], a);
          vfma<V>(accn[q], w[u], xn[u][q]);
        }
      }
  }
}

// Accumulates row (rb, re) of Â_n · act(T) for both branches: per chunk of L
// neighbours each lane loads one (colind, val) pair (+ perm for layer 1),
// broadcast by shuffles, then batches of kU neighbours; the last partial batch
// is one padded batch (measured against a neighbour-at-a-time tail and
// predicated tails).
template <class S, bool BOTH, int ACT, bool PERM, typename T, int KU = kU, class Src>
__device__ __forceinline__ void row_gather(const Src& src, const int32_t* __restrict__ colind,
                                           const float* __restrict__ vals,
                                           const int32_t* __restrict__ perm, int32_t rb,
                                           int32_t re, unsigned gmask, int sl, float a,
                                           float (&accp)[S::NT][S::V],
                                           float (&accn)[S::NT][S::V]) {
  for (int32_t k0 = rb; k0 < re; k0 += S::L) {
    const int32_t cnt = min(S::L, re - k0);
    int32_t cj = 0, cjn = 0;
    float cv = 0.f;
    if (sl < cnt) {
      cj = colind[k0 + sl];
      cv = vals[k0 + sl];
      if (PERM && BOTH) cjn = perm[k0 + sl];   // colperm: pi[colind[k]], no dependent lookup
    }
    for (int t = 0; t < cnt; t += KU)
      gather_batch<S, KU, BOTH, ACT, PERM, T>(src, t, min(KU, cnt - t), cj, cv, cjn, gmask, sl,
                                              a, accp, accn);
  }
}

// Power-of-two row scale (gemm_tc3h.cu) of one stored row held by the L lanes
// of a row group: max |x| over the group, lane 0 of the group writes it.
template <class S, int NV>
__device__ __forceinline__ void row_scale_out(const float (&x)[S::NT][NV], unsigned gmask, int sl,
                                              float* __restrict__ dst) {
  float m = 0.f;
#pragma unroll
  for (int q = 0; q < S::NT; ++q)
#pragma unroll
    for (int e = 0; e < NV; ++e) m = fmaxf(m, fabsf(x[q][e]));
  if constexpr (MARS_SPMM_REDUX && S::L == 32) {
    // |x| >= 0: the unsigned maximum of the bit patterns is the float
    // maximum -- one redux.sync over the warp (a NaN, whose bits exceed
    // +inf's, gives the scale 1 in pow2_scale)
    m = __uint_as_float(__reduce_max_sync(gmask, __float_as_uint(m)));
  } else {
#pragma unroll
    for (int o = S::L / 2; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(gmask, m, o));
  }
  if (sl == 0) *dst = pow2_scale(m);
}

#ifndef MARS_SPMM_PF
#define MARS_SPMM_PF (3 << 20)   // L2-prefetch distance in bytes of one branch's rows (0: off)
#endif
__device__ __forceinline__ void prefetch_l2(const void* p) {
  asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

// Streams the inputs of row i + PF into L2 ahead of its block (PF = 3 MB of
// one branch's rows: 3072 rows of 1 KB, 6144 of 512 B; measured, r1s3_spmm_ab.md): its
// own source rows (pos + neg -- also the first-touch gathers of its
// neighbours) now, and its colind / vals lines once its rowptr entry (loaded
// now, used at the end of this row) has arrived.
template <typename T, int C, bool NEG>
__device__ __forceinline__ int32_t prefetch_rows_ahead(int32_t i, int32_t Nt,
                                                       const int32_t* rowptr, const T* base,
                                                       int sl) {
  constexpr int PF = MARS_SPMM_PF / (C * (int)sizeof(T));
  const int32_t ip = i + PF;
  if (PF <= 0 || ip >= Nt) return -1;
  constexpr int LINES = (C * (int)sizeof(T) + 127) / 128;    // 128-byte lines per branch row
  if (sl < LINES) {
    prefetch_l2(reinterpret_cast<const char*>(base + (int64_t)ip * C) + sl * 128);
    if (NEG) prefetch_l2(reinterpret_cast<const char*>(base + ((int64_t)Nt + ip) * C) + sl * 128);
  }
  return __ldg(rowptr + ip);
}
__device__ __forceinline__ void prefetch_csr_ahead(int32_t rp, const int32_t* colind,
                                                   const float* vals, int sl) {
  if (MARS_SPMM_PF <= 0 || rp < 0) return;
  if (sl == 0) {
    prefetch_l2(colind + rp);
    prefetch_l2(vals + rp);
  }
}

// Row bodies shared by the two kernel shapes below.
// MODE 0: layer 1 (neg rows gather X[perm[j]]), MODE 1: PReLU on load.
// SH: row-sharded graph (layers 2-3): rows are gathered through PeerSrc.
template <int C, int MODE, bool BOTH, bool SH, int ACT, bool LONG, typename Tin, typename Tout>
__device__ __forceinline__ void fwd_row(int32_t i, int32_t long_min,
                                        const int32_t* __restrict__ rowptr,
                                        const int32_t* __restrict__ colind,
                                        const float* __restrict__ vals, const Tin* __restrict__ T,
                                        const int32_t* __restrict__ perm, float a, int32_t Nt,
                                        Tout* __restrict__ Y, float* __restrict__ rs,
                                        const PeerRows& pr, unsigned gmask, int sl) {
  using S = SpmmShape<C, Tin>;
  constexpr int V = S::V;
  const int32_t rb = rowptr[i], re = rowptr[i + 1];
  if (LONG && re - rb > long_min) return;            // long row: segments + k_spmm_long_fin
  const int32_t rp_ahead =
      SH ? -1 : prefetch_rows_ahead<Tin, C, MODE == 1 && BOTH>(i, Nt, rowptr, T, sl);
  float accp[S::NT][V], accn[S::NT][V];
#pragma unroll
  for (int q = 0; q < S::NT; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) accp[q][e] = accn[q][e] = 0.f;
  if (MODE == 0)
    row_gather<S, BOTH, 0, true, Tin>(PermSrc<Tin, C>{T}, colind, vals, perm, rb, re, gmask, sl,
                                      a, accp, accn);
  else if (SH)
    row_gather<S, BOTH, ACT, false, Tin>(PeerSrc<Tin, C>{pr}, colind, vals, perm, rb, re, gmask,
                                         sl, a, accp, accn);
  else
    row_gather<S, BOTH, ACT, false, Tin>(StackedSrc<Tin, C>{T, Nt}, colind, vals, perm, rb, re,
                                         gmask, sl, a, accp, accn);
#pragma unroll
  for (int q = 0; q < S::NT; ++q) {
    const int c = (sl + q * S::L) * V;
    StoreN<Tout, V>::store(Y + (int64_t)i * C + c, accp[q]);
    if (BOTH) StoreN<Tout, V>::store(Y + ((int64_t)Nt + i) * C + c, accn[q]);
  }
  prefetch_csr_ahead(rp_ahead, colind, vals, sl);
  if (rs) {                          // fp32 storage: row scales for the 3xFP16 GEMM
    row_scale_out<S>(accp, gmask, sl, rs + i);
    if (BOTH) row_scale_out<S>(accn, gmask, sl, rs + Nt + i);
  }
}

template <int C, bool SH, bool LONG, typename T>
__device__ __forceinline__ void bwd_row(int32_t i, int32_t long_min,
                                        const int32_t* __restrict__ rowptr,
                                        const int32_t* __restrict__ colind,
                                        const float* __restrict__ vals, const T* __restrict__ dY,
                                        const T* __restrict__ Z, float a, int32_t Nt,
                                        T* __restrict__ dZ, float* __restrict__ rs,
                                        const PeerRows& pr, unsigned gmask, int sl, float& da) {
  using S = SpmmShape<C, T>;
  constexpr int V = S::V;
  const int32_t rb = rowptr[i], re = rowptr[i + 1];
  if (LONG && re - rb > long_min) return;            // long row: segments + k_spmm_long_fin
  const int32_t rp_ahead = SH ? -1 : prefetch_rows_ahead<T, C, true>(i, Nt, rowptr, dY, sl);
  if (MARS_SPMM_PF > 0 && sl < (C * (int)sizeof(T) + 127) / 128) {   // own Z rows (epilogue)
    prefetch_l2(reinterpret_cast<const char*>(Z + (int64_t)i * C) + sl * 128);
    prefetch_l2(reinterpret_cast<const char*>(Z + ((int64_t)Nt + i) * C) + sl * 128);
  }
  float accp[S::NT][V], accn[S::NT][V];
#pragma unroll
  for (int q = 0; q < S::NT; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) accp[q][e] = accn[q][e] = 0.f;
  if (SH)
    row_gather<S, true, false, false, T, kUB<T>>(PeerSrc<T, C>{pr}, colind, vals, nullptr, rb, re, gmask,
                                         sl, a, accp, accn);
  else
    row_gather<S, true, false, false, T, kUB<T>>(StackedSrc<T, C>{dY, Nt}, colind, vals, nullptr, rb, re,
                                         gmask, sl, a, accp, accn);
  float o[2][S::NT][V];
#pragma unroll
  for (int q = 0; q < S::NT; ++q) {
    const int c = (sl + q * S::L) * V;
#pragma unroll
    for (int br = 0; br < 2; ++br) {
      const int64_t row = (int64_t)i + (br ? Nt : 0);
      float z[V];
      Vec<T>::load(Z + row * C + c, z);
#pragma unroll
      for (int e = 0; e < V; ++e) {
        const float h = br ? accn[q][e] : accp[q][e];
        o[br][q][e] = z[e] > 0.f ? h : a * h;
        da += z[e] > 0.f ? 0.f : h * z[e];
      }
      StoreN<T, V>::store(dZ + row * C + c, o[br][q]);
    }
  }
  prefetch_csr_ahead(rp_ahead, colind, vals, sl);
  if (rs) {
    row_scale_out<S>(o[0], gmask, sl, rs + i);
    row_scale_out<S>(o[1], gmask, sl, rs + Nt + i);
  }
}


// ---------------------------------------------------------------- long rows
// Rows with more than long_min entries (hubs: the weight reads of an unrolled
// RNN, fan-out 2T; ~6000 in the 1.1M-op graph) would serialise hundreds of
// gather round trips in one warp and become the kernel's tail.  The row kernels
// skip them; here one warp per segment of kLongSeg entries aggregates into fp32
// partials (same gathers, same activation), and one warp per long row sums its
// segments in order -- deterministic -- and applies the row's epilogue.  The
// sum order differs from a single ascending pass only by the segment
// bracketing (fp32 accumulation either way).
struct LongArgs {
  const int32_t* long_rows;
  const int32_t* long_seg;
  const int32_t* seg_row;
  float* part;
};

// Segment `seg` of a long row, run by the first warp-blocks of the row kernels'
// grid (so the segments overlap the ordinary rows).
template <int C, int MODE, bool BOTH, bool SH, typename Tin>
__device__ __forceinline__ void long_part_dev(int seg, const int32_t* __restrict__ rowptr,
                                              const int32_t* __restrict__ colind,
                                              const float* __restrict__ vals,
                                              const Tin* __restrict__ T,
                                              const int32_t* __restrict__ perm, float a,
                                              int32_t Nt, const LongArgs& la, const PeerRows& pr) {
  using S = SpmmShape<C, Tin>;
  constexpr int V = S::V;
  const int lane = threadIdx.x & 31;
  if (lane >= S::L) return;                          // one row group per warp
  const int sl = lane;
  const unsigned gmask = (S::L == 32) ? kFull : ((1u << S::L) - 1u);
  const int lr = la.seg_row[seg];
  const int32_t i = la.long_rows[lr];
  const int32_t e0 = rowptr[i] + (seg - la.long_seg[lr]) * kLongSeg;
  const int32_t e1 = min(rowptr[i + 1], e0 + kLongSeg);
  float accp[S::NT][V], accn[S::NT][V];
#pragma unroll
  for (int q = 0; q < S::NT; ++q)
#pragma unroll
    for (int e = 0; e < V; ++e) accp[q][e] = accn[q][e] = 0.f;
  if (MODE == 0) {
    row_gather<S, BOTH, 0, true, Tin>(PermSrc<Tin, C>{T}, colind, vals, perm, e0, e1, gmask, sl,
                                      a, accp, accn);
  } else if (MODE == 1) {
    bool done = false;
    if constexpr (std::is_same<Tin, bf16>::value) {
      if (a >= 0.f && a <= 1.f) {
        if (SH)
          row_gather<S, BOTH, 2, false, Tin>(PeerSrc<Tin, C>{pr}, colind, vals, perm, e0, e1, gmask,
                                             sl, a, accp, accn);
        else
          row_gather<S, BOTH, 2, false, Tin>(StackedSrc<Tin, C>{T, Nt}, colind, vals, perm, e0, e1,
                                             gmask, sl, a, accp, accn);
        done = true;
      }
    }
    if (!done) {
      if (SH)
        row_gather<S, BOTH, 1, false, Tin>(PeerSrc<Tin, C>{pr}, colind, vals, perm, e0, e1, gmask,
                                           sl, a, accp, accn);
      else
        row_gather<S, BOTH, 1, false, Tin>(StackedSrc<Tin, C>{T, Nt}, colind, vals, perm, e0, e1,
                                           gmask, sl, a, accp, accn);
    }
  } else {
    if (SH)
      row_gather<S, true, 0, false, Tin>(PeerSrc<Tin, C>{pr}, colind, vals, nullptr, e0, e1, gmask,
                                         sl, a, accp, accn);
    else
      row_gather<S, true, 0, false, Tin>(StackedSrc<Tin, C>{T, Nt}, colind, vals, nullptr, e0, e1,
                                         gmask, sl, a, accp, accn);
  }
  float* out = la.part + (int64_t)seg * 2 * C;
#pragma unroll
  for (int q = 0; q < S::NT; ++q) {
    const int c = (sl + q * S::L) * V;
    StoreN<float, V>::store(out + c, accp[q]);
    StoreN<float, V>::store(out + C + c, accn[q]);
  }
}

// Combine: one warp per long row, segments summed in order.  FWD: store Y (+ the
// row scales); else the backward epilogue (PReLU'(Z), dZ, dalpha partial into
// slots[lr]).
template <int C, bool FWD, bool BOTH, typename Tin, typename Tout>
__global__ void __launch_bounds__(32)
k_spmm_long_fin(const float* __restrict__ alpha, int layer, int32_t Nt, LongArgs la,
                const Tin* __restrict__ Z, Tout* __restrict__ out, float* __restrict__ rs,
                double* __restrict__ slots) {
  using S = SpmmShape<C, Tout>;
  constexpr int V = S::V;
  const int lane = threadIdx.x;
  const int lr = blockIdx.x;
  if (lane >= S::L) return;                          // one row group per warp
  const int sl = lane;
  const unsigned gmask = (S::L == 32) ? kFull : ((1u << S::L) - 1u);
  const int32_t i = la.long_rows[lr];
  float acc[2][S::NT][V];
#pragma unroll
  for (int b = 0; b < 2; ++b)
#pragma unroll
    for (int q = 0; q < S::NT; ++q)
#pragma unroll
      for (int e = 0; e < V; ++e) acc[b][q][e] = 0.f;
  for (int seg = la.long_seg[lr]; seg < la.long_seg[lr + 1]; ++seg) {
    const float* p = la.part + (int64_t)seg * 2 * C;
#pragma unroll
    for (int b = 0; b < 2; ++b)
#pragma unroll
      for (int q = 0; q < S::NT; ++q) {
        const float4* v4 = reinterpret_cast<const float4*>(p + b * C + (sl + q * S::L) * V);
#pragma unroll
        for (int e4 = 0; e4 < V / 4; ++e4) {
          const float4 x = v4[e4];
          acc[b][q][4 * e4] += x.x;
          acc[b][q][4 * e4 + 1] += x.y;
          acc[b][q][4 * e4 + 2] += x.z;
          acc[b][q][4 * e4 + 3] += x.w;
        }
      }
  }
  if constexpr (FWD) {
#pragma unroll
    for (int q = 0; q < S::NT; ++q) {
      const int c = (sl + q * S::L) * V;
      StoreN<Tout, V>::store(out + (int64_t)i * C + c, acc[0][q]);
      if (BOTH) StoreN<Tout, V>::store(out + ((int64_t)Nt + i) * C + c, acc[1][q]);
    }
    if (rs) {
      row_scale_out<S>(acc[0], gmask, sl, rs + i);
      if (BOTH) row_scale_out<S>(acc[1], gmask, sl, rs + Nt + i);
    }
  } else {
  const float a = alpha[layer];
  float da = 0.f;
  float o[2][S::NT][V];
#pragma unroll
  for (int q = 0; q < S::NT; ++q) {
    const int c = (sl + q * S::L) * V;
#pragma unroll
    for (int br = 0; br < 2; ++br) {
      const int64_t row = (int64_t)i + (br ? Nt : 0);
      float z[V];
      Vec<Tin>::load(Z + row * C + c, z);
#pragma unroll
      for (int e = 0; e < V; ++e) {
        const float h = acc[br][q][e];
        o[br][q][e] = z[e] > 0.f ? h : a * h;
        da += z[e] > 0.f ? 0.f : h * z[e];
      }
      StoreN<Tout, V>::store(out + row * C + c, o[br][q]);
    }
  }
  if (rs) {
    row_scale_out<S>(o[0], gmask, sl, rs + i);
    row_scale_out<S>(o[1], gmask, sl, rs + Nt + i);
  }
  double dd = (double)da;
#pragma unroll
  for (int off = S::L / 2; off > 0; off >>= 1) dd += __shfl_xor_sync(gmask, dd, off);
  if (sl == 0) slots[lr] = dd;
  }
}

template <int C, int MODE, bool BOTH, bool SH, typename Tin, typename Tout>
cudaError_t long_fwd(const GraphDev& g, const Tin* T, const int32_t* perm, const float* alpha,
                     int act_layer, Tout* Y, float* rs, cudaStream_t s, const PeerRows& pr) {
  if (g.nlong == 0) return cudaSuccess;
  const LongArgs la{g.long_rows, g.long_seg, g.seg_row, g.long_part};
  k_spmm_long_fin<C, true, BOTH, Tin, Tout><<<g.nlong, 32, 0, s>>>(
      alpha, 0, g.Nt, la, nullptr, Y, rs, nullptr);
  return cudaGetLastError();
}

template <int C, bool SH, typename T>
cudaError_t long_bwd(const GraphDev& g, const T* dY, const T* Z, const float* alpha, int layer,
                     T* dZ, double* slots, float* rs, cudaStream_t s, const PeerRows& pr) {
  if (g.nlong == 0) return cudaSuccess;
  const LongArgs la{g.long_rows, g.long_seg, g.seg_row, g.long_part};
  k_spmm_long_fin<C, false, true, T, T><<<g.nlong, 32, 0, s>>>(alpha, layer, g.Nt, la, Z, dZ, rs,
                                                                 slots);
  return cudaGetLastError();
}

// Rows handled by block b: one warp of RPW row groups (rows b·RPW ...).
// Measured and rejected: multi-warp blocks, a persistent grid
// walking rows i, i + NG, ..., and banded grids of one 1024-thread block per SM.
static_assert(kSpmmThreads == 32, "long-row segments and the row map assume one-warp blocks");

template <int C, int MODE, bool BOTH, bool SH, bool LONG, typename Tin, typename Tout>
__global__ void __launch_bounds__(kSpmmThreads, MARS_SPMM_MINB)
k_spmm_fwd(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
           const float* __restrict__ vals, const Tin* __restrict__ T,
           const int32_t* __restrict__ perm, const float* __restrict__ alpha, int act_layer,
           int32_t Nt, Tout* __restrict__ Y, float* __restrict__ rs,
           const __grid_constant__ PeerRows pr, const __grid_constant__ LongArgs la, int32_t nseg,
           int32_t long_min) {
  using S = SpmmShape<C, Tin>;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int sub = lane / S::L, sl = lane % S::L;
  const unsigned gmask = (S::L == 32) ? kFull : (((1u << S::L) - 1u) << (sub * S::L));
  const float a = (MODE == 1) ? alpha[act_layer] : 1.f;
  if (LONG && (int32_t)blockIdx.x < nseg) {         // long-row segments first
    long_part_dev<C, MODE, BOTH, SH, Tin>(blockIdx.x, rowptr, colind, vals, T, perm, a, Nt, la,
                                          pr);
    return;
  }
  const int32_t bid = LONG ? (int32_t)blockIdx.x - nseg : (int32_t)blockIdx.x;
  const int32_t i = bid * S::RPB + w * S::RPW + sub;
  if (i >= Nt) return;
  // bf16 storage: PReLU on packed pairs when 0 <= a <= 1 (uniform branch)
  if constexpr (MODE == 1 && std::is_same<Tin, bf16>::value) {
    if (a >= 0.f && a <= 1.f) {
      fwd_row<C, MODE, BOTH, SH, 2, LONG>(i, long_min, rowptr, colind, vals, T, perm, a, Nt, Y, rs,
                                          pr, gmask, sl);
      return;
    }
  }
  fwd_row<C, MODE, BOTH, SH, 1, LONG>(i, long_min, rowptr, colind, vals, T, perm, a, Nt, Y, rs, pr,
                                      gmask, sl);
}

template <int C, bool SH, bool LONG, typename T>
__global__ void __launch_bounds__(kSpmmThreads, MARS_SPMM_MINB)
k_spmm_bwd(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
           const float* __restrict__ vals, const T* __restrict__ dY, const T* __restrict__ Z,
           const float* __restrict__ alpha, int layer, int32_t Nt, T* __restrict__ dZ,
           double* __restrict__ slots, float* __restrict__ rs,
           const __grid_constant__ PeerRows pr, const __grid_constant__ LongArgs la, int32_t nseg,
           int32_t long_min) {
  using S = SpmmShape<C, T>;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int sub = lane / S::L, sl = lane % S::L;
  const unsigned gmask = (S::L == 32) ? kFull : (((1u << S::L) - 1u) << (sub * S::L));
  const float a = alpha[layer];
  if (LONG && (int32_t)blockIdx.x < nseg) {         // long-row segments first (no slot)
    long_part_dev<C, 2, true, SH, T>(blockIdx.x, rowptr, colind, vals, dY, nullptr, 1.f, Nt, la,
                                     pr);
    return;
  }
  const int32_t bid = LONG ? (int32_t)blockIdx.x - nseg : (int32_t)blockIdx.x;
  const int32_t i = bid * S::RPB + w * S::RPW + sub;
  float da = 0.f;
  if (i < Nt)
    bwd_row<C, SH, LONG>(i, long_min, rowptr, colind, vals, dY, Z, a, Nt, dZ, rs, pr, gmask, sl, da);
  const double wd = warp_sum((double)da);   // the block is one warp
  if (lane == 0) slots[bid] = wd;
}

// One one-warp block per RPB rows.
template <int C, typename T>
unsigned spmm_blocks(int32_t Nt) {
  return cdiv(Nt, SpmmShape<C, T>::RPB);
}

template <int C, int MODE, bool BOTH, bool SH, typename Tin, typename Tout>
cudaError_t fwd_launch(const GraphDev& g, const Tin* T, const int32_t* perm, const float* alpha,
                       int act_layer, Tout* Y, float* rs, cudaStream_t s, const PeerRows& pr) {
  const LongArgs la{g.long_rows, g.long_seg, g.seg_row, g.long_part};
  const unsigned nb = spmm_blocks<C, Tin>(g.Nt);
  const int al = act_layer < 0 ? 0 : act_layer;
  if (g.nseg > 0)   // long rows: their segments run as the grid's first blocks
    k_spmm_fwd<C, MODE, BOTH, SH, true, Tin, Tout><<<nb + g.nseg, kSpmmThreads, 0, s>>>(
        g.rowptr, g.colind, g.vals, T, perm, alpha, al, g.Nt, Y, rs, pr, la, g.nseg, g.long_min);
  else
    k_spmm_fwd<C, MODE, BOTH, SH, false, Tin, Tout><<<nb, kSpmmThreads, 0, s>>>(
            g.rowptr, g.colind, g.vals, T, perm, alpha, al, g.Nt, Y, rs, pr, la, 0, 0);
  if (cudaError_t e = cudaGetLastError()) return e;
  return long_fwd<C, MODE, BOTH, SH, Tin, Tout>(g, T, perm, alpha, act_layer, Y, rs, s, pr);
}

template <int C, typename Tin, typename Tout>
cudaError_t fwd_c(const GraphDev& g, const Tin* T, const int32_t* perm, const float* alpha,
                  int act_layer, Tout* Y, float* rs, int both, cudaStream_t s,
                  const PeerRows* peers) {
  const PeerRows none{};
  if (act_layer < 0) {
    if (peers) return cudaErrorInvalidValue;    // layer 1 reads the replicated X
    return both ? fwd_launch<C, 0, true, false, Tin, Tout>(g, T, perm, alpha, act_layer, Y, rs, s, none)
                : fwd_launch<C, 0, false, false, Tin, Tout>(g, T, perm, alpha, act_layer, Y, rs, s, none);
  }
  if constexpr ((C == 128 || C == 256) && std::is_same<Tin, Tout>::value) {
    if (peers) {
      if (!both) return cudaErrorInvalidValue;
      return fwd_launch<C, 1, true, true, Tin, Tout>(g, T, perm, alpha, act_layer, Y, rs, s, *peers);
    }
  }
  if (peers) return cudaErrorInvalidValue;
  return both ? fwd_launch<C, 1, true, false, Tin, Tout>(g, T, perm, alpha, act_layer, Y, rs, s, none)
              : fwd_launch<C, 1, false, false, Tin, Tout>(g, T, perm, alpha, act_layer, Y, rs, s, none);
}

template <typename Tin, typename Tout>
cudaError_t fwd_t(const GraphDev& g, int C, const void* T, const int32_t* perm, const float* alpha,
                  int act_layer, void* Y, float* rs, int both, cudaStream_t s, const PeerRows* pr) {
  const Tin* t = static_cast<const Tin*>(T);
  Tout* y = static_cast<Tout*>(Y);
  switch (C) {
    case 16: return fwd_c<16, Tin, Tout>(g, t, perm, alpha, act_layer, y, rs, both, s, pr);
    case 32: return fwd_c<32, Tin, Tout>(g, t, perm, alpha, act_layer, y, rs, both, s, pr);
    case 64: return fwd_c<64, Tin, Tout>(g, t, perm, alpha, act_layer, y, rs, both, s, pr);
    case 128: return fwd_c<128, Tin, Tout>(g, t, perm, alpha, act_layer, y, rs, both, s, pr);
    case 256: return fwd_c<256, Tin, Tout>(g, t, perm, alpha, act_layer, y, rs, both, s, pr);
    default: return cudaErrorInvalidValue;
  }
}

template <int C, typename T>
cudaError_t bwd_c(const GraphDev& g, const T* dY, const T* Z, const float* alpha, int layer,
                  T* dZ, double* slots, int* nslots, float* rs, cudaStream_t s,
                  const PeerRows* peers) {
  const unsigned blocks = spmm_blocks<C, T>(g.Nt);
  const unsigned threads = kSpmmThreads;
  const LongArgs la{g.long_rows, g.long_seg, g.seg_row, g.long_part};
  *nslots = (int)blocks + g.nlong;                   // long rows' dalpha after the blocks'
  if constexpr (C == 128 || C == 256) {
    if (peers) {
      if (g.nseg > 0)
        k_spmm_bwd<C, true, true, T><<<blocks + g.nseg, threads, 0, s>>>(
            g.rowptr, g.colind, g.vals, dY, Z, alpha, layer, g.Nt, dZ, slots, rs, *peers, la,
            g.nseg, g.long_min);
      else
        k_spmm_bwd<C, true, false, T><<<blocks, threads, 0, s>>>(
            g.rowptr, g.colind, g.vals, dY, Z, alpha, layer, g.Nt, dZ, slots, rs, *peers, la, 0, 0);
      if (cudaError_t e = cudaGetLastError()) return e;
      return long_bwd<C, true, T>(g, dY, Z, alpha, layer, dZ, slots + blocks, rs, s, *peers);
    }
  }
  if (peers) return cudaErrorInvalidValue;
  if (g.nseg > 0)
    k_spmm_bwd<C, false, true, T><<<blocks + g.nseg, threads, 0, s>>>(
        g.rowptr, g.colind, g.vals, dY, Z, alpha, layer, g.Nt, dZ, slots, rs, PeerRows{}, la,
        g.nseg, g.long_min);
  else
    k_spmm_bwd<C, false, false, T><<<blocks, threads, 0, s>>>(
        g.rowptr, g.colind, g.vals, dY, Z, alpha, layer, g.Nt, dZ, slots, rs, PeerRows{}, la, 0, 0);
  if (cudaError_t e = cudaGetLastError()) return e;
  return long_bwd<C, false, T>(g, dY, Z, alpha, layer, dZ, slots + blocks, rs, s, PeerRows{});
}

template <typename T>
cudaError_t bwd_t(const GraphDev& g, int C, const void* dY, const void* Z, const float* alpha,
                  int layer, void* dZ, double* slots, int* nslots, float* rs, cudaStream_t s,
                  const PeerRows* pr) {
  const T* d = static_cast<const T*>(dY);
  const T* z = static_cast<const T*>(Z);
  T* o = static_cast<T*>(dZ);
  switch (C) {
    case 32: return bwd_c<32, T>(g, d, z, alpha, layer, o, slots, nslots, rs, s, pr);
    case 64: return bwd_c<64, T>(g, d, z, alpha, layer, o, slots, nslots, rs, s, pr);
    case 128: return bwd_c<128, T>(g, d, z, alpha, layer, o, slots, nslots, rs, s, pr);
    case 256: return bwd_c<256, T>(g, d, z, alpha, layer, o, slots, nslots, rs, s, pr);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace

// act_layer < 0: layer 1 (X with the fused corruption gather through perm).
// in_bf16 / out_bf16 select the storage type of T and Y.
cudaError_t launch_spmm_fwd(const GraphDev& g, int C, const void* T, int in_bf16,
                            const int32_t* perm, const float* alpha_dev, int act_layer, void* Y,
                            int out_bf16, int both, cudaStream_t s, int* launches,
                            const PeerRows* peers, float* rs) {
  count_launch(launches, g.nlong ? 2 : 1);
  if (!in_bf16 && !out_bf16)
    return fwd_t<float, float>(g, C, T, perm, alpha_dev, act_layer, Y, rs, both, s, peers);
  if (!in_bf16 && out_bf16)
    return fwd_t<float, bf16>(g, C, T, perm, alpha_dev, act_layer, Y, nullptr, both, s, peers);
  if (in_bf16 && out_bf16)
    return fwd_t<bf16, bf16>(g, C, T, perm, alpha_dev, act_layer, Y, nullptr, both, s, peers);
  return cudaErrorInvalidValue;
}

// colperm[k] = pi[colind[k]] for the entries of the view's rows (layer 1's
// corrupted gathers read it beside colind instead of a dependent pi lookup).
__global__ void k_colperm(const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
                          const int32_t* __restrict__ perm, int64_t nnz,
                          int32_t* __restrict__ colperm) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= nnz) return;
  const int64_t k = rowptr[0] + t;
  colperm[k] = perm[colind[k]];
}

// max over the view's rows of rowptr[i+1] - rowptr[i] (into *out, zeroed here).
__global__ void k_max_degree(const int32_t* __restrict__ rowptr, int32_t Nt, int32_t* out) {
  int32_t m = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < Nt;
       i += (int64_t)gridDim.x * blockDim.x)
    m = max(m, rowptr[i + 1] - rowptr[i]);
  m = __reduce_max_sync(kFull, (unsigned)m);
  if ((threadIdx.x & 31) == 0 && m > 0) atomicMax(out, m);
}

cudaError_t launch_max_degree(const int32_t* rowptr, int32_t Nt, int32_t* out, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(out, 0, sizeof(int32_t), s);
  if (e != cudaSuccess) return e;
  k_max_degree<<<std::min<unsigned>(cdiv(Nt, 256), 1184), 256, 0, s>>>(rowptr, Nt, out);
  return cudaGetLastError();
}

cudaError_t launch_colperm(const GraphDev& g, const int32_t* perm, int32_t* colperm,
                           cudaStream_t s, int* launches) {
  count_launch(launches);
  if (g.nnz > 0)
    k_colperm<<<cdiv(g.nnz, 256), 256, 0, s>>>(g.rowptr, g.colind, perm, g.nnz, colperm);
  return cudaGetLastError();
}

// fp32 rows per block is the smallest RPB (largest block count) of any config.
// (+ 128 doubles of scratch for the two-stage reduction, head.cu)
int spmm_bwd_slots(const GraphDev& g) {
  return (int)cdiv(g.Nt, SpmmShape<256, float>::RPB) + 1 + g.nlong + 128;
}

cudaError_t launch_spmm_bwd(const GraphDev& g, int C, const void* dY, const void* Z, int bf16_,
                            const float* alpha_dev, int layer, void* dZ, double* slots,
                            int* nslots, cudaStream_t s, int* launches, const PeerRows* peers,
                            float* rs) {
  count_launch(launches, g.nlong ? 2 : 1);
  if (bf16_) return bwd_t<bf16>(g, C, dY, Z, alpha_dev, layer, dZ, slots, nslots, nullptr, s, peers);
  return bwd_t<float>(g, C, dY, Z, alpha_dev, layer, dZ, slots, nslots, rs, s, peers);
}

}  // namespace mars
