// a6 / a12 on the 5th-generation tensor cores: the dense transforms of Eq. 1
// -- Z_l = Y_l·W_l, dY_l = dZ_l·W_lᵀ, dW_l = Y_lᵀ·dZ_l -- at fp32
// accuracy with 3xTF32 (reading c18: the fp32 reference precision).
//
// Each fp32 operand is split a = hi + lo with hi = tf32_rn(a) and lo = a - hi
// (exact in fp32); D += A_hi·B_hi + A_hi·B_lo + A_lo·B_hi on tcgen05.mma
// kind::tf32 with fp32 accumulation in TMEM.  The dropped lo·lo term and the
// tf32 rounding of lo are ~2^-22 relative.
//
// Row-major activations feed both the forward (K-major A) and the weight
// gradient (MN-major A and B, reduction over rows) without transposes: only
// the TMA swizzle mode and the UMMA descriptors differ.  The lo parts are
// written by converter warps beside the TMA tile (position-preserving, so the
// swizzle needs no remapping), then fence.proxy.async hands them to the MMA.
//
// k_tc_rows  : C[M×N] = A[M×K]·Bᵀ, B [N×K] = weights pre-split (hi/lo arrays,
//              k_split_w).  K-blocks of 16 fp32 (64-byte rows, 64B swizzle)
//              so 4 (N = 256) / 6 stages fit; persistent over 128-row tiles;
//              warp 0 TMA, warp 1 MMA issuer, warps 2-3 split A, warps 4-7
//              epilogue (tcgen05.ld -> 128B-swizzled smem slabs -> TMA store);
//              double-buffered TMEM accumulators so the epilogue of tile i
//              overlaps the main loop of tile i+1.
// k_tc_dw2   : dW partials per row chunk (below), MN-major operands with the
//              128B swizzle in 32-byte atoms (layout type SW128_BASE32B).
#include <cudaTypedefs.h>

#include <cstdlib>
#include <mutex>

#include "common.cuh"
#include "internal.cuh"
#include "tc_ptx.cuh"

namespace mars {
namespace {

using namespace tc;

constexpr int kBM = 128;        // tile rows (UMMA M)
constexpr int kBK = 16;         // fp32 elements per K-block = one 64-byte swizzle row
constexpr int kThreads = 256;

// ---------------------------------------------------------------- k_tc_rows
template <int N>
struct RowsCfg {
  // 64-byte K-blocks keep a stage at 48 KB (N = 256) so four stages are in
  // flight: enough to cover TMA latency + the A split ahead of the MMAs.
  static constexpr int kStages = N > 128 ? 4 : 6;
  static constexpr int A_BYTES = kBM * kBK * 4;       // 8 KB
  static constexpr int B_BYTES = N * kBK * 4;
  static constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
  // epilogue staging: per epilogue warp two 32 x 32 fp32 slabs (128-byte swizzle)
  static constexpr int SLAB = 32 * 32 * 4;
  static constexpr int STAGING = 4 * 2 * SLAB;
  static constexpr int SMEM = kStages * STAGE + STAGING + 1024 + 256;
  static constexpr uint32_t TMEM_COLS = (2 * N) <= 32 ? 32 : (2 * N) <= 64 ? 64 : (2 * N) <= 128 ? 128
                                        : (2 * N) <= 256 ? 256 : 512;
};

template <int N>
__global__ void __launch_bounds__(kThreads, 1)
k_tc_rows(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmBhi,
          const __grid_constant__ CUtensorMap tmBlo, const __grid_constant__ CUtensorMap tmC,
          int32_t M, int32_t K) {
  using Cfg = RowsCfg<N>;
  constexpr int S = Cfg::kStages;
  extern __shared__ uint8_t smem_raw[];
  // 1024-byte alignment for the 128-byte swizzle atoms, by pointer arithmetic on
  // the shared array itself so every access stays in the shared window (LDS/STS).
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* staging = smem + S * Cfg::STAGE;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + S * Cfg::STAGE + Cfg::STAGING);
  uint64_t* full = bars;            // TMA landed            (count 1 + tx)
  uint64_t* conv = bars + S;        // A split done          (count 2 warps)
  uint64_t* empty = bars + 2 * S;   // MMA done with stage   (commit)
  uint64_t* tfull = bars + 3 * S;   // accumulator ready     (commit)   [2]
  uint64_t* tempty = bars + 3 * S + 2;  // accumulator drained (4 warps) [2]
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bars + 3 * S + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = (M + kBM - 1) / kBM;
  const int nk = K / kBK;
  auto stA = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stAlo = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES; };
  auto stB = [&](int s) { return smem + s * Cfg::STAGE + 2 * Cfg::A_BYTES; };
  auto stBlo = [&](int s) { return smem + s * Cfg::STAGE + 2 * Cfg::A_BYTES + Cfg::B_BYTES; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&conv[s], 2);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 4);
    }
    fence_mbar_init();
    tma_prefetch(&tmA);
    tma_prefetch(&tmBhi);
    tma_prefetch(&tmBlo);
    tma_prefetch(&tmC);
  }
  if (warp == 1) tmem_alloc(tslot, Cfg::TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tslot;

  if (warp == 0) {
    if (lane == 0) {                                         // ---- TMA producer
      int s = 0;
      uint32_t ph = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x)
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait(&empty[s], ph ^ 1);
          mbar_expect_tx(&full[s], Cfg::A_BYTES + 2 * Cfg::B_BYTES);
          tma_load_2d(stA(s), &tmA, kb * kBK, t * kBM, &full[s]);
          tma_load_2d(stB(s), &tmBhi, kb * kBK, 0, &full[s]);
          tma_load_2d(stBlo(s), &tmBlo, kb * kBK, 0, &full[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                         // ---- MMA issuer
      constexpr uint32_t idesc = idesc_tf32(kBM, N, false, false);
      int s = 0;
      uint32_t ph = 0;
      int acc = 0;
      uint32_t aph = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        mbar_wait(&tempty[acc], aph ^ 1);
        tc_fence_after();
        const uint32_t d = tbase + acc * N;
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait(&conv[s], ph);
          tc_fence_after();
          const uint32_t a = smem_u32(stA(s)), al = smem_u32(stAlo(s));
          const uint32_t b = smem_u32(stB(s)), bl = smem_u32(stBlo(s));
#pragma unroll
          for (int k = 0; k < kBK / 8; ++k) {
            // K-major, 64-byte swizzle: rows 64 B apart, 8-row groups 512 B (SBO)
            const uint64_t ah = sdesc_sw64(a + 32 * k, 16, 512);
            const uint64_t alo = sdesc_sw64(al + 32 * k, 16, 512);
            const uint64_t bh = sdesc_sw64(b + 32 * k, 16, 512);
            const uint64_t blo = sdesc_sw64(bl + 32 * k, 16, 512);
            mma_tf32(d, ah, bh, idesc, (kb | k) != 0);
            mma_tf32(d, ah, blo, idesc, 1);
            mma_tf32(d, alo, bh, idesc, 1);
          }
          mma_commit(&empty[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(&tfull[acc]);
        acc ^= 1;
        if (acc == 0) aph ^= 1;
      }
    }
  } else if (warp < 4) {                                     // ---- split A = hi + lo
    const int ct = threadIdx.x - 64;
    int s = 0;
    uint32_t ph = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x)
      for (int kb = 0; kb < nk; ++kb) {
        mbar_wait(&full[s], ph);
        float4* a = reinterpret_cast<float4*>(stA(s));
        float4* al = reinterpret_cast<float4*>(stAlo(s));
#pragma unroll 4
        for (int i = ct; i < Cfg::A_BYTES / 16; i += 64) {
          float4 v = a[i];
          float4 h = make_float4(to_tf32(v.x), to_tf32(v.y), to_tf32(v.z), to_tf32(v.w));
          a[i] = h;
          al[i] = make_float4(v.x - h.x, v.y - h.y, v.z - h.z, v.w - h.w);
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(&conv[s]);
        if (++s == S) { s = 0; ph ^= 1; }
      }
  } else {                                                   // ---- epilogue
    const int q = warp & 3;
    int acc = 0;
    uint32_t aph = 0;
    // TMEM -> registers -> 128B-swizzled smem slab (conflict-free row-per-lane
    // writes) -> TMA tile store: coalesced full-line writes, tail rows clipped
    uint8_t* slab0 = staging + q * 2 * Cfg::SLAB;
    int nslab = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
      mbar_wait(&tfull[acc], aph);
      tc_fence_after();
#pragma unroll 1
      for (int c0 = 0; c0 < N; c0 += 32, ++nslab) {
        uint32_t r[32];
        tmem_ld32(tbase + ((uint32_t)(q * 32) << 16) + acc * N + c0, r);
        uint8_t* slab = slab0 + (nslab & 1) * Cfg::SLAB;
        if (lane == 0) bulk_wait_read<1>();                // the store issued 2 slabs ago is done
        __syncwarp();
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          float4* dst = reinterpret_cast<float4*>(slab + lane * 128 + ((j ^ (lane & 7)) << 4));
          *dst = make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]),
                             __uint_as_float(r[4 * j + 2]), __uint_as_float(r[4 * j + 3]));
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          tma_store_2d(&tmC, slab, c0, t * kBM + q * 32);
          bulk_commit();
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[acc]);
      acc ^= 1;
      if (acc == 0) aph ^= 1;
    }
    if (lane == 0) bulk_wait<0>();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tbase, Cfg::TMEM_COLS);
  }
}

// ---------------------------------------------------------------- k_tc_dw2 tiling
constexpr int kDwBK = 16;        // rows of R per stage
constexpr int kDwStages = 4;
constexpr int kSubKb = 8;        // k-blocks per work accumulation (128 rows)

// ---------------------------------------------------------------- k_tc_dw2
// Per CTA: one chunk of rows x one CINT-wide tile of C_in.  D = dZᵀ·Y for the
// tile is accumulated by the tensor cores in a TMEM "work" accumulator for
// 128 rows (kSubKb k-blocks) at a time; epilogue warps then fold each run into
// an fp32 master held in their registers with IEEE adds, so the tensor core's
// own fp32 accumulation never runs over more than 128 rows (its truncating
// accumulation error grows with the run length; folding keeps dW at ~1e-6 of
// scale on the bench graphs).  Quadrant q = warp & 3 owns TMEM lanes 32q..,
// column half ch = (warp-4)/4 owns half of the tile's columns; the two TMEM
// work accumulators are double-buffered so the tensor cores fill one run
// while the epilogue folds the previous one.  The chunk result is written as
// an fp32 partial for the fixed-order fp64 reduce (k_dw_reduce).
// 12 warps: 0 TMA, 1 MMA issuer, 2-11 split the tf32 lo parts and fold.
template <int CINT, int HH>
struct Dw2Cfg {
  static constexpr int NH = HH / 128;                 // 128-row halves of H (UMMA M)
  static constexpr int A_BYTES = HH * kDwBK * 4;
  static constexpr int B_BYTES = CINT * kDwBK * 4;
  static constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
  static constexpr int SMEM = kDwStages * STAGE + 1024 + 256;
  static constexpr uint32_t TMEM_COLS = 2 * NH * CINT;  // 2 work buffers x NH halves of H
  static constexpr int BOX = 32 * kDwBK * 4;
  static constexpr int MCOLS = CINT / 2;              // columns per epilogue thread per half
};

template <int CINT, int HH>
__global__ void __launch_bounds__(384, 1)
k_tc_dw2(const __grid_constant__ CUtensorMap tmDZ, const __grid_constant__ CUtensorMap tmY,
         float* __restrict__ part, int32_t R, int32_t rows_per_chunk, int32_t CIN) {
  using Cfg = Dw2Cfg<CINT, HH>;
  constexpr int NH = Cfg::NH;
  constexpr int S = kDwStages;
  constexpr int MC = Cfg::MCOLS;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + S * Cfg::STAGE);
  uint64_t* full = bars;
  uint64_t* conv = bars + S;
  uint64_t* empty = bars + 2 * S;
  uint64_t* tfull = bars + 3 * S;        // [2]
  uint64_t* tempty = bars + 3 * S + 2;   // [2]
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bars + 3 * S + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntile = CIN / CINT;
  const int chunk = blockIdx.x / ntile, c_off = (blockIdx.x % ntile) * CINT;
  const int32_t r0 = chunk * rows_per_chunk;
  const int32_t r1 = min(R, r0 + rows_per_chunk);
  const int nk = r1 > r0 ? (r1 - r0 + kDwBK - 1) / kDwBK : 0;
  const int nsub = (nk + kSubKb - 1) / kSubKb;
  auto stA = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stAlo = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES; };
  auto stB = [&](int s) { return smem + s * Cfg::STAGE + 2 * Cfg::A_BYTES; };
  auto stBlo = [&](int s) { return smem + s * Cfg::STAGE + 2 * Cfg::A_BYTES + Cfg::B_BYTES; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&conv[s], 10);                               // split warps 2..11
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 8);
    }
    fence_mbar_init();
    tma_prefetch(&tmDZ);
    tma_prefetch(&tmY);
  }
  if (warp == 1) tmem_alloc(tslot, Cfg::TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tslot;

  if (warp == 0) {
    if (lane == 0) {                                         // ---- TMA producer
      int s = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < nk; ++kb) {
        mbar_wait(&empty[s], ph ^ 1);
        mbar_expect_tx(&full[s], Cfg::A_BYTES + Cfg::B_BYTES);
        const int32_t row = r0 + kb * kDwBK;
#pragma unroll
        for (int bx = 0; bx < HH / 32; ++bx)
          tma_load_2d(stA(s) + bx * Cfg::BOX, &tmDZ, bx * 32, row, &full[s]);
#pragma unroll
        for (int bx = 0; bx < CINT / 32; ++bx)
          tma_load_2d(stB(s) + bx * Cfg::BOX, &tmY, c_off + bx * 32, row, &full[s]);
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                         // ---- MMA issuer
      constexpr uint32_t idesc = idesc_tf32(kBM, CINT, true, true);
      int s = 0;
      uint32_t ph = 0;
      for (int sub = 0; sub < nsub; ++sub) {
        const int buf = sub & 1;
        mbar_wait(&tempty[buf], ((sub >> 1) & 1) ^ 1);      // previous use of this buffer folded
        tc_fence_after();
        const uint32_t twork = tbase + buf * NH * CINT;
        const int kb1 = min(nk, (sub + 1) * kSubKb);
        for (int kb = sub * kSubKb; kb < kb1; ++kb) {
          mbar_wait(&conv[s], ph);
          tc_fence_after();
          const uint32_t a = smem_u32(stA(s)), al = smem_u32(stAlo(s));
          const uint32_t b = smem_u32(stB(s)), bl = smem_u32(stBlo(s));
#pragma unroll
          for (int k = 0; k < kDwBK / 8; ++k) {
            const uint64_t bh = sdesc_sw128_b32(b + 1024 * k, Cfg::BOX, 512);
            const uint64_t blo = sdesc_sw128_b32(bl + 1024 * k, Cfg::BOX, 512);
            const uint32_t first = (kb == sub * kSubKb && k == 0) ? 0u : 1u;
#pragma unroll
            for (int h = 0; h < NH; ++h) {
              const uint64_t ah = sdesc_sw128_b32(a + h * 4 * Cfg::BOX + 1024 * k, Cfg::BOX, 512);
              const uint64_t alo = sdesc_sw128_b32(al + h * 4 * Cfg::BOX + 1024 * k, Cfg::BOX, 512);
              const uint32_t d = twork + h * CINT;
              mma_tf32(d, ah, bh, idesc, first);
              mma_tf32(d, ah, blo, idesc, 1);
              mma_tf32(d, alo, bh, idesc, 1);
            }
          }
          mma_commit(&empty[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(&tfull[buf]);
      }
    }
  } else {                         // ---- split (warps 2..11); warps 4..11 also fold
    const bool folder = warp >= 4;
    const int ct = (warp - 2) * 32 + lane;
    constexpr int NT = 10 * 32;
    const int q = warp & 3, ch = (warp - 4) >> 2;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    float master[NH][MC];
#pragma unroll
    for (int h = 0; h < NH; ++h)
#pragma unroll
      for (int j = 0; j < MC; ++j) master[h][j] = 0.f;
    int folded = 0;
    // fold work run `sub` (double-buffered in TMEM) into the register master
    auto fold = [&](int sub) {
      const int buf = sub & 1;
      mbar_wait(&tfull[buf], (sub >> 1) & 1);
      tc_fence_after();
      const uint32_t twork = tbase + buf * NH * CINT + ch * MC;
#pragma unroll
      for (int h = 0; h < NH; ++h)
#pragma unroll
        for (int c0 = 0; c0 < MC; c0 += 32) {
          uint32_t w[32];
          tmem_ld32(twork + lane_off + h * CINT + c0, w);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 32; ++j) master[h][c0 + j] += __uint_as_float(w[j]);
        }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[buf]);
    };
    int s = 0;
    uint32_t ph = 0;
    for (int kb = 0; kb < nk; ++kb) {
      mbar_wait(&full[s], ph);
      float4* a = reinterpret_cast<float4*>(stA(s));
      float4* al = reinterpret_cast<float4*>(stAlo(s));
      float4* bb = reinterpret_cast<float4*>(stB(s));
      float4* bl = reinterpret_cast<float4*>(stBlo(s));
      for (int i = ct; i < (Cfg::A_BYTES + Cfg::B_BYTES) / 16; i += NT) {
        const bool isA = i < Cfg::A_BYTES / 16;
        float4* src = isA ? a + i : bb + (i - Cfg::A_BYTES / 16);
        float4* dlo = isA ? al + i : bl + (i - Cfg::A_BYTES / 16);
        const float4 v = *src;
        const float4 hv = make_float4(to_tf32(v.x), to_tf32(v.y), to_tf32(v.z), to_tf32(v.w));
        *src = hv;
        *dlo = make_float4(v.x - hv.x, v.y - hv.y, v.z - hv.z, v.w - hv.w);
      }
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) mbar_arrive(&conv[s]);
      if (++s == S) { s = 0; ph ^= 1; }
      // mid-way through run sub+1 the MMAs of run sub are done: fold it, well
      // before run sub+2 needs its TMEM buffer back
      if (folder && (kb % kSubKb) == kSubKb / 2 && kb / kSubKb >= 1) fold(folded++);
    }
    if (folder) {
      while (folded < nsub) fold(folded++);
      float* out = part + (int64_t)chunk * HH * CIN + c_off + ch * MC;   // chunk partial
#pragma unroll
      for (int h = 0; h < NH; ++h) {
        float4* dst = reinterpret_cast<float4*>(out + (int64_t)(h * 128 + q * 32 + lane) * CIN);
#pragma unroll
        for (int j = 0; j < MC / 4; ++j)
          dst[j] = make_float4(master[h][4 * j], master[h][4 * j + 1], master[h][4 * j + 2],
                               master[h][4 * j + 3]);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tbase, Cfg::TMEM_COLS);
  }
}


// dW[c][h] = Σ_chunk part[chunk][h][c], fixed order, fp64.
__global__ void k_dw_reduce(const float* __restrict__ part, int nchunk, int CIN, int H,
                            float* __restrict__ dW) {
  dw_reduce_body(part, nchunk, CIN, H, dW);
}

// hi / lo split of the weights for the B operand: Bt = Wᵀ [H × Cin] (forward)
// and B = W [Cin × H] (dY), written once per step from the current params.
__global__ void k_split_w(const float* __restrict__ W, int CIN, int H, float* __restrict__ Bt_hi,
                          float* __restrict__ Bt_lo, float* __restrict__ B_hi,
                          float* __restrict__ B_lo) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;   // e = c * H + h
  if (e >= (int64_t)CIN * H) return;
  int c = (int)(e / H), h = (int)(e % H);
  float w = W[e];
  float hi = to_tf32(w), lo = w - hi;
  B_hi[e] = hi;
  B_lo[e] = lo;
  Bt_hi[(int64_t)h * CIN + c] = hi;
  Bt_lo[(int64_t)h * CIN + c] = lo;
}

// ---------------------------------------------------------------- host side
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;
std::once_flag g_encode_once;

bool encode_fn() {
  std::call_once(g_encode_once, [] {
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  });
  return g_encode != nullptr;
}

// Row-major fp32 [rows × cols] boxes for the UMMA operand layouts:
//  mn_major: {32 cols, box_rows}, 128-byte swizzle with 32-byte atoms (MN-major tf32)
//  else    : {kBK = 16 cols, box_rows}, 64-byte swizzle (K-major, 64-byte rows)
bool tmap_2d(CUtensorMap* m, const float* base, int64_t rows, int64_t cols, int box_rows,
             bool mn_major = false) {
  if (!encode_fn()) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
  cuuint32_t box[2] = {mn_major ? 32u : (cuuint32_t)kBK, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  return g_encode(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides,
                  box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  mn_major ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B : CU_TENSOR_MAP_SWIZZLE_64B,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Output [rows × cols] fp32 for the epilogue's TMA stores: {32, 32} boxes, 128B swizzle.
bool tmap_store(CUtensorMap* m, const float* base, int64_t rows, int64_t cols) {
  if (!encode_fn()) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
  cuuint32_t box[2] = {32, 32};
  cuuint32_t es[2] = {1, 1};
  return g_encode(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides,
                  box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

int g_sms = 0;
int num_sms() {
  if (!g_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
    if (!g_sms) g_sms = 148;
  }
  return g_sms;
}

template <int N>
cudaError_t rows_n(const float* A, const float* Bhi, const float* Blo, float* C, int64_t M, int K,
                   cudaStream_t s) {
  using Cfg = RowsCfg<N>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k_tc_rows<N>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap ta, tbh, tbl, tc;
  if (!tmap_2d(&ta, A, M, K, kBM) || !tmap_2d(&tbh, Bhi, N, K, N) ||
      !tmap_2d(&tbl, Blo, N, K, N) || !tmap_store(&tc, C, M, N))
    return cudaErrorInvalidValue;
  int ntiles = (int)((M + kBM - 1) / kBM);
  int grid = std::min(ntiles, num_sms());
  k_tc_rows<N><<<grid, kThreads, Cfg::SMEM, s>>>(ta, tbh, tbl, tc, (int32_t)M, K);
  return cudaGetLastError();
}

template <int CINT, int HH>
cudaError_t dw_c(const float* Y, const float* dZ, float* part, int nchunk, int64_t R, int rows,
                 int CIN, cudaStream_t s) {
  using Cfg = Dw2Cfg<CINT, HH>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k_tc_dw2<CINT, HH>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap tdz, ty;
  if (!tmap_2d(&tdz, dZ, R, HH, kDwBK, true) || !tmap_2d(&ty, Y, R, CIN, kDwBK, true))
    return cudaErrorInvalidValue;
  k_tc_dw2<CINT, HH><<<nchunk * (CIN / CINT), 384, Cfg::SMEM, s>>>(tdz, ty, part, (int32_t)R, rows, CIN);
  return cudaGetLastError();
}

int dw_tile(int CIN) { return CIN >= 128 ? 128 : 64; }

}  // namespace

// Shared with gemm_tc16.cu.
bool tc_tmap(CUtensorMap* m, CUtensorMapDataType dt, int elem_bytes, const void* base, int64_t rows,
             int64_t cols, int box_cols, int box_rows, CUtensorMapSwizzle swz) {
  if (!encode_fn()) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)cols * (cuuint64_t)elem_bytes};
  cuuint32_t box[2] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  return g_encode(m, dt, 2, const_cast<void*>(base), dims, strides, box, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Row-major [rows × cols] matrix viewed as 3-D {128-byte column block, rows,
// column blocks}: one box {128 B, box_rows, nblk} lands as nblk consecutive
// [box_rows × 128 B] blocks with the 128-byte swizzle -- e.g. the MN-major
// 128B-swizzle atom columns of the UMMA layout -- in a single TMA request.
bool tc_tmap_blocks(CUtensorMap* m, CUtensorMapDataType dt, int elem_bytes, const void* base,
                    int64_t rows, int64_t cols, int box_rows, int nblk) {
  if (!encode_fn()) return false;
  const cuuint64_t bc = 128 / elem_bytes;            // columns per 128-byte block
  cuuint64_t dims[3] = {bc, (cuuint64_t)rows, (cuuint64_t)(cols / bc)};
  cuuint64_t strides[2] = {(cuuint64_t)cols * elem_bytes, 128};
  cuuint32_t box[3] = {(cuuint32_t)bc, (cuuint32_t)box_rows, (cuuint32_t)nblk};
  cuuint32_t es[3] = {1, 1, 1};
  return g_encode(m, dt, 3, const_cast<void*>(base), dims, strides, box, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) ==
         CUDA_SUCCESS;
}

int tc_num_sms() { return num_sms(); }

bool tc_supported(int K_or_cin, int N_or_h) {
  return (N_or_h == 128 || N_or_h == 256) && (K_or_cin == 64 || K_or_cin == 128 || K_or_cin == 256);
}

cudaError_t tc_split_weights(const float* W, int CIN, int H, float* Bt_hi, float* Bt_lo,
                             float* B_hi, float* B_lo, cudaStream_t s, int* launches) {
  count_launch(launches);
  k_split_w<<<cdiv((int64_t)CIN * H, 256), 256, 0, s>>>(W, CIN, H, Bt_hi, Bt_lo, B_hi, B_lo);
  return cudaGetLastError();
}

// C[M×N] = A[M×K] · Bᵀ with B = (B_hi + B_lo) [N×K].
cudaError_t tc_gemm_rows(const float* A, const float* B_hi, const float* B_lo, float* C,
                         int64_t M, int N, int K, cudaStream_t s, int* launches) {
  count_launch(launches);
  if (K % kBK) return cudaErrorInvalidValue;
  switch (N) {
    case 64: return rows_n<64>(A, B_hi, B_lo, C, M, K, s);
    case 128: return rows_n<128>(A, B_hi, B_lo, C, M, K, s);
    case 256: return rows_n<256>(A, B_hi, B_lo, C, M, K, s);
    default: return cudaErrorInvalidValue;
  }
}

// Row chunks so that chunks x C_in tiles ~ one CTA per SM.
int tc_dw_chunks(int64_t R, int CIN) {
  const int ntile = std::max(1, CIN / dw_tile(CIN));
  int64_t want = std::max<int64_t>(1, num_sms() / ntile);
  int64_t maxc = std::max<int64_t>(1, R / 256);
  return (int)std::min(want, maxc);
}

size_t tc_dw_partial_floats(int64_t R, int CIN) {
  return (size_t)tc_dw_chunks(R, CIN) * 256 * CIN;
}

// dW [CIN × H] = Yᵀ dZ with Y [R × CIN], dZ [R × H], H in {128, 256}.
cudaError_t tc_gemm_dw(const float* Y, const float* dZ, float* dW, int64_t R, int CIN, int H,
                       float* part, cudaStream_t s, int* launches) {
  count_launch(launches, 2);
  int nchunk = tc_dw_chunks(R, CIN);
  int rows = (int)((R + nchunk - 1) / nchunk);
  rows = (rows + kDwBK - 1) / kDwBK * kDwBK;
  nchunk = (int)((R + rows - 1) / rows);
  cudaError_t e;
  if (H != 128 && H != 256) return cudaErrorInvalidValue;
  switch (CIN) {
    case 64: e = H == 256 ? dw_c<64, 256>(Y, dZ, part, nchunk, R, rows, CIN, s)
                          : dw_c<64, 128>(Y, dZ, part, nchunk, R, rows, CIN, s); break;
    case 128:
    case 256: e = H == 256 ? dw_c<128, 256>(Y, dZ, part, nchunk, R, rows, CIN, s)
                           : dw_c<128, 128>(Y, dZ, part, nchunk, R, rows, CIN, s); break;
    default: return cudaErrorInvalidValue;
  }
  if (e != cudaSuccess) return e;
  k_dw_reduce<<<cdiv((int64_t)H * CIN, 32), 256, 0, s>>>(part, nchunk, CIN, H, dW);
  return cudaGetLastError();
}

}  // namespace mars
