// a6 / a12, fp32 path: the row GEMMs of Eq. 1 -- Z_l = Y_l·W_l and
// dY_l = dZ_l·W_lᵀ -- at fp32 accuracy on the kind::f16 tensor cores, which
// run at twice the kind::tf32 rate (reading c18: fp32 reference precision).
//
// 3xFP16 with exact power-of-two scaling.  Every row r of A is scaled by
// s_r = 2^(14 - e_r) (e_r = exponent of max_k |A[r][k]|) and the weights by
// one per-tensor t = 2^(14 - e_W), so every scaled value lies below 2^15 (fp16
// max 65504) and a value 2^-28 of its row maximum is still a normal fp16.
// Then x = hi + lo with hi = fp16_rn(x), lo = fp16_rn(x - hi) (x - hi exact in
// fp32), and D += A_hi·B_hi + A_hi·B_lo + A_lo·B_hi in fp32 TMEM, C = D / (s_r t)
// (exact).  hi and lo carry 11 significant bits each, so the dropped lo·lo
// term and the rounding of lo are ~2^-22 relative to the row's scale
// (the same budget as a 3xTF32 split, at twice its MMA rate).
//
// k_tc3h_rows: persistent over 128-row tiles.  Warp 0 TMA (fp32 A K-blocks of
// 32 columns, 128-byte swizzle; pre-split fp16 B hi/lo, 64-byte swizzle),
// warp 1 MMA issuer, warps 2-5 convert A in place (fp32 tile -> fp16 hi and lo
// tiles in the UMMA 64-byte-swizzle K-major layout) and compute the next
// tile's row maxima from global memory while doing so, warps 6-9 epilogue
// (tcgen05.ld, per-row unscale, 128B-swizzled smem slabs, TMA store).
#include <cuda_fp16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "internal.cuh"
#include "tc_ptx.cuh"

namespace mars {
namespace {

using namespace tc;

constexpr int kBM = 128;       // tile rows (UMMA M)
constexpr int kBK = 32;        // K elements per stage: 128 B of fp32 staging, 64 B of fp16
constexpr int kThreads = 320;  // 10 warps
constexpr int kScaleSlots = 8; // per-tile row-scale slots in flight (converters run ahead)

// Instruction descriptor, kind::f16 with fp16 A, B and fp32 D, K-major both.
__host__ __device__ constexpr uint32_t idesc_f16(int M, int N) {
  return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

template <int N>
struct H3Cfg {
#ifndef MARS_H3_STAGES256
#define MARS_H3_STAGES256 4
#endif
  // N = 256: 4 stages of 48 KB fit with one epilogue slab per warp; else 5
  static constexpr int kStages = N > 128 ? MARS_H3_STAGES256 : 5;
  static constexpr int NSLAB = (N > 128 && kStages > 3) ? 1 : 2;
  static constexpr int A_BYTES = kBM * kBK * 4;      // fp32 staging, later hi | lo (8 KB each)
  static constexpr int B_BYTES = N * kBK * 2;        // fp16
  static constexpr int STAGE = A_BYTES + 2 * B_BYTES;
  static constexpr int SLAB = 32 * 32 * 4;
  static constexpr int STAGING = 4 * NSLAB * SLAB;
  static constexpr int SCALES = kScaleSlots * kBM * 4;       // 1 / s_r
  static constexpr int SMEM = kStages * STAGE + STAGING + SCALES + 1024 + 256;
  static constexpr uint32_t TMEM_COLS = (2 * N) <= 128 ? 128 : (2 * N) <= 256 ? 256 : 512;
};

__device__ __forceinline__ void conv_bar() {   // the 4 converter warps
  asm volatile("bar.sync 1, 128;" ::: "memory");
}

// x = hi + lo for 8 scaled values: hi = fp16_rn(x) (packed in pairs), read
// back as fp32 to form lo = x - hi exactly, lo rounded to fp16.
__device__ __forceinline__ void split_h8(const float (&x)[8], uint4& hi, uint4& lo) {
  uint32_t hw[4], lw[4];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const __half2 h2 = __floats2half2_rn(x[2 * k], x[2 * k + 1]);
    const float2 hf = __half22float2(h2);
    const __half2 l2 = __floats2half2_rn(x[2 * k] - hf.x, x[2 * k + 1] - hf.y);
    hw[k] = *reinterpret_cast<const uint32_t*>(&h2);
    lw[k] = *reinterpret_cast<const uint32_t*>(&l2);
  }
  hi = make_uint4(hw[0], hw[1], hw[2], hw[3]);
  lo = make_uint4(lw[0], lw[1], lw[2], lw[3]);
}

template <int N>
__global__ void __launch_bounds__(kThreads, 1)
k_tc3h_rows(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmBhi,
            const __grid_constant__ CUtensorMap tmBlo, const __grid_constant__ CUtensorMap tmC,
            const float* __restrict__ rs, const float* __restrict__ inv_tb, int32_t M, int32_t K) {
  using Cfg = H3Cfg<N>;
  constexpr int S = Cfg::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* staging = smem + S * Cfg::STAGE;
  float* rscale = reinterpret_cast<float*>(staging + Cfg::STAGING);     // [slots][128]: 1 / s_r
  uint64_t* bars = reinterpret_cast<uint64_t*>(staging + Cfg::STAGING + Cfg::SCALES);
  uint64_t* full = bars;                 // TMA landed              (1 + tx)
  uint64_t* conv = bars + S;             // A converted             (4 warps)
  uint64_t* empty = bars + 2 * S;        // MMA done with the stage (commit)
  uint64_t* tfull = bars + 3 * S;        // accumulator ready       [2]
  uint64_t* tempty = bars + 3 * S + 2;   // accumulator drained     [2] (4 warps)
  uint64_t* sready = bars + 3 * S + 4;   // 1 / s_r of a tile published [slots] (4 converter warps)
  uint64_t* sfree = sready + kScaleSlots;//   ... read by the epilogue     [slots] (4 epilogue warps)
  uint32_t* tslot = reinterpret_cast<uint32_t*>(sfree + kScaleSlots);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = (M + kBM - 1) / kBM;
  const int nk = (K + kBK - 1) / kBK;    // K = 16: one block, TMA zero-fills the rest
  auto stA = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stB = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES; };
  auto stBlo = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES + Cfg::B_BYTES; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&conv[s], 4);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 4);
    }
    for (int b = 0; b < kScaleSlots; ++b) {
      mbar_init(&sready[b], 4);
      mbar_init(&sfree[b], 4);
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
      constexpr uint32_t idesc = idesc_f16(kBM, N);
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
          const uint32_t a = smem_u32(stA(s)), al = a + kBM * kBK * 2;
          const uint32_t b = smem_u32(stB(s)), bl = smem_u32(stBlo(s));
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k) {
            // K-major, 64-byte swizzle: rows 64 B apart, 8-row groups 512 B (SBO)
            const uint64_t ah = sdesc_sw64(a + 32 * k, 16, 512);
            const uint64_t alo = sdesc_sw64(al + 32 * k, 16, 512);
            const uint64_t bh = sdesc_sw64(b + 32 * k, 16, 512);
            const uint64_t blo = sdesc_sw64(bl + 32 * k, 16, 512);
            mma_f16(d, ah, bh, idesc, (kb | k) != 0);
            mma_f16(d, ah, blo, idesc, 1);
            mma_f16(d, alo, bh, idesc, 1);
          }
          mma_commit(&empty[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(&tfull[acc]);
        acc ^= 1;
        if (acc == 0) aph ^= 1;
      }
    }
  } else if (warp < 6) {                                     // ---- convert A (row ct per thread)
    const int ct = threadIdx.x - 64;
    int s = 0;
    uint32_t ph = 0;
    int it = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
      const int slot = it % kScaleSlots;
      const int64_t row = (int64_t)t * kBM + ct;
      const float scale = row < M ? __ldg(rs + row) : 1.f;  // s_r (power of two) of row ct
      if (it >= kScaleSlots) mbar_wait(&sfree[slot], ((it / kScaleSlots) - 1) & 1);
      rscale[slot * kBM + ct] = 1.f / scale;
      __syncwarp();
      if (lane == 0) mbar_arrive(&sready[slot]);
      for (int kb = 0; kb < nk; ++kb) {
        mbar_wait(&full[s], ph);
        uint8_t* base = stA(s);
        // read row ct of the fp32 staging tile (128-byte swizzle: chunk j of row r
        // at r*128 + ((j ^ (r & 7)) << 4)) -> scaled hi / lo halves
        uint4 hi[kBK / 8], lo[kBK / 8];
#pragma unroll
        for (int c = 0; c < kBK / 8; ++c) {
          float x[8];
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int j = 2 * c + h;
            const float4 v =
                *reinterpret_cast<const float4*>(base + ct * 128 + ((j ^ (ct & 7)) << 4));
            x[4 * h] = v.x * scale;
            x[4 * h + 1] = v.y * scale;
            x[4 * h + 2] = v.z * scale;
            x[4 * h + 3] = v.w * scale;
          }
          split_h8(x, hi[c], lo[c]);
        }
        conv_bar();                  // every converter has read its row before any write
        // hi tile [0, 8 KB), lo tile [8 KB, 16 KB): 64-byte rows, 16-byte chunk c of
        // row r at r*64 + ((c ^ ((r >> 1) & 3)) << 4)
#pragma unroll
        for (int c = 0; c < kBK / 8; ++c) {
          const int off = ct * 64 + ((c ^ ((ct >> 1) & 3)) << 4);
          *reinterpret_cast<uint4*>(base + off) = hi[c];
          *reinterpret_cast<uint4*>(base + kBM * kBK * 2 + off) = lo[c];
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(&conv[s]);
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp < 10) {                                    // ---- epilogue
    const int q = warp & 3;
    int acc = 0;
    uint32_t aph = 0;
    const float itb = *inv_tb;
    uint8_t* slab0 = staging + q * Cfg::NSLAB * Cfg::SLAB;
    int nslab = 0;
    int it = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
      const int slot = it % kScaleSlots;
      mbar_wait(&sready[slot], (it / kScaleSlots) & 1);
      const float f = rscale[slot * kBM + q * 32 + lane] * itb;
      __syncwarp();
      if (lane == 0) mbar_arrive(&sfree[slot]);
      mbar_wait(&tfull[acc], aph);
      tc_fence_after();
#pragma unroll 1
      for (int c0 = 0; c0 < N; c0 += 32, ++nslab) {
        uint32_t r[32];
        tmem_ld32(tbase + ((uint32_t)(q * 32) << 16) + acc * N + c0, r);
        uint8_t* slab = slab0 + (Cfg::NSLAB == 2 ? (nslab & 1) * Cfg::SLAB : 0);
        if (lane == 0) {   // the store that last read this slab is done
          if (Cfg::NSLAB == 2) bulk_wait_read<1>();
          else bulk_wait_read<0>();
        }
        __syncwarp();
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          float4* dst = reinterpret_cast<float4*>(slab + lane * 128 + ((j ^ (lane & 7)) << 4));
          *dst = make_float4(__uint_as_float(r[4 * j]) * f, __uint_as_float(r[4 * j + 1]) * f,
                             __uint_as_float(r[4 * j + 2]) * f, __uint_as_float(r[4 * j + 3]) * f);
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

// ---------------------------------------------------------------- k_tc3h_rows_pair
// Z = A·Bᵀ for N = 256 on CTA pairs (cta_group::2): each CTA of a pair owns
// one 128-row tile of A and HALF of the weight operand (N rows 128r ..
// 128r + 127), so per K-block a CTA loads 16 KB of A and 16 KB of B hi / lo
// instead of 16 + 32 KB, and every pair MMA (M = 256: both CTAs' A tiles;
// N = 256: both CTAs' B halves) reads each B half from the CTA that holds it
// -- a third less shared-memory traffic per row tile than k_tc3h_rows.
// Roles as in k_tc3h_rows (warp 0 TMA, warp 1 MMA -- the even CTA issues --
// warps 2-5 convert their own A rows in place, warps 6-9 drain their own
// TMEM rows); the odd CTA's converters and epilogue warps meet at a named
// barrier and one thread arrives on the even CTA's conv / tempty barrier.
#ifndef MARS_ROWS_PAIR
#define MARS_ROWS_PAIR 1
#endif
#ifndef MARS_RP_STAGES
#define MARS_RP_STAGES 6
#endif
#ifndef MARS_RP_SLABS
#define MARS_RP_SLABS 1
#endif
#ifndef MARS_RP_NARROW
#define MARS_RP_NARROW 1      // K <= 64: 4 stages, 4 epilogue slabs per warp (output-bound launches)
#endif
template <int SS, int NS>
struct H3RowsPairCfg {
  static constexpr int N = 256, NHALF = 128;
  static constexpr int A_BYTES = kBM * kBK * 4;       // fp32 staging, later hi | lo (8 KB each)
  static constexpr int B_BYTES = NHALF * kBK * 2;     // one fp16 half tile (8 KB)
  static constexpr int STAGE = A_BYTES + 2 * B_BYTES; // 32 KB
  static constexpr int SLAB = 32 * 32 * 4;
  static constexpr int S = SS;
  static constexpr int NSLAB = NS;
  static constexpr int STAGING = 4 * NSLAB * SLAB;    // slabs per epilogue warp
  static constexpr int SCALES = kScaleSlots * kBM * 4;
  static constexpr int SMEM = SS * STAGE + STAGING + SCALES + 1024 + 512;
  static constexpr uint32_t TMEM_COLS = 512;
};

__device__ __forceinline__ void rp_epi_bar() {     // the 4 epilogue warps
  asm volatile("bar.sync 2, 128;" ::: "memory");
}

template <class Cfg>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
k_tc3h_rows_pair(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmBhi,
                 const __grid_constant__ CUtensorMap tmBlo, const __grid_constant__ CUtensorMap tmC,
                 const float* __restrict__ rs, const float* __restrict__ inv_tb, int32_t M,
                 int32_t K) {
  constexpr int S = Cfg::S, N = Cfg::N;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* staging = smem + S * Cfg::STAGE;
  float* rscale = reinterpret_cast<float*>(staging + Cfg::STAGING);
  uint64_t* bars = reinterpret_cast<uint64_t*>(staging + Cfg::STAGING + Cfg::SCALES);
  uint64_t* full = bars;                 // TMA landed (this CTA)
  uint64_t* conv = bars + S;             // even CTA: both CTAs' converters (4 + 1)
  uint64_t* empty = bars + 2 * S;        // pair MMAs done with the stage (multicast commit)
  uint64_t* tfull = bars + 3 * S;        // [2] accumulator ready (multicast commit)
  uint64_t* tempty = bars + 3 * S + 2;   // [2] even CTA: both CTAs' epilogues (4 + 1)
  uint64_t* sready = bars + 3 * S + 4;   // [slots] local
  uint64_t* sfree = sready + kScaleSlots;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(sfree + kScaleSlots);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_rank();
  const int ntiles = (M + kBM - 1) / kBM;
  const int npair = (ntiles + 1) / 2;
  const int nclu = gridDim.x / 2, clu = blockIdx.x / 2;
  const int nk = (K + kBK - 1) / kBK;
  auto stA = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stB = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES; };
  auto stBlo = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES + Cfg::B_BYTES; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&conv[s], 5);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 5);
    }
    for (int b = 0; b < kScaleSlots; ++b) {
      mbar_init(&sready[b], 4);
      mbar_init(&sfree[b], 4);
    }
    fence_mbar_init();
    tma_prefetch(&tmA);
    tma_prefetch(&tmBhi);
    tma_prefetch(&tmBlo);
    tma_prefetch(&tmC);
  }
  if (warp == 1) tmem_alloc_pair(tslot, Cfg::TMEM_COLS);
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tbase = *tslot;

  if (warp == 0) {
    if (lane == 0) {                                         // ---- TMA producer (both CTAs)
      int s = 0;
      uint32_t ph = 0;
      for (int pt = clu; pt < npair; pt += nclu) {
        const int t = 2 * pt + (int)rank;
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait(&empty[s], ph ^ 1);
          mbar_expect_tx(&full[s], Cfg::A_BYTES + 2 * Cfg::B_BYTES);
          tma_load_2d(stA(s), &tmA, kb * kBK, t * kBM, &full[s]);
          tma_load_2d(stB(s), &tmBhi, kb * kBK, (int)rank * Cfg::NHALF, &full[s]);
          tma_load_2d(stBlo(s), &tmBlo, kb * kBK, (int)rank * Cfg::NHALF, &full[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {                            // ---- pair MMA issuer
      constexpr uint32_t idesc = idesc_f16(2 * kBM, N);
      int s = 0;
      uint32_t ph = 0;
      int acc = 0;
      uint32_t aph = 0;
      for (int pt = clu; pt < npair; pt += nclu) {
        mbar_wait_cluster(&tempty[acc], aph ^ 1);
        tc_fence_after();
        const uint32_t d = tbase + acc * N;
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait_cluster(&conv[s], ph);
          tc_fence_after();
          const uint32_t a = smem_u32(stA(s)), al = a + kBM * kBK * 2;
          const uint32_t b = smem_u32(stB(s)), bl = smem_u32(stBlo(s));
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k) {
            const uint64_t ah = sdesc_sw64(a + 32 * k, 16, 512);
            const uint64_t alo = sdesc_sw64(al + 32 * k, 16, 512);
            const uint64_t bh = sdesc_sw64(b + 32 * k, 16, 512);
            const uint64_t blo = sdesc_sw64(bl + 32 * k, 16, 512);
            mma_f16_pair(d, ah, bh, idesc, (kb | k) != 0);
            mma_f16_pair(d, ah, blo, idesc, 1);
            mma_f16_pair(d, alo, bh, idesc, 1);
          }
          mma_commit_pair(&empty[s], 0x3);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit_pair(&tfull[acc], 0x3);
        acc ^= 1;
        if (acc == 0) aph ^= 1;
      }
    }
  } else if (warp < 6) {                                     // ---- convert own A rows
    const int ct = threadIdx.x - 64;
    const uint32_t conv0 = mapa_u32(conv, 0);
    int s = 0;
    uint32_t ph = 0;
    int it = 0;
    for (int pt = clu; pt < npair; pt += nclu, ++it) {
      const int t = 2 * pt + (int)rank;
      const int slot = it % kScaleSlots;
      const int64_t row = (int64_t)t * kBM + ct;
      const float scale = row < M ? __ldg(rs + row) : 1.f;
      if (it >= kScaleSlots) mbar_wait(&sfree[slot], ((it / kScaleSlots) - 1) & 1);
      rscale[slot * kBM + ct] = 1.f / scale;
      __syncwarp();
      if (lane == 0) mbar_arrive(&sready[slot]);
      for (int kb = 0; kb < nk; ++kb) {
        mbar_wait(&full[s], ph);
        uint8_t* base = stA(s);
        uint4 hi[kBK / 8], lo[kBK / 8];
#pragma unroll
        for (int c = 0; c < kBK / 8; ++c) {
          float x[8];
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int j = 2 * c + h;
            const float4 v =
                *reinterpret_cast<const float4*>(base + ct * 128 + ((j ^ (ct & 7)) << 4));
            x[4 * h] = v.x * scale;
            x[4 * h + 1] = v.y * scale;
            x[4 * h + 2] = v.z * scale;
            x[4 * h + 3] = v.w * scale;
          }
          split_h8(x, hi[c], lo[c]);
        }
        conv_bar();                  // every converter has read its row before any write
#pragma unroll
        for (int c = 0; c < kBK / 8; ++c) {
          const int off = ct * 64 + ((c ^ ((ct >> 1) & 3)) << 4);
          *reinterpret_cast<uint4*>(base + off) = hi[c];
          *reinterpret_cast<uint4*>(base + kBM * kBK * 2 + off) = lo[c];
        }
        fence_proxy_async_smem();
        if (rank == 0) {
          __syncwarp();
          if (lane == 0) mbar_arrive(&conv[s]);
        } else {
          conv_bar();                                        // the 4 converter warps
          if (threadIdx.x == 64) mbar_arrive_cluster(conv0 + s * 8);
        }
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp < 10) {                                    // ---- epilogue (own rows)
    const int q = warp & 3;
    const uint32_t tempty0 = mapa_u32(tempty, 0);
    int acc = 0;
    uint32_t aph = 0;
    const float itb = *inv_tb;
    uint8_t* slab0 = staging + q * Cfg::NSLAB * Cfg::SLAB;
    int nslab = 0;
    int it = 0;
    for (int pt = clu; pt < npair; pt += nclu, ++it) {
      const int t = 2 * pt + (int)rank;
      const int slot = it % kScaleSlots;
      mbar_wait(&sready[slot], (it / kScaleSlots) & 1);
      const float f = rscale[slot * kBM + q * 32 + lane] * itb;
      __syncwarp();
      if (lane == 0) mbar_arrive(&sfree[slot]);
      mbar_wait(&tfull[acc], aph);
      tc_fence_after();
#pragma unroll 1
      for (int c0 = 0; c0 < N; c0 += 32, ++nslab) {
        uint32_t r[32];
        tmem_ld32(tbase + ((uint32_t)(q * 32) << 16) + acc * N + c0, r);
        uint8_t* slab = slab0 + (nslab % Cfg::NSLAB) * Cfg::SLAB;
        if (lane == 0) bulk_wait_read<Cfg::NSLAB - 1>();   // the store that last read this slab is done
        __syncwarp();
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          float4* dst = reinterpret_cast<float4*>(slab + lane * 128 + ((j ^ (lane & 7)) << 4));
          *dst = make_float4(__uint_as_float(r[4 * j]) * f, __uint_as_float(r[4 * j + 1]) * f,
                             __uint_as_float(r[4 * j + 2]) * f, __uint_as_float(r[4 * j + 3]) * f);
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          tma_store_2d(&tmC, slab, c0, t * kBM + q * 32);
          bulk_commit();
        }
      }
      tc_fence_before();
      if (rank == 0) {
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
      } else {
        rp_epi_bar();
        if (threadIdx.x == 6 * 32) mbar_arrive_cluster(tempty0 + acc * 8);
      }
      acc ^= 1;
      if (acc == 0) aph ^= 1;
    }
    if (lane == 0) bulk_wait<0>();
  }
  tc_fence_before();
  cluster_sync();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc_pair(tbase, Cfg::TMEM_COLS);
  }
}

using RpWide = H3RowsPairCfg<MARS_RP_STAGES, MARS_RP_SLABS>;
using RpNarrow = H3RowsPairCfg<4, 4>;

template <class Cfg>
int rows_pair_clusters_t() {
  static int n = 0;
  if (!n) {
    cudaFuncSetAttribute(k_tc3h_rows_pair<Cfg>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         Cfg::SMEM);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2 * 74, 1, 1);
    cfg.blockDim = dim3(kThreads, 1, 1);
    cfg.dynamicSmemBytes = Cfg::SMEM;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int c = 0;
    if (cudaOccupancyMaxActiveClusters(&c, k_tc3h_rows_pair<Cfg>, &cfg) != cudaSuccess || c < 1) {
      cudaGetLastError();
      c = tc_num_sms() / 2;
    }
    n = c;
  }
  return n;
}

template <class Cfg>
cudaError_t rows3h_pair_t(const float* A, const float* rs, const __half* Bhi, const __half* Blo,
                          const float* inv_tb, float* C, int64_t M, int K, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k_tc3h_rows_pair<Cfg>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap ta, tbh, tbl, tc;
  if (!tc_tmap(&ta, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, A, M, K, kBK, kBM,
               CU_TENSOR_MAP_SWIZZLE_128B) ||
      !tc_tmap(&tbh, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, Bhi, Cfg::N, K, kBK, Cfg::NHALF,
               CU_TENSOR_MAP_SWIZZLE_64B) ||
      !tc_tmap(&tbl, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, Blo, Cfg::N, K, kBK, Cfg::NHALF,
               CU_TENSOR_MAP_SWIZZLE_64B) ||
      !tc_tmap(&tc, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, C, M, Cfg::N, 32, 32,
               CU_TENSOR_MAP_SWIZZLE_128B))
    return cudaErrorInvalidValue;
  const int ntiles = (int)((M + kBM - 1) / kBM);
  const int npair = (ntiles + 1) / 2;
  const int nclu = std::min(npair, rows_pair_clusters_t<Cfg>());
  k_tc3h_rows_pair<Cfg><<<2 * nclu, kThreads, Cfg::SMEM, s>>>(ta, tbh, tbl, tc, rs, inv_tb,
                                                               (int32_t)M, K);
  return cudaGetLastError();
}

// K <= 64 launches write four times the bytes they read: the epilogue's slab
// round trips bound them, so they run with 4 slabs per epilogue warp.
cudaError_t rows3h_pair(const float* A, const float* rs, const __half* Bhi, const __half* Blo,
                        const float* inv_tb, float* C, int64_t M, int K, cudaStream_t s) {
  if (MARS_RP_NARROW && K <= 64) return rows3h_pair_t<RpNarrow>(A, rs, Bhi, Blo, inv_tb, C, M, K, s);
  return rows3h_pair_t<RpWide>(A, rs, Bhi, Blo, inv_tb, C, M, K, s);
}

// ---------------------------------------------------------------- row scales
// rs[r] = 2^(14 - e_r) of max_k |A[r][k]| (warp per row), for A not produced by
// a kernel that writes its own row scales.
__global__ void k_row_scale(const float* __restrict__ A, int64_t M, int K, float* __restrict__ rs) {
  const int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= M) return;
  float m = 0.f;
  for (int k = lane; k < K; k += 32) m = fmaxf(m, fabsf(A[r * K + k]));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(kFull, m, o));
  if (lane == 0) rs[r] = pow2_scale(m);
}

// ---------------------------------------------------------------- weights
// max |W| -> 1 / t (one block; W has at most 256 x 256 entries)
__global__ void __launch_bounds__(1024) k_wscale(const float* __restrict__ W, int n,
                                                 float* __restrict__ wsc) {
  __shared__ float sh[32];
  float m = 0.f;
  for (int e = threadIdx.x; e < n; e += 1024) m = fmaxf(m, fabsf(W[e]));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(kFull, m, o));
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = m;
  __syncthreads();
  if (threadIdx.x < 32) {
    m = sh[threadIdx.x];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(kFull, m, o));
    if (threadIdx.x == 0) {
      const float t = pow2_scale(m);
      wsc[0] = t;
      wsc[1] = 1.f / t;
    }
  }
}

// Scaled fp16 hi / lo of Bt = Wᵀ [H × Cin] (forward) and B = W [Cin × H] (dY).
__global__ void k_split_w3h(const float* __restrict__ W, int CIN, int H,
                            const float* __restrict__ wsc, __half* __restrict__ Bt_hi,
                            __half* __restrict__ Bt_lo, __half* __restrict__ B_hi,
                            __half* __restrict__ B_lo) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;   // e = c * H + h
  if (e >= (int64_t)CIN * H) return;
  const int c = (int)(e / H), h = (int)(e % H);
  const float x = W[e] * wsc[0];
  const __half hi = __float2half_rn(x);
  const __half lo = __float2half_rn(x - __half2float(hi));
  B_hi[e] = hi;
  B_lo[e] = lo;
  Bt_hi[(int64_t)h * CIN + c] = hi;
  Bt_lo[(int64_t)h * CIN + c] = lo;
}

// All layers' weights in one launch (grid: kSplitBlocks x layers): every block
// forms its layer's max |W| itself (at most 256 KB, read from L2), block 0
// publishes {t, 1/t}, and each block splits its share of the entries --
// the same values as k_wscale + k_split_w3h per layer, in one graph node
// instead of six.
constexpr int kSplitBlocks = 8;
__global__ void __launch_bounds__(1024) k_split_w3h_all(const W3Split a) {
  __shared__ float sh[32];
  __shared__ float ts;
  const int l = blockIdx.y;
  const float* __restrict__ W = a.W[l];
  const int CIN = a.cin[l], H = a.H, n = CIN * H;
  float m = 0.f;
  for (int e = threadIdx.x; e < n; e += 1024) m = fmaxf(m, fabsf(W[e]));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(kFull, m, o));
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = m;
  __syncthreads();
  if (threadIdx.x < 32) {
    m = sh[threadIdx.x];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(kFull, m, o));
    if (threadIdx.x == 0) {
      const float t = pow2_scale(m);
      ts = t;
      if (blockIdx.x == 0) {
        a.wsc[l][0] = t;
        a.wsc[l][1] = 1.f / t;
      }
    }
  }
  __syncthreads();
  const float t = ts;
  for (int e = blockIdx.x * 1024 + threadIdx.x; e < n; e += kSplitBlocks * 1024) {
    const int c = e / H, h = e % H;
    const float x = W[e] * t;
    const __half hi = __float2half_rn(x);
    const __half lo = __float2half_rn(x - __half2float(hi));
    static_cast<__half*>(a.b_hi[l])[e] = hi;
    static_cast<__half*>(a.b_lo[l])[e] = lo;
    static_cast<__half*>(a.bt_hi[l])[(int64_t)h * CIN + c] = hi;
    static_cast<__half*>(a.bt_lo[l])[(int64_t)h * CIN + c] = lo;
  }
}

template <int N>
// N = the tile width (64, 128, 256); n = the actual output width (n <= N: the
// weight rows beyond n are zero-filled by TMA and the store is clipped to n).
cudaError_t rows3h_n(const float* A, const float* rs, const __half* Bhi, const __half* Blo,
                     const float* inv_tb, float* C, int64_t M, int K, int n, cudaStream_t s) {
  using Cfg = H3Cfg<N>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k_tc3h_rows<N>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap ta, tbh, tbl, tc;
  if (!tc_tmap(&ta, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, A, M, K, kBK, kBM,
               CU_TENSOR_MAP_SWIZZLE_128B) ||
      !tc_tmap(&tbh, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, Bhi, n, K, kBK, N,
               CU_TENSOR_MAP_SWIZZLE_64B) ||
      !tc_tmap(&tbl, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, Blo, n, K, kBK, N,
               CU_TENSOR_MAP_SWIZZLE_64B) ||
      !tc_tmap(&tc, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, C, M, n, 32, 32,
               CU_TENSOR_MAP_SWIZZLE_128B))
    return cudaErrorInvalidValue;
  const int ntiles = (int)((M + kBM - 1) / kBM);
  const int grid = std::min(ntiles, tc_num_sms());
  k_tc3h_rows<N><<<grid, kThreads, Cfg::SMEM, s>>>(ta, tbh, tbl, tc, rs, inv_tb, (int32_t)M, K);
  return cudaGetLastError();
}

// ---------------------------------------------------------------- k_tc3h_dw
// dW partials per row chunk, 3xFP16: D[h][c] += Σ_r dZ[r][h]·Y[r][c] with both
// operands MN-major (row-major activations, reduction over rows, no
// transpose).  Scaling: one power of two per CTA and operand, the smallest row
// scale of its chunk (min_r rs[r], rs written by the producing kernels), so
// the chunk's largest |value| maps into [2^14, 2^15); the partial is unscaled
// (exactly) before it is written.  TMA brings fp32 row tiles (one 3-D box of
// 16 rows x all 32-column 128B-swizzled blocks per operand and stage);
// converter warps 2..11 write scaled fp16
// hi / lo tiles in the MN-major 128B-swizzle layout (64-column atoms, 8-row
// groups); warps 4..11 also fold the 128-row TMEM work runs into an fp32
// register master (as k_tc_dw2: bounded tensor-core accumulation runs).
constexpr int kDwBK = 16;        // rows per stage = one K = 16 MMA step
constexpr int kDwStages = 4;
constexpr int kDwSub = 8;        // stages per TMEM work run (128 rows)
#ifndef MARS_DW_PAIR
#define MARS_DW_PAIR 1
#endif
constexpr bool kDwPair = MARS_DW_PAIR != 0;
#ifndef MARS_DW_NG
#define MARS_DW_NG 1          // converter groups of k_tc3h_dw working on alternate stages
#endif   // C_in = H = 256 on a CTA pair (k_tc3h_dw_pair)

template <int CINT, int HH>
struct H3DwCfg {
  static constexpr int NH = HH / 128;                 // 128-row halves of H (UMMA M)
  static constexpr int ATOM = 64 * kDwBK * 2;         // fp16 MN atom column: 64 cols x 16 rows
  static constexpr int BOX32 = 32 * kDwBK * 4;        // one 32-column fp32 block: 16 rows x 128 B
  static constexpr int A32 = (HH / 32) * BOX32;
  static constexpr int B32 = (CINT / 32) * BOX32;
  static constexpr int A16 = (HH / 64) * ATOM;
  static constexpr int B16 = (CINT / 64) * ATOM;
  static constexpr int STAGE = A32 + B32 + 2 * A16 + 2 * B16;
  static constexpr int SMEM = kDwStages * STAGE + 1024 + 512;
  static constexpr uint32_t TMEM_COLS = 2 * NH * CINT;
  static constexpr int MCOLS = CINT / 2;              // columns per folding thread per half
};

__device__ __forceinline__ void dwconv_bar() {      // converter warps 2..11
  asm volatile("bar.sync 2, 320;" ::: "memory");
}

template <int CINT, int HH>
__global__ void __launch_bounds__(384, 1)
k_tc3h_dw(const __grid_constant__ CUtensorMap tmDZ, const __grid_constant__ CUtensorMap tmY,
          const float* __restrict__ rs_dz, const float* __restrict__ rs_y,
          float* __restrict__ part, int32_t R, int32_t rows_per_chunk, int32_t CIN, int32_t Hn) {
  // Hn <= HH, CIN: the actual widths (narrower operands are zero-filled by TMA;
  // the partial [chunk][Hn][CIN] is written for the actual widths only)
  using Cfg = H3DwCfg<CINT, HH>;
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
  float* wmin = reinterpret_cast<float*>(bars + 3 * S + 6);   // [2][10] per-warp minima

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntile = (CIN + CINT - 1) / CINT;
  const int chunk = blockIdx.x / ntile, c_off = (blockIdx.x % ntile) * CINT;
  const int32_t r0 = chunk * rows_per_chunk;
  const int32_t r1 = min(R, r0 + rows_per_chunk);
  const int nk = r1 > r0 ? (r1 - r0 + kDwBK - 1) / kDwBK : 0;
  const int nsub = (nk + kDwSub - 1) / kDwSub;
  auto stA32 = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stB32 = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A32; };
  auto stA16 = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A32 + Cfg::B32; };  // hi, lo
  auto stB16 = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A32 + Cfg::B32 + 2 * Cfg::A16; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&conv[s], 10 / MARS_DW_NG);   // the converter warps of the stage's group
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
        mbar_expect_tx(&full[s], Cfg::A32 + Cfg::B32);
        const int32_t row = r0 + kb * kDwBK;
        // one 3-D box per operand: all 32-column (128-byte, swizzled) blocks of
        // the stage in a single TMA request
        tma_load_3d(stA32(s), &tmDZ, 0, row, 0, &full[s]);
        tma_load_3d(stB32(s), &tmY, 0, row, c_off / 32, &full[s]);
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                         // ---- MMA issuer
      constexpr uint32_t idesc = idesc_f16(kBM, CINT) | (1u << 15) | (1u << 16);   // MN-major
      int s = 0;
      uint32_t ph = 0;
      for (int sub = 0; sub < nsub; ++sub) {
        const int buf = sub & 1;
        mbar_wait(&tempty[buf], ((sub >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t twork = tbase + buf * NH * CINT;
        const int kb1 = min(nk, (sub + 1) * kDwSub);
        for (int kb = sub * kDwSub; kb < kb1; ++kb) {
          mbar_wait(&conv[s], ph);
          tc_fence_after();
          const uint32_t a = smem_u32(stA16(s)), al = a + Cfg::A16;
          const uint32_t b = smem_u32(stB16(s)), bl = b + Cfg::B16;
          // MN-major fp16, 128B swizzle: 8-row atoms (1 KB, SBO), 64-column
          // blocks one atom column apart (LBO); one MMA (K = 16) spans two atoms
          const uint64_t bh = sdesc_sw128(b, Cfg::ATOM, 1024);
          const uint64_t blo = sdesc_sw128(bl, Cfg::ATOM, 1024);
          const uint32_t first = kb == sub * kDwSub ? 0u : 1u;
#pragma unroll
          for (int h = 0; h < NH; ++h) {
            const uint64_t ah = sdesc_sw128(a + h * 2 * Cfg::ATOM, Cfg::ATOM, 1024);
            const uint64_t alo = sdesc_sw128(al + h * 2 * Cfg::ATOM, Cfg::ATOM, 1024);
            const uint32_t d = twork + h * CINT;
            mma_f16(d, ah, bh, idesc, first);
            mma_f16(d, ah, blo, idesc, 1);
            mma_f16(d, alo, bh, idesc, 1);
          }
          mma_commit(&empty[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(&tfull[buf]);
      }
    }
  } else {                         // ---- convert (warps 2..11); warps 4..11 also fold
    const bool folder = warp >= 4;
    const int ct = (warp - 2) * 32 + lane;
    constexpr int NT = 10 * 32;
    // chunk scales: min over the chunk's row scales of each operand
    float mz = INFINITY, my = INFINITY;
    for (int32_t r = r0 + ct; r < r1; r += NT) {
      mz = fminf(mz, __ldg(rs_dz + r));
      my = fminf(my, __ldg(rs_y + r));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      mz = fminf(mz, __shfl_xor_sync(kFull, mz, o));
      my = fminf(my, __shfl_xor_sync(kFull, my, o));
    }
    if (lane == 0) {
      wmin[warp - 2] = mz;
      wmin[10 + warp - 2] = my;
    }
    dwconv_bar();
    float sz = INFINITY, sy = INFINITY;
#pragma unroll
    for (int k = 0; k < 10; ++k) {
      sz = fminf(sz, wmin[k]);
      sy = fminf(sy, wmin[10 + k]);
    }
    if (!(sz < INFINITY)) sz = 1.f;          // empty chunk
    if (!(sy < INFINITY)) sy = 1.f;

    const int q = warp & 3, ch = (warp - 4) >> 2;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    float master[NH][MC];
#pragma unroll
    for (int h = 0; h < NH; ++h)
#pragma unroll
      for (int j = 0; j < MC; ++j) master[h][j] = 0.f;
    int folded = 0;
    auto fold = [&](int sub) {
      const int buf = sub & 1;
      mbar_wait(&tfull[buf], (sub >> 1) & 1);
      tc_fence_after();
      const uint32_t twork = tbase + buf * NH * CINT + ch * MC;
#pragma unroll
      for (int h = 0; h < NH; ++h)
#pragma unroll
        for (int c0 = 0; c0 < MC; c0 += 16) {          // 16 columns at a time: register budget
          uint32_t w[16];
          tmem_ld16(twork + lane_off + h * CINT + c0, w);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 16; ++j) master[h][c0 + j] += __uint_as_float(w[j]);
        }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[buf]);
    };
    // converter group: warps 2 + GW g .. 2 + GW g + GW - 1 convert stages kb = g (mod NG)
    constexpr int NG = MARS_DW_NG, GW = 10 / NG, GT = GW * 32;
    static_assert(10 % NG == 0 && NG <= kDwStages && NG <= kDwSub, "converter groups");
    const int grp = (warp - 2) / GW;
    const int gt = ct - grp * GT;                        // thread index within the group
    constexpr int NTA = kDwBK * HH / 8;                 // 8-column tasks of dZ per stage
    constexpr int NTT = NTA + kDwBK * CINT / 8;
    constexpr int MAXT = (NTT + GT - 1) / GT;             // tasks per thread
    // a thread's tasks are the same in every stage: their offsets from the
    // stage base are computed once (the second 16-byte source chunk is the
    // first's chunk index ^ 1: w0 is even)
    uint32_t so0[MAXT], dof[MAXT];
    int ntask = 0;
#pragma unroll
    for (int t = 0; t < MAXT; ++t) {
      const int i = gt + t * GT;
      so0[t] = dof[t] = 0;
      if (i < NTT) {
        const bool isA = i < NTA;
        const int ii = isA ? i : i - NTA;
        const int r = ii % kDwBK, c0 = (ii / kDwBK) * 8;
        const uint32_t sb = (isA ? 0u : (uint32_t)Cfg::A32) + (c0 / 32) * Cfg::BOX32 + r * 128;
        const int w0 = (c0 % 32) / 4;
        so0[t] = sb + ((w0 ^ (r & 7)) << 4);
        dof[t] = Cfg::A32 + Cfg::B32 + (isA ? 0u : 2u * Cfg::A16) + (c0 / 64) * Cfg::ATOM +
                 r * 128 + ((((c0 % 64) / 8) ^ (r & 7)) << 4);
        ntask = t + 1;
      }
    }
    int s = grp;
    uint32_t ph = 0;
    for (int kb = grp; kb < nk; kb += NG) {
      mbar_wait(&full[s], ph);
      uint8_t* stage = smem + s * Cfg::STAGE;
#pragma unroll
      for (int t = 0; t < MAXT; ++t) {
        if (t >= ntask) break;
        const bool isA = so0[t] < (uint32_t)Cfg::A32;
        const float4 v0 = *reinterpret_cast<const float4*>(stage + so0[t]);
        const float4 v1 = *reinterpret_cast<const float4*>(stage + (so0[t] ^ 16u));
        const float sc = isA ? sz : sy;
        const float x[8] = {v0.x * sc, v0.y * sc, v0.z * sc, v0.w * sc,
                            v1.x * sc, v1.y * sc, v1.z * sc, v1.w * sc};
        uint4 hv, lv;
        split_h8(x, hv, lv);
        *reinterpret_cast<uint4*>(stage + dof[t]) = hv;
        *reinterpret_cast<uint4*>(stage + dof[t] + (isA ? Cfg::A16 : Cfg::B16)) = lv;
      }
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) mbar_arrive(&conv[s]);
      s += NG;
      if (s >= S) { s -= S; ph ^= 1; }
      // fold run j once the conversion has passed the middle of run j + 1
      while (folder && folded < nsub && kb >= (folded + 1) * kDwSub + kDwSub / 2) fold(folded++);
    }
    if (folder) {
      while (folded < nsub) fold(folded++);
      const float inv = 1.f / (sz * sy);                   // exact (powers of two)
      float* out = part + (int64_t)chunk * Hn * CIN + c_off + ch * MC;
      const int cend = CIN - (c_off + ch * MC);            // columns of this thread that exist
#pragma unroll
      for (int h = 0; h < NH; ++h) {
        const int hr = h * 128 + q * 32 + lane;
        if (hr >= Hn) continue;
        float4* dst = reinterpret_cast<float4*>(out + (int64_t)hr * CIN);
#pragma unroll
        for (int j = 0; j < MC / 4; ++j)
          if (4 * j < cend)
            dst[j] = make_float4(master[h][4 * j] * inv, master[h][4 * j + 1] * inv,
                                 master[h][4 * j + 2] * inv, master[h][4 * j + 3] * inv);
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

// ---------------------------------------------------------------- k_tc3h_dw_pair
// The C_in = H = 256 weight gradient on a CTA pair (cta_group::2), so that no
// operand is converted twice.  With one CTA per 128-column tile of C_in (the
// kernel above), both tiles of a row chunk convert the whole dZ tile: 1.5x the
// conversion work the GEMM needs, and the fp32 -> fp16 hi / lo conversion is
// what bounds this kernel.  Here the pair splits both operands instead: CTA r
// converts dZ columns (h) [128r, 128r + 128) and Y columns (c) [128r, 128r +
// 128) of every BK-row stage (32 by default: a stage is one synchronisation
// chain of the converters, and the chain, not the bandwidth, set the 16-row
// kernel's pace); the even CTA issues BK / 16 M = 256 (h), N = 256 (c) K = 16
// pair MMAs per product that read the A half and the B half of each CTA from
// the same shared-memory offsets; CTA r's TMEM accumulates D[h][c] for its 128
// h rows and all 256 c columns (256 fp32 columns, double-buffered).
// Synchronisation: the MMA commits multicast to both CTAs' empty / tfull
// barriers; the even CTA's converter (folder) warps arrive on its own conv
// (tempty) barrier; the odd CTA's converters (folders) first meet at a named
// barrier, then ONE thread arrives on the even CTA's barrier (remote arrive).
// Scaling, folding and the partial layout are those of k_tc3h_dw.
#ifndef MARS_PAIR_STAGES
#define MARS_PAIR_STAGES 6
#endif
#ifndef MARS_DWP_BK
#define MARS_DWP_BK 32        // rows per pair stage (BK / 16 MMA K-steps per stage)
#endif
#ifndef MARS_DWP_NG
#define MARS_DWP_NG 1         // converter groups working on alternate stages
#endif
#ifndef MARS_DWP_RUN
#define MARS_DWP_RUN 128      // rows per tensor-core accumulation run before the fp32 fold
#endif

#define MARS_DWP_WARPS 10     // TMA + MMA + 8 converter / folder warps
constexpr int kDwpThreads = MARS_DWP_WARPS * 32;
// one CTA per SM: warps are spread over the 4 SM sub-partitions, each with a
// quarter of the register file (16384), so the busiest one bounds the count
constexpr int kDwpRegs = (16384 / (32 * ((MARS_DWP_WARPS + 3) / 4))) / 8 * 8;
template <int NCW>
__device__ __forceinline__ void dwp_conv_bar() {    // the converter warps
  asm volatile("bar.sync 2, %0;" ::"n"(NCW * 32) : "memory");
}

template <int BK>
struct H3PairCfg {
  static constexpr int ATOM = 64 * BK * 2;             // fp16 MN atom column: 64 cols x BK rows
  static constexpr int BOX32 = 32 * BK * 4;            // one 32-column fp32 block: BK rows x 128 B
  static constexpr int HALF = 128;                     // columns of each operand per CTA
  static constexpr int A32 = (HALF / 32) * BOX32;
  static constexpr int B32 = (HALF / 32) * BOX32;
  static constexpr int A16 = (HALF / 64) * ATOM;       // hi; lo follows
  static constexpr int B16 = (HALF / 64) * ATOM;
  static constexpr int STAGE = A32 + B32 + 2 * A16 + 2 * B16;   // 2 KB per row
  static constexpr int S = BK == 16 ? MARS_PAIR_STAGES : (200 * 1024) / STAGE;
  static constexpr int SMEM = S * STAGE + 1024 + 512;
  static constexpr int SUB = MARS_DWP_RUN / BK;        // stages per TMEM work run (MARS_DWP_RUN rows)
  static constexpr uint32_t TMEM_COLS = 512;           // 2 buffers x 256 fp32 columns
  static constexpr int MC = 128;                       // columns per folding thread
};

template <int BK, int NG>
__global__ void __cluster_dims__(2, 1, 1) __maxnreg__(kDwpRegs)
k_tc3h_dw_pair(const __grid_constant__ CUtensorMap tmDZ, const __grid_constant__ CUtensorMap tmY,
               const float* __restrict__ rs_dz, const float* __restrict__ rs_y,
               float* __restrict__ part, int32_t R, int32_t rows_per_chunk) {
  using Cfg = H3PairCfg<BK>;
  constexpr int S = Cfg::S;
  constexpr int SUB = Cfg::SUB;
  constexpr int MC = Cfg::MC;
  constexpr int CIN = 256, HH = 256;
  constexpr int NCW = kDwpThreads / 32 - 2;              // converter (and folder) warps
  constexpr int GW = NCW / NG;                           // converter warps per group
  static_assert(NCW % NG == 0 && SUB >= NG, "converter groups");
  static_assert(NCW == 8, "8 folder warps: 4 TMEM lane quadrants x 2 column halves");
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + S * Cfg::STAGE);
  uint64_t* full = bars;
  uint64_t* conv = bars + S;             // even CTA: both CTAs' converters
  uint64_t* empty = bars + 2 * S;
  uint64_t* tfull = bars + 3 * S;        // [2]
  uint64_t* tempty = bars + 3 * S + 2;   // [2] even CTA: both CTAs' folders
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bars + 3 * S + 4);
  float* wmin = reinterpret_cast<float*>(bars + 3 * S + 6);   // [2][NCW] per-warp minima

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_rank();
  const int chunk = blockIdx.x >> 1;
  const int32_t r0 = chunk * rows_per_chunk;
  const int32_t r1 = min(R, r0 + rows_per_chunk);
  const int nk = r1 > r0 ? (r1 - r0 + BK - 1) / BK : 0;
  const int nsub = (nk + SUB - 1) / SUB;
  auto stA32 = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stB32 = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A32; };
  auto stA16 = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A32 + Cfg::B32; };  // hi, lo
  auto stB16 = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A32 + Cfg::B32 + 2 * Cfg::A16; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&conv[s], GW + 1);     // the group's local converter warps + 1 from the odd CTA
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], NCW + 1);  // the local folder warps + 1 from the odd CTA
    }
    fence_mbar_init();
    tma_prefetch(&tmDZ);
    tma_prefetch(&tmY);
  }
  if (warp == 1) tmem_alloc_pair(tslot, Cfg::TMEM_COLS);
  tc_fence_before();
  cluster_sync();                        // peers' barriers initialised, TMEM allocated
  tc_fence_after();
  const uint32_t tbase = *tslot;

  if (warp == 0) {
    if (lane == 0) {                                         // ---- TMA producer (both CTAs)
      int s = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < nk; ++kb) {
        mbar_wait(&empty[s], ph ^ 1);
        mbar_expect_tx(&full[s], Cfg::A32 + Cfg::B32);
        const int32_t row = r0 + kb * BK;
        tma_load_3d(stA32(s), &tmDZ, 0, row, (int)rank * (Cfg::HALF / 32), &full[s]);
        tma_load_3d(stB32(s), &tmY, 0, row, (int)rank * (Cfg::HALF / 32), &full[s]);
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {                            // ---- pair MMA issuer
      constexpr uint32_t idesc = idesc_f16(2 * Cfg::HALF, CIN) | (1u << 15) | (1u << 16);
      int s = 0;
      uint32_t ph = 0;
      for (int sub = 0; sub < nsub; ++sub) {
        const int buf = sub & 1;
        mbar_wait_cluster(&tempty[buf], ((sub >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t twork = tbase + buf * CIN;
        const int kb1 = min(nk, (sub + 1) * SUB);
        for (int kb = sub * SUB; kb < kb1; ++kb) {
          mbar_wait_cluster(&conv[s], ph);
          tc_fence_after();
#pragma unroll
          for (int j = 0; j < BK / 16; ++j) {                // K = 16 steps: 16 rows = 2 KB of an atom column
            const uint32_t a = smem_u32(stA16(s)) + j * 2048, al = a + Cfg::A16;
            const uint32_t b = smem_u32(stB16(s)) + j * 2048, bl = b + Cfg::B16;
            const uint64_t ah = sdesc_sw128(a, Cfg::ATOM, 1024);
            const uint64_t alo = sdesc_sw128(al, Cfg::ATOM, 1024);
            const uint64_t bh = sdesc_sw128(b, Cfg::ATOM, 1024);
            const uint64_t blo = sdesc_sw128(bl, Cfg::ATOM, 1024);
            const uint32_t first = (kb == sub * SUB && j == 0) ? 0u : 1u;
            mma_f16_pair(twork, ah, bh, idesc, first);
            mma_f16_pair(twork, ah, blo, idesc, 1);
            mma_f16_pair(twork, alo, bh, idesc, 1);
          }
          mma_commit_pair(&empty[s], 0x3);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit_pair(&tfull[buf], 0x3);
      }
    }
  } else {                         // ---- convert and fold (warps 2 .. 2 + NCW - 1)
    constexpr bool folder = true;
    const int ct = (warp - 2) * 32 + lane;
    constexpr int NT = NCW * 32;
    float mz = INFINITY, my = INFINITY;
    for (int32_t r = r0 + ct; r < r1; r += NT) {
      mz = fminf(mz, __ldg(rs_dz + r));
      my = fminf(my, __ldg(rs_y + r));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      mz = fminf(mz, __shfl_xor_sync(kFull, mz, o));
      my = fminf(my, __shfl_xor_sync(kFull, my, o));
    }
    if (lane == 0) {
      wmin[warp - 2] = mz;
      wmin[NCW + warp - 2] = my;
    }
    dwp_conv_bar<NCW>();
    float sz = INFINITY, sy = INFINITY;
#pragma unroll
    for (int k = 0; k < NCW; ++k) {
      sz = fminf(sz, wmin[k]);
      sy = fminf(sy, wmin[NCW + k]);
    }
    if (!(sz < INFINITY)) sz = 1.f;          // empty chunk
    if (!(sy < INFINITY)) sy = 1.f;
    const uint32_t conv0 = mapa_u32(conv, 0), tempty0 = mapa_u32(tempty, 0);

    const int q = warp & 3, ch = (warp - 2) >> 2;     // TMEM lane quadrant, column half
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    float master[MC];
#pragma unroll
    for (int j = 0; j < MC; ++j) master[j] = 0.f;
    int folded = 0;
    auto fold = [&](int sub) {
      const int buf = sub & 1;
      mbar_wait(&tfull[buf], (sub >> 1) & 1);
      tc_fence_after();
      const uint32_t twork = tbase + buf * CIN + ch * MC;
#pragma unroll
      for (int c0 = 0; c0 < MC; c0 += 16) {            // 16 columns at a time: register budget
        uint32_t w[16];
        tmem_ld16(twork + lane_off + c0, w);
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 16; ++j) master[c0 + j] += __uint_as_float(w[j]);
      }
      tc_fence_before();
      if (rank == 0) {
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[buf]);
      } else {
        asm volatile("bar.sync 3, %0;" ::"r"(NT) : "memory");   // the folder warps
        if (threadIdx.x == 2 * 32) mbar_arrive_cluster(tempty0 + buf * 8);
      }
    };
    // converter group: warps 2 + GW g .. 2 + GW g + GW - 1 convert stages kb = g (mod NG)
    const int grp = (warp - 2) / GW;
    const int gt = ct - grp * GW * 32;                   // thread index within the group
    constexpr int GT = GW * 32;
    constexpr int NTA = BK * Cfg::HALF / 8;              // 8-column tasks of dZ per stage
    constexpr int NTT = 2 * NTA;
    constexpr int MAXT = (NTT + GT - 1) / GT;            // tasks per thread
    // a thread's tasks are the same in every stage: their offsets from the
    // stage base (swizzled source chunks, destination chunk) are computed once
    // (the second 16-byte chunk of a task is the first's chunk index ^ 1: w0 is even)
    uint32_t so0[MAXT], dof[MAXT];
    int ntask = 0;
#pragma unroll
    for (int t = 0; t < MAXT; ++t) {
      const int i = gt + t * GT;
      so0[t] = dof[t] = 0;
      if (i < NTT) {
        const bool isA = i < NTA;
        const int ii = isA ? i : i - NTA;
        const int r = ii % BK, c0 = (ii / BK) * 8;
        const uint32_t sb = (isA ? 0u : (uint32_t)Cfg::A32) + (c0 / 32) * Cfg::BOX32 + r * 128;
        const int w0 = (c0 % 32) / 4;
        so0[t] = sb + ((w0 ^ (r & 7)) << 4);
        dof[t] = Cfg::A32 + Cfg::B32 + (isA ? 0u : 2u * Cfg::A16) + (c0 / 64) * Cfg::ATOM +
                 r * 128 + ((((c0 % 64) / 8) ^ (r & 7)) << 4);
        ntask = t + 1;
      }
    }
    int s = grp;
    uint32_t ph = 0;
    for (int kb = grp; kb < nk; kb += NG) {
      mbar_wait(&full[s], ph);
      uint8_t* stage = smem + s * Cfg::STAGE;
#pragma unroll
      for (int t = 0; t < MAXT; ++t) {
        if (t >= ntask) break;
        const float4 v0 = *reinterpret_cast<const float4*>(stage + so0[t]);
        const float4 v1 = *reinterpret_cast<const float4*>(stage + (so0[t] ^ 16u));
        const float sc = so0[t] < (uint32_t)Cfg::A32 ? sz : sy;
        const float x[8] = {v0.x * sc, v0.y * sc, v0.z * sc, v0.w * sc,
                            v1.x * sc, v1.y * sc, v1.z * sc, v1.w * sc};
        uint4 hv, lv;
        split_h8(x, hv, lv);
        *reinterpret_cast<uint4*>(stage + dof[t]) = hv;
        *reinterpret_cast<uint4*>(stage + dof[t] + Cfg::A16) = lv;      // A16 == B16
      }
      fence_proxy_async_smem();
      if (rank == 0) {
        __syncwarp();
        if (lane == 0) mbar_arrive(&conv[s]);
      } else {
        if (NG == 1) {
          dwp_conv_bar<NCW>();                               // the converter warps
        } else {
          asm volatile("bar.sync %0, %1;" ::"r"(4 + grp), "r"(GT) : "memory");
        }
        if (gt == 0) mbar_arrive_cluster(conv0 + s * 8);
      }
      s += NG;
      if (s >= S) { s -= S; ph ^= 1; }
      // fold run j once the conversion has passed the middle of run j + 1
      while (folder && folded < nsub && kb >= (folded + 1) * SUB + SUB / 2) fold(folded++);
    }
    if (folder) {
      while (folded < nsub) fold(folded++);
      const float inv = 1.f / (sz * sy);                   // exact (powers of two)
      float* out = part + (int64_t)chunk * HH * CIN +
                   (int64_t)(rank * Cfg::HALF + q * 32 + lane) * CIN + ch * MC;
      float4* dst = reinterpret_cast<float4*>(out);
#pragma unroll
      for (int j = 0; j < MC / 4; ++j)
        dst[j] = make_float4(master[4 * j] * inv, master[4 * j + 1] * inv,
                             master[4 * j + 2] * inv, master[4 * j + 3] * inv);
    }
  }
  tc_fence_before();
  cluster_sync();                        // both CTAs done with TMEM and the peer's barriers
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc_pair(tbase, Cfg::TMEM_COLS);
  }
}

constexpr int kDwpBK = MARS_DWP_BK;
#define K_DW_PAIR k_tc3h_dw_pair<MARS_DWP_BK, MARS_DWP_NG>

__global__ void k_dw3h_reduce(const float* __restrict__ part, int nchunk, int CIN, int H,
                              float* __restrict__ dW) {
  dw_reduce_body(part, nchunk, CIN, H, dW);
}

template <int CINT, int HH>
cudaError_t dw3h_c(const float* Y, const float* rs_y, const float* dZ, const float* rs_dz,
                   float* part, int nchunk, int64_t R, int rows, int CIN, int H, cudaStream_t s) {
  using Cfg = H3DwCfg<CINT, HH>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k_tc3h_dw<CINT, HH>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap tdz, ty;
  if (!tc_tmap_blocks(&tdz, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, dZ, R, H, kDwBK, HH / 32) ||
      !tc_tmap_blocks(&ty, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, Y, R, CIN, kDwBK, CINT / 32))
    return cudaErrorInvalidValue;
  k_tc3h_dw<CINT, HH><<<nchunk * ((CIN + CINT - 1) / CINT), 384, Cfg::SMEM, s>>>(
      tdz, ty, rs_dz, rs_y, part, (int32_t)R, rows, CIN, H);
  return cudaGetLastError();
}

// Co-resident CTA pairs of k_tc3h_dw_pair (cudaOccupancyMaxActiveClusters).
int dw_pair_clusters() {
  static int n = 0;
  if (!n) {
    cudaFuncSetAttribute(K_DW_PAIR, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         H3PairCfg<kDwpBK>::SMEM);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2 * 74, 1, 1);
    cfg.blockDim = dim3(kDwpThreads, 1, 1);
    cfg.dynamicSmemBytes = H3PairCfg<kDwpBK>::SMEM;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int c = 0;
    if (cudaOccupancyMaxActiveClusters(&c, K_DW_PAIR, &cfg) != cudaSuccess || c < 1) {
      cudaGetLastError();
      c = tc_num_sms() / 2;
    }
    n = c;
    if (getenv("MARS_DEBUG_DW")) fprintf(stderr, "k_tc3h_dw_pair: %d co-resident CTA pairs\n", n);
  }
  return n;
}

cudaError_t dw3h_pair(const float* Y, const float* rs_y, const float* dZ, const float* rs_dz,
                      float* part, int nchunk, int64_t R, int rows, cudaStream_t s) {
  using Cfg = H3PairCfg<kDwpBK>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(K_DW_PAIR, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap tdz, ty;
  if (!tc_tmap_blocks(&tdz, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, dZ, R, 256, kDwpBK, Cfg::HALF / 32) ||
      !tc_tmap_blocks(&ty, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, Y, R, 256, kDwpBK, Cfg::HALF / 32))
    return cudaErrorInvalidValue;
  K_DW_PAIR<<<2 * nchunk, kDwpThreads, Cfg::SMEM, s>>>(tdz, ty, rs_dz, rs_y, part, (int32_t)R, rows);
  return cudaGetLastError();
}

}  // namespace

// wsc[2] = {t, 1/t}; Bt_* [H × CIN], B_* [CIN × H], fp16.
cudaError_t tc3h_split_weights(const float* W, int CIN, int H, float* wsc, void* Bt_hi,
                               void* Bt_lo, void* B_hi, void* B_lo, cudaStream_t s,
                               int* launches) {
  count_launch(launches, 2);
  k_wscale<<<1, 1024, 0, s>>>(W, CIN * H, wsc);
  k_split_w3h<<<cdiv((int64_t)CIN * H, 256), 256, 0, s>>>(
      W, CIN, H, wsc, static_cast<__half*>(Bt_hi), static_cast<__half*>(Bt_lo),
      static_cast<__half*>(B_hi), static_cast<__half*>(B_lo));
  return cudaGetLastError();
}

cudaError_t tc3h_split_weights_all(const W3Split& a, int nl, cudaStream_t s, int* launches) {
  if (nl < 1 || nl > 3) return cudaErrorInvalidValue;
  count_launch(launches);
  k_split_w3h_all<<<dim3(kSplitBlocks, nl), 1024, 0, s>>>(a);
  return cudaGetLastError();
}

cudaError_t tc3h_row_scales(const float* A, int64_t M, int K, float* rs, cudaStream_t s,
                            int* launches) {
  count_launch(launches);
  k_row_scale<<<cdiv(M * 32, 256), 256, 0, s>>>(A, M, K, rs);
  return cudaGetLastError();
}

// C[M×N] = A[M×K] · Bᵀ, B = (B_hi + B_lo) / t [N×K] (fp16, scaled by t = 1 / inv_tb[0]),
// rs[M] = the power-of-two row scales of A (2^(14 - e_r), see k_row_scale).
cudaError_t tc3h_gemm_rows(const float* A, const float* rs, const void* B_hi, const void* B_lo,
                           const float* inv_tb, float* C, int64_t M, int N, int K, cudaStream_t s,
                           int* launches) {
  count_launch(launches);
  if (K % 16 || K > 256) return cudaErrorInvalidValue;
  const __half* bh = static_cast<const __half*>(B_hi);
  const __half* bl = static_cast<const __half*>(B_lo);
  switch (N) {
    case 32:
    case 64: return rows3h_n<64>(A, rs, bh, bl, inv_tb, C, M, K, N, s);
    case 128: return rows3h_n<128>(A, rs, bh, bl, inv_tb, C, M, K, N, s);
    case 256:
      if (MARS_ROWS_PAIR && M >= 2 * kBM * tc_num_sms())   // CTA pairs for the large launches
        return rows3h_pair(A, rs, bh, bl, inv_tb, C, M, K, s);
      return rows3h_n<256>(A, rs, bh, bl, inv_tb, C, M, K, N, s);
    default: return cudaErrorInvalidValue;
  }
}

// dW [CIN × H] = Yᵀ dZ, Y [R × CIN], dZ [R × H] (H in {128, 256}), with the
// power-of-two row scales rs_y / rs_dz of both operands (see k_tc3h_dw).
cudaError_t tc3h_gemm_dw(const float* Y, const float* rs_y, const float* dZ, const float* rs_dz,
                         float* dW, int64_t R, int CIN, int H, float* part, cudaStream_t s,
                         int* launches) {
  count_launch(launches, 2);
  int nchunk = tc_dw_chunks(R, CIN);
  int rows = (int)((R + nchunk - 1) / nchunk);
  rows = (rows + kDwBK - 1) / kDwBK * kDwBK;
  nchunk = (int)((R + rows - 1) / rows);
  cudaError_t e;
  if (H != 32 && H != 64 && H != 128 && H != 256) return cudaErrorInvalidValue;
  if (CIN == 256 && H == 256 && kDwPair) {
    // one wave: as many row chunks as CTA pairs can be co-resident (a pair
    // needs both SMs of a TPC free; not every SM can be paired)
    nchunk = std::min(tc_dw_chunks(R, CIN), dw_pair_clusters());
    rows = (int)((R + nchunk - 1) / nchunk);
    rows = (rows + kDwpBK - 1) / kDwpBK * kDwpBK;
    nchunk = (int)((R + rows - 1) / rows);
    e = dw3h_pair(Y, rs_y, dZ, rs_dz, part, nchunk, R, rows, s);
    if (e != cudaSuccess) return e;
    k_dw3h_reduce<<<dw_reduce_blocks((int64_t)H * CIN), 256, 0, s>>>(part, nchunk, CIN, H, dW);
    return cudaGetLastError();
  }
  // H in {32, 64} runs the H = 128 tiles and C_in in {16, 32} the 64-column
  // tiles (TMA zero-fills the missing columns; only the real ones are written)
  switch (CIN) {
    case 16:
    case 32:
    case 64: e = H == 256 ? dw3h_c<64, 256>(Y, rs_y, dZ, rs_dz, part, nchunk, R, rows, CIN, H, s)
                          : dw3h_c<64, 128>(Y, rs_y, dZ, rs_dz, part, nchunk, R, rows, CIN, H, s); break;
    case 128:
    case 256: e = H == 256 ? dw3h_c<128, 256>(Y, rs_y, dZ, rs_dz, part, nchunk, R, rows, CIN, H, s)
                           : dw3h_c<128, 128>(Y, rs_y, dZ, rs_dz, part, nchunk, R, rows, CIN, H, s); break;
    default: return cudaErrorInvalidValue;
  }
  if (e != cudaSuccess) return e;
  k_dw3h_reduce<<<dw_reduce_blocks((int64_t)H * CIN), 256, 0, s>>>(part, nchunk, CIN, H, dW);
  return cudaGetLastError();
}

}  // namespace mars
