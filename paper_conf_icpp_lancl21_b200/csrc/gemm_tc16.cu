// a6 / a12 on tcgen05 for the bf16 path (MARS_BF16; BASELINE.json's "2e-2
// relative for bf16 tensor-core paths"): bf16 activations and weights, one
// kind::f16 MMA per 16-element k-step, fp32 accumulation in TMEM.
//
// k_tc16_rows : C[M×N] (bf16) = A[M×K]·Bᵀ, A activations, B = bf16 weights [N×K].
//               K-major operands, 128-byte rows (64 bf16) with 128B swizzle;
//               persistent over 128-row tiles; warp 0 TMA, warp 1 MMA issuer,
//               warps 4-7 epilogue (TMEM -> bf16 -> swizzled smem slab -> TMA
//               store) with double-buffered accumulators.
// k_tc16_dw   : per CTA a chunk of rows x a CINT tile of C_in, D = dZᵀ·Y with
//               MN-major operands (row-major activations, 128B swizzle, 16-byte
//               atoms); runs of 128 rows accumulate in a double-buffered TMEM
//               work accumulator and are folded into fp32 registers by eight
//               epilogue warps; fp32 chunk partials, fixed-order fp64 reduce.
#include "common.cuh"
#include "internal.cuh"
#include "tc_ptx.cuh"
#include "vec.cuh"

namespace mars {
namespace {

using namespace tc;

constexpr int kBM = 128;
constexpr int kBK = 64;          // bf16 elements per 128-byte K-block
constexpr int kThreads = 256;

template <int N>
struct R16Cfg {
  static constexpr int kStages = N > 128 ? 4 : 6;
  static constexpr int A_BYTES = kBM * kBK * 2;       // 16 KB
  static constexpr int B_BYTES = N * kBK * 2;
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int SLAB = 32 * 64 * 2;            // 32 rows x 64 bf16 (128 B rows)
  static constexpr int STAGING = 4 * 2 * SLAB;
  static constexpr int SMEM = kStages * STAGE + STAGING + 1024 + 256;
  static constexpr uint32_t TMEM_COLS = (2 * N) <= 32 ? 32 : (2 * N) <= 64 ? 64 : (2 * N) <= 128 ? 128
                                        : (2 * N) <= 256 ? 256 : 512;
};

template <int N>
__global__ void __launch_bounds__(kThreads, 1)
k_tc16_rows(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
            const __grid_constant__ CUtensorMap tmC, int32_t M, int32_t K) {
  using Cfg = R16Cfg<N>;
  constexpr int S = Cfg::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* staging = smem + S * Cfg::STAGE;
  uint64_t* bars = reinterpret_cast<uint64_t*>(staging + Cfg::STAGING);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* tfull = bars + 2 * S;
  uint64_t* tempty = bars + 2 * S + 2;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bars + 2 * S + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = (M + kBM - 1) / kBM;
  const int nk = K / kBK;
  auto stA = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stB = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 4);
    }
    fence_mbar_init();
    tma_prefetch(&tmA);
    tma_prefetch(&tmB);
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
          mbar_expect_tx(&full[s], Cfg::A_BYTES + Cfg::B_BYTES);
          tma_load_2d(stA(s), &tmA, kb * kBK, t * kBM, &full[s]);
          tma_load_2d(stB(s), &tmB, kb * kBK, 0, &full[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                         // ---- MMA issuer
      constexpr uint32_t idesc = idesc_bf16(kBM, N, false, false);
      int s = 0;
      uint32_t ph = 0;
      int acc = 0;
      uint32_t aph = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        mbar_wait(&tempty[acc], aph ^ 1);
        tc_fence_after();
        const uint32_t d = tbase + acc * N;
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait(&full[s], ph);
          tc_fence_after();
          const uint32_t a = smem_u32(stA(s)), b = smem_u32(stB(s));
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k)
            mma_f16(d, sdesc_sw128(a + 32 * k, 16, 1024), sdesc_sw128(b + 32 * k, 16, 1024), idesc,
                    (kb | k) != 0);
          mma_commit(&empty[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(&tfull[acc]);
        acc ^= 1;
        if (acc == 0) aph ^= 1;
      }
    }
  } else if (warp >= 4) {                                    // ---- epilogue
    const int q = warp & 3;
    uint8_t* slab0 = staging + q * 2 * Cfg::SLAB;
    int nslab = 0;
    int acc = 0;
    uint32_t aph = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
      mbar_wait(&tfull[acc], aph);
      tc_fence_after();
#pragma unroll 1
      for (int c0 = 0; c0 < N; c0 += 64, ++nslab) {
        uint32_t r0[32], r1[32];
        tmem_ld32(tbase + ((uint32_t)(q * 32) << 16) + acc * N + c0, r0);
        tmem_ld32(tbase + ((uint32_t)(q * 32) << 16) + acc * N + c0 + 32, r1);
        uint8_t* slab = slab0 + (nslab & 1) * Cfg::SLAB;
        if (lane == 0) bulk_wait_read<1>();
        __syncwarp();
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 8; ++j) {           // 16-byte chunk j = columns 8j .. 8j+7
          const uint32_t* src = j < 4 ? r0 + 8 * j : r1 + 8 * (j - 4);
          uint4 v = make_uint4(pack_bf16x2(__uint_as_float(src[0]), __uint_as_float(src[1])),
                               pack_bf16x2(__uint_as_float(src[2]), __uint_as_float(src[3])),
                               pack_bf16x2(__uint_as_float(src[4]), __uint_as_float(src[5])),
                               pack_bf16x2(__uint_as_float(src[6]), __uint_as_float(src[7])));
          *reinterpret_cast<uint4*>(slab + lane * 128 + ((j ^ (lane & 7)) << 4)) = v;
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

// ---------------------------------------------------------------- k_tc16_dw
#ifndef MARS_DW16_3D
#define MARS_DW16_3D 1   // one 3-D TMA box per operand and stage (vs one per 64-column atom)
#endif
constexpr int kDwBK = 16;        // rows per stage (one K = 16 MMA)
constexpr int kDwStages = 8;
constexpr int kSubKb = 8;        // stages per TMEM work run (128 rows)

template <int CINT, int HH>
struct D16Cfg {
  static constexpr int NH = HH / 128;                 // 128-row halves of H (UMMA M)
  static constexpr int BOX = 64 * kDwBK * 2;          // 64 bf16 cols x 16 rows = 2 KB
  static constexpr int A_BYTES = (HH / 64) * BOX;     // dZ: HH cols
  static constexpr int B_BYTES = (CINT / 64) * BOX;   // Y : CINT cols
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int SMEM = kDwStages * STAGE + 1024 + 256;
  static constexpr uint32_t TMEM_COLS = 2 * NH * CINT;
  static constexpr int MCOLS = CINT / 2;
};

template <int CINT, int HH>
__global__ void __launch_bounds__(384, 1)
k_tc16_dw(const __grid_constant__ CUtensorMap tmDZ, const __grid_constant__ CUtensorMap tmY,
          float* __restrict__ part, int32_t R, int32_t rows_per_chunk, int32_t CIN) {
  using Cfg = D16Cfg<CINT, HH>;
  constexpr int NH = Cfg::NH;
  constexpr int S = kDwStages;
  constexpr int MC = Cfg::MCOLS;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + S * Cfg::STAGE);
  uint64_t* full = bars;
  uint64_t* empty = bars + S;
  uint64_t* tfull = bars + 2 * S;        // [2]
  uint64_t* tempty = bars + 2 * S + 2;   // [2]
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bars + 2 * S + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntile = CIN / CINT;
  const int chunk = blockIdx.x / ntile, c_off = (blockIdx.x % ntile) * CINT;
  const int32_t r0 = chunk * rows_per_chunk;
  const int32_t r1 = min(R, r0 + rows_per_chunk);
  const int nk = r1 > r0 ? (r1 - r0 + kDwBK - 1) / kDwBK : 0;
  const int nsub = (nk + kSubKb - 1) / kSubKb;
  auto stA = [&](int s) { return smem + s * Cfg::STAGE; };
  auto stB = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
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
#if MARS_DW16_3D
        // one 3-D box per operand: all 64-column atom columns of the stage
        tma_load_3d(stA(s), &tmDZ, 0, row, 0, &full[s]);
        tma_load_3d(stB(s), &tmY, 0, row, c_off / 64, &full[s]);
#else
#pragma unroll
        for (int bx = 0; bx < HH / 64; ++bx)
          tma_load_2d(stA(s) + bx * Cfg::BOX, &tmDZ, bx * 64, row, &full[s]);
#pragma unroll
        for (int bx = 0; bx < CINT / 64; ++bx)
          tma_load_2d(stB(s) + bx * Cfg::BOX, &tmY, c_off + bx * 64, row, &full[s]);
#endif
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                         // ---- MMA issuer
      constexpr uint32_t idesc = idesc_bf16(kBM, CINT, true, true);
      int s = 0;
      uint32_t ph = 0;
      for (int sub = 0; sub < nsub; ++sub) {
        const int buf = sub & 1;
        mbar_wait(&tempty[buf], ((sub >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t twork = tbase + buf * NH * CINT;
        const int kb1 = min(nk, (sub + 1) * kSubKb);
        for (int kb = sub * kSubKb; kb < kb1; ++kb) {
          mbar_wait(&full[s], ph);
          tc_fence_after();
          const uint32_t a = smem_u32(stA(s)), b = smem_u32(stB(s));
          // MN-major bf16, 128B swizzle: 8-row atoms (1 KB, SBO), 64-element MN
          // blocks one box apart (LBO); one MMA (K = 16) spans two atoms.
          const uint64_t bd = sdesc_sw128(b, Cfg::BOX, 1024);
          const uint32_t first = kb == sub * kSubKb ? 0u : 1u;
#pragma unroll
          for (int h = 0; h < NH; ++h)
            mma_f16(twork + h * CINT, sdesc_sw128(a + h * 2 * Cfg::BOX, Cfg::BOX, 1024), bd, idesc,
                    first);
          mma_commit(&empty[s]);
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(&tfull[buf]);
      }
    }
  } else if (warp >= 4) {                                    // ---- fold (warps 4..11)
    const int q = warp & 3, ch = (warp - 4) >> 2;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    float master[NH][MC];
#pragma unroll
    for (int h = 0; h < NH; ++h)
#pragma unroll
      for (int j = 0; j < MC; ++j) master[h][j] = 0.f;
    for (int sub = 0; sub < nsub; ++sub) {
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
    }
    float* out = part + (int64_t)chunk * HH * CIN + c_off + ch * MC;
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      float4* dst = reinterpret_cast<float4*>(out + (int64_t)(h * 128 + q * 32 + lane) * CIN);
#pragma unroll
      for (int j = 0; j < MC / 4; ++j)
        dst[j] = make_float4(master[h][4 * j], master[h][4 * j + 1], master[h][4 * j + 2],
                             master[h][4 * j + 3]);
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
__global__ void k_dw16_reduce(const float* __restrict__ part, int nchunk, int CIN, int H,
                              float* __restrict__ dW) {
  dw_reduce_body(part, nchunk, CIN, H, dW);
}

__global__ void k_w16(const float* __restrict__ W, int CIN, int H, bf16* __restrict__ Bt,
                      bf16* __restrict__ B) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;   // e = c * H + h
  if (e >= (int64_t)CIN * H) return;
  int c = (int)(e / H), h = (int)(e % H);
  const bf16 w = __float2bfloat16_rn(W[e]);
  B[e] = w;
  Bt[(int64_t)h * CIN + c] = w;
}

bool tmap16(CUtensorMap* m, const void* base, int64_t rows, int64_t cols, int box_cols,
            int box_rows) {
  return tc_tmap(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, base, rows, cols, box_cols, box_rows,
                 CU_TENSOR_MAP_SWIZZLE_128B);
}

template <int N>
cudaError_t rows16_n(const void* A, const void* B, void* C, int64_t M, int K, cudaStream_t s) {
  using Cfg = R16Cfg<N>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k_tc16_rows<N>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap ta, tb, tc_;
  if (!tmap16(&ta, A, M, K, kBK, kBM) || !tmap16(&tb, B, N, K, kBK, N) ||
      !tmap16(&tc_, C, M, N, 64, 32))
    return cudaErrorInvalidValue;
  const int ntiles = (int)((M + kBM - 1) / kBM);
  const int grid = std::min(ntiles, tc_num_sms());
  k_tc16_rows<N><<<grid, kThreads, Cfg::SMEM, s>>>(ta, tb, tc_, (int32_t)M, K);
  return cudaGetLastError();
}

int dw16_tile(int CIN) { return CIN >= 128 ? 128 : 64; }

int dw16_chunks(int64_t R, int CIN) {
  const int ntile = std::max(1, CIN / dw16_tile(CIN));
  int64_t want = std::max<int64_t>(1, tc_num_sms() / ntile);
  int64_t maxc = std::max<int64_t>(1, R / 256);
  return (int)std::min(want, maxc);
}

template <int CINT, int HH>
cudaError_t dw16_c(const void* Y, const void* dZ, float* part, int nchunk, int64_t R, int rows,
                   int CIN, cudaStream_t s) {
  using Cfg = D16Cfg<CINT, HH>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k_tc16_dw<CINT, HH>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  CUtensorMap tdz, ty;
#if MARS_DW16_3D
  if (!tc_tmap_blocks(&tdz, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, dZ, R, HH, kDwBK, HH / 64) ||
      !tc_tmap_blocks(&ty, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, Y, R, CIN, kDwBK, CINT / 64))
    return cudaErrorInvalidValue;
#else
  if (!tmap16(&tdz, dZ, R, HH, 64, kDwBK) || !tmap16(&ty, Y, R, CIN, 64, kDwBK))
    return cudaErrorInvalidValue;
#endif
  k_tc16_dw<CINT, HH><<<nchunk * (CIN / CINT), 384, Cfg::SMEM, s>>>(tdz, ty, part, (int32_t)R, rows,
                                                               CIN);
  return cudaGetLastError();
}

}  // namespace

cudaError_t tc16_weights(const float* W, int CIN, int H, void* Bt16, void* B16, cudaStream_t s,
                         int* launches) {
  count_launch(launches);
  k_w16<<<cdiv((int64_t)CIN * H, 256), 256, 0, s>>>(W, CIN, H, static_cast<bf16*>(Bt16),
                                                     static_cast<bf16*>(B16));
  return cudaGetLastError();
}

cudaError_t tc16_gemm_rows(const void* A, const void* B, void* C, int64_t M, int N, int K,
                           cudaStream_t s, int* launches) {
  count_launch(launches);
  if (K % kBK) return cudaErrorInvalidValue;
  switch (N) {
    case 64: return rows16_n<64>(A, B, C, M, K, s);
    case 128: return rows16_n<128>(A, B, C, M, K, s);
    case 256: return rows16_n<256>(A, B, C, M, K, s);
    default: return cudaErrorInvalidValue;
  }
}

size_t tc16_dw_partial_floats(int64_t R, int CIN) {
  return (size_t)dw16_chunks(R, CIN) * 256 * CIN;
}

cudaError_t tc16_gemm_dw(const void* Y, const void* dZ, float* dW, int64_t R, int CIN, int H,
                         float* part, cudaStream_t s, int* launches) {
  count_launch(launches, 2);
  int nchunk = dw16_chunks(R, CIN);
  int rows = (int)((R + nchunk - 1) / nchunk);
  rows = (rows + kDwBK - 1) / kDwBK * kDwBK;
  nchunk = (int)((R + rows - 1) / rows);
  cudaError_t e;
  if (H != 128 && H != 256) return cudaErrorInvalidValue;
  switch (CIN) {
    case 64: e = H == 256 ? dw16_c<64, 256>(Y, dZ, part, nchunk, R, rows, CIN, s)
                          : dw16_c<64, 128>(Y, dZ, part, nchunk, R, rows, CIN, s); break;
    case 128:
    case 256: e = H == 256 ? dw16_c<128, 256>(Y, dZ, part, nchunk, R, rows, CIN, s)
                           : dw16_c<128, 128>(Y, dZ, part, nchunk, R, rows, CIN, s); break;
    default: return cudaErrorInvalidValue;
  }
  if (e != cudaSuccess) return e;
  k_dw16_reduce<<<dw_reduce_blocks((int64_t)H * CIN), 256, 0, s>>>(part, nchunk, CIN, H, dW);
  return cudaGetLastError();
}

}  // namespace mars
