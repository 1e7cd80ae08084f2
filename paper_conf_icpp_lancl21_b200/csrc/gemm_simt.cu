// a6 / a12: the dense transforms of Eq. 1 (Z_l = Y_l · W_l) and their
// backward (dY_l = dZ_l · W_lᵀ, dW_l = Y_lᵀ · dZ_l) in fp32 FFMA -- the fp32
// reference-precision path (reading c18) for the widths the tcgen05 kernels do
// not cover (H in {32, 64}, C_in in {16, 32}: the tiny configuration) and for
// MARS_GEMM_SIMT A/B runs; plain tf32 tensor cores could not meet the 1e-5
// bar.
//
// gemm_nn / gemm_nt: 128-row CTA tiles, the whole W tile column block staged
// through shared memory 16 K-rows at a time, 8×8 (or 8×4 / 4×4) register
// micro-tiles.  gemm_tn (dW): reduction over the R = 2ΣN stacked rows, split
// into row chunks; each thread accumulates 64-row blocks in fp32 and flushes
// them into fp64 accumulators, chunk partials are combined in a fixed order
// (deterministic, fp64), so the cancellation between the positive and the
// corrupted branch does not eat the fp32 budget.
#include <algorithm>

#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

constexpr int kBK = 16;
constexpr int kThreads = 256;

// C[M×N] = A[M×K] · op(B); op(B) = B [K×N] (BT = false) or Bᵀ with B [N×K].
template <int BM, int BN, int TM, int TN, bool BT>
__global__ void __launch_bounds__(kThreads)
k_gemm(const float* __restrict__ A, const float* __restrict__ B, float* __restrict__ C,
       int64_t M, int N, int K) {
  static_assert((BM / TM) * (BN / TN) == kThreads, "thread tiling");
  static_assert(TM % 4 == 0 && TN % 4 == 0, "float4 micro-tiles");
  __shared__ __align__(16) float As[kBK][BM];
  __shared__ __align__(16) float Bs[kBK][BN];
  constexpr int TX = BN / TN;
  constexpr int GM = TM / 4, GN = TN / 4;          // float4 groups per thread
  const int tid = threadIdx.x;
  const int tx = tid % TX, ty = tid / TX;
  const int64_t m0 = (int64_t)blockIdx.x * BM;
  const int n0 = blockIdx.y * BN;
  float acc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; ++i)
#pragma unroll
    for (int j = 0; j < TN; ++j) acc[i][j] = 0.f;

  for (int k0 = 0; k0 < K; k0 += kBK) {
    for (int e = tid; e < BM * kBK / 4; e += kThreads) {
      int r = e / (kBK / 4), c4 = e % (kBK / 4);
      int64_t gm = m0 + r;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (gm < M) v = __ldg(reinterpret_cast<const float4*>(A + gm * K + k0) + c4);
      As[c4 * 4 + 0][r] = v.x;
      As[c4 * 4 + 1][r] = v.y;
      As[c4 * 4 + 2][r] = v.z;
      As[c4 * 4 + 3][r] = v.w;
    }
    if (!BT) {
      for (int e = tid; e < kBK * BN / 4; e += kThreads) {
        int r = e / (BN / 4), c4 = e % (BN / 4);
        *reinterpret_cast<float4*>(&Bs[r][c4 * 4]) =
            __ldg(reinterpret_cast<const float4*>(B + (int64_t)(k0 + r) * N + n0) + c4);
      }
    } else {
      for (int e = tid; e < BN * kBK / 4; e += kThreads) {
        int r = e / (kBK / 4), c4 = e % (kBK / 4);
        float4 v = __ldg(reinterpret_cast<const float4*>(B + (int64_t)(n0 + r) * K + k0) + c4);
        Bs[c4 * 4 + 0][r] = v.x;
        Bs[c4 * 4 + 1][r] = v.y;
        Bs[c4 * 4 + 2][r] = v.z;
        Bs[c4 * 4 + 3][r] = v.w;
      }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBK; ++k) {
      float a[TM], b[TN];
#pragma unroll
      for (int g = 0; g < GM; ++g) {
        float4 v = *reinterpret_cast<const float4*>(&As[k][g * (BM / GM) + ty * 4]);
        a[g * 4 + 0] = v.x; a[g * 4 + 1] = v.y; a[g * 4 + 2] = v.z; a[g * 4 + 3] = v.w;
      }
#pragma unroll
      for (int g = 0; g < GN; ++g) {
        float4 v = *reinterpret_cast<const float4*>(&Bs[k][g * (BN / GN) + tx * 4]);
        b[g * 4 + 0] = v.x; b[g * 4 + 1] = v.y; b[g * 4 + 2] = v.z; b[g * 4 + 3] = v.w;
      }
#pragma unroll
      for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int gi = 0; gi < GM; ++gi)
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      int64_t gm = m0 + gi * (BM / GM) + ty * 4 + i;
      if (gm >= M) continue;
#pragma unroll
      for (int gj = 0; gj < GN; ++gj) {
        float4 v = make_float4(acc[gi * 4 + i][gj * 4 + 0], acc[gi * 4 + i][gj * 4 + 1],
                               acc[gi * 4 + i][gj * 4 + 2], acc[gi * 4 + i][gj * 4 + 3]);
        *reinterpret_cast<float4*>(C + gm * N + n0 + gj * (BN / GN) + tx * 4) = v;
      }
    }
}

template <bool BT>
cudaError_t gemm_dispatch(const float* A, const float* B, float* C, int64_t M, int N, int K,
                          cudaStream_t s) {
  if (K % kBK) return cudaErrorInvalidValue;
  if (N >= 128 && N % 128 == 0) {
    dim3 grid(cdiv(M, 128), N / 128);
    k_gemm<128, 128, 8, 8, BT><<<grid, kThreads, 0, s>>>(A, B, C, M, N, K);
  } else if (N == 64) {
    dim3 grid(cdiv(M, 128), 1);
    k_gemm<128, 64, 8, 4, BT><<<grid, kThreads, 0, s>>>(A, B, C, M, N, K);
  } else if (N == 32) {
    dim3 grid(cdiv(M, 128), 1);
    k_gemm<128, 32, 4, 4, BT><<<grid, kThreads, 0, s>>>(A, B, C, M, N, K);
  } else {
    return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

// ---------------------------------------------------------------- dW = Aᵀ B
constexpr int kTnBM = 64;
constexpr int kTnFlush = 4;     // BK tiles (64 rows) per fp32 -> fp64 flush

template <int BN, int TN>
__global__ void __launch_bounds__(kThreads)
k_gemm_tn(const float* __restrict__ A, const float* __restrict__ B, double* __restrict__ part,
          int64_t R, int M, int N, int64_t rows_per_split) {
  constexpr int TM = 4;
  constexpr int TX = BN / TN, TY = kTnBM / TM;
  static_assert(TX * TY == kThreads, "thread tiling");
  __shared__ __align__(16) float As[kBK][kTnBM];
  __shared__ __align__(16) float Bs[kBK][BN];
  const int tid = threadIdx.x;
  const int tx = tid % TX, ty = tid / TX;
  const int m0 = blockIdx.x * kTnBM, n0 = blockIdx.y * BN;
  const int64_t r0 = (int64_t)blockIdx.z * rows_per_split;
  const int64_t r1 = min(R, r0 + rows_per_split);
  float acc[TM][TN];
  double dacc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; ++i)
#pragma unroll
    for (int j = 0; j < TN; ++j) { acc[i][j] = 0.f; dacc[i][j] = 0.0; }
  int tile = 0;
  for (int64_t k0 = r0; k0 < r1; k0 += kBK, ++tile) {
    for (int e = tid; e < kBK * kTnBM; e += kThreads) {
      int r = e / kTnBM, c = e % kTnBM;
      int64_t gr = k0 + r;
      As[r][c] = (gr < r1 && m0 + c < M) ? __ldg(A + gr * M + m0 + c) : 0.f;
    }
    for (int e = tid; e < kBK * BN; e += kThreads) {
      int r = e / BN, c = e % BN;
      int64_t gr = k0 + r;
      Bs[r][c] = (gr < r1 && n0 + c < N) ? __ldg(B + gr * N + n0 + c) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBK; ++k) {
      float a[TM], b[TN];
#pragma unroll
      for (int i = 0; i < TM; ++i) a[i] = As[k][ty * TM + i];
#pragma unroll
      for (int j = 0; j < TN; ++j) b[j] = Bs[k][tx * TN + j];
#pragma unroll
      for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
    if ((tile % kTnFlush) == kTnFlush - 1) {
#pragma unroll
      for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) { dacc[i][j] += (double)acc[i][j]; acc[i][j] = 0.f; }
    }
  }
  double* out = part + (int64_t)blockIdx.z * M * N;
#pragma unroll
  for (int i = 0; i < TM; ++i) {
    int m = m0 + ty * TM + i;
    if (m >= M) continue;
#pragma unroll
    for (int j = 0; j < TN; ++j) {
      int n = n0 + tx * TN + j;
      if (n < N) out[(int64_t)m * N + n] = dacc[i][j] + (double)acc[i][j];
    }
  }
}

__global__ void k_reduce_splits(const double* __restrict__ part, int nsplit, int64_t MN,
                                float* __restrict__ out) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= MN) return;
  double t = 0.0;
  for (int s = 0; s < nsplit; ++s) t += part[(int64_t)s * MN + e];
  out[e] = (float)t;
}

int tn_nsplit(int64_t R, int M, int N) {
  int bn = N >= 128 ? 128 : N;
  int tiles = (int)(cdiv(M, kTnBM) * cdiv(N, bn));
  int64_t want = std::max<int64_t>(1, (2 * 148 + tiles - 1) / tiles);
  int64_t maxs = std::max<int64_t>(1, R / 256);
  return (int)std::min(want, maxs);
}

}  // namespace

cudaError_t gemm_nn(const float* A, const float* B, float* C, int64_t M, int N, int K,
                    cudaStream_t s, int* launches) {
  count_launch(launches);
  return gemm_dispatch<false>(A, B, C, M, N, K, s);
}

cudaError_t gemm_nt(const float* A, const float* B, float* C, int64_t M, int N, int K,
                    cudaStream_t s, int* launches) {
  count_launch(launches);
  return gemm_dispatch<true>(A, B, C, M, N, K, s);
}

size_t gemm_tn_partial_floats(int64_t R, int M, int N) {
  return (size_t)tn_nsplit(R, M, N) * (size_t)M * (size_t)N;
}

// out[M×N] = Aᵀ B with A [R×M], B [R×N]; partial: gemm_tn_partial_floats doubles.
cudaError_t gemm_tn(const float* A, const float* B, float* out, int64_t R, int M, int N,
                    double* partial, cudaStream_t s, int* launches) {
  int ns = tn_nsplit(R, M, N);
  int64_t rows = cdiv(R, ns);
  rows = (rows + kBK - 1) / kBK * kBK;
  ns = (int)cdiv(R, rows);
  if (N >= 128) {
    dim3 grid(cdiv(M, kTnBM), cdiv(N, 128), ns);
    k_gemm_tn<128, 8><<<grid, kThreads, 0, s>>>(A, B, partial, R, M, N, rows);
  } else if (N == 64) {
    dim3 grid(cdiv(M, kTnBM), 1, ns);
    k_gemm_tn<64, 4><<<grid, kThreads, 0, s>>>(A, B, partial, R, M, N, rows);
  } else if (N == 32) {
    dim3 grid(cdiv(M, kTnBM), 1, ns);
    k_gemm_tn<32, 2><<<grid, kThreads, 0, s>>>(A, B, partial, R, M, N, rows);
  } else {
    return cudaErrorInvalidValue;
  }
  int64_t MN = (int64_t)M * N;
  k_reduce_splits<<<cdiv(MN, 256), 256, 0, s>>>(partial, ns, MN, out);
  count_launch(launches, 2);
  return cudaGetLastError();
}

}  // namespace mars
