// Host-side helpers shared by the tcgen05 GEMM translation units
// (gemm_tc3h.cu: 3xFP16 fp32 path; gemm_tc16.cu: bf16 path): TMA tensor-map
// encoding, the SM count, the shape support condition and the split-K chunking
// of the weight-gradient GEMMs (a12, dW_l = Y_lᵀ dZ_l; Eq. 1).
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>

#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

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

int g_sms = 0;

}  // namespace

// Row-major [rows × cols] matrix, {box_cols, box_rows} boxes, swizzle `swz`.
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
  // a row narrower than one block (C_in = 16 fp32): one partial block; the
  // box's remaining columns and blocks are zero-filled
  cuuint64_t dims[3] = {std::min<cuuint64_t>(bc, (cuuint64_t)cols), (cuuint64_t)rows,
                        std::max<cuuint64_t>(1, (cuuint64_t)cols / bc)};
  cuuint64_t strides[2] = {(cuuint64_t)cols * elem_bytes, 128};
  cuuint32_t box[3] = {(cuuint32_t)bc, (cuuint32_t)box_rows, (cuuint32_t)nblk};
  cuuint32_t es[3] = {1, 1, 1};
  return g_encode(m, dt, 3, const_cast<void*>(base), dims, strides, box, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) ==
         CUDA_SUCCESS;
}

int tc_num_sms() {
  if (!g_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
    if (!g_sms) g_sms = 148;
  }
  return g_sms;
}

bool tc_supported(int K_or_cin, int N_or_h) {
  return (N_or_h == 128 || N_or_h == 256) && (K_or_cin == 64 || K_or_cin == 128 || K_or_cin == 256);
}

// The 3xFP16 kernels also take the narrow widths of the tiny configuration
// (H in {32, 64}, C_in in {16, 32}) on zero-filled wider tiles.
bool tc3h_supported(int K_or_cin, int N_or_h) {
  const bool n = N_or_h == 32 || N_or_h == 64 || N_or_h == 128 || N_or_h == 256;
  const bool k = K_or_cin == 16 || K_or_cin == 32 || K_or_cin == 64 || K_or_cin == 128 ||
                 K_or_cin == 256;
  return n && k;
}

// Row chunks of the split-K weight gradient so that chunks x C_in tiles is
// about one CTA per SM (C_in tiles of 128 columns, 64 for C_in = 64).
int tc_dw_chunks(int64_t R, int CIN) {
  const int tile = CIN >= 128 ? 128 : 64;
  const int ntile = std::max(1, CIN / tile);
  int64_t want = std::max<int64_t>(1, tc_num_sms() / ntile);
  int64_t maxc = std::max<int64_t>(1, R / 256);
  return (int)std::min(want, maxc);
}

size_t tc_dw_partial_floats(int64_t R, int CIN) {
  return (size_t)tc_dw_chunks(R, CIN) * 256 * CIN;
}

}  // namespace mars
