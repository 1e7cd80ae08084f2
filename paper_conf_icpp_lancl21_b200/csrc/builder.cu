// a1-a3: CSR / normalisation builder for Â_n = D̂^-1/2 (A ∨ Aᵀ + I) D̂^-1/2
// (Eq. 1; Â = A + I, D̂_ii = Σ_j Â_ij; readings c1-c4).
//
// Load-time only (the op graph is static across pre-training steps).  All
// steps are deterministic so the result is bit-exact against the oracle:
//   1. count (with duplicates) row lengths of S = {(u,v),(v,u): u->v, u≠v} ∪ {(i,i)}
//   2. exclusive scan -> segment offsets
//   3. scatter every member of S into its row segment (atomic cursor; order
//      inside a segment is arbitrary)
//   4. per row: stable rank-sort + dedupe (warp kernel for rows ≤ 32, block
//      kernel for longer rows) -> unique counts = degrees
//   5. exclusive scan -> rowptr
//   6. compact colind; deg, dinv = f32(1/√d), vals = f32(1/√(d_i d_j)) in double.
#include <climits>

#include "common.cuh"
#include "internal.cuh"

namespace mars {

// ---------------------------------------------------------------- scan
namespace {
constexpr int kScanT = 512;
constexpr int kScanIpt = 4;
constexpr int kScanTile = kScanT * kScanIpt;

__device__ __forceinline__ int32_t block_excl_scan(int32_t x, int32_t* total) {
  __shared__ int32_t warp_tot[kScanT / 32];
  int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int32_t inc = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int32_t y = __shfl_up_sync(kFull, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) warp_tot[wid] = inc;
  __syncthreads();
  if (wid == 0) {
    int32_t t = lane < kScanT / 32 ? warp_tot[lane] : 0;
    int32_t ti = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int32_t y = __shfl_up_sync(kFull, ti, o);
      if (lane >= o) ti += y;
    }
    if (lane < kScanT / 32) warp_tot[lane] = ti - t;
    if (lane == kScanT / 32 - 1) *total = ti;
  }
  __syncthreads();
  int32_t r = warp_tot[wid] + inc - x;
  __syncthreads();
  return r;
}

__global__ void k_scan_tile(const int32_t* __restrict__ in, int32_t* __restrict__ out, int64_t n,
                            int32_t* __restrict__ block_sums) {
  __shared__ int32_t tot;
  int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanIpt;
  int32_t v[kScanIpt];
  int32_t local = 0;
#pragma unroll
  for (int k = 0; k < kScanIpt; ++k) {
    v[k] = (base + k < n) ? in[base + k] : 0;
    local += v[k];
  }
  int32_t run = block_excl_scan(local, &tot);
#pragma unroll
  for (int k = 0; k < kScanIpt; ++k) {
    if (base + k < n) out[base + k] = run;
    run += v[k];
  }
  if (threadIdx.x == 0) block_sums[blockIdx.x] = tot;
}

__global__ void k_scan_add(int32_t* __restrict__ out, int64_t n, const int32_t* __restrict__ off,
                           int64_t nb) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] += off[i / kScanTile];
  if (i == 0) out[n] = off[nb];
}

__global__ void k_scan_total(const int32_t* __restrict__ block_sums, int32_t* __restrict__ out,
                             int64_t n) {
  out[n] = block_sums[0];
}
}  // namespace

size_t scan_tmp_bytes(int64_t n) {
  size_t b = 0;
  while (n > kScanTile) {
    int64_t nb = (n + kScanTile - 1) / kScanTile;
    b += sizeof(int32_t) * (size_t)(2 * nb + 2);
    n = nb;
  }
  return b + 64;
}

// out[0..n) = exclusive scan of in, out[n] = total.  in may alias out.
cudaError_t scan_exclusive_i32(const int32_t* in, int32_t* out, int64_t n, void* tmp,
                               cudaStream_t s, int* launches) {
  int32_t* t = static_cast<int32_t*>(tmp);
  if (n <= kScanTile) {
    k_scan_tile<<<1, kScanT, 0, s>>>(in, out, n, t);
    k_scan_total<<<1, 1, 0, s>>>(t, out, n);
    count_launch(launches, 2);
    return cudaGetLastError();
  }
  int64_t nb = (n + kScanTile - 1) / kScanTile;
  int32_t* sums = t;
  int32_t* offs = t + nb + 1;
  k_scan_tile<<<(unsigned)nb, kScanT, 0, s>>>(in, out, n, sums);
  count_launch(launches);
  cudaError_t e = scan_exclusive_i32(sums, offs, nb, offs + nb + 1, s, launches);
  if (e != cudaSuccess) return e;
  k_scan_add<<<cdiv(n, 256), 256, 0, s>>>(out, n, offs, nb);
  count_launch(launches);
  return cudaGetLastError();
}

// ---------------------------------------------------------------- builder kernels
namespace {

// kRG lanes per row (mean directed out-degree ~1.7, mean |S| row ~4.4: a whole
// warp per row left most lanes idle; round 2 measured warp-per-row at ~2.4x
// the time of these kernels).
constexpr int kRG = 8;
constexpr int kRGW = 32 / kRG;          // rows per warp

// kRG lanes per directed-CSR row u.  Validates, and counts row lengths of S
// with duplicates (pass == 0) or scatters S into the row segments (pass == 1).
template <int kPass>
__global__ void k_count_scatter(BuilderIO io) {
  int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / kRG;
  int gl = threadIdx.x % kRG;
  if (w >= io.Nt) return;
  int32_t u = (int32_t)w;
  int32_t g = io.node_graph[u];
  int32_t off = io.node_off[g];
  int32_t Ng = io.node_off[g + 1] - off;
  int32_t ul = u - off;
  int64_t Eg = io.edge_off[g + 1] - io.edge_off[g];
  const int64_t* ip = io.indptr + off + g;           // graph g's indptr array
  int64_t b = ip[ul], e = ip[ul + 1];
  if (kPass == 0) {
    if (gl == 0) {
      bool bad = b > e || e > Eg || b < 0 || (ul == 0 && b != 0) || (ul == Ng - 1 && e != Eg);
      if (bad) atomicOr(io.err, 1);
      atomicAdd(&io.cnt[u], 1);                       // + I
    }
  } else if (gl == 0) {
    io.buf[atomicAdd(&io.cursor[u], 1)] = u;
  }
  if (b > e || e > Eg || b < 0) return;               // malformed row: only the diagonal
  const int32_t* idx = io.indices + io.edge_off[g];
  for (int64_t k = b + gl; k < e; k += kRG) {
    int32_t vl = idx[k];
    if (vl < 0 || vl >= Ng) {
      if (kPass == 0) atomicOr(io.err, 2);
      continue;
    }
    if (vl == ul) continue;                           // c2: drop input self-loops
    int32_t v = off + vl;
    if (kPass == 0) {
      atomicAdd(&io.cnt[u], 1);
      atomicAdd(&io.cnt[v], 1);
    } else {
      io.buf[atomicAdd(&io.cursor[u], 1)] = v;       // c1: u->v and v->u
      io.buf[atomicAdd(&io.cursor[v], 1)] = u;
    }
  }
}

// Stable rank sort + dedupe of one row of length L <= W held by W lanes
// (x = INT_MAX past L), in place at buf[base ..]; returns the unique count.
// gmask: the converged lanes (every group of the warp runs this together).
template <int W>
__device__ __forceinline__ int32_t sort_dedupe_row(int32_t* __restrict__ buf, int32_t base,
                                                   int32_t L, int32_t x, int gl, unsigned gmask,
                                                   int32_t* sm) {
  int r = 0;
#pragma unroll
  for (int j = 0; j < W; ++j) {
    int32_t y = __shfl_sync(gmask, x, j, W);
    r += (y < x) || (y == x && j < gl);
  }
  sm[r] = x;                                          // r is a bijection on the group's lanes
  __syncwarp(gmask);
  int32_t sv = sm[gl];
  int32_t pv = gl > 0 ? sm[gl - 1] : INT_MIN;
  bool uniq = gl < L && (gl == 0 || sv != pv);
  unsigned m = __ballot_sync(gmask, uniq);
  const int sh = (threadIdx.x & 31) & ~(W - 1);        // the group's first lane
  unsigned mine = W == 32 ? m : (m >> sh) & ((1u << W) - 1u);
  int pos = __popc(mine & ((1u << gl) - 1u));
  if (uniq) buf[base + pos] = sv;
  return __popc(mine);
}

// Rows of length <= 32, kRGW consecutive rows per warp: when all of them have
// length <= kRG, each kRG-lane group sorts its own row; otherwise the warp
// sorts them one after the other.  Longer rows go to big_rows for k_sort_big.
__global__ void k_sort_small(BuilderIO io, int32_t* big_rows, int32_t* nbig) {
  __shared__ int32_t sm[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32 * kRGW;  // first row
  if (w0 >= io.Nt) return;
  const int gi = lane / kRG, gl = lane % kRG;
  const int64_t ug = w0 + gi;
  int32_t Lg = -1, bg = 0;
  if (ug < io.Nt) {
    bg = io.off_dup[ug];
    Lg = io.off_dup[ug + 1] - bg;
  }
  const bool narrow = __all_sync(kFull, Lg <= kRG);   // absent rows count as narrow
  if (narrow) {
    int32_t x = gl < Lg ? io.buf[bg + gl] : INT_MAX;   // (the whole warp is converged here)
    int32_t c = sort_dedupe_row<kRG>(io.buf, bg, Lg < 0 ? 0 : Lg, x, gl, kFull, &sm[wib][gi * kRG]);
    if (ug < io.Nt && gl == 0) io.ucnt[ug] = c;
    return;
  }
  for (int k = 0; k < kRGW; ++k) {
    const int64_t u = w0 + k;
    if (u >= io.Nt) break;
    const int32_t base = __shfl_sync(kFull, bg, k * kRG);
    const int32_t L = __shfl_sync(kFull, Lg, k * kRG);
    if (L > 32) {
      if (lane == 0) big_rows[atomicAdd(nbig, 1)] = (int32_t)u;
      continue;
    }
    int32_t x = lane < L ? io.buf[base + lane] : INT_MAX;
    int32_t c = sort_dedupe_row<32>(io.buf, base, L, x, lane, kFull, sm[wib]);
    if (lane == 0) io.ucnt[u] = c;
    __syncwarp();
  }
}

// Rows longer than 32 (hubs): one block per row.  Stable rank by comparison
// against shared-memory tiles of the row (O(L^2 / threads)), sorted copy into
// buf2, then ordered unique-compaction back into buf.
constexpr int kBigT = 256;
constexpr int kBigTile = 2048;
__global__ void k_sort_big(BuilderIO io, const int32_t* big_rows, const int32_t* nbig) {
  __shared__ int32_t tile[kBigTile];
  __shared__ int32_t carry, wsum[kBigT / 32];
  int nb = *nbig;
  for (int rI = blockIdx.x; rI < nb; rI += gridDim.x) {
    int32_t u = big_rows[rI];
    int32_t base = io.off_dup[u];
    int32_t L = io.off_dup[u + 1] - base;
    const int32_t* a = io.buf + base;
    for (int p0 = 0; p0 < L; p0 += kBigT) {
      int p = p0 + threadIdx.x;
      int32_t x = p < L ? a[p] : INT_MAX;
      int r = 0;
      for (int q0 = 0; q0 < L; q0 += kBigTile) {
        int n = min(kBigTile, L - q0);
        __syncthreads();
        for (int t = threadIdx.x; t < n; t += kBigT) tile[t] = a[q0 + t];
        __syncthreads();
        for (int t = 0; t < n; ++t) {
          int32_t y = tile[t];
          r += (y < x) || (y == x && q0 + t < p);
        }
      }
      if (p < L) io.buf2[base + r] = x;
    }
    __syncthreads();
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    const int32_t* s = io.buf2 + base;
    for (int p0 = 0; p0 < L; p0 += kBigT) {
      int p = p0 + threadIdx.x;
      bool uq = p < L && (p == 0 || s[p] != s[p - 1]);
      int32_t val = p < L ? s[p] : 0;
      unsigned m = __ballot_sync(kFull, uq);
      int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
      if (lane == 0) wsum[wid] = __popc(m);
      __syncthreads();
      int pre = 0, tot = 0;
      for (int k = 0; k < kBigT / 32; ++k) {
        if (k < wid) pre += wsum[k];
        tot += wsum[k];
      }
      pre += __popc(m & ((1u << lane) - 1u));
      if (uq) io.buf[base + carry + pre] = val;
      __syncthreads();
      if (threadIdx.x == 0) carry += tot;
      __syncthreads();
    }
    if (threadIdx.x == 0) io.ucnt[u] = carry;
    __syncthreads();
  }
}

// kRG lanes per row: compact colind; deg, dinv, vals (c4: double, rounded once).
__global__ void k_compact(BuilderIO io, int32_t* __restrict__ colind, float* __restrict__ vals) {
  int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / kRG;
  int lane = threadIdx.x % kRG;
  if (w >= io.Nt) return;
  int32_t u = (int32_t)w;
  int32_t rb = io.rowptr[u], re = io.rowptr[u + 1];
  int32_t du = re - rb;
  double ddu = (double)du;
  if (lane == 0) {
    io.deg[u] = du;
    io.dinv[u] = __double2float_rn(__ddiv_rn(1.0, __dsqrt_rn(ddu)));
  }
  const int32_t* src = io.buf + io.off_dup[u];
  for (int k = lane; k < du; k += kRG) {
    int32_t v = src[k];
    colind[rb + k] = v;
    double dv = (double)(io.rowptr[v + 1] - io.rowptr[v]);
    vals[rb + k] = __double2float_rn(__ddiv_rn(1.0, __dsqrt_rn(__dmul_rn(ddu, dv))));
  }
}

}  // namespace

// Phase 1: counts, scatter, per-row sort/dedupe, rowptr.  The caller reads
// rowptr[Nt] (= nnz) and err before phase 2.
cudaError_t build_csr_phase1(const BuilderIO& io, cudaStream_t s) {
  cudaError_t e;
  int32_t* nbig = io.err + 1;
  int32_t* big_rows = io.cursor;  // reused after the scatter pass (cursor no longer needed)
  if ((e = cudaMemsetAsync(io.cnt, 0, sizeof(int32_t) * (size_t)(io.Nt + 1), s))) return e;
  if ((e = cudaMemsetAsync(io.err, 0, sizeof(int32_t) * 2, s))) return e;
  const unsigned gblocks = cdiv((int64_t)io.Nt * kRG, 256);   // kRG lanes per row
  k_count_scatter<0><<<gblocks, 256, 0, s>>>(io);
  if ((e = scan_exclusive_i32(io.cnt, io.off_dup, io.Nt, io.scan_tmp, s, nullptr))) return e;
  if ((e = cudaMemcpyAsync(io.cursor, io.off_dup, sizeof(int32_t) * (size_t)io.Nt,
                           cudaMemcpyDeviceToDevice, s)))
    return e;
  k_count_scatter<1><<<gblocks, 256, 0, s>>>(io);
  k_sort_small<<<gblocks, 256, 0, s>>>(io, big_rows, nbig);
  k_sort_big<<<592, kBigT, 0, s>>>(io, big_rows, nbig);
  if ((e = cudaGetLastError())) return e;
  return scan_exclusive_i32(io.ucnt, io.rowptr, io.Nt, io.scan_tmp, s, nullptr);
}

cudaError_t build_csr_phase2(const BuilderIO& io, int32_t* colind, float* vals, cudaStream_t s) {
  k_compact<<<cdiv((int64_t)io.Nt * kRG, 256), 256, 0, s>>>(io, colind, vals);
  return cudaGetLastError();
}

}  // namespace mars
