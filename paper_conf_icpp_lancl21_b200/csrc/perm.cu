// a4: corruption permutation (Eq. 2; reading c12).
//
// pi_g = node indices of graph g sorted ascending by (key_i, i) with
// key_i = sm64(k_g ^ i), k_g = sm64(sm64(sm64(seed) ^ step) ^ (pair_base + g)).
// Instead of a comparison sort, every node's final position is its exact rank:
// keys are uniform 64-bit hashes, so bucketing by the top bits (≈2-4 keys per
// bucket) plus an in-bucket comparison count gives the same total order as a
// full sort in O(N) parallel work -- no global sort, no per-graph serialisation.
//   k_perm_keys    key, bucket id, bucket histogram (atomic int: deterministic)
//   scan           bucket starts (graph g's buckets start at node_off[g])
//   k_perm_scatter bucket membership lists (order arbitrary)
//   k_perm_rank    pos = bucket start + #{j in bucket: (key_j, j) < (key_i, i)}
// The X~ = X[pi] gather itself is fused into the first SpMM (spmm.cu).
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

__global__ void k_perm_keys(const int32_t* __restrict__ node_graph,
                            const int32_t* __restrict__ node_off,
                            const int64_t* __restrict__ pair_off,
                            const int32_t* __restrict__ bucket_off,
                            const int32_t* __restrict__ bucket_log2, int32_t Nt, uint64_t seed,
                            const StepParams* __restrict__ sp, uint64_t* __restrict__ keys,
                            int32_t* __restrict__ bucket, int32_t* __restrict__ bcnt) {
  int32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= Nt) return;
  int32_t g = node_graph[i];
  uint64_t kg = sm64(sm64(sm64(seed) ^ sp->step_index) ^ (uint64_t)(sp->pair_base + pair_off[g]));
  uint64_t key = sm64(kg ^ (uint64_t)(i - node_off[g]));
  int lb = bucket_log2[g];
  int32_t b = bucket_off[g] + (lb ? (int32_t)(key >> (64 - lb)) : 0);
  keys[i] = key;
  bucket[i] = b;
  atomicAdd(&bcnt[b], 1);
}

__global__ void k_perm_scatter(const int32_t* __restrict__ bucket, int32_t Nt,
                               int32_t* __restrict__ bcur, int32_t* __restrict__ members) {
  int32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= Nt) return;
  members[atomicAdd(&bcur[bucket[i]], 1)] = i;
}

__global__ void k_perm_rank(const uint64_t* __restrict__ keys, const int32_t* __restrict__ bucket,
                            const int32_t* __restrict__ bstart,
                            const int32_t* __restrict__ members, int32_t Nt,
                            int32_t* __restrict__ perm_global) {
  int32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= Nt) return;
  uint64_t k = keys[i];
  int32_t b = bucket[i];
  int32_t q0 = bstart[b], q1 = bstart[b + 1];
  int32_t r = 0;
  for (int32_t q = q0; q < q1; ++q) {
    int32_t j = members[q];
    uint64_t kj = keys[j];
    r += (kj < k) || (kj == k && j < i);
  }
  perm_global[q0 + r] = i;  // X~ row (q0 + r) takes X row i
}

// The permutation of one graph per CTA (graphs of up to 2^15 nodes): bucket
// counts, starts and cursors and the bucket members live in shared memory,
// the phases are separated by __syncthreads instead of kernel boundaries, and
// the CTA finishes with colperm over its graph's CSR entries (block-diagonal:
// they reference only this graph's nodes).  Keys, buckets, starts and ranks
// are those of the kernels above (graph g's buckets start at node_off[g]), so
// the permutation is the same.
#ifndef MARS_PERM_GRAPH_MAXN
#define MARS_PERM_GRAPH_MAXN 4096   // largest graph (nodes) the per-graph kernel takes
#endif
constexpr int kPgT = 1024;
constexpr int kPgMaxLog2 = 13;                 // 2^13 buckets, 2^15 nodes per graph
__global__ void __launch_bounds__(kPgT) k_perm_graph(
    const int32_t* __restrict__ node_off, const int64_t* __restrict__ pair_off,
    const int32_t* __restrict__ bucket_log2, uint64_t seed, const StepParams* __restrict__ sp,
    uint64_t* __restrict__ keys, int32_t* __restrict__ perm_global,
    const int32_t* __restrict__ rowptr, const int32_t* __restrict__ colind,
    int32_t* __restrict__ colperm) {
  extern __shared__ int32_t psm[];
  __shared__ int32_t wsum[kPgT / 32];
  const int g = blockIdx.x, tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int32_t off = node_off[g], N = node_off[g + 1] - off;
  const int lb = bucket_log2[g];
  const int nbk = 1 << lb;
  int32_t* bst = psm;                  // [nbk + 1] bucket starts (graph-local)
  int32_t* bcur = psm + nbk + 1;       // [nbk]     counts, then cursors
  int32_t* mem = bcur + nbk;           // [N]       members of each bucket
  const uint64_t kg = sm64(sm64(sm64(seed) ^ sp->step_index) ^ (uint64_t)(sp->pair_base + pair_off[g]));
  for (int b = tid; b < nbk; b += kPgT) bcur[b] = 0;
  __syncthreads();
  for (int32_t i = tid; i < N; i += kPgT) {
    const uint64_t key = sm64(kg ^ (uint64_t)i);
    keys[off + i] = key;
    atomicAdd(&bcur[lb ? (int32_t)(key >> (64 - lb)) : 0], 1);
  }
  __syncthreads();
  // exclusive scan of the counts: thread t owns buckets [t per, (t + 1) per)
  const int per = (nbk + kPgT - 1) / kPgT;
  const int b0 = min(tid * per, nbk), b1 = min(b0 + per, nbk);
  int32_t run = 0;
  for (int b = b0; b < b1; ++b) run += bcur[b];
  int32_t inc = run;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int32_t y = __shfl_up_sync(kFull, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) wsum[wid] = inc;
  __syncthreads();
  int32_t base = inc - run;
  for (int k = 0; k < wid; ++k) base += wsum[k];
  for (int b = b0; b < b1; ++b) {
    const int32_t c = bcur[b];
    bst[b] = base;
    bcur[b] = base;
    base += c;
  }
  if (tid == 0) bst[nbk] = N;
  __syncthreads();
  for (int32_t i = tid; i < N; i += kPgT) {
    const uint64_t key = keys[off + i];
    mem[atomicAdd(&bcur[lb ? (int32_t)(key >> (64 - lb)) : 0], 1)] = i;
  }
  __syncthreads();
  for (int32_t i = tid; i < N; i += kPgT) {
    const uint64_t k = keys[off + i];
    const int32_t b = lb ? (int32_t)(k >> (64 - lb)) : 0;
    const int32_t q0 = bst[b], q1 = bst[b + 1];
    int32_t r = 0;
    for (int32_t q = q0; q < q1; ++q) {
      const int32_t j = mem[q];
      const uint64_t kj = keys[off + j];
      r += (kj < k) || (kj == k && j < i);
    }
    perm_global[off + q0 + r] = off + i;   // X~ row (off + q0 + r) takes X row off + i
  }
  if (!colperm) return;
  __syncthreads();                         // this CTA's perm entries are complete
  const int32_t e0 = rowptr[off], e1 = rowptr[off + N];
  for (int32_t k = e0 + tid; k < e1; k += kPgT) colperm[k] = perm_global[colind[k]];
}

}  // namespace

cudaError_t launch_perm_graph(const GraphDev& g, uint64_t seed, const StepParams* sp,
                              const PermWork& w, int32_t* perm_global, int32_t* colperm,
                              cudaStream_t s, int* launches) {
  // measured (tools/step_series.py, captured replays): Inception x16 (3.4k
  // nodes per graph) 0.501 -> 0.491 ms per step; GNMT x16 (6.8k-16.7k) +1 %,
  // BERT x8 (15k) +2 %: one CTA per graph only pays for small graphs
  if (g.G < 1 || g.max_bucket_log2 > kPgMaxLog2 || g.max_graph_nodes > MARS_PERM_GRAPH_MAXN)
    return cudaErrorNotSupported;
  const int nbk = 1 << g.max_bucket_log2;
  const size_t smem = sizeof(int32_t) * ((size_t)2 * nbk + 1 + (size_t)g.max_graph_nodes);
  static size_t attr = 0;
  if (smem > 48 * 1024 && smem > attr) {
    cudaError_t e = cudaFuncSetAttribute(k_perm_graph, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return e;
    attr = smem;
  }
  count_launch(launches);
  k_perm_graph<<<g.G, kPgT, smem, s>>>(g.node_off, g.pair_off, g.bucket_log2, seed, sp, w.keys,
                                       perm_global, g.rowptr, g.colind, colperm);
  return cudaGetLastError();
}

cudaError_t launch_perm(const GraphDev& g, uint64_t seed, const StepParams* sp, const PermWork& w,
                        int32_t* perm_global, cudaStream_t s, int* launches) {
  cudaError_t e;
  if ((e = cudaMemsetAsync(w.bcnt, 0, sizeof(int32_t) * (size_t)(g.nbuckets + 1), s))) return e;
  unsigned nb = cdiv(g.Nt, 256);
  k_perm_keys<<<nb, 256, 0, s>>>(g.node_graph, g.node_off, g.pair_off, g.bucket_off, g.bucket_log2, g.Nt,
                                 seed, sp, w.keys, w.bucket, w.bcnt);
  count_launch(launches);
  if ((e = scan_exclusive_i32(w.bcnt, w.bstart, g.nbuckets, w.scan_tmp, s, launches))) return e;
  if ((e = cudaMemcpyAsync(w.bcur, w.bstart, sizeof(int32_t) * (size_t)g.nbuckets,
                           cudaMemcpyDeviceToDevice, s)))
    return e;
  k_perm_scatter<<<nb, 256, 0, s>>>(w.bucket, g.Nt, w.bcur, w.members);
  k_perm_rank<<<nb, 256, 0, s>>>(w.keys, w.bucket, w.bstart, w.members, g.Nt, perm_global);
  count_launch(launches, 2);
  return cudaGetLastError();
}

}  // namespace mars
