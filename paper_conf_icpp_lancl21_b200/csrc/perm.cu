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

}  // namespace

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
