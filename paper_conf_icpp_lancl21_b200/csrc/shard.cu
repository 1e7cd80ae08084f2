// Row-sharded single graph: the exchange steps between the
// shards of one op graph that is too large (or too slow) for one GPU.
//
// A GCN layer Y = Â_n act(T) (Eq. 1) on shard p needs the rows of T
// owned by other shards wherever row i of Â_n has a column outside p's block
// (the halo).  Instead of packing halo rows and exchanging them with NCCL
// send/recv, every shard's activation buffers are mapped into every other
// shard's address space (same-process peer access, or CUDA IPC across
// processes) and the SpMM kernels gather remote rows directly by global column
// id over NVLink (spmm.cu, PeerSrc): the transfer is fused into the
// aggregation and overlaps it row by row.  What remains here is ordering and
// the two small per-graph reductions of the head:
//   - k_barrier: a device-side barrier across shards (release/acquire flags at
//     system scope in peer memory), placed wherever a shard is about to read
//     buffers its peers wrote in this step (Z_1, Z_2, dY_3, dY_2, head
//     partials, gradient partials);
//   - k_head_xsum: readout column sums (Eq. 4) and dv / loss (Eqs. 5-6) summed
//     over shards in rank order (deterministic, identical on every shard);
//   - k_grad_sum: the gradient reduction over shards in rank order (fp64), so
//     replicated Adam stays bit-identical across shards; the same kernel is
//     the data-parallel gradient exchange over peer memory (a13, mars_dp_*),
//     where every entry including the loss is a per-rank partial.
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

constexpr unsigned long long kBarrierTimeoutNs = 20ull * 1000 * 1000 * 1000;

__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// One warp: lane q < P signals shard q and waits for shard q's signal.
__global__ void k_barrier(const __grid_constant__ ShardSync s) {
  const int q = threadIdx.x;
  const unsigned long long e = *s.epoch + 1;
  if (q < s.P) {
    __threadfence_system();                      // this shard's prior writes, visible system-wide
    st_release_sys(s.flags[q] + s.me, e);
    const unsigned long long* mine = s.flags[s.me] + q;
    const unsigned long long t0 = globaltimer();
    while (ld_acquire_sys(mine) < e) {
      if (globaltimer() - t0 > kBarrierTimeoutNs) {
        atomicExch(s.err, 1);
        break;
      }
      __nanosleep(64);
    }
  }
  __syncwarp();
  if (q == 0) *s.epoch = e;
}

// grid (H/32 + 1): block b < H/32 sums 32 columns over shards; the last block
// sums the loss slot.  Rank order, fp64.
__global__ void k_head_xsum(const __grid_constant__ PeerPtrs x, int P, int H, int mode,
                            const int32_t* __restrict__ gsize, double* __restrict__ outd,
                            float* __restrict__ outf, double* __restrict__ loss_g) {
  const int c = blockIdx.x * 32 + threadIdx.x;
  if (blockIdx.x * 32 >= H) {
    if (threadIdx.x == 0 && loss_g) {
      double t = 0.0;
      for (int p = 0; p < P; ++p) t += static_cast<const double*>(x.p[p])[H];
      *loss_g = t;
    }
    return;
  }
  double t = 0.0;
  for (int p = 0; p < P; ++p) t += static_cast<const double*>(x.p[p])[c];
  if (mode == 0) t = 1.0 / (1.0 + exp(-(t / (double)gsize[0])));
  outd[c] = t;
  outf[c] = (float)t;
}

__global__ void k_grad_sum(const __grid_constant__ PeerPtrs g, int P, int me, int64_t n,
                           int64_t keep_b, int64_t keep_e, int sum_last, float* __restrict__ out) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  if ((k >= keep_b && k < keep_e) || (!sum_last && k == n - 1)) {
    out[k] = static_cast<const float*>(g.p[me])[k];
    return;
  }
  double t = 0.0;
  for (int p = 0; p < P; ++p) t += (double)static_cast<const float*>(g.p[p])[k];
  out[k] = (float)t;
}

}  // namespace

cudaError_t launch_shard_barrier(const ShardSync& s, cudaStream_t st, int* launches) {
  count_launch(launches);
  k_barrier<<<1, 32, 0, st>>>(s);
  return cudaGetLastError();
}

cudaError_t launch_head_xsum(const PeerPtrs& x, int P, int H, int mode, const int32_t* gsize,
                             double* outd, float* outf, double* loss_g, cudaStream_t st,
                             int* launches) {
  count_launch(launches);
  k_head_xsum<<<H / 32 + 1, 32, 0, st>>>(x, P, H, mode, gsize, outd, outf, loss_g);
  return cudaGetLastError();
}

cudaError_t launch_grad_sum(const PeerPtrs& g, int P, int me, int64_t n, int64_t keep_b,
                            int64_t keep_e, int sum_last, float* out, cudaStream_t st,
                            int* launches) {
  count_launch(launches);
  k_grad_sum<<<cdiv(n, 256), 256, 0, st>>>(g, P, me, n, keep_b, keep_e, sum_last, out);
  return cudaGetLastError();
}

}  // namespace mars
