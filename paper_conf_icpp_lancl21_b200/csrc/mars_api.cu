// libmars.so runtime and C ABI (include/mars.h): handle management, graph-set
// ingest, workspaces, the per-step kernel schedule captured once
// into a CUDA Graph and replayed, NCCL data parallelism, test hooks.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/mars.h"
#include "common.cuh"
#include "internal.cuh"

using namespace mars;

namespace {

constexpr uint64_t kTagGraph = 0x4D41525347524150ULL;  // "MARSGRAP"
constexpr uint64_t kTagDgi = 0x4D41525344474931ULL;    // "MARSDGI1"
constexpr uint64_t kTagDead = 0xDEADDEADDEADDEADULL;
constexpr uint64_t kTagPlacer = 0x4D415253504C4331ULL;  // "MARSPLC1"
constexpr uint64_t kTagPpo = 0x4D41525350504F31ULL;     // "MARSPPO1"
constexpr int kChunkRows = 256;   // deterministic reduction chunk (rows, within one graph)

thread_local std::string g_err;

mars_status fail(mars_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

#define CK(call)                                                                   \
  do {                                                                             \
    cudaError_t e_ = (call);                                                       \
    if (e_ != cudaSuccess) {                                                       \
      cudaGetLastError();                                                          \
      return fail(e_ == cudaErrorMemoryAllocation ? MARS_ENOMEM : MARS_ECUDA,       \
                  "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
    }                                                                              \
  } while (0)

bool valid_F(int F) { return F == 16 || F == 32 || F == 64 || F == 128 || F == 256; }
bool valid_H(int H) { return H == 32 || H == 64 || H == 128 || H == 256; }

template <typename T>
cudaError_t dalloc(T** p, size_t n) {
  return cudaMalloc(reinterpret_cast<void**>(p), sizeof(T) * (n ? n : 1));
}

// Stream-ordered allocation from the device's default pool (graph sets are
// loaded and freed per batch when op graphs are streamed; the pool keeps the
// memory instead of returning it to the driver).
template <typename T>
cudaError_t palloc(T** p, size_t n, cudaStream_t s) {
  return cudaMallocAsync(reinterpret_cast<void**>(p), sizeof(T) * (n ? n : 1), s);
}

void pool_init(int device) {
  static std::mutex mu;
  static bool done[64] = {};
  std::lock_guard<std::mutex> lk(mu);
  if (device < 0 || device >= 64 || done[device]) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  cudaGetLastError();
  done[device] = true;
}

bool is_pinned(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeHost;
}

// ---------------------------------------------------------------- NCCL (dlopen)
struct NcclApi {
  bool tried = false, ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

bool nccl_load() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.tried) return g_nccl.ok;
  g_nccl.tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) return false;
  g_nccl.GetUniqueId = reinterpret_cast<decltype(g_nccl.GetUniqueId)>(dlsym(h, "ncclGetUniqueId"));
  g_nccl.CommInitRank = reinterpret_cast<decltype(g_nccl.CommInitRank)>(dlsym(h, "ncclCommInitRank"));
  g_nccl.AllReduce = reinterpret_cast<decltype(g_nccl.AllReduce)>(dlsym(h, "ncclAllReduce"));
  g_nccl.CommDestroy = reinterpret_cast<decltype(g_nccl.CommDestroy)>(dlsym(h, "ncclCommDestroy"));
  g_nccl.GetErrorString =
      reinterpret_cast<decltype(g_nccl.GetErrorString)>(dlsym(h, "ncclGetErrorString"));
  g_nccl.ok = g_nccl.GetUniqueId && g_nccl.CommInitRank && g_nccl.AllReduce && g_nccl.CommDestroy;
  return g_nccl.ok;
}

// ---------------------------------------------------------------- pinned staging
struct Pinned {
  std::mutex mu;
  void* p = nullptr;
  size_t cap = 0;
  void* get(size_t n) {
    if (n > cap) {
      if (p) cudaFreeHost(p);
      p = nullptr;
      cap = 0;
      size_t want = n + n / 4 + 4096;
      if (cudaMallocHost(&p, want) != cudaSuccess) return nullptr;
      cap = want;
    }
    return p;
  }
};
Pinned g_stage;

// ---------------------------------------------------------------- kernels local to the runtime
__global__ void k_node_graph(const int32_t* __restrict__ node_off, int G, int32_t Nt,
                             int32_t* __restrict__ node_graph) {
  int32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= Nt) return;
  int lo = 0, hi = G - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (node_off[mid] <= i) lo = mid; else hi = mid - 1;
  }
  node_graph[i] = lo;
}

// Xavier-uniform init (c14): w = f32((2u-1) b), u = (sm64(sm64(seed^tag)^idx) >> 40) 2^-24.
__global__ void k_xavier(float* __restrict__ p, int64_t n, uint64_t seed, uint64_t tag, float b) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint64_t base = sm64(seed ^ tag);
  double u = (double)(sm64(base ^ (uint64_t)i) >> 40) * (1.0 / 16777216.0);
  p[i] = __double2float_rn(__dmul_rn(__dsub_rn(__dmul_rn(2.0, u), 1.0), (double)b));
}

__global__ void k_gather_rowptr(const int32_t* __restrict__ rowptr,
                                const int32_t* __restrict__ node_off, int G,
                                int32_t* __restrict__ out) {
  int g = blockIdx.x * blockDim.x + threadIdx.x;
  if (g <= G) out[g] = rowptr[node_off[g]];
}

__global__ void k_fill(float* __restrict__ p, int64_t n, float v) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = v;
}

}  // namespace

// ---------------------------------------------------------------- handles
std::atomic<uint64_t> g_graph_uid{1};

struct mars_graph {
  uint64_t tag = kTagGraph;
  uint64_t uid = g_graph_uid.fetch_add(1);
  int device = 0;
  int G = 0, F = 0;
  int32_t Nt = 0;
  int64_t Et = 0, nnz = 0;
  std::vector<int32_t> h_node_off;
  std::vector<int64_t> h_nnz_off;
  int32_t *node_off = nullptr, *node_graph = nullptr, *rowptr = nullptr, *colind = nullptr;
  int32_t *deg = nullptr, *chunk_row = nullptr, *chunk_graph = nullptr, *graph_chunk = nullptr;
  int32_t *bucket_off = nullptr, *bucket_log2 = nullptr;
  float *vals = nullptr, *dinv = nullptr, *X = nullptr;
  int32_t* gsize = nullptr;
  int64_t* pair_off = nullptr;      // [G] global pair index offsets (c15), default 0..G-1
  GraphDev dev{};
  // Row-sharded graph (mars_graph_load_shard): dev is the
  // view of this shard's rows [row_begin, row_end) (local row ids, global
  // column ids, the whole X); dev_full the whole graph (corruption permutation).
  bool sharded = false;
  int32_t P = 1, me = 0, row_begin = 0, row_end = 0;
  int64_t halo_rows = 0, local_nnz = 0;
  std::vector<int32_t> starts;
  GraphDev dev_full{};
  int32_t *l_node_off = nullptr, *l_node_graph = nullptr, *l_chunk_row = nullptr,
          *l_chunk_graph = nullptr, *l_graph_chunk = nullptr;
  std::vector<void*> extra;         // long-row tables (pool memory)
  std::vector<int32_t> h_long[3];   // host copies: long rows, segment offsets, segment rows
  int64_t nnz_cap = 0;              // entries colind / vals can hold (mars_graph_reload)
  int64_t Et_load = 0;
  // Last use per stream: every step / encode that reads this graph records an
  // event on its stream, so mars_free waits for exactly those uses (not for the
  // whole device, which would serialise against other models' steps).
  mutable std::mutex use_mu;
  mutable std::vector<std::pair<cudaStream_t, cudaEvent_t>> uses;
  void note_use(cudaStream_t s) const {
    std::lock_guard<std::mutex> lk(use_mu);
    for (auto& u : uses)
      if (u.first == s) {
        cudaEventRecord(u.second, s);
        return;
      }
    cudaEvent_t e;
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) {
      cudaGetLastError();
      cudaStreamSynchronize(s);           // no event: wait for the stream instead
      return;
    }
    cudaEventRecord(e, s);
    uses.emplace_back(s, e);
  }
  ~mars_graph() {   // pool memory, freed on a private stream after the recorded uses
    for (auto& u : uses) {
      cudaEventSynchronize(u.second);
      cudaEventDestroy(u.second);
    }
    cudaStream_t fs = nullptr;
    if (cudaStreamCreateWithFlags(&fs, cudaStreamNonBlocking) != cudaSuccess) fs = nullptr;
    for (void* p : extra) cudaFreeAsync(p, fs);
    for (void* p : {(void*)node_off, (void*)node_graph, (void*)rowptr, (void*)colind, (void*)deg,
                    (void*)chunk_row, (void*)chunk_graph, (void*)graph_chunk, (void*)bucket_off,
                    (void*)bucket_log2, (void*)vals, (void*)dinv, (void*)X, (void*)gsize,
                    (void*)pair_off, (void*)l_node_off, (void*)l_node_graph, (void*)l_chunk_row,
                    (void*)l_chunk_graph, (void*)l_graph_chunk})
      if (p) cudaFreeAsync(p, fs);
    if (fs) cudaStreamDestroy(fs);
  }
  const GraphDev& perm_view() const { return sharded ? dev_full : dev; }
};

// Long rows of a view (degree > long_min, spmm.cu): host scan of its rowptr and
// the segment tables on the device (read-only; the fp32 partial-sum scratch
// the segments write belongs to each model's Workspace, so models stepping the
// same graph concurrently never share it).
// Everything on the loader's non-blocking stream `s` (no legacy-stream copies or
// cudaMalloc, which would wait for a model's step running concurrently).
static cudaError_t build_long_rows(mars_graph* gr, GraphDev& v, cudaStream_t s,
                                   bool* changed = nullptr) {
  const GraphDev old = v;
  if (changed) *changed = true;
  v.nlong = v.nseg = 0;
  v.long_min = 0x7fffffff;
  v.long_rows = v.long_seg = v.seg_row = nullptr;
  v.long_part = nullptr;
  if (v.Nt < 1) return cudaSuccess;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t per_slot = (int64_t)v.Nt / std::max(1, sms * 32);
  const int32_t long_min =
      (int32_t)std::min<int64_t>(kLongMax, std::max<int64_t>(kLongMin, kLongFactor * per_slot));
  {   // most graphs have no long row: 4 bytes back instead of the whole rowptr
    int32_t* dmax = nullptr;
    int32_t hmax = 0;
    cudaError_t e0 = cudaMallocAsync(&dmax, sizeof(int32_t), s);
    if (e0 == cudaSuccess) e0 = launch_max_degree(v.rowptr, v.Nt, dmax, s);
    if (e0 == cudaSuccess)
      e0 = cudaMemcpyAsync(&hmax, dmax, sizeof(int32_t), cudaMemcpyDeviceToHost, s);
    if (dmax) cudaFreeAsync(dmax, s);
    if (e0 == cudaSuccess) e0 = cudaStreamSynchronize(s);
    if (e0 != cudaSuccess) return e0;
    if (hmax <= long_min) {
      if (changed) *changed = old.nlong != 0;
      for (auto& h : gr->h_long) h.clear();
      return cudaSuccess;
    }
  }
  std::vector<int32_t> rp((size_t)v.Nt + 1);
  cudaError_t e = cudaMemcpyAsync(rp.data(), v.rowptr, sizeof(int32_t) * rp.size(),
                                  cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return e;
  v.long_min = long_min;
  std::vector<int32_t> rows, seg{0}, segrow;
  for (int32_t i = 0; i < v.Nt; ++i) {
    const int32_t d = rp[i + 1] - rp[i];
    if (d <= v.long_min) continue;
    const int32_t ns = (d + kLongSeg - 1) / kLongSeg;
    for (int32_t k = 0; k < ns; ++k) segrow.push_back((int32_t)rows.size());
    rows.push_back(i);
    seg.push_back(seg.back() + ns);
  }
  if (rows.empty()) {
    if (changed) *changed = old.nlong != 0;
    for (auto& h : gr->h_long) h.clear();
    return cudaSuccess;
  }
  if (old.nlong == (int32_t)rows.size() && old.long_min == long_min && gr->h_long[0] == rows &&
      gr->h_long[1] == seg && gr->h_long[2] == segrow) {   // reload: tables unchanged
    v = old;
    if (changed) *changed = false;
    return cudaSuccess;
  }
  gr->h_long[0] = rows;
  gr->h_long[1] = seg;
  gr->h_long[2] = segrow;
  auto up = [&](const std::vector<int32_t>& h, const int32_t** d) -> cudaError_t {
    void* p = nullptr;
    cudaError_t e2 = cudaMallocAsync(&p, sizeof(int32_t) * h.size(), s);
    if (e2 != cudaSuccess) return e2;
    gr->extra.push_back(p);
    *d = static_cast<const int32_t*>(p);
    return cudaMemcpyAsync(p, h.data(), sizeof(int32_t) * h.size(), cudaMemcpyHostToDevice, s);
  };
  if ((e = up(rows, &v.long_rows)) || (e = up(seg, &v.long_seg)) || (e = up(segrow, &v.seg_row)))
    return e;
  v.nlong = (int32_t)rows.size();
  v.nseg = seg.back();
  return cudaStreamSynchronize(s);   // the host vectors go out of scope
}

#ifndef MARS_PERM_GRAPH
#define MARS_PERM_GRAPH 1  // a4: one CTA per graph (launch_perm_graph)
#endif
#ifndef MARS_PERM_GRAPH_COLPERM
#define MARS_PERM_GRAPH_COLPERM 0   // colperm inside that kernel (16 CTAs) or over the whole GPU
#endif

struct Workspace {
  int32_t Nt = 0, G = 0, nchunks = 0, nbuckets = 0, F = 0, H = 0;
  int32_t Nperm = 0;      // rows of the permutation (the whole graph when row-sharded)
  int64_t nnz_perm = 0;   // entries of the permuted view (colperm)
  int32_t nlong = 0;      // long rows (dalpha slots of the backward aggregation)
  int32_t nseg = 0;       // long-row segments (long_part)
  float* long_part = nullptr;   // [nseg * 2 * 256] fp32 segment partial sums (spmm.cu)
  float *Y1 = nullptr, *Z[3] = {nullptr, nullptr, nullptr}, *Y23[2] = {nullptr, nullptr};
  float *dZ = nullptr, *dY = nullptr;
  int32_t* perm = nullptr;
  int32_t* colperm = nullptr;         // [nnz of the permuted view] pi[colind[k]] (layer 1)
  PermWork pw{};
  HeadWork hw{};
  double *slots[3] = {nullptr, nullptr, nullptr};
  double* tn_part = nullptr;
  size_t tn_part_n = 0;
  // 3xFP16 row GEMMs: scaled fp16 hi/lo splits + {t, 1/t} per layer
  void *h3_wt_hi[3] = {}, *h3_wt_lo[3] = {}, *h3_w_hi[3] = {}, *h3_w_lo[3] = {};
  float* h3_wsc[3] = {};
  float* h3_rsY[3] = {};              // [R] power-of-two row scales of Y_l (written by the SpMM)
  float* h3_rsdZ = nullptr;           // [R] ... of dZ_l (written by the head / backward SpMM)
  float* dw_part = nullptr;
  // bf16 path: bf16 weight copies (Wᵀ for the forward, W for dY), dW partials.
  // (Activation buffers are sized for fp32 and hold bf16 in that mode.)
  void *w16t[3] = {}, *w16[3] = {};
  float* dw16_part = nullptr;
  // NEXT-4 variants (contrast.cu): nb stacked blocks, K corruption samples,
  // materialised layer-1 inputs Xs [nb*Nt x F], per-sample pair offsets,
  // SAGE-GCN values (forward Â, backward Âᵀ), PReLU slope 1 for layer 1
  int32_t nb = 2, K = 1;
  bool has_xs = false;
  int64_t nnz_vals = 0;
  float* Xs = nullptr;
  int64_t* pair_off_k = nullptr;
  float *valsR = nullptr, *valsC = nullptr;
  float* one = nullptr;
  // SAGE-mean encoder (c38): U = [U_n; U_s] and V = [V_n; V_s] ([2 nb Nt x H]),
  // the redirected CSR (colS) and its three value arrays, G's row scales,
  // the six weight matrices' 3xFP16 splits
  float *sU = nullptr, *sV = nullptr;
  int32_t* sColS = nullptr;
  float *sVf = nullptr, *sVb = nullptr, *sVn = nullptr;
  float* rsG = nullptr;
  void *s3_wt_hi[6] = {}, *s3_wt_lo[6] = {}, *s3_w_hi[6] = {}, *s3_w_lo[6] = {};
  float* s3_wsc[6] = {};
  // SAGE-pool encoder (c40): per layer U_p = A W_p, the max aggregation, its
  // argmax and row scales; scratch U_s / V (forward) = dA_s / dA_p (backward),
  // dU_p and its row scales, a ones column (the pool-bias gradient), the nine
  // weight matrices' 3xFP16 splits
  float *pUP[3] = {}, *pAGG[3] = {}, *pRsAGG[3] = {};
  int32_t* pIDX[3] = {};
  float *pUS = nullptr, *pVV = nullptr, *pDUP = nullptr, *pRsDUP = nullptr, *pOnes = nullptr;
  void *p3_wt_hi[9] = {}, *p3_wt_lo[9] = {}, *p3_w_hi[9] = {}, *p3_w_lo[9] = {};
  float* p3_wsc[9] = {};
  std::vector<void*> owned;
  void release() {
    for (void* p : owned) cudaFree(p);
    owned.clear();
    *this = Workspace();
  }
};

struct mars_dgi {
  uint64_t tag = kTagDgi;
  mars_dgi_config cfg{};
  int F = 0, H = 0;
  int64_t P = 0;
  cudaStream_t own_stream = nullptr, stream = nullptr;
  float *params = nullptr, *adam_m = nullptr, *adam_v = nullptr, *grads = nullptr;
  double* guard_part = nullptr;      // [adam_guard_doubles()] finiteness / clip-norm partials
  AdamDev* adam_st = nullptr;        // device-resident Adam step count + bias corrections
  int32_t skipped_seen = 0;          // skipped updates already reported (MARS_ENUMERIC)
  StepParams* d_sp = nullptr;
  StepParams* h_sp = nullptr;       // pinned ring
  cudaEvent_t* sp_ev = nullptr;
  int sp_ring = 32, sp_next = 0;
  // asynchronous loss read-back (mars_dgi_enqueue_loss / mars_dgi_wait_loss):
  // pinned {loss, skipped count} slots, one event each, tickets modulo the ring
  struct LossSlot {
    float loss;
    int32_t skipped;
  };
  static constexpr int kLossRing = 16;
  LossSlot* loss_ring = nullptr;
  cudaEvent_t loss_ev[kLossRing] = {};
  int64_t loss_next = 0;
  Workspace ws;
  const mars_graph* ws_graph = nullptr;
  mars_contrastive ct{1, MARS_CORRUPT_PERMUTE, 0.f, MARS_READOUT_SIGMOID_MEAN, MARS_AGG_GCN,
                      MARS_LOSS_BCE};
  bool sage = false;                // MARS_ENCODER_SAGE (c38)
  bool pool = false;                // MARS_ENCODER_SAGE_POOL (c40)
  int ct_nb() const { return (ct.num_neg + 2) & ~1; }     // K + 1 blocks, rounded up to even
  bool ct_materialise() const {
    return sage || pool || ct.num_neg > 1 || ct.corruption != MARS_CORRUPT_PERMUTE;
  }
  bool capture = true;
  int gemm_impl = 0;                // 0 auto (tcgen05 3xFP16 when supported), 1 SIMT FFMA
  // Captured steps, one per (graph set, stream), least recently used evicted:
  // a loader that alternates a few graph handles (mars_graph_reload) replays
  // each handle's graph instead of launching the step's kernels eagerly.
  struct ExecEntry {
    uint64_t uid;
    cudaStream_t stream;
    cudaGraphExec_t exec;
    int64_t launches;
    uint64_t last;
  };
  static constexpr int kExecCache = 4;
  std::vector<ExecEntry> execs;
  uint64_t exec_clock = 0;
  uint64_t seen[kExecCache] = {};   // uids of recent steps (capture on a set's second step)
  int seen_next = 0;
  int64_t last_launches = 0;
  void drop_execs() {
    for (auto& e : execs) cudaGraphExecDestroy(e.exec);
    execs.clear();
  }
  ExecEntry* find_exec(uint64_t uid, cudaStream_t s) {
    for (auto& e : execs)
      if (e.uid == uid && e.stream == s) return &e;
    return nullptr;
  }
  bool seen_recently(uint64_t uid) const {
    for (uint64_t u : seen)
      if (u == uid) return true;
    return false;
  }
  void note_seen(uint64_t uid) {
    if (seen_recently(uid)) return;
    seen[seen_next] = uid;
    seen_next = (seen_next + 1) % kExecCache;
  }
  ExecEntry* add_exec(uint64_t uid, cudaStream_t s, cudaGraphExec_t ex, int64_t launches) {
    if ((int)execs.size() >= kExecCache) {
      auto lru = std::min_element(execs.begin(), execs.end(),
                                  [](const ExecEntry& a, const ExecEntry& b) { return a.last < b.last; });
      cudaGraphExecDestroy(lru->exec);
      execs.erase(lru);
    }
    execs.push_back(ExecEntry{uid, s, ex, launches, ++exec_clock});
    return &execs.back();
  }
  int32_t last_Nt = 0;              // node count of the last step's graph set (export hook)
  // keep_backward test hook: copies of dZ3, dZ2, dZ1 (kb_dZ[l]) and dY3, dY2
  // (kb_dY[l - 1]) of the last step, 2 * kb_rows rows each
  bool keep_bwd = false;
  void *kb_dZ[3] = {}, *kb_dY[2] = {};
  int64_t kb_rows = 0;              // rows per branch the buffers hold
  int32_t kb_valid_Nt = 0;          // last_Nt of the step that filled them (0: none)
  void kb_release() {
    for (void*& p : kb_dZ) { if (p) cudaFree(p); p = nullptr; }
    for (void*& p : kb_dY) { if (p) cudaFree(p); p = nullptr; }
    kb_rows = 0;
    kb_valid_Nt = 0;
  }
  ncclComm_t comm = nullptr;
  // Row-sharded graph: the shard this model is attached to,
  // its peer-visible buffers, and the peers' buffers once connected.
  struct Shard {
    const mars_graph* g = nullptr;
    uint64_t guid = 0;
    bool connected = false;
    unsigned long long* flags = nullptr;   // [kMaxShards] arrival slots (peer-visible)
    unsigned long long* epoch = nullptr;   // barrier counter (local)
    int32_t* err = nullptr;                // barrier timeout flag (local)
    double* xbuf = nullptr;                // [2][H+1] head exchange (peer-visible)
    void* dY2 = nullptr;                   // layer-2 dY (layer 3 uses ws.dY), peer-visible
    float* gsum = nullptr;                 // [P+1] gradients summed over shards
    ShardSync sync{};
    PeerRows z[2]{}, dy[2]{};
    PeerPtrs x[2]{}, grads{};
    std::vector<void*> ipc;                // pointers opened with cudaIpcOpenMemHandle
    std::vector<void*> owned;
  } sh;
  // Data parallelism over peer memory (mars_dp_*): rank-ordered sum of the
  // ranks' partial gradients (+ loss) between two device barriers.
  struct Dp {
    int32_t R = 1, me = 0;                 // world size, rank (R > 1: peer mode)
    bool connected = false;
    unsigned long long* flags = nullptr;   // [kMaxShards] arrival slots (peer-visible)
    unsigned long long* epoch = nullptr;
    int32_t* err = nullptr;
    float* gsum = nullptr;                 // [P + 1] global gradient + loss
    ShardSync sync{};
    PeerPtrs grads{};
    std::vector<void*> ipc, owned;
  } dp;
  float* grads_final() const {
    return sh.connected ? sh.gsum : dp.connected ? dp.gsum : grads;
  }
  ~mars_dgi() {
    drop_execs();
    kb_release();
    for (void* p : sh.ipc) cudaIpcCloseMemHandle(p);
    for (void* p : sh.owned) cudaFree(p);
    for (void* p : dp.ipc) cudaIpcCloseMemHandle(p);
    for (void* p : dp.owned) cudaFree(p);
    ws.release();
    for (void* p : {(void*)params, (void*)adam_m, (void*)adam_v, (void*)grads, (void*)guard_part,
                    (void*)adam_st, (void*)d_sp})
      if (p) cudaFree(p);
    if (sp_ev) {
      for (int i = 0; i < sp_ring; ++i) cudaEventDestroy(sp_ev[i]);
      delete[] sp_ev;
    }
    if (h_sp) cudaFreeHost(h_sp);
    for (cudaEvent_t e : loss_ev)
      if (e) cudaEventDestroy(e);
    if (loss_ring) cudaFreeHost(loss_ring);
    if (comm && g_nccl.CommDestroy) g_nccl.CommDestroy(comm);
    if (own_stream) cudaStreamDestroy(own_stream);
  }
};

// ---------------------------------------------------------------- misc ABI
extern "C" const char* mars_last_error(void) { return g_err.c_str(); }
extern "C" const char* mars_version(void) { return "mars-b200 0.1 sm_100a"; }
extern "C" int64_t mars_num_params(int32_t F, int32_t H) {
  return (int64_t)F * H + 3LL * H * H + 3;
}

extern "C" void mars_dgi_config_default(mars_dgi_config* c) {
  if (!c) return;
  memset(c, 0, sizeof *c);
  c->in_dim = 64;
  c->hidden_dim = 256;
  c->num_layers = 3;
  c->precision = MARS_FP32;
  c->lr = 1e-3;
  c->beta1 = 0.9;
  c->beta2 = 0.999;
  c->eps = 1e-8;
  c->clip_norm = 0.0;
  c->seed = 0;
  c->init_params = nullptr;
  c->device = 0;
  c->world_size = 1;
  c->rank = 0;
  c->nccl_unique_id = nullptr;
}

static mars_status check_graph(const mars_graph* g) {
  if (!g || g->tag != kTagGraph) return fail(MARS_ESTATE, "invalid or freed mars_graph handle");
  return MARS_OK;
}
static mars_status check_dgi(const mars_dgi* m) {
  if (!m || m->tag != kTagDgi) return fail(MARS_ESTATE, "invalid or freed mars_dgi handle");
  return MARS_OK;
}

// ---------------------------------------------------------------- graph load (a1-a3)
extern "C" mars_status mars_graph_load(const mars_graph_desc* descs, int32_t G, int32_t device,
                                       mars_graph** out) {
  if (!out) return fail(MARS_EINVAL, "out is NULL");
  *out = nullptr;
  if (!descs || G < 1) return fail(MARS_EINVAL, "need at least one graph");
  int F = descs[0].feat_dim;
  if (!valid_F(F)) return fail(MARS_EINVAL, "feat_dim %d not in {16,32,64,128,256}", F);
  int64_t Nt = 0, Et = 0;
  for (int g = 0; g < G; ++g) {
    const mars_graph_desc& d = descs[g];
    if (d.num_nodes < 1) return fail(MARS_EINVAL, "graph %d: num_nodes < 1", g);
    if (!d.indptr || !d.features || (!d.indices && d.indptr[d.num_nodes] > 0))
      return fail(MARS_EINVAL, "graph %d: NULL array", g);
    if (d.feat_dim != F) return fail(MARS_EINVAL, "graph %d: feat_dim mismatch", g);
    if (d.indptr[0] != 0 || d.indptr[d.num_nodes] < 0)
      return fail(MARS_EINVAL, "graph %d: malformed indptr", g);
    Nt += d.num_nodes;
    Et += d.indptr[d.num_nodes];
  }
  if (Nt + 2 * Et >= (int64_t)INT32_MAX - 1) return fail(MARS_EINVAL, "graph set too large");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(MARS_ECUDA, "no CUDA device (libmars has no CPU fallback)");
  }
  if (device < 0 || device >= ndev) return fail(MARS_EINVAL, "bad device %d", device);
  CK(cudaSetDevice(device));

  auto* gr = new mars_graph();
  std::unique_ptr<mars_graph> guard(gr);
  gr->device = device;
  gr->G = G;
  gr->F = F;
  gr->Nt = (int32_t)Nt;
  gr->Et = Et;
  // host-side small tables: node/edge offsets, reduction chunks, permutation buckets
  gr->h_node_off.resize(G + 1);
  std::vector<int64_t> edge_off(G + 1);
  std::vector<int32_t> chunk_row, chunk_graph, graph_chunk(G + 1), bucket_off(G + 1),
      bucket_log2(G);
  gr->h_node_off[0] = 0;
  edge_off[0] = 0;
  for (int g = 0; g < G; ++g) {
    int32_t N = descs[g].num_nodes;
    gr->h_node_off[g + 1] = gr->h_node_off[g] + N;
    edge_off[g + 1] = edge_off[g] + descs[g].indptr[N];
    graph_chunk[g] = (int32_t)chunk_graph.size();
    for (int32_t r = 0; r < N; r += kChunkRows) {
      chunk_row.push_back(gr->h_node_off[g] + r);
      chunk_graph.push_back(g);
    }
    int lb = 0;
    while ((1LL << lb) < N) ++lb;
    lb = lb > 2 ? lb - 2 : 0;
    bucket_log2[g] = lb;
    bucket_off[g + 1] = bucket_off[g] + (1 << lb);
  }
  bucket_off[0] = 0;
  graph_chunk[G] = (int32_t)chunk_graph.size();
  chunk_row.push_back((int32_t)Nt);
  int nchunks = (int)chunk_graph.size();

  cudaStream_t s = nullptr;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{s};
  pool_init(device);

  size_t b_indptr = sizeof(int64_t) * (size_t)(Nt + G);
  size_t b_idx = sizeof(int32_t) * (size_t)Et;
  size_t b_X = sizeof(float) * (size_t)Nt * F;
  int64_t* d_indptr;
  int32_t* d_idx;
  int64_t* d_edge_off;
  struct F1 { void* p; ~F1() { if (p) cudaFreeAsync(p, nullptr); } };
  CK(palloc(&d_indptr, (size_t)(Nt + G), s));
  F1 f1{d_indptr};
  CK(palloc(&d_idx, (size_t)Et, s));
  F1 f2{d_idx};
  CK(palloc(&d_edge_off, (size_t)G + 1, s));
  F1 f3{d_edge_off};
  CK(palloc(&gr->X, (size_t)Nt * F, s));
  CK(palloc(&gr->node_off, (size_t)G + 1, s));
  CK(palloc(&gr->node_graph, (size_t)Nt, s));
  CK(palloc(&gr->rowptr, (size_t)Nt + 1, s));
  CK(palloc(&gr->deg, (size_t)Nt, s));
  CK(palloc(&gr->dinv, (size_t)Nt, s));
  CK(palloc(&gr->chunk_row, (size_t)nchunks + 1, s));
  CK(palloc(&gr->chunk_graph, (size_t)nchunks, s));
  CK(palloc(&gr->graph_chunk, (size_t)G + 1, s));
  CK(palloc(&gr->bucket_off, (size_t)G + 1, s));
  CK(palloc(&gr->bucket_log2, (size_t)G, s));
  CK(palloc(&gr->gsize, (size_t)G, s));
  CK(palloc(&gr->pair_off, (size_t)G, s));

  // Inputs in page-locked host memory are copied straight to the device;
  // otherwise they are packed into a pinned staging buffer first.
  bool pinned = true;
  for (int g = 0; g < G && pinned; ++g)
    pinned = is_pinned(descs[g].indptr) && is_pinned(descs[g].features) &&
             (descs[g].indptr[descs[g].num_nodes] == 0 || is_pinned(descs[g].indices));
  std::unique_lock<std::mutex> lk(g_stage.mu, std::defer_lock);
  if (pinned) {
    for (int g = 0; g < G; ++g) {
      const mars_graph_desc& d = descs[g];
      int32_t N = d.num_nodes;
      CK(cudaMemcpyAsync(d_indptr + gr->h_node_off[g] + g, d.indptr, sizeof(int64_t) * (N + 1),
                         cudaMemcpyHostToDevice, s));
      if (d.indptr[N] > 0)
        CK(cudaMemcpyAsync(d_idx + edge_off[g], d.indices, sizeof(int32_t) * d.indptr[N],
                           cudaMemcpyHostToDevice, s));
      CK(cudaMemcpyAsync(gr->X + (int64_t)gr->h_node_off[g] * F, d.features,
                         sizeof(float) * (size_t)N * F, cudaMemcpyHostToDevice, s));
    }
  } else {
    lk.lock();
    char* stage = static_cast<char*>(g_stage.get(b_indptr + b_idx + b_X + 64));
    if (!stage) return fail(MARS_ENOMEM, "pinned staging allocation failed");
    int64_t* s_indptr = reinterpret_cast<int64_t*>(stage);
    int32_t* s_idx = reinterpret_cast<int32_t*>(stage + b_indptr);
    float* s_X = reinterpret_cast<float*>(stage + b_indptr + b_idx);
    for (int g = 0; g < G; ++g) {
      const mars_graph_desc& d = descs[g];
      int32_t N = d.num_nodes;
      memcpy(s_indptr + gr->h_node_off[g] + g, d.indptr, sizeof(int64_t) * (size_t)(N + 1));
      if (d.indptr[N] > 0)
        memcpy(s_idx + edge_off[g], d.indices, sizeof(int32_t) * (size_t)d.indptr[N]);
      memcpy(s_X + (int64_t)gr->h_node_off[g] * F, d.features, sizeof(float) * (size_t)N * F);
    }
    CK(cudaMemcpyAsync(d_indptr, s_indptr, b_indptr, cudaMemcpyHostToDevice, s));
    if (Et) CK(cudaMemcpyAsync(d_idx, s_idx, b_idx, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(gr->X, s_X, b_X, cudaMemcpyHostToDevice, s));
  }
  CK(cudaMemcpyAsync(d_edge_off, edge_off.data(), sizeof(int64_t) * (G + 1), cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(gr->node_off, gr->h_node_off.data(), sizeof(int32_t) * (G + 1), cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(gr->chunk_row, chunk_row.data(), sizeof(int32_t) * (nchunks + 1), cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(gr->chunk_graph, chunk_graph.data(), sizeof(int32_t) * nchunks, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(gr->graph_chunk, graph_chunk.data(), sizeof(int32_t) * (G + 1), cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(gr->bucket_off, bucket_off.data(), sizeof(int32_t) * (G + 1), cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(gr->bucket_log2, bucket_log2.data(), sizeof(int32_t) * G, cudaMemcpyHostToDevice, s));
  std::vector<int32_t> gsize(G);
  for (int g = 0; g < G; ++g) gsize[g] = descs[g].num_nodes;
  CK(cudaMemcpyAsync(gr->gsize, gsize.data(), sizeof(int32_t) * G, cudaMemcpyHostToDevice, s));
  std::vector<int64_t> poff(G);
  for (int g = 0; g < G; ++g) poff[g] = g;
  CK(cudaMemcpyAsync(gr->pair_off, poff.data(), sizeof(int64_t) * G, cudaMemcpyHostToDevice, s));
  k_node_graph<<<cdiv(Nt, 256), 256, 0, s>>>(gr->node_off, G, (int32_t)Nt, gr->node_graph);
  CK(cudaGetLastError());

  // builder scratch
  BuilderIO io{};
  io.G = G;
  io.Nt = (int32_t)Nt;
  io.Et = Et;
  io.indptr = d_indptr;
  io.indices = d_idx;
  io.node_off = gr->node_off;
  io.edge_off = d_edge_off;
  io.node_graph = gr->node_graph;
  int64_t cap = Nt + 2 * Et;
  std::vector<void*> scratch;
  struct SF {
    std::vector<void*>* v;
    cudaStream_t s;
    ~SF() { for (void* p : *v) cudaFreeAsync(p, s); }
  } sf{&scratch, s};
  auto salloc = [&](void** p, size_t bytes) -> cudaError_t {
    cudaError_t e = cudaMallocAsync(p, bytes ? bytes : 4, s);
    if (e == cudaSuccess) scratch.push_back(*p);
    return e;
  };
  CK(salloc((void**)&io.cnt, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.off_dup, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.cursor, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.buf, sizeof(int32_t) * cap));
  CK(salloc((void**)&io.buf2, sizeof(int32_t) * cap));
  CK(salloc((void**)&io.ucnt, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.err, sizeof(int32_t) * 2));
  io.scan_tmp_bytes = scan_tmp_bytes(Nt + 1);
  CK(salloc(&io.scan_tmp, io.scan_tmp_bytes));
  io.rowptr = gr->rowptr;
  io.deg = gr->deg;
  io.dinv = gr->dinv;
  CK(build_csr_phase1(io, s));
  // per-graph nnz offsets rowptr[node_off[g]] (+ the error flags) in one small D2H
  std::vector<int32_t> hbuf((size_t)G + 3);
  int32_t* d_nnzoff = io.ucnt;                         // ucnt is free after the scan
  k_gather_rowptr<<<cdiv(G + 1, 256), 256, 0, s>>>(gr->rowptr, gr->node_off, G, d_nnzoff);
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(hbuf.data(), d_nnzoff, sizeof(int32_t) * (G + 1), cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(hbuf.data() + G + 1, io.err, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  const int32_t herr = hbuf[G + 1];
  if (herr) return fail(MARS_EINVAL, "malformed graph input (code %d): %s", herr,
                        (herr & 2) ? "edge index out of range" : "indptr inconsistent");
  gr->h_nnz_off.resize(G + 1);
  for (int g = 0; g <= G; ++g) gr->h_nnz_off[g] = hbuf[g];
  gr->nnz = gr->h_nnz_off[G];
  CK(palloc(&gr->colind, (size_t)gr->nnz, s));
  CK(palloc(&gr->vals, (size_t)gr->nnz, s));
  gr->nnz_cap = gr->nnz;
  gr->Et_load = Et;
  CK(build_csr_phase2(io, gr->colind, gr->vals, s));
  CK(cudaStreamSynchronize(s));

  GraphDev& v = gr->dev;
  v.G = G;
  v.Nt = (int32_t)Nt;
  v.nnz = gr->nnz;
  v.F = F;
  v.node_off = gr->node_off;
  v.node_graph = gr->node_graph;
  v.rowptr = gr->rowptr;
  v.colind = gr->colind;
  v.vals = gr->vals;
  v.X = gr->X;
  v.nchunks = nchunks;
  v.chunk_row = gr->chunk_row;
  v.chunk_graph = gr->chunk_graph;
  v.graph_chunk = gr->graph_chunk;
  v.nbuckets = bucket_off[G];
  v.bucket_off = gr->bucket_off;
  v.bucket_log2 = gr->bucket_log2;
  for (int g = 0; g < G; ++g) {
    v.max_bucket_log2 = std::max(v.max_bucket_log2, bucket_log2[g]);
    v.max_graph_nodes = std::max(v.max_graph_nodes, gr->h_node_off[g + 1] - gr->h_node_off[g]);
  }
  v.gsize = gr->gsize;
  v.pair_off = gr->pair_off;
  CK(build_long_rows(gr, v, s));
  *out = guard.release();
  return MARS_OK;
}

// In-place reload (a1-a3 again) of a graph set with the same graphs' node
// counts and feature width: new edges and features into the existing device
// buffers, on a private stream that first waits (on the device) for every
// recorded use of the old contents.  The handle keeps its identity -- and the
// steps models captured for it stay valid -- unless the stored-entry count or
// the long-row structure changed (then it gets a new identity).
extern "C" mars_status mars_graph_reload(mars_graph* gr, const mars_graph_desc* descs, int32_t G) {
  if (mars_status st = check_graph(gr)) return st;
  if (gr->sharded) return fail(MARS_EINVAL, "a row-sharded graph cannot be reloaded");
  if (!descs || G != gr->G) return fail(MARS_EINVAL, "reload needs the same number of graphs");
  const int F = gr->F;
  int64_t Et = 0;
  for (int g = 0; g < G; ++g) {
    const mars_graph_desc& d = descs[g];
    if (d.num_nodes != gr->h_node_off[g + 1] - gr->h_node_off[g])
      return fail(MARS_EINVAL, "graph %d: reload needs the same node count", g);
    if (d.feat_dim != F) return fail(MARS_EINVAL, "graph %d: feat_dim mismatch", g);
    if (!d.indptr || !d.features || (!d.indices && d.indptr[d.num_nodes] > 0))
      return fail(MARS_EINVAL, "graph %d: NULL array", g);
    if (d.indptr[0] != 0 || d.indptr[d.num_nodes] < 0)
      return fail(MARS_EINVAL, "graph %d: malformed indptr", g);
    Et += d.indptr[d.num_nodes];
  }
  const int64_t Nt = gr->Nt;
  if (Nt + 2 * Et >= (int64_t)INT32_MAX - 1) return fail(MARS_EINVAL, "graph set too large");
  CK(cudaSetDevice(gr->device));
  cudaStream_t s = nullptr;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{s};
  {   // the old contents stay until every recorded use of them has run
    std::lock_guard<std::mutex> lk(gr->use_mu);
    for (auto& u : gr->uses) CK(cudaStreamWaitEvent(s, u.second, 0));
  }
  std::vector<int64_t> edge_off(G + 1, 0);
  for (int g = 0; g < G; ++g) edge_off[g + 1] = edge_off[g] + descs[g].indptr[descs[g].num_nodes];
  std::vector<void*> scratch;
  struct SF {
    std::vector<void*>* v;
    cudaStream_t s;
    ~SF() { for (void* p : *v) cudaFreeAsync(p, s); }
  } sf{&scratch, s};
  auto salloc = [&](void** p, size_t bytes) -> cudaError_t {
    cudaError_t e = cudaMallocAsync(p, bytes ? bytes : 4, s);
    if (e == cudaSuccess) scratch.push_back(*p);
    return e;
  };
  int64_t* d_indptr = nullptr;
  int32_t* d_idx = nullptr;
  int64_t* d_edge_off = nullptr;
  CK(salloc((void**)&d_indptr, sizeof(int64_t) * (size_t)(Nt + G)));
  CK(salloc((void**)&d_idx, sizeof(int32_t) * (size_t)std::max<int64_t>(Et, 1)));
  CK(salloc((void**)&d_edge_off, sizeof(int64_t) * (G + 1)));
  for (int g = 0; g < G; ++g) {   // pinned inputs are copied directly, pageable ones staged by CUDA
    const mars_graph_desc& d = descs[g];
    const int32_t N = d.num_nodes;
    CK(cudaMemcpyAsync(d_indptr + gr->h_node_off[g] + g, d.indptr, sizeof(int64_t) * (N + 1),
                       cudaMemcpyHostToDevice, s));
    if (d.indptr[N] > 0)
      CK(cudaMemcpyAsync(d_idx + edge_off[g], d.indices, sizeof(int32_t) * d.indptr[N],
                         cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(gr->X + (int64_t)gr->h_node_off[g] * F, d.features,
                       sizeof(float) * (size_t)N * F, cudaMemcpyHostToDevice, s));
  }
  CK(cudaMemcpyAsync(d_edge_off, edge_off.data(), sizeof(int64_t) * (G + 1), cudaMemcpyHostToDevice, s));
  BuilderIO io{};
  io.G = G;
  io.Nt = (int32_t)Nt;
  io.Et = Et;
  io.indptr = d_indptr;
  io.indices = d_idx;
  io.node_off = gr->node_off;
  io.edge_off = d_edge_off;
  io.node_graph = gr->node_graph;
  const int64_t cap = Nt + 2 * Et;
  CK(salloc((void**)&io.cnt, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.off_dup, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.cursor, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.buf, sizeof(int32_t) * cap));
  CK(salloc((void**)&io.buf2, sizeof(int32_t) * cap));
  CK(salloc((void**)&io.ucnt, sizeof(int32_t) * (Nt + 1)));
  CK(salloc((void**)&io.err, sizeof(int32_t) * 2));
  io.scan_tmp_bytes = scan_tmp_bytes(Nt + 1);
  CK(salloc(&io.scan_tmp, io.scan_tmp_bytes));
  io.rowptr = gr->rowptr;
  io.deg = gr->deg;
  io.dinv = gr->dinv;
  CK(build_csr_phase1(io, s));
  std::vector<int32_t> hbuf((size_t)G + 3);
  int32_t* d_nnzoff = io.ucnt;
  k_gather_rowptr<<<cdiv(G + 1, 256), 256, 0, s>>>(gr->rowptr, gr->node_off, G, d_nnzoff);
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(hbuf.data(), d_nnzoff, sizeof(int32_t) * (G + 1), cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(hbuf.data() + G + 1, io.err, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (hbuf[G + 1]) {
    gr->uid = g_graph_uid.fetch_add(1);   // contents undefined until a successful reload
    return fail(MARS_EINVAL, "malformed graph input (code %d): %s", hbuf[G + 1],
                (hbuf[G + 1] & 2) ? "edge index out of range" : "indptr inconsistent");
  }
  const int64_t nnz_old = gr->nnz;
  for (int g = 0; g <= G; ++g) gr->h_nnz_off[g] = hbuf[g];
  gr->nnz = gr->h_nnz_off[G];
  bool same = gr->nnz == nnz_old;
  if (gr->nnz > gr->nnz_cap) {          // more stored entries than the buffers hold
    cudaFreeAsync(gr->colind, s);
    cudaFreeAsync(gr->vals, s);
    gr->colind = nullptr;
    gr->vals = nullptr;
    CK(palloc(&gr->colind, (size_t)gr->nnz, s));
    CK(palloc(&gr->vals, (size_t)gr->nnz, s));
    gr->nnz_cap = gr->nnz;
    same = false;
  }
  CK(build_csr_phase2(io, gr->colind, gr->vals, s));
  GraphDev& v = gr->dev;
  v.nnz = gr->nnz;
  v.colind = gr->colind;
  v.vals = gr->vals;
  bool lchanged = true;
  CK(build_long_rows(gr, v, s, &lchanged));
  CK(cudaStreamSynchronize(s));
  gr->Et = Et;
  if (!same || lchanged) gr->uid = g_graph_uid.fetch_add(1);   // captured steps are stale
  return MARS_OK;
}

extern "C" mars_status mars_graph_info(const mars_graph* g, int32_t* G, int64_t* Nt, int64_t* nnz,
                                       int32_t* F) {
  if (mars_status st = check_graph(g)) return st;
  if (G) *G = g->G;
  if (Nt) *Nt = g->Nt;
  if (nnz) *nnz = g->nnz;
  if (F) *F = g->F;
  return MARS_OK;
}

extern "C" mars_status mars_graph_size(const mars_graph* g, int32_t idx, int32_t* N, int64_t* nnz) {
  if (mars_status st = check_graph(g)) return st;
  if (idx < 0 || idx >= g->G) return fail(MARS_EINVAL, "graph index out of range");
  if (N) *N = g->h_node_off[idx + 1] - g->h_node_off[idx];
  if (nnz) *nnz = g->h_nnz_off[idx + 1] - g->h_nnz_off[idx];
  return MARS_OK;
}

extern "C" mars_status mars_graph_export_csr(const mars_graph* g, int32_t idx, int32_t* rowptr,
                                             int32_t* colind, int32_t* deg, float* dinv,
                                             float* vals) {
  if (mars_status st = check_graph(g)) return st;
  if (idx < 0 || idx >= g->G) return fail(MARS_EINVAL, "graph index out of range");
  CK(cudaSetDevice(g->device));
  int32_t n0 = g->h_node_off[idx], N = g->h_node_off[idx + 1] - n0;
  int64_t z0 = g->h_nnz_off[idx], Z = g->h_nnz_off[idx + 1] - z0;
  if (rowptr) {
    CK(cudaMemcpy(rowptr, g->rowptr + n0, sizeof(int32_t) * (N + 1), cudaMemcpyDeviceToHost));
    for (int32_t i = 0; i <= N; ++i) rowptr[i] -= (int32_t)z0;
  }
  if (colind) {
    CK(cudaMemcpy(colind, g->colind + z0, sizeof(int32_t) * Z, cudaMemcpyDeviceToHost));
    for (int64_t k = 0; k < Z; ++k) colind[k] -= n0;
  }
  if (deg) CK(cudaMemcpy(deg, g->deg + n0, sizeof(int32_t) * N, cudaMemcpyDeviceToHost));
  if (dinv) CK(cudaMemcpy(dinv, g->dinv + n0, sizeof(float) * N, cudaMemcpyDeviceToHost));
  if (vals) CK(cudaMemcpy(vals, g->vals + z0, sizeof(float) * Z, cudaMemcpyDeviceToHost));
  return MARS_OK;
}

// ---------------------------------------------------------------- featuriser (NEXT-1)
extern "C" mars_status mars_featurize(const int32_t* types, const int64_t* dims, int32_t N,
                                      int32_t F, int32_t device, float* X) {
  if (!types || !dims || !X) return fail(MARS_EINVAL, "NULL argument");
  if (N < 1) return fail(MARS_EINVAL, "N < 1");
  if (!valid_F(F)) return fail(MARS_EINVAL, "feat_dim %d not in {16,32,64,128,256}", F);
  for (int32_t i = 0; i < N; ++i)
    if (types[i] < 0) return fail(MARS_EINVAL, "op %d: negative type", i);
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(MARS_ECUDA, "no CUDA device (libmars has no CPU fallback)");
  }
  if (device < 0 || device >= ndev) return fail(MARS_EINVAL, "bad device %d", device);
  CK(cudaSetDevice(device));
  cudaStream_t s = nullptr;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{s};
  int32_t* d_types = nullptr;
  int64_t* d_dims = nullptr;
  float* d_X = nullptr;
  unsigned long long* d_max = nullptr;
  struct F1 { void* p; cudaStream_t s; ~F1() { if (p) cudaFreeAsync(p, s); } };
  CK(palloc(&d_types, (size_t)N, s));
  F1 f1{d_types, s};
  CK(palloc(&d_dims, 8 * (size_t)N, s));
  F1 f2{d_dims, s};
  CK(palloc(&d_X, (size_t)N * F, s));
  F1 f3{d_X, s};
  CK(palloc(&d_max, 1, s));
  F1 f4{d_max, s};
  CK(cudaMemcpyAsync(d_types, types, sizeof(int32_t) * N, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(d_dims, dims, sizeof(int64_t) * 8 * N, cudaMemcpyHostToDevice, s));
  CK(launch_featurize(d_types, d_dims, N, F, d_max, d_X, s));
  CK(cudaMemcpyAsync(X, d_X, sizeof(float) * (size_t)N * F, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  return MARS_OK;
}

// ---------------------------------------------------------------- model create
extern "C" int64_t mars_dgi_num_params(const mars_dgi* m) {
  return (m && m->tag == kTagDgi) ? m->P : -1;
}

extern "C" mars_status mars_nccl_get_unique_id(void* out128) {
  if (!out128) return fail(MARS_EINVAL, "out is NULL");
  if (!nccl_load()) return fail(MARS_ENCCL, "libnccl.so.2 not loadable");
  ncclUniqueId id;
  ncclResult_t r = g_nccl.GetUniqueId(&id);
  if (r != ncclSuccess) return fail(MARS_ENCCL, "ncclGetUniqueId failed (%d)", (int)r);
  memcpy(out128, &id, sizeof id);
  return MARS_OK;
}

extern "C" mars_status mars_dgi_create(const mars_dgi_config* cfg, mars_dgi** out) {
  if (!cfg || !out) return fail(MARS_EINVAL, "NULL argument");
  *out = nullptr;
  if (!valid_F(cfg->in_dim)) return fail(MARS_EINVAL, "in_dim %d unsupported", cfg->in_dim);
  if (!valid_H(cfg->hidden_dim)) return fail(MARS_EINVAL, "hidden_dim %d unsupported", cfg->hidden_dim);
  if (cfg->num_layers != 3) return fail(MARS_EINVAL, "num_layers must be 3 (P:L101, c10)");
  if (cfg->precision != MARS_FP32 && cfg->precision != MARS_BF16)
    return fail(MARS_EINVAL, "unknown precision %d", cfg->precision);
  if (cfg->precision == MARS_BF16 &&
      !(tc_supported(cfg->in_dim, cfg->hidden_dim) && tc_supported(cfg->hidden_dim, cfg->hidden_dim)))
    return fail(MARS_EINVAL, "MARS_BF16 needs hidden_dim in {128, 256} and in_dim in {64, 128, 256}");
  if (cfg->world_size < 1 || cfg->rank < 0 || cfg->rank >= cfg->world_size)
    return fail(MARS_EINVAL, "bad world_size/rank");
  if (cfg->encoder != MARS_ENCODER_GCN && cfg->encoder != MARS_ENCODER_SAGE &&
      cfg->encoder != MARS_ENCODER_SAGE_POOL)
    return fail(MARS_EINVAL, "unknown encoder %d", cfg->encoder);
  if (cfg->encoder != MARS_ENCODER_GCN && cfg->precision != MARS_FP32)
    return fail(MARS_EINVAL, "the SAGE encoders run MARS_FP32 only");
  if (cfg->world_size > kMaxShards && !cfg->nccl_unique_id)
    return fail(MARS_EINVAL, "peer-memory data parallelism supports world_size <= %d", kMaxShards);
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(MARS_ECUDA, "no CUDA device (libmars has no CPU fallback)");
  }
  if (cfg->device < 0 || cfg->device >= ndev) return fail(MARS_EINVAL, "bad device");
  CK(cudaSetDevice(cfg->device));
  auto* m = new mars_dgi();
  std::unique_ptr<mars_dgi> guard(m);
  m->cfg = *cfg;
  m->cfg.init_params = nullptr;
  m->cfg.nccl_unique_id = nullptr;
  m->F = cfg->in_dim;
  m->H = cfg->hidden_dim;
  m->sage = cfg->encoder == MARS_ENCODER_SAGE;
  m->pool = cfg->encoder == MARS_ENCODER_SAGE_POOL;
  m->P = m->pool ? 2LL * m->F * m->H + 8LL * m->H * m->H + 3LL * m->H + 3
                 : mars_num_params(m->F, m->H) +
                       (m->sage ? (int64_t)m->F * m->H + 2LL * m->H * m->H : 0);
  CK(cudaStreamCreateWithFlags(&m->own_stream, cudaStreamNonBlocking));
  m->stream = m->own_stream;
  CK(dalloc(&m->params, m->P));
  CK(dalloc(&m->adam_m, m->P));
  CK(dalloc(&m->adam_v, m->P));
  CK(dalloc(&m->grads, m->P + 1));
  CK(dalloc(&m->guard_part, (size_t)adam_guard_doubles()));
  CK(dalloc(&m->adam_st, 1));
  CK(dalloc(&m->d_sp, 1));
  CK(cudaMallocHost(&m->h_sp, sizeof(StepParams) * m->sp_ring));
  m->sp_ev = new cudaEvent_t[m->sp_ring];
  for (int i = 0; i < m->sp_ring; ++i) {
    CK(cudaEventCreateWithFlags(&m->sp_ev[i], cudaEventDisableTiming));
    CK(cudaEventRecord(m->sp_ev[i], m->stream));
  }
  cudaStream_t s = m->stream;
  CK(cudaMemsetAsync(m->adam_m, 0, sizeof(float) * m->P, s));
  CK(cudaMemsetAsync(m->adam_v, 0, sizeof(float) * m->P, s));
  CK(cudaMemsetAsync(m->grads, 0, sizeof(float) * (m->P + 1), s));
  CK(cudaMemsetAsync(m->adam_st, 0, sizeof(AdamDev), s));
  if (cfg->init_params) {
    CK(cudaMemcpyAsync(m->params, cfg->init_params, sizeof(float) * m->P, cudaMemcpyHostToDevice, s));
  } else if (m->pool) {            // c40: per layer W_s, W_n, W_p (tags 3l+1..3l+3), b_p = 0; M
    const int F = m->F, H = m->H;
    int64_t off = 0;
    auto xav = [&](int tag, int64_t n, double fan) {
      const float b = (float)std::sqrt(6.0 / fan);
      k_xavier<<<cdiv(n, 256), 256, 0, s>>>(m->params + off, n, cfg->seed, (uint64_t)tag, b);
      off += n;
    };
    for (int l = 0; l < 3; ++l) {
      const int C = l == 0 ? F : H;
      xav(3 * l + 1, (int64_t)C * H, (double)C + 2.0 * H);
      xav(3 * l + 2, (int64_t)H * H, (double)C + 2.0 * H);
      xav(3 * l + 3, (int64_t)C * H, (double)C + H);
      CK(cudaMemsetAsync(m->params + off, 0, sizeof(float) * H, s));
      off += H;
    }
    xav(10, (int64_t)H * H, 2.0 * H);
    k_fill<<<1, 32, 0, s>>>(m->params + off, 3, 0.25f);
    CK(cudaGetLastError());
  } else if (!m->sage) {
    int64_t off = 0;
    for (int t = 1; t <= 4; ++t) {
      int fin = t == 1 ? m->F : m->H;
      int64_t n = (int64_t)fin * m->H;
      float b = (float)std::sqrt(6.0 / (double)(fin + m->H));
      k_xavier<<<cdiv(n, 256), 256, 0, s>>>(m->params + off, n, cfg->seed, (uint64_t)t, b);
      off += n;
    }
    k_fill<<<1, 32, 0, s>>>(m->params + off, 3, 0.25f);
    CK(cudaGetLastError());
  } else {                         // c38: W1s W1n W2s W2n W3s W3n M, tags 1..7
    int64_t off = 0;
    for (int t = 1; t <= 7; ++t) {
      const int fin = t <= 2 ? m->F : m->H;
      const int64_t n = (int64_t)fin * m->H;
      const double fan = t == 7 ? 2.0 * m->H : 2.0 * fin + m->H;
      const float b = (float)std::sqrt(6.0 / fan);
      k_xavier<<<cdiv(n, 256), 256, 0, s>>>(m->params + off, n, cfg->seed, (uint64_t)t, b);
      off += n;
    }
    k_fill<<<1, 32, 0, s>>>(m->params + off, 3, 0.25f);
    CK(cudaGetLastError());
  }
  CK(cudaStreamSynchronize(s));
  if (cfg->world_size > 1 && !cfg->nccl_unique_id) {      // peer-memory exchange
    mars_dgi::Dp& d = m->dp;
    d.R = cfg->world_size;
    d.me = cfg->rank;
    auto al = [&](void** p, size_t bytes) -> cudaError_t {
      cudaError_t e = cudaMalloc(p, bytes);
      if (e == cudaSuccess) d.owned.push_back(*p);
      return e;
    };
    CK(al((void**)&d.flags, sizeof(unsigned long long) * kMaxShards));
    CK(al((void**)&d.epoch, sizeof(unsigned long long)));
    CK(al((void**)&d.err, sizeof(int32_t)));
    CK(al((void**)&d.gsum, sizeof(float) * (m->P + 1)));
    CK(cudaMemset(d.flags, 0, sizeof(unsigned long long) * kMaxShards));
    CK(cudaMemset(d.epoch, 0, sizeof(unsigned long long)));
    CK(cudaMemset(d.err, 0, sizeof(int32_t)));
    CK(cudaMemset(d.gsum, 0, sizeof(float) * (m->P + 1)));
    CK(cudaDeviceSynchronize());
  }
  // an NCCL id makes the exchange an NCCL allreduce; with world_size == 1 an
  // id may still be passed to run the (identity) allreduce path (tests).
  if (cfg->nccl_unique_id) {
    if (!nccl_load()) return fail(MARS_ENCCL, "libnccl.so.2 not loadable");
    ncclUniqueId id;
    memcpy(&id, cfg->nccl_unique_id, sizeof id);
    ncclResult_t r = g_nccl.CommInitRank(&m->comm, cfg->world_size, id, cfg->rank);
    if (r != ncclSuccess)
      return fail(MARS_ENCCL, "ncclCommInitRank: %s",
                  g_nccl.GetErrorString ? g_nccl.GetErrorString(r) : "error");
  }
  *out = guard.release();
  return MARS_OK;
}

extern "C" mars_status mars_dgi_set_stream(mars_dgi* m, void* stream) {
  if (mars_status st = check_dgi(m)) return st;
  m->stream = stream ? static_cast<cudaStream_t>(stream) : m->own_stream;
  return MARS_OK;
}

extern "C" mars_status mars_dgi_set_gemm_impl(mars_dgi* m, int32_t impl) {
  if (mars_status st = check_dgi(m)) return st;
  if (impl != MARS_GEMM_AUTO && impl != MARS_GEMM_SIMT)
    return fail(MARS_EINVAL, "bad gemm impl");
  if (impl != m->gemm_impl) m->drop_execs();
  m->gemm_impl = impl;
  return MARS_OK;
}

extern "C" mars_status mars_dgi_set_graph_capture(mars_dgi* m, int32_t enable) {
  if (mars_status st = check_dgi(m)) return st;
  m->capture = enable != 0;
  return MARS_OK;
}

extern "C" mars_status mars_dgi_set_contrastive(mars_dgi* m, const mars_contrastive* c) {
  if (mars_status st = check_dgi(m)) return st;
  if (!c) return fail(MARS_EINVAL, "config is NULL");
  if (c->num_neg < 1 || c->num_neg > 64) return fail(MARS_EINVAL, "num_neg must be in [1, 64]");
  if (c->corruption != MARS_CORRUPT_PERMUTE && c->corruption != MARS_CORRUPT_MASK)
    return fail(MARS_EINVAL, "unknown corruption");
  if (!(c->mask_rate >= 0.f && c->mask_rate <= 1.f)) return fail(MARS_EINVAL, "mask_rate not in [0, 1]");
  if (c->readout != MARS_READOUT_SIGMOID_MEAN && c->readout != MARS_READOUT_MEAN)
    return fail(MARS_EINVAL, "unknown readout");
  if (c->aggregator != MARS_AGG_GCN && c->aggregator != MARS_AGG_SAGE_GCN)
    return fail(MARS_EINVAL, "unknown aggregator");
  if (c->loss != MARS_LOSS_BCE && c->loss != MARS_LOSS_INFONCE) return fail(MARS_EINVAL, "unknown loss");
  const bool dflt = c->num_neg == 1 && c->corruption == MARS_CORRUPT_PERMUTE &&
                    c->readout == MARS_READOUT_SIGMOID_MEAN && c->aggregator == MARS_AGG_GCN &&
                    c->loss == MARS_LOSS_BCE;
  if (m->sh.g && !dflt) return fail(MARS_ESTATE, "a row-sharded model runs the default step only");
  if (memcmp(c, &m->ct, sizeof *c) == 0) return MARS_OK;     // unchanged: keep workspace and graphs
  if ((m->sage || m->pool) && c->aggregator != MARS_AGG_GCN)
    return fail(MARS_EINVAL, "the SAGE encoders have their own aggregation (aggregator must be GCN)");
  CK(cudaSetDevice(m->cfg.device));
  m->drop_execs();                 // captured steps bake the variant in
  CK(cudaStreamSynchronize(m->stream));
  m->ws.release();                 // re-sized on the next step / encode
  m->last_Nt = 0;
  m->kb_valid_Nt = 0;
  m->ct = *c;
  return MARS_OK;
}

extern "C" mars_status mars_dgi_get_contrastive(const mars_dgi* m, mars_contrastive* c) {
  if (mars_status st = check_dgi(m)) return st;
  if (!c) return fail(MARS_EINVAL, "config is NULL");
  *c = m->ct;
  return MARS_OK;
}

// ---------------------------------------------------------------- workspaces
static mars_status ensure_kb(mars_dgi* m, const mars_graph* g) {
  if (!m->keep_bwd || m->kb_rows >= g->dev.Nt) return MARS_OK;
  m->drop_execs();                 // a captured step without the copies
  CK(cudaStreamSynchronize(m->stream));
  m->kb_release();
  const size_t bytes = sizeof(float) * 2 * (size_t)g->dev.Nt * m->H;
  for (void*& p : m->kb_dZ) CK(cudaMalloc(&p, bytes));
  for (void*& p : m->kb_dY) CK(cudaMalloc(&p, bytes));
  m->kb_rows = g->dev.Nt;
  return MARS_OK;
}

static mars_status ensure_ws(mars_dgi* m, const mars_graph* g) {
  if (mars_status st = ensure_kb(m, g)) return st;
  Workspace& w = m->ws;
  const GraphDev& pv = g->perm_view();
  const int nbk = m->ct_nb(), K = m->ct.num_neg;
  const bool xs = m->ct_materialise(), sage = m->ct.aggregator == MARS_AGG_SAGE_GCN;
  const bool smean = m->sage, spool = m->pool;
  if (w.Nt >= g->dev.Nt && w.Nperm >= pv.Nt && w.G >= g->G && w.nchunks >= g->dev.nchunks &&
      w.nbuckets >= pv.nbuckets && w.nnz_perm >= pv.nnz && w.nlong >= g->dev.nlong &&
      w.nseg >= g->dev.nseg && w.F == m->F && w.H == m->H && w.nb == nbk && w.K == K &&
      (w.has_xs || !xs) && (!sage || w.nnz_vals >= g->dev.nnz) &&
      (!smean || (w.sU && w.nnz_vals >= g->dev.nnz)) && (!spool || w.pUS))
    return MARS_OK;
  if (m->sh.g) return fail(MARS_ESTATE, "workspace of a shard-attached model cannot grow");
  m->drop_execs();
  CK(cudaStreamSynchronize(m->stream));
  w.release();
  int64_t Nt = g->dev.Nt, R = nbk * Nt, Np = pv.Nt;
  int F = m->F, H = m->H, G = g->G, nch = g->dev.nchunks, nb = pv.nbuckets;
  auto al = [&](void** p, size_t bytes) -> cudaError_t {
    cudaError_t e = cudaMalloc(p, bytes ? bytes : 8);
    if (e == cudaSuccess) w.owned.push_back(*p);
    return e;
  };
  CK(al((void**)&w.Y1, sizeof(float) * R * F));
  for (int l = 0; l < 3; ++l) CK(al((void**)&w.Z[l], sizeof(float) * R * H));
  for (int l = 0; l < 2; ++l) CK(al((void**)&w.Y23[l], sizeof(float) * R * H));
  CK(al((void**)&w.dZ, sizeof(float) * R * H));
  CK(al((void**)&w.dY, sizeof(float) * R * H));
  if (nbk > K + 1) {               // the padding block stays zero (enqueue_step)
    CK(cudaMemset(w.Y1, 0, sizeof(float) * R * F));
    for (int l = 0; l < 3; ++l) CK(cudaMemset(w.Z[l], 0, sizeof(float) * R * H));
    for (int l = 0; l < 2; ++l) CK(cudaMemset(w.Y23[l], 0, sizeof(float) * R * H));
    CK(cudaMemset(w.dZ, 0, sizeof(float) * R * H));
    CK(cudaMemset(w.dY, 0, sizeof(float) * R * H));
  }
  CK(al((void**)&w.perm, sizeof(int32_t) * Np * K));
  CK(al((void**)&w.pair_off_k, sizeof(int64_t) * (size_t)G * K));
  if (xs) CK(al((void**)&w.Xs, sizeof(float) * R * F));
  if (sage) {
    CK(al((void**)&w.valsR, sizeof(float) * (size_t)std::max<int64_t>(1, g->dev.nnz)));
    CK(al((void**)&w.valsC, sizeof(float) * (size_t)std::max<int64_t>(1, g->dev.nnz)));
  }
  if (smean) {
    const size_t z = (size_t)std::max<int64_t>(1, g->dev.nnz);
    CK(al((void**)&w.sU, sizeof(float) * 2 * R * H));
    CK(al((void**)&w.sV, sizeof(float) * 2 * R * H));
    CK(cudaMemset(w.sU, 0, sizeof(float) * 2 * R * H));    // padding rows stay zero
    CK(cudaMemset(w.sV, 0, sizeof(float) * 2 * R * H));
    CK(al((void**)&w.sColS, sizeof(int32_t) * z));
    CK(al((void**)&w.sVf, sizeof(float) * z));
    CK(al((void**)&w.sVb, sizeof(float) * z));
    CK(al((void**)&w.sVn, sizeof(float) * z));
    CK(al((void**)&w.rsG, sizeof(float) * R));
    for (int t = 0; t < 6; ++t) {
      const int64_t n = (int64_t)(t < 2 ? F : H) * H;
      CK(al(&w.s3_wt_hi[t], 2 * n));
      CK(al(&w.s3_wt_lo[t], 2 * n));
      CK(al(&w.s3_w_hi[t], 2 * n));
      CK(al(&w.s3_w_lo[t], 2 * n));
      CK(al((void**)&w.s3_wsc[t], sizeof(float) * 2));
    }
  }
  if (spool) {
    for (int l = 0; l < 3; ++l) {
      CK(al((void**)&w.pUP[l], sizeof(float) * R * H));
      CK(al((void**)&w.pAGG[l], sizeof(float) * R * H));
      CK(al((void**)&w.pIDX[l], sizeof(int32_t) * R * H));
      CK(al((void**)&w.pRsAGG[l], sizeof(float) * R));
    }
    CK(al((void**)&w.pUS, sizeof(float) * R * H));
    CK(al((void**)&w.pVV, sizeof(float) * R * H));
    CK(al((void**)&w.pDUP, sizeof(float) * R * H));
    CK(al((void**)&w.pRsDUP, sizeof(float) * R));
    CK(al((void**)&w.pOnes, sizeof(float) * R));
    k_fill<<<cdiv(R, 256), 256>>>(w.pOnes, R, 1.f);
    CK(cudaGetLastError());
    for (int t = 0; t < 9; ++t) {
      const int64_t n = (int64_t)(t < 3 && t != 1 ? F : H) * H;    // layer 1: W_s, W_p are F x H
      CK(al(&w.p3_wt_hi[t], 2 * n));
      CK(al(&w.p3_wt_lo[t], 2 * n));
      CK(al(&w.p3_w_hi[t], 2 * n));
      CK(al(&w.p3_w_lo[t], 2 * n));
      CK(al((void**)&w.p3_wsc[t], sizeof(float) * 2));
    }
    CK(cudaDeviceSynchronize());
  }
  CK(al((void**)&w.one, sizeof(float)));
  {
    const float one = 1.f;
    CK(cudaMemcpy(w.one, &one, sizeof one, cudaMemcpyHostToDevice));
  }
  CK(al((void**)&w.long_part, sizeof(float) * (size_t)g->dev.nseg * 2 * 256));
  CK(al((void**)&w.colperm, sizeof(int32_t) * (size_t)std::max<int64_t>(1, pv.nnz)));
  CK(al((void**)&w.pw.keys, sizeof(uint64_t) * Np));
  CK(al((void**)&w.pw.bucket, sizeof(int32_t) * Np));
  CK(al((void**)&w.pw.bcnt, sizeof(int32_t) * (nb + 1)));
  CK(al((void**)&w.pw.bstart, sizeof(int32_t) * (nb + 1)));
  CK(al((void**)&w.pw.bcur, sizeof(int32_t) * (nb + 1)));
  CK(al((void**)&w.pw.members, sizeof(int32_t) * Np));
  CK(al(&w.pw.scan_tmp, scan_tmp_bytes(nb + 1)));
  HeadWork& h = w.hw;
  CK(al((void**)&h.colsum_part, sizeof(double) * nch * H));
  CK(al((void**)&h.dv_part, sizeof(double) * nch * nbk * H));
  CK(al((void**)&h.loss_part, sizeof(double) * nch * nbk));
  CK(al((void**)&h.s, sizeof(float) * G * H));
  CK(al((void**)&h.v, sizeof(float) * G * H));
  CK(al((void**)&h.dm, sizeof(float) * G * H));
  CK(al((void**)&h.dv, sizeof(float) * G * H));
  CK(al((void**)&h.dvd, sizeof(double) * G * H));
  CK(al((void**)&h.sd, sizeof(double) * G * H));
  CK(al((void**)&h.dl, sizeof(float) * R));
  CK(al((void**)&h.loss_g, sizeof(double) * G));
  int nsl = std::max(head_slots(g->dev, nbk), (nbk / 2) * spmm_bwd_slots(g->dev));
  for (int l = 0; l < 3; ++l) CK(al((void**)&w.slots[l], sizeof(double) * nsl));
  h.slots = w.slots[2];
  size_t tn = std::max(gemm_tn_partial_floats(R, F, H), gemm_tn_partial_floats(R, H, H));
  CK(al((void**)&w.tn_part, sizeof(double) * tn));
  w.tn_part_n = tn;
  for (int l = 0; l < 3; ++l) {
    int64_t n = (int64_t)(l == 0 ? F : H) * H;
    CK(al(&w.h3_wt_hi[l], 2 * n));
    CK(al(&w.h3_wt_lo[l], 2 * n));
    CK(al(&w.h3_w_hi[l], 2 * n));
    CK(al(&w.h3_w_lo[l], 2 * n));
    CK(al((void**)&w.h3_wsc[l], sizeof(float) * 2));
  }
  for (int l = 0; l < 3; ++l) CK(al((void**)&w.h3_rsY[l], sizeof(float) * R));
  CK(al((void**)&w.h3_rsdZ, sizeof(float) * R));
  CK(al((void**)&w.dw_part, sizeof(float) * std::max(tc_dw_partial_floats(R, F),
                                                      tc_dw_partial_floats(R, H))));
  if (m->cfg.precision == MARS_BF16) {
    for (int l = 0; l < 3; ++l) {
      const int64_t n = (int64_t)(l == 0 ? F : H) * H;
      CK(al(&w.w16t[l], 2 * n));
      CK(al(&w.w16[l], 2 * n));
    }
    CK(al((void**)&w.dw16_part, sizeof(float) * std::max(tc16_dw_partial_floats(R, F),
                                                          tc16_dw_partial_floats(R, H))));
  }
  w.Nt = (int32_t)Nt;
  w.Nperm = (int32_t)Np;
  w.nnz_perm = pv.nnz;
  w.nlong = g->dev.nlong;
  w.nseg = g->dev.nseg;
  w.G = G;
  w.nchunks = nch;
  w.nbuckets = nb;
  w.F = F;
  w.H = H;
  w.nb = nbk;
  w.K = K;
  w.has_xs = xs;
  w.nnz_vals = (sage || smean) ? g->dev.nnz : 0;
  h.nb = nbk;
  h.K = K;
  h.readout = m->ct.readout;
  h.loss = m->ct.loss;
  return MARS_OK;
}

// ---------------------------------------------------------------- the step schedule
// Optional per-phase event profiler (mars_dgi_profile_step): an event is
// recorded on the launching stream after every kernel group.
struct Profiler {
  std::vector<cudaEvent_t> ev;
  std::vector<int32_t> phase;
  cudaError_t mark(int ph, cudaStream_t s) {
    cudaEvent_t e;
    cudaError_t r = cudaEventCreate(&e);
    if (r != cudaSuccess) return r;
    ev.push_back(e);
    phase.push_back(ph);
    return cudaEventRecord(e, s);
  }
  ~Profiler() {
    for (cudaEvent_t e : ev) cudaEventDestroy(e);
  }
};

// Parameter blocks of the SAGE-pool encoder (c40): W_s, W_n, W_p, b_p of
// layer l, then M and α.
struct PoolParams {
  float *Ws[3], *Wn[3], *Wp[3], *bp[3], *M, *alpha;
};
static PoolParams pool_params(float* P, int F, int H) {
  PoolParams q{};
  int64_t o = 0;
  for (int l = 0; l < 3; ++l) {
    const int64_t C = l == 0 ? F : H;
    q.Ws[l] = P + o; o += C * H;
    q.Wn[l] = P + o; o += (int64_t)H * H;
    q.Wp[l] = P + o; o += C * H;
    q.bp[l] = P + o; o += H;
  }
  q.M = P + o;
  q.alpha = P + o + (int64_t)H * H;
  return q;
}

// Row GEMM out[R x N] = A[R x K] W (W [K x N]) on the 3xFP16 tensor cores when
// the widths allow (split t of the workspace), else FFMA.
static cudaError_t pool_gemm(Workspace& w, bool tc, int t, const float* A, const float* rsA,
                             const float* W, float* out, int64_t R, int N, int K, cudaStream_t s,
                             int* nl) {
  if (tc) return tc3h_gemm_rows(A, rsA, w.p3_wt_hi[t], w.p3_wt_lo[t], w.p3_wsc[t] + 1, out, R, N, K, s, nl);
  return gemm_nn(A, W, out, R, N, K, s, nl);
}
// out[R x K] = D[R x N] Wᵀ (W [K x N]).
static cudaError_t pool_gemm_t(Workspace& w, bool tc, int t, const float* D, const float* rsD,
                               const float* W, float* out, int64_t R, int K, int N, cudaStream_t s,
                               int* nl) {
  if (tc) return tc3h_gemm_rows(D, rsD, w.p3_w_hi[t], w.p3_w_lo[t], w.p3_wsc[t] + 1, out, R, K, N, s, nl);
  return gemm_nt(D, W, out, R, K, N, s, nl);
}
// dW [K x N] = Aᵀ D.
static cudaError_t pool_dw(Workspace& w, bool tc, const float* A, const float* rsA, const float* D,
                           const float* rsD, float* dW, int64_t R, int K, int N, cudaStream_t s,
                           int* nl) {
  if (tc) return tc3h_gemm_dw(A, rsA, D, rsD, dW, R, K, N, w.dw_part, s, nl);
  return gemm_tn(A, D, dW, R, K, N, w.tn_part, s, nl);
}

// One SAGE-pool layer forward over R rows of A (C columns): Z = A W_s +
// maxagg(ReLU(A W_p + b_p)) W_n.
static cudaError_t pool_layer_fwd(mars_dgi* m, const GraphDev& g, const PoolParams& q, int l,
                                  const float* A, const float* rsA, float* Z, int64_t R,
                                  cudaStream_t s, int* nl) {
  Workspace& w = m->ws;
  const int H = m->H, C = l == 0 ? m->F : H;
  const bool tcC = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(C, H);
  const bool tcH = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(H, H);
  cudaError_t e;
  if ((e = pool_gemm(w, tcC, 3 * l + 2, A, rsA, q.Wp[l], w.pUP[l], R, H, C, s, nl))) return e;
  if ((e = launch_maxagg(g, w.pUP[l], q.bp[l], R, H, w.pAGG[l], w.pIDX[l],
                         tcH ? w.pRsAGG[l] : nullptr, s, nl)))
    return e;
  if ((e = pool_gemm(w, tcC, 3 * l, A, rsA, q.Ws[l], w.pUS, R, H, C, s, nl))) return e;
  if ((e = pool_gemm(w, tcH, 3 * l + 1, w.pAGG[l], w.pRsAGG[l], q.Wn[l], w.pVV, R, H, H, s, nl)))
    return e;
  return launch_add(w.pUS, w.pVV, Z, R * H, s, nl);
}

static cudaError_t pool_splits(mars_dgi* m, const PoolParams& q, cudaStream_t s, int* nl) {
  Workspace& w = m->ws;
  const int F = m->F, H = m->H;
  cudaError_t e;
  for (int l = 0; l < 3; ++l) {
    const int C = l == 0 ? F : H;
    const bool tcC = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(C, H);
    const bool tcH = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(H, H);
    const float* Wm[3] = {q.Ws[l], q.Wn[l], q.Wp[l]};
    for (int h = 0; h < 3; ++h) {
      const int K = h == 1 ? H : C;
      if (!(h == 1 ? tcH : tcC)) continue;
      const int t = 3 * l + h;
      if ((e = tc3h_split_weights(Wm[h], K, H, w.p3_wsc[t], w.p3_wt_hi[t], w.p3_wt_lo[t],
                                  w.p3_w_hi[t], w.p3_w_lo[t], s, nl)))
        return e;
    }
  }
  return cudaSuccess;
}

// The SAGE-pool encoder's step (c40).  Forward per layer as pool_layer_fwd;
// the head as in the GCN step; backward per layer, from dZ:
//   dW_s = Aᵀ dZ, dW_n = aggᵀ dZ, dagg = dZ W_nᵀ, dU_p = maxagg_bwd(dagg),
//   dW_p = Aᵀ dU_p, db_p = 1ᵀ dU_p, and for l > 1
//   dZ_{l-1} = (dZ W_sᵀ + dU_p W_pᵀ) ⊙ PReLU'(Z_{l-1}) with dα fused.
static cudaError_t enqueue_step_pool(mars_dgi* m, const mars_graph* gr, cudaStream_t s, int* nl,
                                     Profiler* prof) {
  Workspace& w = m->ws;
  GraphDev g = gr->dev;
  g.long_part = w.long_part;
  const int F = m->F, H = m->H;
  const int nb = w.nb, K = m->ct.num_neg;
  const int64_t Nt = g.Nt, R = (int64_t)(K + 1) * Nt;
  const PoolParams q = pool_params(m->params, F, H), gq = pool_params(m->grads, F, H);
  float* gloss = m->grads + m->P;
  float* A[3] = {w.Xs, w.Y23[0], w.Y23[1]};
  cudaError_t e;
#define RET(x)                                  \
  do {                                          \
    if ((e = (x)) != cudaSuccess) return e;     \
  } while (0)
#define MARK(ph)                                \
  do {                                          \
    if (prof) RET(prof->mark(ph, s));           \
  } while (0)
  MARK(-1);
  w.hw.nb = nb;
  w.hw.K = K;
  w.hw.readout = m->ct.readout;
  w.hw.loss = m->ct.loss;
  RET(launch_pair_off_k(g.pair_off, g.G, K, w.pair_off_k, s, nl));
  if (m->ct.corruption == MARS_CORRUPT_PERMUTE)
    for (int k = 0; k < K; ++k) {
      GraphDev pv = g;
      pv.pair_off = w.pair_off_k + (int64_t)k * g.G;
      RET(launch_perm(pv, m->cfg.seed, m->d_sp, w.pw, w.perm + (int64_t)k * Nt, s, nl));
    }
  RET(launch_corrupt(g, K, nb, m->ct.corruption, m->ct.mask_rate, m->cfg.seed, m->d_sp,
                     w.pair_off_k, w.perm, w.Xs, s, nl));
  MARK(MARS_PH_PERM);
  RET(pool_splits(m, q, s, nl));
  MARK(MARS_PH_GEMM_FWD);
  for (int l = 0; l < 3; ++l) {
    const int C = l == 0 ? F : H;
    const bool tcC = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(C, H);
    if (l == 0) {
      if (tcC) RET(launch_rowprep(w.Xs, R, F, w.one, nullptr, w.h3_rsY[0], s, nl));
    } else {
      RET(launch_rowprep(w.Z[l - 1], R, H, q.alpha + (l - 1), A[l], tcC ? w.h3_rsY[l] : nullptr,
                         s, nl));
    }
    RET(pool_layer_fwd(m, g, q, l, A[l], w.h3_rsY[l], w.Z[l], R, s, nl));
    MARK(MARS_PH_GEMM_FWD);
  }
  const bool tcH = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(H, H);
  int ns = 0;
  w.hw.rs_dz3 = tcH ? w.h3_rsdZ : nullptr;
  RET(launch_head(g, H, w.Z[2], 0, q.M, q.alpha, m->d_sp, w.hw, w.dZ, gq.M, gloss, &ns, s, nl,
                  nullptr));
  RET(launch_reduce_slots(w.slots[2], ns, gq.alpha + 2, s, nl));
  MARK(MARS_PH_HEAD);
  for (int l = 2; l >= 0; --l) {
    const int C = l == 0 ? F : H;
    const bool tcC = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(C, H);
    RET(pool_dw(w, tcC, A[l], w.h3_rsY[l], w.dZ, w.h3_rsdZ, gq.Ws[l], R, C, H, s, nl));
    RET(pool_dw(w, tcH, w.pAGG[l], w.pRsAGG[l], w.dZ, w.h3_rsdZ, gq.Wn[l], R, H, H, s, nl));
    MARK(MARS_PH_GEMM_DW);
    RET(pool_gemm_t(w, tcH, 3 * l + 1, w.dZ, w.h3_rsdZ, q.Wn[l], w.dY, R, H, H, s, nl));   // dagg
    MARK(MARS_PH_GEMM_DY);
    RET(launch_maxagg_bwd(g, w.dY, w.pIDX[l], w.pUP[l], q.bp[l], R, H, w.pDUP,
                          tcC ? w.pRsDUP : nullptr, s, nl));
    MARK(MARS_PH_SPMM_BWD);
    RET(pool_dw(w, tcC, A[l], w.h3_rsY[l], w.pDUP, w.pRsDUP, gq.Wp[l], R, C, H, s, nl));
    RET(gemm_tn(w.pOnes, w.pDUP, gq.bp[l], R, 1, H, w.tn_part, s, nl));               // db_p
    MARK(MARS_PH_GEMM_DW);
    if (l > 0) {
      RET(pool_gemm_t(w, tcC, 3 * l, w.dZ, w.h3_rsdZ, q.Ws[l], w.pUS, R, C, H, s, nl));     // dA_s
      RET(pool_gemm_t(w, tcC, 3 * l + 2, w.pDUP, w.pRsDUP, q.Wp[l], w.pVV, R, C, H, s, nl));  // dA_p
      MARK(MARS_PH_GEMM_DY);
      const bool tcP = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(l - 1 == 0 ? F : H, H);
      RET(launch_add_prelu_bwd(w.pUS, w.pVV, w.Z[l - 1], q.alpha, l - 1, R, H, w.dZ,
                               tcP || tcH ? w.h3_rsdZ : nullptr, w.slots[l - 1], &ns, s, nl));
      MARK(MARS_PH_SPMM_BWD);
      RET(launch_reduce_slots(w.slots[l - 1], ns, gq.alpha + (l - 1), s, nl));
      MARK(MARS_PH_REDUCE);
    }
  }
  if (m->comm) {
    ncclResult_t r = g_nccl.AllReduce(m->grads, m->grads, (size_t)(m->P + 1), ncclFloat32, ncclSum,
                                      m->comm, s);
    if (r != ncclSuccess) return cudaErrorUnknown;
    MARK(MARS_PH_ALLREDUCE);
  }
  if (m->dp.connected) {
    RET(launch_shard_barrier(m->dp.sync, s, nl));
    RET(launch_grad_sum(m->dp.grads, m->dp.R, m->dp.me, m->P + 1, 0, 0, 1, m->dp.gsum, s, nl));
    RET(launch_shard_barrier(m->dp.sync, s, nl));
    MARK(MARS_PH_ALLREDUCE);
  }
  RET(launch_adam(m->params, m->adam_m, m->adam_v, m->grads_final(), m->P, m->cfg.lr,
                  m->cfg.beta1, m->cfg.beta2, m->cfg.eps, m->cfg.clip_norm, m->guard_part,
                  m->adam_st, s, nl));
  MARK(MARS_PH_ADAM);
#undef MARK
#undef RET
  return cudaSuccess;
}

// The SAGE-mean encoder's step (c38, MARS_ENCODER_SAGE), GEMM-first per layer:
//   A_0 = X~ stacked (materialised, c34/c35), A_l = PReLU(Z_l) (+ row scales)
//   U_n = A W_n, U_s = A W_s                    (rows [0, R) / [nb Nt, nb Nt + R) of U)
//   Z   = one aggregation over the redirected CSR: Z_i = U_s[i] + Σ_j U_n[j] / deg_N(i)
// head as in the GCN step; backward per layer, from dZ:
//   G   = Â_Nᵀ dZ (neighbour-only transpose; its row scales for the GEMM)
//   dW_s = Aᵀ dZ, dW_n = Aᵀ G
//   V_n = dZ W_nᵀ, V_s = dZ W_sᵀ; dZ_{l-1} = (V_s[i] + Σ_j V_n[j] / deg_N(j)) ⊙ PReLU'(Z_{l-1})
//   (the same redirected CSR with the transpose's values, PReLU' and dα fused).
static cudaError_t enqueue_step_sage(mars_dgi* m, const mars_graph* gr, cudaStream_t s, int* nl,
                                     Profiler* prof) {
  Workspace& w = m->ws;
  GraphDev g = gr->dev;
  g.long_part = w.long_part;
  const int F = m->F, H = m->H;
  const int nb = w.nb, K = m->ct.num_neg, nbp = nb / 2;
  const int64_t Nt = g.Nt, Rb = (int64_t)nb * Nt, R = (int64_t)(K + 1) * Nt;
  float* P = m->params;
  float* Gd = m->grads;
  const int64_t o1 = (int64_t)F * H, o2 = (int64_t)H * H;
  // W[l][0] = W_ls, W[l][1] = W_ln (layout c38)
  float* W[3][2] = {{P, P + o1}, {P + 2 * o1, P + 2 * o1 + o2}, {P + 2 * o1 + 2 * o2, P + 2 * o1 + 3 * o2}};
  float* gW[3][2] = {{Gd, Gd + o1}, {Gd + 2 * o1, Gd + 2 * o1 + o2},
                     {Gd + 2 * o1 + 2 * o2, Gd + 2 * o1 + 3 * o2}};
  float* Mp = P + 2 * o1 + 4 * o2;
  float* alpha = Mp + o2;
  float* gM = Gd + 2 * o1 + 4 * o2;
  float* galpha = gM + o2;
  float* gloss = Gd + m->P;
  float* A[3] = {w.Xs, w.Y23[0], w.Y23[1]};       // GEMM inputs of the three layers
  cudaError_t e;
#define RET(x)                                  \
  do {                                          \
    if ((e = (x)) != cudaSuccess) return e;     \
  } while (0)
#define MARK(ph)                                \
  do {                                          \
    if (prof) RET(prof->mark(ph, s));           \
  } while (0)
  MARK(-1);
  w.hw.nb = nb;
  w.hw.K = K;
  w.hw.readout = m->ct.readout;
  w.hw.loss = m->ct.loss;
  // corrupted inputs + the redirected CSR (self entry -> row Rb + i)
  RET(launch_pair_off_k(g.pair_off, g.G, K, w.pair_off_k, s, nl));
  if (m->ct.corruption == MARS_CORRUPT_PERMUTE)
    for (int k = 0; k < K; ++k) {
      GraphDev pv = g;
      pv.pair_off = w.pair_off_k + (int64_t)k * g.G;
      RET(launch_perm(pv, m->cfg.seed, m->d_sp, w.pw, w.perm + (int64_t)k * Nt, s, nl));
    }
  RET(launch_corrupt(g, K, nb, m->ct.corruption, m->ct.mask_rate, m->cfg.seed, m->d_sp,
                     w.pair_off_k, w.perm, w.Xs, s, nl));
  RET(launch_sage_csr(g, Rb, w.sColS, w.sVf, w.sVb, w.sVn, s, nl));
  MARK(MARS_PH_PERM);
  GraphDev gf = g, gbk = g, gn = g;
  gf.colind = w.sColS;
  gf.vals = w.sVf;
  gbk.colind = w.sColS;
  gbk.vals = w.sVb;
  gn.vals = w.sVn;
  bool tc[3];
  for (int l = 0; l < 3; ++l) {
    const int Cin = l == 0 ? F : H;
    tc[l] = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(Cin, H);
    if (tc[l])
      for (int h = 0; h < 2; ++h) {
        const int t = 2 * l + h;
        RET(tc3h_split_weights(W[l][h], Cin, H, w.s3_wsc[t], w.s3_wt_hi[t], w.s3_wt_lo[t],
                               w.s3_w_hi[t], w.s3_w_lo[t], s, nl));
      }
  }
  MARK(MARS_PH_GEMM_FWD);
  float* U[2] = {w.sU + Rb * H, w.sU};           // [0]: U_s, [1]: U_n
  float* Vv[2] = {w.sV + Rb * H, w.sV};          // [0]: V_s, [1]: V_n
  auto blk = [&](float* base, int p, int C) { return base + (int64_t)2 * p * Nt * C; };
  // forward
  for (int l = 0; l < 3; ++l) {
    const int Cin = l == 0 ? F : H;
    if (l == 0) {
      if (tc[0]) RET(launch_rowprep(w.Xs, R, F, w.one, nullptr, w.h3_rsY[0], s, nl));
    } else {
      RET(launch_rowprep(w.Z[l - 1], R, H, alpha + (l - 1), A[l], tc[l] ? w.h3_rsY[l] : nullptr,
                         s, nl));
    }
    for (int h = 0; h < 2; ++h) {
      const int t = 2 * l + h;
      if (tc[l])
        RET(tc3h_gemm_rows(A[l], w.h3_rsY[l], w.s3_wt_hi[t], w.s3_wt_lo[t], w.s3_wsc[t] + 1, U[h],
                           R, H, Cin, s, nl));
      else RET(gemm_nn(A[l], W[l][h], U[h], R, H, Cin, s, nl));
    }
    MARK(MARS_PH_GEMM_FWD);
    for (int p = 0; p < nbp; ++p)
      RET(launch_spmm_fwd(gf, H, blk(w.sU, p, H), 0, nullptr, w.one, 0, blk(w.Z[l], p, H), 0,
                          2 * p + 1 <= K, s, nl, nullptr, nullptr));
    MARK(MARS_PH_SPMM_FWD);
  }
  // head (a8-a11) -> dZ3
  int ns = 0;
  w.hw.rs_dz3 = tc[2] ? w.h3_rsdZ : nullptr;
  RET(launch_head(g, H, w.Z[2], 0, Mp, alpha, m->d_sp, w.hw, w.dZ, gM, gloss, &ns, s, nl, nullptr));
  RET(launch_reduce_slots(w.slots[2], ns, galpha + 2, s, nl));
  MARK(MARS_PH_HEAD);
  // backward
  for (int l = 2; l >= 0; --l) {
    const int Cin = l == 0 ? F : H;
    for (int p = 0; p < nbp; ++p)        // G = Â_Nᵀ dZ
      RET(launch_spmm_fwd(gn, H, blk(w.dZ, p, H), 0, nullptr, w.one, 0, blk(w.dY, p, H), 0,
                          2 * p + 1 <= K, s, nl, nullptr, tc[l] ? w.rsG + 2LL * p * Nt : nullptr));
    MARK(MARS_PH_SPMM_BWD);
    if (tc[l]) {
      RET(tc3h_gemm_dw(A[l], w.h3_rsY[l], w.dZ, w.h3_rsdZ, gW[l][0], R, Cin, H, w.dw_part, s, nl));
      RET(tc3h_gemm_dw(A[l], w.h3_rsY[l], w.dY, w.rsG, gW[l][1], R, Cin, H, w.dw_part, s, nl));
    } else {
      RET(gemm_tn(A[l], w.dZ, gW[l][0], R, Cin, H, w.tn_part, s, nl));
      RET(gemm_tn(A[l], w.dY, gW[l][1], R, Cin, H, w.tn_part, s, nl));
    }
    MARK(MARS_PH_GEMM_DW);
    if (l > 0) {
      for (int h = 0; h < 2; ++h) {
        const int t = 2 * l + h;
        if (tc[l])
          RET(tc3h_gemm_rows(w.dZ, w.h3_rsdZ, w.s3_w_hi[t], w.s3_w_lo[t], w.s3_wsc[t] + 1, Vv[h], R,
                             Cin, H, s, nl));
        else RET(gemm_nt(w.dZ, W[l][h], Vv[h], R, Cin, H, s, nl));
      }
      MARK(MARS_PH_GEMM_DY);
      ns = 0;
      for (int p = 0; p < nbp; ++p) {
        int nsp = 0;
        RET(launch_spmm_bwd(gbk, Cin, blk(w.sV, p, Cin), blk(w.Z[l - 1], p, Cin), 0, alpha, l - 1,
                            blk(w.dZ, p, Cin), w.slots[l - 1] + ns, &nsp, s, nl, nullptr,
                            tc[l - 1] ? w.h3_rsdZ + 2LL * p * Nt : nullptr));
        ns += nsp;
      }
      MARK(MARS_PH_SPMM_BWD);
      RET(launch_reduce_slots(w.slots[l - 1], ns, galpha + (l - 1), s, nl));
      MARK(MARS_PH_REDUCE);
    }
  }
  if (m->comm) {
    ncclResult_t r = g_nccl.AllReduce(m->grads, m->grads, (size_t)(m->P + 1), ncclFloat32, ncclSum,
                                      m->comm, s);
    if (r != ncclSuccess) return cudaErrorUnknown;
    MARK(MARS_PH_ALLREDUCE);
  }
  if (m->dp.connected) {
    RET(launch_shard_barrier(m->dp.sync, s, nl));
    RET(launch_grad_sum(m->dp.grads, m->dp.R, m->dp.me, m->P + 1, 0, 0, 1, m->dp.gsum, s, nl));
    RET(launch_shard_barrier(m->dp.sync, s, nl));
    MARK(MARS_PH_ALLREDUCE);
  }
  RET(launch_adam(m->params, m->adam_m, m->adam_v, m->grads_final(), m->P, m->cfg.lr,
                  m->cfg.beta1, m->cfg.beta2, m->cfg.eps, m->cfg.clip_norm, m->guard_part,
                  m->adam_st, s, nl));
  MARK(MARS_PH_ADAM);
#undef MARK
#undef RET
  return cudaSuccess;
}

// Enqueues one full DGI step (a4-a14) on stream s.  Reads step scalars from m->d_sp.
static cudaError_t enqueue_step(mars_dgi* m, const mars_graph* gr, cudaStream_t s, int* nl,
                                Profiler* prof = nullptr) {
  if (m->sage) return enqueue_step_sage(m, gr, s, nl, prof);
  if (m->pool) return enqueue_step_pool(m, gr, s, nl, prof);
  Workspace& w = m->ws;
  GraphDev g = gr->dev;
  g.long_part = w.long_part;
  const int F = m->F, H = m->H;
  // NEXT-4 variants (c34-c37): nb stacked blocks [pos; neg_1..neg_K; pad];
  // the default DGI step has nb = 2 and the fused layer-1 corruption gather
  const int nb = w.nb, K = m->ct.num_neg, nbp = nb / 2;
  const bool mat = m->ct_materialise();
  // GEMM rows: the K + 1 real blocks.  A padding block (K even) is zero from
  // allocation and never written: its forward aggregation is skipped (the last
  // pair runs one branch), and the backward aggregation's pass over it gathers
  // zeros into zeros.
  const int64_t R = (int64_t)(K + 1) * g.Nt;
  GraphDev gb = g;                       // the backward aggregation's view (Âᵀ)
  w.hw.nb = nb;
  w.hw.K = K;
  w.hw.readout = m->ct.readout;
  w.hw.loss = m->ct.loss;
  float* W[3] = {m->params, m->params + (int64_t)F * H, m->params + (int64_t)F * H + (int64_t)H * H};
  float* Mp = m->params + (int64_t)F * H + 2LL * H * H;
  float* alpha = m->params + (int64_t)F * H + 3LL * H * H;
  float* gW[3] = {m->grads, m->grads + (int64_t)F * H, m->grads + (int64_t)F * H + (int64_t)H * H};
  float* gM = m->grads + (int64_t)F * H + 2LL * H * H;
  float* galpha = m->grads + (int64_t)F * H + 3LL * H * H;
  float* gloss = m->grads + m->P;
  float* Ys[3] = {w.Y1, w.Y23[0], w.Y23[1]};
  cudaError_t e;
#define RET(x)                                  \
  do {                                          \
    if ((e = (x)) != cudaSuccess) return e;     \
  } while (0)
#define MARK(ph)                                \
  do {                                          \
    if (prof) RET(prof->mark(ph, s));           \
  } while (0)
  MARK(-1);
  // Row-sharded graph: exchange steps between the shards (shard.cu).  A
  // barrier precedes every read of buffers the peers wrote in this step.
  const bool shard = m->sh.connected && gr->uid == m->sh.guid;
  if (m->ct.aggregator == MARS_AGG_SAGE_GCN) {
    RET(launch_sage_vals(g, w.valsR, w.valsC, s, nl));
    g.vals = w.valsR;
    gb.vals = w.valsC;
  }
  if (!mat) {
    // a4: corruption permutation (the X~ gather is fused into layer 1's SpMM);
    // a row-sharded graph permutes the whole graph on every shard
    cudaError_t pe = cudaErrorNotSupported;
    if (MARS_PERM_GRAPH && !shard && !gr->sharded)
      pe = launch_perm_graph(g, m->cfg.seed, m->d_sp, w.pw, w.perm,
                             MARS_PERM_GRAPH_COLPERM ? w.colperm : nullptr, s, nl);
    if (pe == cudaErrorNotSupported) {
      RET(launch_perm(gr->perm_view(), m->cfg.seed, m->d_sp, w.pw, w.perm, s, nl));
      RET(launch_colperm(g, w.perm, w.colperm, s, nl));
    } else {
      RET(pe);
      if (!MARS_PERM_GRAPH_COLPERM) RET(launch_colperm(g, w.perm, w.colperm, s, nl));
    }
  } else {
    // K samples (c34): sample k of graph g is pair pair_off[g] K + k; the
    // corrupted layer-1 inputs are materialised block by block (c35)
    RET(launch_pair_off_k(g.pair_off, g.G, K, w.pair_off_k, s, nl));
    if (m->ct.corruption == MARS_CORRUPT_PERMUTE)
      for (int k = 0; k < K; ++k) {
        GraphDev pv = g;
        pv.pair_off = w.pair_off_k + (int64_t)k * g.G;
        RET(launch_perm(pv, m->cfg.seed, m->d_sp, w.pw, w.perm + (int64_t)k * g.Nt, s, nl));
      }
    RET(launch_corrupt(g, K, nb, m->ct.corruption, m->ct.mask_rate, m->cfg.seed, m->d_sp,
                       w.pair_off_k, w.perm, w.Xs, s, nl));
  }
  MARK(MARS_PH_PERM);
  const bool b16 = m->cfg.precision == MARS_BF16;        // bf16 storage + bf16 MMAs
  bool tc[3];
  for (int l = 0; l < 3; ++l)
    tc[l] = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(l == 0 ? F : H, H);
  if (!b16 && tc[0] && tc[1] && tc[2]) {                  // one launch for the three splits
    W3Split a{};
    a.H = H;
    for (int l = 0; l < 3; ++l) {
      a.W[l] = W[l];
      a.cin[l] = l == 0 ? F : H;
      a.wsc[l] = w.h3_wsc[l];
      a.bt_hi[l] = w.h3_wt_hi[l];
      a.bt_lo[l] = w.h3_wt_lo[l];
      a.b_hi[l] = w.h3_w_hi[l];
      a.b_lo[l] = w.h3_w_lo[l];
    }
    RET(tc3h_split_weights_all(a, 3, s, nl));
  } else {
    for (int l = 0; l < 3; ++l) {
      int Cin = l == 0 ? F : H;
      if (b16) RET(tc16_weights(W[l], Cin, H, w.w16t[l], w.w16[l], s, nl));
      else if (tc[l])
        RET(tc3h_split_weights(W[l], Cin, H, w.h3_wsc[l], w.h3_wt_hi[l], w.h3_wt_lo[l],
                               w.h3_w_hi[l], w.h3_w_lo[l], s, nl));
    }
  }
  MARK(MARS_PH_GEMM_FWD);
  const size_t es = b16 ? 2 : 4;                         // storage bytes per element
  // rows [2p Nt, (2p + 2) Nt) of a stacked buffer of C columns (block pair p)
  auto blk = [&](const void* base, int p, int C, size_t bytes) -> char* {
    return (char*)base + (size_t)2 * p * g.Nt * C * bytes;
  };
  // a5-a7: forward, l = 1..3
  for (int l = 0; l < 3; ++l) {
    int Cin = l == 0 ? F : H;
    const void* T = l == 0 ? (const void*)g.X : (const void*)w.Z[l - 1];
    if (shard && l > 0) {
      RET(launch_shard_barrier(m->sh.sync, s, nl));   // peers' Z_{l-1} complete
      MARK(MARS_PH_EXCHANGE);
    }
    if (!mat || l > 0) {
      // one aggregation per block pair (the positive / corrupted pair of the
      // default step): both halves of the pair share each CSR entry read
      for (int p = 0; p < nbp; ++p)
        RET(launch_spmm_fwd(g, Cin, l == 0 ? T : blk(T, p, Cin, es), b16 && l > 0, w.colperm,
                            alpha, l - 1, blk(Ys[l], p, Cin, es), b16, 2 * p + 1 <= K, s, nl,
                            shard && l > 0 ? &m->sh.z[l - 1] : nullptr,
                            tc[l] ? w.h3_rsY[l] + 2LL * p * g.Nt : nullptr));
    } else {
      // materialised layer-1 inputs: the stacked aggregation with slope-1 PReLU
      for (int p = 0; p < nbp; ++p)
        RET(launch_spmm_fwd(g, Cin, blk(w.Xs, p, F, 4), 0, nullptr, w.one, 0,
                            blk(Ys[0], p, Cin, es), b16, 2 * p + 1 <= K, s, nl, nullptr,
                            tc[0] ? w.h3_rsY[0] + 2LL * p * g.Nt : nullptr));
    }
    MARK(MARS_PH_SPMM_FWD);
    if (b16) RET(tc16_gemm_rows(Ys[l], w.w16t[l], w.Z[l], R, H, Cin, s, nl));
    else if (tc[l])
      RET(tc3h_gemm_rows(Ys[l], w.h3_rsY[l], w.h3_wt_hi[l], w.h3_wt_lo[l], w.h3_wsc[l] + 1,
                         w.Z[l], R, H, Cin, s, nl));
    else RET(gemm_nn(Ys[l], W[l], w.Z[l], R, H, Cin, s, nl));
    MARK(MARS_PH_GEMM_FWD);
  }
  // a8-a11 + dZ3
  int ns = 0;
  HeadShard hs{};
  if (shard) {
    hs.sync = &m->sh.sync;
    hs.x_own[0] = m->sh.xbuf;
    hs.x_own[1] = m->sh.xbuf + H + 1;
    hs.x_peers[0] = m->sh.x[0];
    hs.x_peers[1] = m->sh.x[1];
  }
  w.hw.rs_dz3 = !b16 && tc[2] ? w.h3_rsdZ : nullptr;   // dZ3 row scales (3xFP16 dY GEMM)
  RET(launch_head(g, H, w.Z[2], b16, Mp, alpha, m->d_sp, w.hw, w.dZ, gM, gloss, &ns, s, nl,
                  shard ? &hs : nullptr));
  RET(launch_reduce_slots(w.slots[2], ns, galpha + 2, s, nl));
  const size_t kb_bytes = (size_t)2 * g.Nt * H * es;     // test hook: blocks 0 and 1
  const bool kb = m->keep_bwd && m->kb_rows >= g.Nt;
  if (kb) RET(cudaMemcpyAsync(m->kb_dZ[2], w.dZ, kb_bytes, cudaMemcpyDeviceToDevice, s));
  MARK(MARS_PH_HEAD);
  // a12: backward, l = 3..1
  for (int l = 2; l >= 0; --l) {
    int Cin = l == 0 ? F : H;
    if (b16) RET(tc16_gemm_dw(Ys[l], w.dZ, gW[l], R, Cin, H, w.dw16_part, s, nl));
    else if (tc[l])
      RET(tc3h_gemm_dw(Ys[l], w.h3_rsY[l], w.dZ, w.h3_rsdZ, gW[l], R, Cin, H, w.dw_part, s, nl));
    else RET(gemm_tn(Ys[l], w.dZ, gW[l], R, Cin, H, w.tn_part, s, nl));
    MARK(MARS_PH_GEMM_DW);
    if (l > 0) {
      // sharded: the two backward aggregations use separate peer-visible dY buffers
      float* dYl = (shard && l == 1) ? static_cast<float*>(m->sh.dY2) : w.dY;
      if (b16) RET(tc16_gemm_rows(w.dZ, w.w16[l], dYl, R, Cin, H, s, nl));
      else if (tc[l])
        RET(tc3h_gemm_rows(w.dZ, w.h3_rsdZ, w.h3_w_hi[l], w.h3_w_lo[l], w.h3_wsc[l] + 1, dYl, R,
                           Cin, H, s, nl));
      else RET(gemm_nt(w.dZ, W[l], dYl, R, Cin, H, s, nl));
      if (kb) RET(cudaMemcpyAsync(m->kb_dY[l - 1], dYl, kb_bytes, cudaMemcpyDeviceToDevice, s));
      MARK(MARS_PH_GEMM_DY);
      if (shard) {
        RET(launch_shard_barrier(m->sh.sync, s, nl));  // peers' dY_l complete
        MARK(MARS_PH_EXCHANGE);
      }
      ns = 0;
      for (int p = 0; p < nbp; ++p) {
        int nsp = 0;
        RET(launch_spmm_bwd(gb, Cin, blk(dYl, p, Cin, es), blk(w.Z[l - 1], p, Cin, es), b16,
                            alpha, l - 1, blk(w.dZ, p, Cin, es), w.slots[l - 1] + ns, &nsp, s, nl,
                            shard ? &m->sh.dy[l == 2 ? 0 : 1] : nullptr,
                            tc[l - 1] ? w.h3_rsdZ + 2LL * p * g.Nt : nullptr));
        ns += nsp;
      }
      if (kb) RET(cudaMemcpyAsync(m->kb_dZ[l - 1], w.dZ, kb_bytes, cudaMemcpyDeviceToDevice, s));
      MARK(MARS_PH_SPMM_BWD);
      RET(launch_reduce_slots(w.slots[l - 1], ns, galpha + (l - 1), s, nl));
      MARK(MARS_PH_REDUCE);
    }
  }
  // a13: data-parallel gradient allreduce (grads + loss, pre-scaled by 1/B)
  if (m->comm) {
    ncclResult_t r = g_nccl.AllReduce(m->grads, m->grads, (size_t)(m->P + 1), ncclFloat32, ncclSum,
                                      m->comm, s);
    if (r != ncclSuccess) return cudaErrorUnknown;
    MARK(MARS_PH_ALLREDUCE);
  }
  // a13 over peer memory: barrier (every rank's partials complete), rank-ordered
  // fp64 sum of the partial gradients + loss, barrier (every rank has read
  // them, so the next step may overwrite its own)
  if (m->dp.connected) {
    RET(launch_shard_barrier(m->dp.sync, s, nl));
    RET(launch_grad_sum(m->dp.grads, m->dp.R, m->dp.me, m->P + 1, 0, 0, 1, m->dp.gsum, s, nl));
    RET(launch_shard_barrier(m->dp.sync, s, nl));
    MARK(MARS_PH_ALLREDUCE);
  }
  // row-sharded: sum the shards' W / alpha partials in rank order (dM and the
  // loss are already global on every shard after the head exchange)
  if (shard) {
    RET(launch_shard_barrier(m->sh.sync, s, nl));
    const int64_t mb = (int64_t)F * H + 2LL * H * H;
    RET(launch_grad_sum(m->sh.grads, m->sh.sync.P, m->sh.sync.me, m->P + 1, mb, mb + (int64_t)H * H,
                        0, m->sh.gsum, s, nl));
    MARK(MARS_PH_EXCHANGE);
  }
  // a14: Adam
  RET(launch_adam(m->params, m->adam_m, m->adam_v, m->grads_final(), m->P, m->cfg.lr,
                  m->cfg.beta1, m->cfg.beta2, m->cfg.eps, m->cfg.clip_norm, m->guard_part,
                  m->adam_st, s, nl));
  MARK(MARS_PH_ADAM);
#undef MARK
#undef RET
  return cudaSuccess;
}

// Writes the step scalars for the next step into a pinned ring slot and
// enqueues their copy to the device (the captured graph reads them there).
static mars_status push_step_params(mars_dgi* m, uint64_t step_index, int64_t pair_base,
                                    int64_t global_batch) {
  cudaStream_t s = m->stream;
  int slot = m->sp_next;
  m->sp_next = (m->sp_next + 1) % m->sp_ring;
  CK(cudaEventSynchronize(m->sp_ev[slot]));
  StepParams& sp = m->h_sp[slot];
  sp.step_index = step_index;
  sp.pair_base = pair_base;
  sp.inv_batch = (float)(1.0 / (double)global_batch);
  CK(cudaMemcpyAsync(m->d_sp, &sp, sizeof sp, cudaMemcpyHostToDevice, s));
  CK(cudaEventRecord(m->sp_ev[slot], s));
  return MARS_OK;
}

// A guarded Adam update was skipped (non-finite loss or gradient, adam.cu)
// since the last report: MARS_ENUMERIC once per skipped batch of steps.
static mars_status check_skipped(mars_dgi* m, int32_t skipped) {
  if (skipped <= m->skipped_seen) return MARS_OK;
  const int32_t n = skipped - m->skipped_seen;
  m->skipped_seen = skipped;
  return fail(MARS_ENUMERIC, "non-finite loss or gradient: %d Adam update(s) skipped", n);
}

static mars_status check_step_args(mars_dgi* m, const mars_graph* g, int64_t global_batch) {
  if (mars_status st = check_dgi(m)) return st;
  if (mars_status st = check_graph(g)) return st;
  if (g->F != m->F) return fail(MARS_EINVAL, "graph feat_dim %d != model in_dim %d", g->F, m->F);
  if (g->device != m->cfg.device) return fail(MARS_EINVAL, "graph and model on different devices");
  if (global_batch < g->G) return fail(MARS_EINVAL, "global_batch < graphs in this set");
  if (m->dp.R > 1 && !m->dp.connected)
    return fail(MARS_ESTATE, "peer-memory data parallelism: mars_dp_connect first");
  return MARS_OK;
}

extern "C" mars_status mars_dgi_profile_step(mars_dgi* m, const mars_graph* g, uint64_t step_index,
                                             int64_t pair_base, int64_t global_batch,
                                             int32_t* phase_ids, float* phase_ms,
                                             int32_t max_phases, int32_t* n_phases) {
  if (mars_status st = check_step_args(m, g, global_batch)) return st;
  if (!phase_ids || !phase_ms || !n_phases) return fail(MARS_EINVAL, "NULL output");
  CK(cudaSetDevice(m->cfg.device));
  if (mars_status st = ensure_ws(m, g)) return st;
  if (mars_status st = push_step_params(m, step_index, pair_base, global_batch)) return st;
  Profiler prof;
  int nl = 0;
  cudaError_t e = enqueue_step(m, g, m->stream, &nl, &prof);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(MARS_ECUDA, "profile step: %s", cudaGetErrorString(e));
  }
  g->note_use(m->stream);
  CK(cudaStreamSynchronize(m->stream));
  int n = 0;
  for (size_t k = 1; k < prof.ev.size() && n < max_phases; ++k, ++n) {
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, prof.ev[k - 1], prof.ev[k]));
    phase_ids[n] = prof.phase[k];
    phase_ms[n] = ms;
  }
  *n_phases = n;
  m->last_launches = nl;
  m->last_Nt = g->dev.Nt;
  m->kb_valid_Nt = m->keep_bwd ? g->dev.Nt : 0;
  return MARS_OK;
}

static mars_status run_step(mars_dgi* m, const mars_graph* g, uint64_t step_index,
                            int64_t pair_base, int64_t global_batch);

extern "C" mars_status mars_dgi_step(mars_dgi* m, const mars_graph* g, uint64_t step_index,
                                     int64_t pair_base, int64_t global_batch, mars_step_out* out) {
  if (mars_status st = check_step_args(m, g, global_batch)) return st;
  if (out && out->perms && m->ct.corruption != MARS_CORRUPT_PERMUTE)
    return fail(MARS_EINVAL, "no permutations: the corruption is feature masking");
  CK(cudaSetDevice(m->cfg.device));
  if (mars_status st = ensure_ws(m, g)) return st;
  if (mars_status st = run_step(m, g, step_index, pair_base, global_batch)) return st;
  cudaStream_t s = m->stream;
  if (out && (out->loss || out->grads || out->perms)) {
    float loss = 0.f;
    int32_t skipped = 0;
    CK(cudaMemcpyAsync(&loss, m->grads_final() + m->P, sizeof(float), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&skipped, &m->adam_st->skipped, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    if (out->grads)
      CK(cudaMemcpyAsync(out->grads, m->grads_final(), sizeof(float) * m->P,
                         cudaMemcpyDeviceToHost, s));
    const int K = m->ct.num_neg;
    if (out->perms)
      CK(cudaMemcpyAsync(out->perms, m->ws.perm, sizeof(int32_t) * g->Nt * K,
                         cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (out->perms)
      for (int k = 0; k < K; ++k)
        for (int gi = 0; gi < g->G; ++gi)
          for (int32_t i = g->h_node_off[gi]; i < g->h_node_off[gi + 1]; ++i)
            out->perms[(int64_t)k * g->Nt + i] -= g->h_node_off[gi];
    if (out->loss) *out->loss = loss;
    if (mars_status st = check_skipped(m, skipped)) return st;
    if (!std::isfinite(loss)) return fail(MARS_ENUMERIC, "non-finite loss");
  }
  return MARS_OK;
}

namespace {
// NEXT-1 best-loss tracking (c17): strict < keeps the earliest minimum.
__global__ void k_track_decide(const float* __restrict__ loss, int64_t t, float* __restrict__ losses,
                               float* __restrict__ best_loss, int64_t* __restrict__ best_step,
                               int32_t* __restrict__ flag) {
  const float l = *loss;
  losses[t] = l;
  const bool better = l < *best_loss;
  *flag = better ? 1 : 0;
  if (better) {
    *best_loss = l;
    *best_step = t;
  }
}
__global__ void k_track_copy(const int32_t* __restrict__ flag, const float* __restrict__ prev,
                             float* __restrict__ best, int64_t P) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < P && *flag) best[i] = prev[i];
}
__global__ void k_init_best(float* best_loss, int64_t* best_step) {
  *best_loss = INFINITY;
  *best_step = -1;
}
}  // namespace

extern "C" mars_status mars_dgi_pretrain(mars_dgi* m, const mars_graph* g, uint64_t step0,
                                         int32_t n_steps, int64_t pair_base, int64_t global_batch,
                                         float* losses, float* best_params, float* best_loss,
                                         int64_t* best_step) {
  if (mars_status st = check_step_args(m, g, global_batch)) return st;
  if (n_steps < 1) return fail(MARS_EINVAL, "n_steps < 1");
  CK(cudaSetDevice(m->cfg.device));
  if (mars_status st = ensure_ws(m, g)) return st;
  cudaStream_t s = m->stream;
  float *prev = nullptr, *best = nullptr, *d_losses = nullptr, *d_bl = nullptr;
  int64_t* d_bs = nullptr;
  int32_t* d_flag = nullptr;
  struct FreeAll {
    std::vector<void*> v;
    ~FreeAll() { for (void* p : v) cudaFree(p); }
  } fa;
  CK(dalloc(&prev, m->P)); fa.v.push_back(prev);
  CK(dalloc(&best, m->P)); fa.v.push_back(best);
  CK(dalloc(&d_losses, (size_t)n_steps)); fa.v.push_back(d_losses);
  CK(dalloc(&d_bl, 1)); fa.v.push_back(d_bl);
  CK(dalloc(&d_bs, 1)); fa.v.push_back(d_bs);
  CK(dalloc(&d_flag, 1)); fa.v.push_back(d_flag);
  k_init_best<<<1, 1, 0, s>>>(d_bl, d_bs);
  CK(cudaMemcpyAsync(best, m->params, sizeof(float) * m->P, cudaMemcpyDeviceToDevice, s));
  for (int32_t t = 0; t < n_steps; ++t) {
    // the parameters a step's loss is computed with are the ones before its Adam update
    CK(cudaMemcpyAsync(prev, m->params, sizeof(float) * m->P, cudaMemcpyDeviceToDevice, s));
    if (mars_status st = run_step(m, g, step0 + (uint64_t)t, pair_base, global_batch)) return st;
    k_track_decide<<<1, 1, 0, s>>>(m->grads_final() + m->P, t, d_losses, d_bl, d_bs, d_flag);
    k_track_copy<<<cdiv(m->P, 256), 256, 0, s>>>(d_flag, prev, best, m->P);
    CK(cudaGetLastError());
  }
  int64_t bs = -1;
  float bl = 0.f;
  if (losses) CK(cudaMemcpyAsync(losses, d_losses, sizeof(float) * n_steps, cudaMemcpyDeviceToHost, s));
  if (best_params) CK(cudaMemcpyAsync(best_params, best, sizeof(float) * m->P, cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(&bl, d_bl, sizeof(float), cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(&bs, d_bs, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  int32_t skipped = 0;
  CK(cudaMemcpyAsync(&skipped, &m->adam_st->skipped, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (best_loss) *best_loss = bl;
  if (best_step) *best_step = bs;
  if (bs < 0) return fail(MARS_ENUMERIC, "no finite loss during pre-training");
  return check_skipped(m, skipped);
}

// Enqueues one step (graph replay or eager) after the step scalars.
static mars_status run_step(mars_dgi* m, const mars_graph* g, uint64_t step_index,
                            int64_t pair_base, int64_t global_batch) {
  cudaStream_t s = m->stream;
  if (mars_status st = push_step_params(m, step_index, pair_base, global_batch)) return st;

  int nl = 0;
  // Capture once a graph set is stepped twice in a row (pre-training reuses one
  // set for many steps); a set seen once (streamed batches) runs eagerly.
  mars_dgi::ExecEntry* ent = m->capture ? m->find_exec(g->uid, s) : nullptr;
  const bool replay = m->capture && (ent || m->seen_recently(g->uid));
  m->note_seen(g->uid);
  if (replay) {
    if (!ent) {
      cudaGraph_t graph;
      CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
      cudaError_t e = enqueue_step(m, g, s, &nl);
      cudaError_t e2 = cudaStreamEndCapture(s, &graph);
      if (e != cudaSuccess || e2 != cudaSuccess) {
        if (e2 == cudaSuccess) cudaGraphDestroy(graph);
        cudaGetLastError();
        return fail(MARS_ECUDA, "step capture failed: %s",
                    cudaGetErrorString(e != cudaSuccess ? e : e2));
      }
      cudaGraphExec_t ex = nullptr;
      cudaError_t e3 = cudaGraphInstantiate(&ex, graph, 0);
      cudaGraphDestroy(graph);
      CK(e3);
      ent = m->add_exec(g->uid, s, ex, nl);
    }
    ent->last = ++m->exec_clock;
    CK(cudaGraphLaunch(ent->exec, s));
    nl = (int)ent->launches;
  } else {
    cudaError_t e = enqueue_step(m, g, s, &nl);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(m->comm && e == cudaErrorUnknown ? MARS_ENCCL : MARS_ECUDA, "step: %s",
                  cudaGetErrorString(e));
    }
  }
  g->note_use(s);
  m->last_launches = nl;
  m->last_Nt = g->dev.Nt;
  m->kb_valid_Nt = m->keep_bwd ? g->dev.Nt : 0;
  return MARS_OK;
}

extern "C" int64_t mars_dgi_last_launches(const mars_dgi* m) {
  return (m && m->tag == kTagDgi) ? m->last_launches : -1;
}

// ---------------------------------------------------------------- encode (a15)
// Forward of the positive branch only (a15): Y_l, Z_l of rows [0, ΣN) and
// H3 = PReLU(Z3) into w.dY (the embeddings, device).
// a15 under the SAGE-mean encoder (c38): the positive branch only, the
// redirected CSR's self entries pointing at row Nt + i of [U_n; U_s].
static cudaError_t enqueue_encode_sage(mars_dgi* m, const mars_graph* gr, cudaStream_t s, int* nl) {
  Workspace& w = m->ws;
  GraphDev g = gr->dev;
  g.long_part = w.long_part;
  const int F = m->F, H = m->H;
  const int64_t Nt = g.Nt, o1 = (int64_t)F * H, o2 = (int64_t)H * H;
  float* P = m->params;
  float* W[3][2] = {{P, P + o1}, {P + 2 * o1, P + 2 * o1 + o2}, {P + 2 * o1 + 2 * o2, P + 2 * o1 + 3 * o2}};
  float* alpha = P + 2 * o1 + 5 * o2;
  const float* A[3] = {g.X, w.Y23[0], w.Y23[1]};
  float* U[2] = {w.sU + Nt * H, w.sU};
  cudaError_t e;
  if ((e = launch_sage_csr(g, Nt, w.sColS, w.sVf, nullptr, nullptr, s, nl))) return e;
  GraphDev gf = g;
  gf.colind = w.sColS;
  gf.vals = w.sVf;
  for (int l = 0; l < 3; ++l) {
    const int Cin = l == 0 ? F : H;
    const bool tc = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(Cin, H);
    if (l == 0) {
      if (tc && (e = launch_rowprep(g.X, Nt, F, w.one, nullptr, w.h3_rsY[0], s, nl))) return e;
    } else if ((e = launch_rowprep(w.Z[l - 1], Nt, H, alpha + (l - 1), w.Y23[l - 1],
                                   tc ? w.h3_rsY[l] : nullptr, s, nl))) {
      return e;
    }
    for (int h = 0; h < 2; ++h) {
      const int t = 2 * l + h;
      if (tc) {
        if ((e = tc3h_split_weights(W[l][h], Cin, H, w.s3_wsc[t], w.s3_wt_hi[t], w.s3_wt_lo[t],
                                    w.s3_w_hi[t], w.s3_w_lo[t], s, nl)))
          return e;
        if ((e = tc3h_gemm_rows(A[l], w.h3_rsY[l], w.s3_wt_hi[t], w.s3_wt_lo[t], w.s3_wsc[t] + 1,
                                U[h], Nt, H, Cin, s, nl)))
          return e;
      } else if ((e = gemm_nn(A[l], W[l][h], U[h], Nt, H, Cin, s, nl))) {
        return e;
      }
    }
    if ((e = launch_spmm_fwd(gf, H, w.sU, 0, nullptr, w.one, 0, w.Z[l], 0, 0, s, nl, nullptr,
                             nullptr)))
      return e;
  }
  return launch_prelu(w.Z[2], 0, alpha, 2, w.dY, Nt * H, s, nl);
}

// a15 under the SAGE-pool encoder (c40): the positive rows only.
static cudaError_t enqueue_encode_pool(mars_dgi* m, const mars_graph* gr, cudaStream_t s, int* nl) {
  Workspace& w = m->ws;
  GraphDev g = gr->dev;
  g.long_part = w.long_part;
  const int F = m->F, H = m->H;
  const int64_t Nt = g.Nt;
  const PoolParams q = pool_params(m->params, F, H);
  const float* A[3] = {g.X, w.Y23[0], w.Y23[1]};
  cudaError_t e;
  if ((e = pool_splits(m, q, s, nl))) return e;
  for (int l = 0; l < 3; ++l) {
    const int C = l == 0 ? F : H;
    const bool tcC = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(C, H);
    if (l == 0) {
      if (tcC && (e = launch_rowprep(g.X, Nt, F, w.one, nullptr, w.h3_rsY[0], s, nl))) return e;
    } else if ((e = launch_rowprep(w.Z[l - 1], Nt, H, q.alpha + (l - 1), w.Y23[l - 1],
                                   tcC ? w.h3_rsY[l] : nullptr, s, nl))) {
      return e;
    }
    if ((e = pool_layer_fwd(m, g, q, l, A[l], w.h3_rsY[l], w.Z[l], Nt, s, nl))) return e;
  }
  return launch_prelu(w.Z[2], 0, q.alpha, 2, w.dY, Nt * H, s, nl);
}

static cudaError_t enqueue_encode(mars_dgi* m, const mars_graph* g, cudaStream_t s, int* nl) {
  if (m->sage) return enqueue_encode_sage(m, g, s, nl);
  if (m->pool) return enqueue_encode_pool(m, g, s, nl);
  Workspace& w = m->ws;
  GraphDev gd = g->dev;
  gd.long_part = w.long_part;
  const int F = m->F, H = m->H;
  float* W[3] = {m->params, m->params + (int64_t)F * H, m->params + (int64_t)F * H + (int64_t)H * H};
  float* alpha = m->params + (int64_t)F * H + 3LL * H * H;
  float* Ys[3] = {w.Y1, w.Y23[0], w.Y23[1]};
  const bool b16 = m->cfg.precision == MARS_BF16;
  cudaError_t e;
  if (m->ct.aggregator == MARS_AGG_SAGE_GCN) {          // c37: Â = D^-1 (A + I)
    if ((e = launch_sage_vals(gd, w.valsR, w.valsC, s, nl))) return e;
    gd.vals = w.valsR;
  }
  for (int l = 0; l < 3; ++l) {
    int Cin = l == 0 ? F : H;
    const void* T = l == 0 ? (const void*)gd.X : (const void*)w.Z[l - 1];
    const bool h3l = !b16 && m->gemm_impl == MARS_GEMM_AUTO && tc3h_supported(Cin, H);
    if ((e = launch_spmm_fwd(gd, Cin, T, b16 && l > 0, nullptr, alpha, l - 1, Ys[l], b16, 0, s, nl,
                             nullptr, h3l ? w.h3_rsY[l] : nullptr)))
      return e;
    if (b16) {
      if ((e = tc16_weights(W[l], Cin, H, w.w16t[l], w.w16[l], s, nl))) return e;
      if ((e = tc16_gemm_rows(Ys[l], w.w16t[l], w.Z[l], gd.Nt, H, Cin, s, nl))) return e;
    } else if (h3l) {
      if ((e = tc3h_split_weights(W[l], Cin, H, w.h3_wsc[l], w.h3_wt_hi[l], w.h3_wt_lo[l],
                                  w.h3_w_hi[l], w.h3_w_lo[l], s, nl)))
        return e;
      if ((e = tc3h_gemm_rows(Ys[l], w.h3_rsY[l], w.h3_wt_hi[l], w.h3_wt_lo[l], w.h3_wsc[l] + 1,
                              w.Z[l], gd.Nt, H, Cin, s, nl)))
        return e;
    } else if ((e = gemm_nn(Ys[l], W[l], w.Z[l], gd.Nt, H, Cin, s, nl))) {
      return e;
    }
  }
  return launch_prelu(w.Z[2], b16, alpha, 2, w.dY, (int64_t)gd.Nt * H, s, nl);
}

extern "C" mars_status mars_encode(mars_dgi* m, const mars_graph* g, float* emb) {
  if (mars_status st = check_dgi(m)) return st;
  if (mars_status st = check_graph(g)) return st;
  if (!emb) return fail(MARS_EINVAL, "embeddings is NULL");
  if (g->sharded) return fail(MARS_EINVAL, "mars_encode runs on an unsharded graph");
  if (g->F != m->F) return fail(MARS_EINVAL, "feat_dim mismatch");
  CK(cudaSetDevice(m->cfg.device));
  if (mars_status st = ensure_ws(m, g)) return st;
  cudaStream_t s = m->stream;
  int nl = 0;
  CK(enqueue_encode(m, g, s, &nl));
  CK(cudaMemcpyAsync(emb, m->ws.dY, sizeof(float) * (size_t)g->dev.Nt * m->H,
                     cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  g->note_use(s);
  m->last_Nt = 0;
  return MARS_OK;
}

namespace {
// Joint training (NEXT-3): dZ3 of the stacked layout from dL/dH3 of the
// positive rows: rows r < Nt: dE ⊙ PReLU'(Z3), rows >= Nt: 0; the 3xFP16 row
// scales; per-row dalpha3 terms sum_c dE min(Z3, 0) into slots[r] (fixed order).
__global__ void k_dz3_from_dE(const float* __restrict__ dE, const float* __restrict__ Z3,
                              const float* __restrict__ alpha, int32_t Nt, int H,
                              float* __restrict__ dZ, float* __restrict__ rs,
                              double* __restrict__ slots) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= 2 * Nt) return;
  const int64_t r = warp;
  const float a = alpha[2];
  float mx = 0.f;
  double da = 0.0;
  for (int c = lane; c < H; c += 32) {
    float d = 0.f;
    if (r < Nt) {
      const float z = Z3[r * H + c], g = dE[r * H + c];
      d = z > 0.f ? g : a * g;
      if (!(z > 0.f)) da += (double)g * (double)z;
    }
    dZ[r * H + c] = d;
    mx = fmaxf(mx, fabsf(d));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(kFull, mx, o));
  da = warp_sum(da);
  if (lane == 0) {
    if (rs) rs[r] = pow2_scale(mx);
    if (r < Nt) slots[r] = da;
  }
}
__global__ void k_fill_f(float* __restrict__ p, int64_t n, float v) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = v;
}
}  // namespace

// Backward of the encoder from dL/dH3 of the positive rows (the placer's dE):
// gradients of W1..3 and alpha into m->grads (dM = 0, loss slot 0), by the
// stacked backward chain of the step with a zero corrupted half.  fp32 models.
static cudaError_t enqueue_encoder_backward(mars_dgi* m, const mars_graph* gr, const float* dE,
                                            cudaStream_t s, int* nl) {
  Workspace& w = m->ws;
  GraphDev g = gr->dev;
  g.long_part = w.long_part;
  const int F = m->F, H = m->H;
  const int64_t Nt = g.Nt, R = 2 * Nt;
  float* W[3] = {m->params, m->params + (int64_t)F * H, m->params + (int64_t)F * H + (int64_t)H * H};
  float* alpha = m->params + (int64_t)F * H + 3LL * H * H;
  float* gW[3] = {m->grads, m->grads + (int64_t)F * H, m->grads + (int64_t)F * H + (int64_t)H * H};
  float* galpha = m->grads + (int64_t)F * H + 3LL * H * H;
  float* Ys[3] = {w.Y1, w.Y23[0], w.Y23[1]};
  cudaError_t e;
  if (m->ct.aggregator == MARS_AGG_SAGE_GCN) g.vals = w.valsC;   // Âᵀ (c37; set by the encode)
  // the corrupted half of the saved activations is zero (and its row scales neutral)
  if ((e = cudaMemsetAsync(w.Y1 + Nt * F, 0, sizeof(float) * Nt * F, s))) return e;
  for (int l = 0; l < 2; ++l)
    if ((e = cudaMemsetAsync(w.Y23[l] + Nt * H, 0, sizeof(float) * Nt * H, s))) return e;
  for (int l = 0; l < 3; ++l) {
    if ((e = cudaMemsetAsync(w.Z[l] + Nt * H, 0, sizeof(float) * Nt * H, s))) return e;
    k_fill_f<<<cdiv(Nt, 256), 256, 0, s>>>(w.h3_rsY[l] + Nt, Nt, 0x1p100f);
  }
  if ((e = cudaMemsetAsync(m->grads, 0, sizeof(float) * (m->P + 1), s))) return e;
  bool tc[3];
  for (int l = 0; l < 3; ++l) tc[l] = m->gemm_impl != MARS_GEMM_SIMT && tc3h_supported(l == 0 ? F : H, H);
  k_dz3_from_dE<<<cdiv(R * 32, 256), 256, 0, s>>>(dE, w.Z[2], alpha, (int32_t)Nt, H, w.dZ,
                                                   tc[2] ? w.h3_rsdZ : nullptr, w.slots[2]);
  count_launch(nl, 2 + 3);
  if ((e = launch_reduce_slots(w.slots[2], (int)Nt, galpha + 2, s, nl))) return e;
  int ns = 0;
  for (int l = 2; l >= 0; --l) {
    const int Cin = l == 0 ? F : H;
    if (tc[l]) e = tc3h_gemm_dw(Ys[l], w.h3_rsY[l], w.dZ, w.h3_rsdZ, gW[l], R, Cin, H, w.dw_part, s, nl);
    else e = gemm_tn(Ys[l], w.dZ, gW[l], R, Cin, H, w.tn_part, s, nl);
    if (e) return e;
    if (l > 0) {
      if (tc[l]) e = tc3h_gemm_rows(w.dZ, w.h3_rsdZ, w.h3_w_hi[l], w.h3_w_lo[l], w.h3_wsc[l] + 1,
                                    w.dY, R, Cin, H, s, nl);
      else e = gemm_nt(w.dZ, W[l], w.dY, R, Cin, H, s, nl);
      if (e) return e;
      if ((e = launch_spmm_bwd(g, Cin, w.dY, w.Z[l - 1], 0, alpha, l - 1, w.dZ, w.slots[l - 1], &ns,
                               s, nl, nullptr, tc[l - 1] ? w.h3_rsdZ : nullptr)))
        return e;
      if ((e = launch_reduce_slots(w.slots[l - 1], ns, galpha + (l - 1), s, nl))) return e;
    }
  }
  return cudaSuccess;
}

// ---------------------------------------------------------------- hooks / state
extern "C" mars_status mars_dgi_export_activations(const mars_dgi* m, int32_t layer, float* Y,
                                                   float* Z) {
  if (mars_status st = check_dgi(m)) return st;
  if (layer < 1 || layer > 3) return fail(MARS_EINVAL, "layer must be 1..3");
  if (!m->ws.Y1 || !m->last_Nt) return fail(MARS_ESTATE, "no step has run since the last encode");
  CK(cudaSetDevice(m->cfg.device));
  CK(cudaStreamSynchronize(m->stream));
  int64_t R = 2LL * m->last_Nt;
  const float* Ys[3] = {(m->sage || m->pool) ? m->ws.Xs : m->ws.Y1, m->ws.Y23[0], m->ws.Y23[1]};
  int Cin = layer == 1 ? m->F : m->H;
  if (m->cfg.precision == MARS_BF16) {     // upcast bf16 storage through a scratch buffer
    float* tmp = nullptr;
    CK(cudaMalloc(&tmp, sizeof(float) * R * std::max(Cin, m->H)));
    struct FT { float* p; ~FT() { cudaFree(p); } } ft{tmp};
    if (Y) {
      CK(launch_upcast(Ys[layer - 1], tmp, R * Cin, nullptr));
      CK(cudaMemcpy(Y, tmp, sizeof(float) * R * Cin, cudaMemcpyDeviceToHost));
    }
    if (Z) {
      CK(launch_upcast(m->ws.Z[layer - 1], tmp, R * m->H, nullptr));
      CK(cudaMemcpy(Z, tmp, sizeof(float) * R * m->H, cudaMemcpyDeviceToHost));
    }
    return MARS_OK;
  }
  if (Y) CK(cudaMemcpy(Y, Ys[layer - 1], sizeof(float) * R * Cin, cudaMemcpyDeviceToHost));
  if (Z) CK(cudaMemcpy(Z, m->ws.Z[layer - 1], sizeof(float) * R * m->H, cudaMemcpyDeviceToHost));
  return MARS_OK;
}

extern "C" mars_status mars_dgi_saved_rows(const mars_dgi* m, int64_t* rows) {
  if (mars_status st = check_dgi(m)) return st;
  if (!rows) return fail(MARS_EINVAL, "rows is NULL");
  *rows = m->last_Nt;
  return MARS_OK;
}

extern "C" mars_status mars_dgi_set_keep_backward(mars_dgi* m, int32_t keep) {
  if (mars_status st = check_dgi(m)) return st;
  if ((m->sage || m->pool) && keep) return fail(MARS_EINVAL, "no backward hook for the SAGE encoders");
  CK(cudaSetDevice(m->cfg.device));
  m->drop_execs();                 // recapture with / without the copies
  CK(cudaStreamSynchronize(m->stream));
  m->keep_bwd = keep != 0;
  if (!m->keep_bwd) m->kb_release();
  m->kb_valid_Nt = 0;
  return MARS_OK;
}

extern "C" mars_status mars_dgi_export_backward(const mars_dgi* m, int32_t layer, float* dY,
                                                float* dZ) {
  if (mars_status st = check_dgi(m)) return st;
  if (layer < 1 || layer > 3) return fail(MARS_EINVAL, "layer must be 1..3");
  if (layer == 1 && dY) return fail(MARS_EINVAL, "there is no dY_1");
  if (!m->kb_valid_Nt || m->kb_valid_Nt != m->last_Nt)
    return fail(MARS_ESTATE, "the last step did not keep its backward intermediates");
  CK(cudaSetDevice(m->cfg.device));
  CK(cudaStreamSynchronize(m->stream));
  const int64_t n = 2LL * m->kb_valid_Nt * m->H;
  const void* srcs[2] = {layer >= 2 ? m->kb_dY[layer - 2] : nullptr, m->kb_dZ[layer - 1]};
  float* dsts[2] = {dY, dZ};
  for (int k = 0; k < 2; ++k) {
    if (!dsts[k]) continue;
    if (m->cfg.precision == MARS_BF16) {
      float* tmp = nullptr;
      CK(cudaMalloc(&tmp, sizeof(float) * n));
      struct FT { float* p; ~FT() { cudaFree(p); } } ft{tmp};
      CK(launch_upcast(srcs[k], tmp, n, nullptr));
      CK(cudaMemcpy(dsts[k], tmp, sizeof(float) * n, cudaMemcpyDeviceToHost));
    } else {
      CK(cudaMemcpy(dsts[k], srcs[k], sizeof(float) * n, cudaMemcpyDeviceToHost));
    }
  }
  return MARS_OK;
}

extern "C" mars_status mars_dgi_get_state(const mars_dgi* m, float* params, float* am, float* av,
                                          int64_t* t) {
  if (mars_status st = check_dgi(m)) return st;
  CK(cudaSetDevice(m->cfg.device));
  CK(cudaStreamSynchronize(m->stream));
  if (params) CK(cudaMemcpy(params, m->params, sizeof(float) * m->P, cudaMemcpyDeviceToHost));
  if (am) CK(cudaMemcpy(am, m->adam_m, sizeof(float) * m->P, cudaMemcpyDeviceToHost));
  if (av) CK(cudaMemcpy(av, m->adam_v, sizeof(float) * m->P, cudaMemcpyDeviceToHost));
  if (t) CK(cudaMemcpy(t, &m->adam_st->t, sizeof(int64_t), cudaMemcpyDeviceToHost));
  return MARS_OK;
}

extern "C" mars_status mars_dgi_set_state(mars_dgi* m, const float* params, const float* am,
                                          const float* av, int64_t t) {
  if (mars_status st = check_dgi(m)) return st;
  if (t < 0) return fail(MARS_EINVAL, "t < 0");
  CK(cudaSetDevice(m->cfg.device));
  CK(cudaStreamSynchronize(m->stream));
  if (params) CK(cudaMemcpy(m->params, params, sizeof(float) * m->P, cudaMemcpyHostToDevice));
  if (am) CK(cudaMemcpy(m->adam_m, am, sizeof(float) * m->P, cudaMemcpyHostToDevice));
  if (av) CK(cudaMemcpy(m->adam_v, av, sizeof(float) * m->P, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(&m->adam_st->t, &t, sizeof(int64_t), cudaMemcpyHostToDevice));
  return MARS_OK;
}

extern "C" mars_status mars_debug_gemm(int32_t device, int32_t op, int32_t impl, const float* A,
                                       const float* B, float* C, int64_t M, int32_t N, int32_t K,
                                       int32_t iters, float* ms) {
  if (!A || !B || !C || M < 1 || N < 1 || K < 1 || (op != 0 && op != 1))
    return fail(MARS_EINVAL, "bad debug_gemm arguments");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(MARS_ECUDA, "no CUDA device");
  }
  CK(cudaSetDevice(device));
  const bool tcp = impl != MARS_GEMM_SIMT && (op == 0 ? tc3h_supported(K, N) || tc3h_supported(N, K)
                                                     : tc3h_supported(K, N));
  float *wsc = nullptr, *rs = nullptr, *rs2 = nullptr;
  CK(dalloc(&wsc, 2));
  CK(dalloc(&rs, (size_t)M));
  CK(dalloc(&rs2, (size_t)M));
  size_t nA = (size_t)M * K, nB = op == 0 ? (size_t)N * K : (size_t)M * N;
  size_t nC = op == 0 ? (size_t)M * N : (size_t)K * N;
  float *dA, *dB, *dC, *part;
  void *bh, *bl, *bth, *btl;
  double* tpart;
  CK(dalloc(&dA, nA));
  CK(dalloc(&dB, nB));
  CK(dalloc(&dC, nC));
  CK(dalloc((char**)&bh, (size_t)N * K * 2));
  CK(dalloc((char**)&bl, (size_t)N * K * 2));
  CK(dalloc((char**)&bth, (size_t)N * K * 2));
  CK(dalloc((char**)&btl, (size_t)N * K * 2));
  size_t np = std::max(tc_dw_partial_floats(M, K), (size_t)1);
  CK(dalloc(&part, np));
  CK(dalloc(&tpart, gemm_tn_partial_floats(M, K, N)));
  CK(cudaMemcpy(dA, A, sizeof(float) * nA, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, B, sizeof(float) * nB, cudaMemcpyHostToDevice));
  cudaStream_t s = nullptr;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  auto run = [&]() -> cudaError_t {
    if (op == 0) {
      if (tcp) {   // B [N×K] = "W" with CIN = N, H = K: the dY orientation
        cudaError_t e = tc3h_split_weights(dB, N, K, wsc, bth, btl, bh, bl, s, nullptr);
        if (e != cudaSuccess) return e;
        if ((e = tc3h_row_scales(dA, M, K, rs, s, nullptr)) != cudaSuccess) return e;
        return tc3h_gemm_rows(dA, rs, bh, bl, wsc + 1, dC, M, N, K, s, nullptr);
      }
      return gemm_nt(dA, dB, dC, M, N, K, s, nullptr);
    }
    if (tcp) {
      cudaError_t e = tc3h_row_scales(dA, M, K, rs, s, nullptr);
      if (e != cudaSuccess) return e;
      if ((e = tc3h_row_scales(dB, M, N, rs2, s, nullptr)) != cudaSuccess) return e;
      return tc3h_gemm_dw(dA, rs, dB, rs2, dC, M, K, N, part, s, nullptr);
    }
    return gemm_tn(dA, dB, dC, M, K, N, tpart, s, nullptr);
  };
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(run());
  CK(cudaEventRecord(e0, s));
  for (int i = 0; i < iters; ++i) CK(run());
  CK(cudaEventRecord(e1, s));
  CK(cudaStreamSynchronize(s));
  float t = 0.f;
  CK(cudaEventElapsedTime(&t, e0, e1));
  if (ms) *ms = iters > 0 ? t / iters : 0.f;
  CK(cudaMemcpy(C, dC, sizeof(float) * nC, cudaMemcpyDeviceToHost));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaStreamDestroy(s);
  for (void* p : {(void*)dA, (void*)dB, (void*)dC, (void*)bh, (void*)bl, (void*)bth, (void*)btl,
                  (void*)part, (void*)tpart, (void*)wsc, (void*)rs, (void*)rs2})
    cudaFree(p);
  return MARS_OK;
}

// ---------------------------------------------------------------- row-sharded graph (§8(e)(ii))
namespace {
constexpr uint64_t kShardBlobMagic = 0x4D41525353484431ULL;   // "MARSSHD1"
constexpr int kShardBufs = 7;     // Z1, Z2, dY (layer 3), dY2 (layer 2), xbuf, flags, grads
struct ShardBlob {
  uint64_t magic;
  int32_t P, me, device, H;
  uint64_t graph_key;               // N, nnz and the row split must agree across shards
  cudaIpcMemHandle_t h[kShardBufs];
};

uint64_t shard_key(const mars_graph* g) {
  uint64_t k = sm64((uint64_t)g->Nt) ^ sm64((uint64_t)g->nnz + 0x51ULL);
  for (int32_t v : g->starts) k = sm64(k ^ (uint64_t)(uint32_t)v);
  return k;
}

void* shard_buf(const mars_dgi* m, int k) {
  switch (k) {
    case 0: return m->ws.Z[0];
    case 1: return m->ws.Z[1];
    case 2: return m->ws.dY;
    case 3: return m->sh.dY2;
    case 4: return m->sh.xbuf;
    case 5: return m->sh.flags;
    default: return m->grads;
  }
}

// Fills the peer tables of m from the P shards' buffer pointers bufs[q][k].
void shard_wire(mars_dgi* m, void* const (*bufs)[kShardBufs]) {
  mars_dgi::Shard& sh = m->sh;
  const mars_graph* g = sh.g;
  PeerRows rows{};
  for (int q = 0; q <= kMaxShards; ++q)
    rows.start[q] = q < g->P ? g->starts[q] : (q == g->P ? g->Nt : INT32_MAX);
  sh.z[0] = sh.z[1] = sh.dy[0] = sh.dy[1] = rows;
  sh.sync.P = g->P;
  sh.sync.me = g->me;
  sh.sync.epoch = sh.epoch;
  sh.sync.err = sh.err;
  for (int q = 0; q < g->P; ++q) {
    sh.z[0].base[q] = bufs[q][0];
    sh.z[1].base[q] = bufs[q][1];
    sh.dy[0].base[q] = bufs[q][2];
    sh.dy[1].base[q] = bufs[q][3];
    sh.x[0].p[q] = bufs[q][4];
    sh.x[1].p[q] = static_cast<double*>(bufs[q][4]) + (m->H + 1);
    sh.sync.flags[q] = static_cast<unsigned long long*>(bufs[q][5]);
    sh.grads.p[q] = bufs[q][6];
  }
  sh.connected = true;
  m->drop_execs();          // a captured step of this graph predates the wiring
}

// Captures the sharded step once at connect time and forces every kernel it
// launches to load (cudaFuncGetAttributes).  With CUDA's lazy module loading a
// kernel's first launch may wait for the whole context to go idle; inside a
// sharded step that would wait on a barrier kernel spinning for a peer whose
// launches are queued behind it (several shards in one process).  The
// instantiated graph is kept, so the first step already replays it.
mars_status shard_prepare(mars_dgi* m) {
  const mars_graph* g = m->sh.g;
  cudaStream_t s = m->stream;
  int nl = 0;
  cudaGraph_t graph;
  CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
  cudaError_t e = enqueue_step(m, g, s, &nl);
  cudaError_t e2 = cudaStreamEndCapture(s, &graph);
  if (e != cudaSuccess || e2 != cudaSuccess) {
    if (e2 == cudaSuccess) cudaGraphDestroy(graph);
    cudaGetLastError();
    return fail(MARS_ECUDA, "sharded step capture failed: %s",
                cudaGetErrorString(e != cudaSuccess ? e : e2));
  }
  struct GD { cudaGraph_t g; ~GD() { cudaGraphDestroy(g); } } gd{graph};
  size_t n = 0;
  CK(cudaGraphGetNodes(graph, nullptr, &n));
  std::vector<cudaGraphNode_t> nodes(n);
  CK(cudaGraphGetNodes(graph, nodes.data(), &n));
  for (cudaGraphNode_t node : nodes) {
    cudaGraphNodeType t;
    CK(cudaGraphNodeGetType(node, &t));
    if (t != cudaGraphNodeTypeKernel) continue;
    cudaKernelNodeParams kp;
    CK(cudaGraphKernelNodeGetParams(node, &kp));
    cudaFuncAttributes fa;
    CK(cudaFuncGetAttributes(&fa, kp.func));
  }
  m->drop_execs();
  cudaGraphExec_t ex = nullptr;
  CK(cudaGraphInstantiate(&ex, graph, 0));
  m->add_exec(g->uid, s, ex, nl);
  return MARS_OK;
}
}  // namespace

extern "C" mars_status mars_shard_partition(const int32_t* rowptr, int32_t N, int32_t P,
                                            int32_t* starts) {
  if (!rowptr || !starts || N < 1 || P < 1 || P > kMaxShards || N < P)
    return fail(MARS_EINVAL, "bad partition arguments");
  const int64_t nnz = rowptr[N];
  starts[0] = 0;
  for (int p = 1; p < P; ++p) {
    const int64_t target = nnz * p / P;
    int32_t r = (int32_t)(std::lower_bound(rowptr, rowptr + N + 1, (int32_t)target) - rowptr);
    r = std::max(r, starts[p - 1] + 1);          // every shard owns >= 1 row
    r = std::min(r, N - (P - p));
    starts[p] = r;
  }
  starts[P] = N;
  return MARS_OK;
}

extern "C" mars_status mars_graph_load_shard(const mars_graph_desc* desc, int32_t P, int32_t me,
                                             int32_t device, mars_graph** out) {
  if (!out) return fail(MARS_EINVAL, "out is NULL");
  *out = nullptr;
  if (!desc) return fail(MARS_EINVAL, "graph is NULL");
  if (P < 1 || P > kMaxShards || me < 0 || me >= P)
    return fail(MARS_EINVAL, "bad shard %d of %d (1 <= P <= %d)", me, P, kMaxShards);
  if (desc->num_nodes < P) return fail(MARS_EINVAL, "fewer nodes than shards");
  mars_graph* g = nullptr;
  if (mars_status st = mars_graph_load(desc, 1, device, &g)) return st;
  std::unique_ptr<mars_graph> guard(g);
  const int32_t N = g->Nt;
  // contiguous row blocks balanced by nnz (mars_shard_partition)
  std::vector<int32_t> rp((size_t)N + 1);
  CK(cudaMemcpy(rp.data(), g->rowptr, sizeof(int32_t) * (N + 1), cudaMemcpyDeviceToHost));
  g->starts.assign(P + 1, 0);
  if (mars_status st = mars_shard_partition(rp.data(), N, P, g->starts.data())) return st;
  g->starts.resize(P);
  const int32_t r0 = g->starts[me], r1 = me + 1 < P ? g->starts[me + 1] : N;
  const int32_t n = r1 - r0;
  g->sharded = true;
  g->P = P;
  g->me = me;
  g->row_begin = r0;
  g->row_end = r1;
  g->local_nnz = (int64_t)rp[r1] - rp[r0];
  {   // halo: distinct columns of the local rows owned by other shards
    std::vector<int32_t> col((size_t)g->local_nnz);
    CK(cudaMemcpy(col.data(), g->colind + rp[r0], sizeof(int32_t) * col.size(),
                  cudaMemcpyDeviceToHost));
    std::vector<uint8_t> seen((size_t)N, 0);
    int64_t h = 0;
    for (int32_t j : col)
      if ((j < r0 || j >= r1) && !seen[j]) { seen[j] = 1; ++h; }
    g->halo_rows = h;
  }
  // local view: rows [r0, r1) with local ids, global columns, the whole X
  std::vector<int32_t> node_off = {0, n}, chunk_row, chunk_graph, graph_chunk = {0, 0};
  for (int32_t r = 0; r < n; r += kChunkRows) {
    chunk_row.push_back(r);
    chunk_graph.push_back(0);
  }
  chunk_row.push_back(n);
  graph_chunk[1] = (int32_t)chunk_graph.size();
  const int nch = (int)chunk_graph.size();
  cudaStream_t s = nullptr;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{s};
  CK(palloc(&g->l_node_off, 2, s));
  CK(palloc(&g->l_node_graph, (size_t)n, s));
  CK(palloc(&g->l_chunk_row, (size_t)nch + 1, s));
  CK(palloc(&g->l_chunk_graph, (size_t)nch, s));
  CK(palloc(&g->l_graph_chunk, 2, s));
  CK(cudaMemcpyAsync(g->l_node_off, node_off.data(), sizeof(int32_t) * 2, cudaMemcpyHostToDevice, s));
  CK(cudaMemsetAsync(g->l_node_graph, 0, sizeof(int32_t) * n, s));
  CK(cudaMemcpyAsync(g->l_chunk_row, chunk_row.data(), sizeof(int32_t) * (nch + 1), cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(g->l_chunk_graph, chunk_graph.data(), sizeof(int32_t) * nch, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(g->l_graph_chunk, graph_chunk.data(), sizeof(int32_t) * 2, cudaMemcpyHostToDevice, s));
  CK(cudaStreamSynchronize(s));
  g->dev_full = g->dev;
  GraphDev& v = g->dev;
  v.Nt = n;
  v.nnz = g->local_nnz;
  v.node_off = g->l_node_off;
  v.node_graph = g->l_node_graph;
  v.rowptr = g->rowptr + r0;             // global nnz offsets into the whole colind / vals
  v.nchunks = nch;
  v.chunk_row = g->l_chunk_row;
  v.chunk_graph = g->l_chunk_graph;
  v.graph_chunk = g->l_graph_chunk;
  v.gsize = g->gsize;                    // N of the whole graph (readout mean, loss scale)
  CK(build_long_rows(g, v, s));          // of the local rows
  *out = guard.release();
  return MARS_OK;
}

extern "C" mars_status mars_graph_shard_info(const mars_graph* g, int32_t* P, int32_t* me,
                                             int32_t* row_begin, int32_t* row_end,
                                             int64_t* local_nnz, int64_t* halo_rows) {
  if (mars_status st = check_graph(g)) return st;
  if (P) *P = g->P;
  if (me) *me = g->me;
  if (row_begin) *row_begin = g->sharded ? g->row_begin : 0;
  if (row_end) *row_end = g->sharded ? g->row_end : g->Nt;
  if (local_nnz) *local_nnz = g->sharded ? g->local_nnz : g->nnz;
  if (halo_rows) *halo_rows = g->sharded ? g->halo_rows : 0;
  return MARS_OK;
}

extern "C" mars_status mars_shard_attach(mars_dgi* m, const mars_graph* g) {
  if (mars_status st = check_dgi(m)) return st;
  if (mars_status st = check_graph(g)) return st;
  if (!g->sharded) return fail(MARS_EINVAL, "graph was not loaded with mars_graph_load_shard");
  if (m->sh.g) return fail(MARS_ESTATE, "model already attached to a shard");
  if (m->sage || m->pool) return fail(MARS_EINVAL, "row sharding runs the GCN encoder only");
  if (m->ct.num_neg != 1 || m->ct.corruption != MARS_CORRUPT_PERMUTE ||
      m->ct.readout != MARS_READOUT_SIGMOID_MEAN || m->ct.aggregator != MARS_AGG_GCN ||
      m->ct.loss != MARS_LOSS_BCE)
    return fail(MARS_ESTATE, "a row-sharded model runs the default step only");
  if (m->comm) return fail(MARS_EINVAL, "a shard-attached model cannot also be data-parallel");
  if (g->F != m->F || g->device != m->cfg.device) return fail(MARS_EINVAL, "F / device mismatch");
  if (!(m->H == 128 || m->H == 256) || m->gemm_impl == MARS_GEMM_SIMT)
    return fail(MARS_EINVAL, "row sharding needs hidden_dim in {128, 256} and the tcgen05 GEMMs");
  CK(cudaSetDevice(m->cfg.device));
  if (mars_status st = ensure_ws(m, g)) return st;
  mars_dgi::Shard& sh = m->sh;
  auto al = [&](void** p, size_t bytes) -> cudaError_t {
    cudaError_t e = cudaMalloc(p, bytes);
    if (e == cudaSuccess) sh.owned.push_back(*p);
    return e;
  };
  CK(al((void**)&sh.flags, sizeof(unsigned long long) * kMaxShards));
  CK(al((void**)&sh.epoch, sizeof(unsigned long long)));
  CK(al((void**)&sh.err, sizeof(int32_t)));
  CK(al((void**)&sh.xbuf, sizeof(double) * 2 * (m->H + 1)));
  CK(al(&sh.dY2, sizeof(float) * 2 * (size_t)g->dev.Nt * m->H));
  CK(al((void**)&sh.gsum, sizeof(float) * (m->P + 1)));
  // zeroed before any shard can connect (connecting is collective), so no
  // early arrival signal is lost
  CK(cudaMemset(sh.flags, 0, sizeof(unsigned long long) * kMaxShards));
  CK(cudaMemset(sh.epoch, 0, sizeof(unsigned long long)));
  CK(cudaMemset(sh.err, 0, sizeof(int32_t)));
  CK(cudaMemset(sh.gsum, 0, sizeof(float) * (m->P + 1)));
  CK(cudaDeviceSynchronize());
  sh.g = g;
  sh.guid = g->uid;
  return MARS_OK;
}

extern "C" int64_t mars_shard_blob_bytes(void) { return (int64_t)sizeof(ShardBlob); }

extern "C" mars_status mars_shard_export(const mars_dgi* m, void* blob) {
  if (mars_status st = check_dgi(m)) return st;
  if (!blob) return fail(MARS_EINVAL, "blob is NULL");
  if (!m->sh.g) return fail(MARS_ESTATE, "mars_shard_attach first");
  CK(cudaSetDevice(m->cfg.device));
  ShardBlob b{};
  b.magic = kShardBlobMagic;
  b.P = m->sh.g->P;
  b.me = m->sh.g->me;
  b.device = m->cfg.device;
  b.H = m->H;
  b.graph_key = shard_key(m->sh.g);
  for (int k = 0; k < kShardBufs; ++k) CK(cudaIpcGetMemHandle(&b.h[k], shard_buf(m, k)));
  memcpy(blob, &b, sizeof b);
  return MARS_OK;
}

extern "C" mars_status mars_shard_connect(mars_dgi* m, const void* blobs) {
  if (mars_status st = check_dgi(m)) return st;
  if (!blobs) return fail(MARS_EINVAL, "blobs is NULL");
  if (!m->sh.g) return fail(MARS_ESTATE, "mars_shard_attach first");
  if (m->sh.connected) return fail(MARS_ESTATE, "already connected");
  CK(cudaSetDevice(m->cfg.device));
  const mars_graph* g = m->sh.g;
  const ShardBlob* b = static_cast<const ShardBlob*>(blobs);
  void* bufs[kMaxShards][kShardBufs] = {};
  for (int q = 0; q < g->P; ++q) {
    if (b[q].magic != kShardBlobMagic || b[q].P != g->P || b[q].me != q || b[q].H != m->H ||
        b[q].graph_key != shard_key(g))
      return fail(MARS_EINVAL, "shard blob %d does not match this graph / model", q);
    for (int k = 0; k < kShardBufs; ++k) {
      if (q == g->me) {
        bufs[q][k] = shard_buf(m, k);
        continue;
      }
      void* p = nullptr;
      CK(cudaIpcOpenMemHandle(&p, b[q].h[k], cudaIpcMemLazyEnablePeerAccess));
      m->sh.ipc.push_back(p);
      bufs[q][k] = p;
    }
  }
  shard_wire(m, bufs);
  return shard_prepare(m);
}

extern "C" mars_status mars_shard_connect_local(mars_dgi* const* models, int32_t P) {
  if (!models || P < 1 || P > kMaxShards) return fail(MARS_EINVAL, "bad model list");
  void* bufs[kMaxShards][kShardBufs] = {};
  for (int q = 0; q < P; ++q) {
    mars_dgi* m = models[q];
    if (mars_status st = check_dgi(m)) return st;
    if (!m->sh.g) return fail(MARS_ESTATE, "model %d: mars_shard_attach first", q);
    if (m->sh.connected) return fail(MARS_ESTATE, "model %d already connected", q);
    if (m->sh.g->P != P || m->sh.g->me != q || m->H != models[0]->H ||
        shard_key(m->sh.g) != shard_key(models[0]->sh.g))
      return fail(MARS_EINVAL, "model %d is not shard %d of the same graph", q, q);
    for (int k = 0; k < kShardBufs; ++k) bufs[q][k] = shard_buf(m, k);
  }
  for (int q = 0; q < P; ++q)          // peer access between distinct devices
    for (int r = 0; r < P; ++r) {
      const int dq = models[q]->cfg.device, dr = models[r]->cfg.device;
      if (dq == dr) continue;
      CK(cudaSetDevice(dq));
      cudaError_t e = cudaDeviceEnablePeerAccess(dr, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
        return fail(MARS_ECUDA, "peer access %d -> %d: %s", dq, dr, cudaGetErrorString(e));
      cudaGetLastError();
    }
  for (int q = 0; q < P; ++q) shard_wire(models[q], bufs);
  for (int q = 0; q < P; ++q) {
    CK(cudaSetDevice(models[q]->cfg.device));
    if (mars_status st = shard_prepare(models[q])) return st;
  }
  return MARS_OK;
}

// ---------------------------------------------------------------- data parallel over peer memory
namespace {
constexpr uint64_t kDpBlobMagic = 0x4D41525344504231ULL;   // "MARSDPB1"
struct DpBlob {
  uint64_t magic;
  int32_t R, me, device, pad;
  int64_t P;
  cudaIpcMemHandle_t grads, flags;
};
}  // namespace

extern "C" int64_t mars_dp_blob_bytes(void) { return (int64_t)sizeof(DpBlob); }

extern "C" mars_status mars_dp_export(const mars_dgi* m, void* blob) {
  if (mars_status st = check_dgi(m)) return st;
  if (!blob) return fail(MARS_EINVAL, "blob is NULL");
  if (m->dp.R < 2) return fail(MARS_ESTATE, "model was not created for peer-memory data parallelism");
  CK(cudaSetDevice(m->cfg.device));
  DpBlob b{};
  b.magic = kDpBlobMagic;
  b.R = m->dp.R;
  b.me = m->dp.me;
  b.device = m->cfg.device;
  b.P = m->P;
  CK(cudaIpcGetMemHandle(&b.grads, m->grads));
  CK(cudaIpcGetMemHandle(&b.flags, m->dp.flags));
  memcpy(blob, &b, sizeof b);
  return MARS_OK;
}

extern "C" mars_status mars_dp_connect(mars_dgi* m, const void* blobs) {
  if (mars_status st = check_dgi(m)) return st;
  if (!blobs) return fail(MARS_EINVAL, "blobs is NULL");
  mars_dgi::Dp& d = m->dp;
  if (d.R < 2) return fail(MARS_ESTATE, "model was not created for peer-memory data parallelism");
  if (d.connected) return fail(MARS_ESTATE, "already connected");
  CK(cudaSetDevice(m->cfg.device));
  const DpBlob* b = static_cast<const DpBlob*>(blobs);
  for (int q = 0; q < d.R; ++q)
    if (b[q].magic != kDpBlobMagic || b[q].R != d.R || b[q].me != q || b[q].P != m->P)
      return fail(MARS_EINVAL, "data-parallel blob %d does not match this job", q);
  d.sync.P = d.R;
  d.sync.me = d.me;
  d.sync.epoch = d.epoch;
  d.sync.err = d.err;
  for (int q = 0; q < d.R; ++q) {
    if (q == d.me) {
      d.grads.p[q] = m->grads;
      d.sync.flags[q] = d.flags;
      continue;
    }
    void* pg = nullptr;
    void* pf = nullptr;
    CK(cudaIpcOpenMemHandle(&pg, b[q].grads, cudaIpcMemLazyEnablePeerAccess));
    d.ipc.push_back(pg);
    CK(cudaIpcOpenMemHandle(&pf, b[q].flags, cudaIpcMemLazyEnablePeerAccess));
    d.ipc.push_back(pf);
    d.grads.p[q] = pg;
    d.sync.flags[q] = static_cast<unsigned long long*>(pf);
  }
  d.connected = true;
  m->drop_execs();
  // One process per rank: each barrier signals its peers before it waits, so a
  // host thread blocked in a lazy module load (which waits for its own context
  // to go idle) cannot deadlock the ranks.
  return MARS_OK;
}

extern "C" mars_status mars_graph_set_pair_offsets(mars_graph* g, const int64_t* off) {
  if (mars_status st = check_graph(g)) return st;
  if (!off) return fail(MARS_EINVAL, "pair_offsets is NULL");
  for (int i = 0; i < g->G; ++i)
    if (off[i] < 0) return fail(MARS_EINVAL, "negative pair offset");
  CK(cudaSetDevice(g->device));
  CK(cudaMemcpy(g->pair_off, off, sizeof(int64_t) * g->G, cudaMemcpyHostToDevice));
  return MARS_OK;
}

extern "C" mars_status mars_dgi_read_step(mars_dgi* m, float* loss, float* grads) {
  if (mars_status st = check_dgi(m)) return st;
  CK(cudaSetDevice(m->cfg.device));
  cudaStream_t s = m->stream;
  float l = 0.f;
  int32_t err = 0, skipped = 0;
  CK(cudaMemcpyAsync(&l, m->grads_final() + m->P, sizeof(float), cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(&skipped, &m->adam_st->skipped, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  if (grads)
    CK(cudaMemcpyAsync(grads, m->grads_final(), sizeof(float) * m->P, cudaMemcpyDeviceToHost, s));
  if (m->sh.err) CK(cudaMemcpyAsync(&err, m->sh.err, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  int32_t derr = 0;
  if (m->dp.err) CK(cudaMemcpyAsync(&derr, m->dp.err, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (err) return fail(MARS_ECUDA, "shard barrier timed out (a peer shard did not step)");
  if (derr) return fail(MARS_ECUDA, "data-parallel barrier timed out (a peer rank did not step)");
  if (loss) *loss = l;
  return check_skipped(m, skipped);
}

extern "C" mars_status mars_dgi_enqueue_loss(mars_dgi* m, int64_t* ticket) {
  if (mars_status st = check_dgi(m)) return st;
  if (!ticket) return fail(MARS_EINVAL, "ticket is NULL");
  CK(cudaSetDevice(m->cfg.device));
  if (!m->loss_ring) {
    CK(cudaMallocHost(&m->loss_ring, sizeof(mars_dgi::LossSlot) * mars_dgi::kLossRing));
    for (cudaEvent_t& e : m->loss_ev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  const int slot = (int)(m->loss_next % mars_dgi::kLossRing);
  // the slot's previous copy must have landed before it is overwritten
  CK(cudaEventSynchronize(m->loss_ev[slot]));
  cudaStream_t s = m->stream;
  mars_dgi::LossSlot* d = m->loss_ring + slot;
  CK(cudaMemcpyAsync(&d->loss, m->grads_final() + m->P, sizeof(float), cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(&d->skipped, &m->adam_st->skipped, sizeof(int32_t), cudaMemcpyDeviceToHost,
                     s));
  CK(cudaEventRecord(m->loss_ev[slot], s));
  *ticket = m->loss_next++;
  return MARS_OK;
}

extern "C" mars_status mars_dgi_wait_loss(mars_dgi* m, int64_t ticket, float* loss) {
  if (mars_status st = check_dgi(m)) return st;
  if (ticket < 0 || ticket >= m->loss_next || ticket < m->loss_next - mars_dgi::kLossRing)
    return fail(MARS_EINVAL, "loss ticket %lld is not one of the last %d enqueued",
                (long long)ticket, mars_dgi::kLossRing);
  CK(cudaSetDevice(m->cfg.device));
  const int slot = (int)(ticket % mars_dgi::kLossRing);
  CK(cudaEventSynchronize(m->loss_ev[slot]));
  const mars_dgi::LossSlot d = m->loss_ring[slot];
  if (loss) *loss = d.loss;
  return check_skipped(m, d.skipped);
}

// ---------------------------------------------------------------- placer (NEXT-2)
struct mars_placer {
  uint64_t tag = kTagPlacer;
  mars_placer_config cfg{};
  PlacerDims d{};
  int64_t P = 0;
  float* params = nullptr;
  PlacerParams w{};
  PlacerWork ws{};
  int64_t ws_N = 0, ws_S = 0, ws_seg = 0;
  std::vector<void*> owned;
  // training (NEXT-3): saved activations, backward state, gradient vector
  PlacerTrain tr{};
  PlacerBwd bw{};
  float *grads = nullptr, *wT = nullptr, *X = nullptr, *tmpNH = nullptr, *ebuf = nullptr;
  double* part = nullptr;
  int32_t* order_b = nullptr;
  int64_t tr_N = 0, tr_S = 0;
  std::vector<void*> tr_owned;
  // the BPTT's per-op kernel chain (~6 N + 2 N launches) captured once per
  // workspace and replayed (launch cost ~1-2 us per node instead of ~5-8 eager)
  cudaGraphExec_t bwd_exec = nullptr;
  const void* bwd_key[3] = {};
  int64_t bwd_launches = 0;
  float* Ein = nullptr;               // [N x H] the embeddings the captured backward reads
  void release_tr() {
    if (bwd_exec) cudaGraphExecDestroy(bwd_exec);
    bwd_exec = nullptr;
    for (const void*& k : bwd_key) k = nullptr;
    for (void* q : tr_owned) cudaFree(q);
    tr_owned.clear();
    tr = PlacerTrain{};
    bw = PlacerBwd{};
    tr_N = tr_S = 0;
  }
  cudaStream_t stream = nullptr;
  void release_ws() {
    for (void* p : owned) cudaFree(p);
    owned.clear();
    ws = PlacerWork{};
    ws_N = ws_S = ws_seg = 0;
  }
  ~mars_placer() {
    if (stream) cudaStreamSynchronize(stream);
    release_ws();
    release_tr();
    if (params) cudaFree(params);
    if (stream) cudaStreamDestroy(stream);
  }
};

static PlacerDims placer_dims(const mars_placer_config* c) {
  return PlacerDims{c->in_dim, c->enc_hidden, c->attn_dim, c->dev_embed, c->num_devices};
}

extern "C" void mars_placer_config_default(mars_placer_config* c) {
  if (!c) return;
  memset(c, 0, sizeof *c);
  c->in_dim = 256;
  c->enc_hidden = 256;
  c->attn_dim = 512;
  c->dev_embed = 64;
  c->num_devices = 4;
  c->segment = 128;
}

extern "C" int64_t mars_placer_num_params(const mars_placer_config* c) {
  return c ? placer_num_params(placer_dims(c)) : -1;
}

static mars_status check_placer_cfg(const mars_placer_config* c) {
  if (!c) return fail(MARS_EINVAL, "NULL config");
  if (c->in_dim < 16 || c->in_dim % 16) return fail(MARS_EINVAL, "in_dim must be a multiple of 16");
  if (c->enc_hidden != 64 && c->enc_hidden != 128 && c->enc_hidden != 256)
    return fail(MARS_EINVAL, "enc_hidden must be 64, 128 or 256");
  if (c->attn_dim < 128 || c->attn_dim % 128) return fail(MARS_EINVAL, "attn_dim must be a multiple of 128");
  if (c->dev_embed < 1 || c->dev_embed > 256) return fail(MARS_EINVAL, "dev_embed in [1, 256]");
  if (c->num_devices < 2 || c->num_devices > 64) return fail(MARS_EINVAL, "num_devices in [2, 64]");
  if (c->segment < 1 || c->segment > 1024) return fail(MARS_EINVAL, "segment in [1, 1024]");
  return MARS_OK;
}

extern "C" mars_status mars_placer_create(const mars_placer_config* cfg, mars_placer** out) {
  if (!out) return fail(MARS_EINVAL, "out is NULL");
  *out = nullptr;
  if (mars_status st = check_placer_cfg(cfg)) return st;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(MARS_ECUDA, "no CUDA device (libmars has no CPU fallback)");
  }
  if (cfg->device < 0 || cfg->device >= ndev) return fail(MARS_EINVAL, "bad device");
  CK(cudaSetDevice(cfg->device));
  auto* p = new mars_placer();
  std::unique_ptr<mars_placer> guard(p);
  p->cfg = *cfg;
  p->cfg.init_params = nullptr;
  p->d = placer_dims(cfg);
  p->P = placer_num_params(p->d);
  CK(cudaStreamCreateWithFlags(&p->stream, cudaStreamNonBlocking));
  CK(dalloc(&p->params, (size_t)p->P));
  p->w = placer_views(p->d, p->params);
  if (cfg->init_params)
    CK(cudaMemcpyAsync(p->params, cfg->init_params, sizeof(float) * p->P, cudaMemcpyHostToDevice,
                       p->stream));
  else
    CK(placer_init(p->d, p->params, cfg->seed, p->stream));
  CK(placer_prepare(p->d));
  CK(cudaStreamSynchronize(p->stream));
  *out = guard.release();
  return MARS_OK;
}

static mars_status check_placer(const mars_placer* p) {
  if (!p || p->tag != kTagPlacer) return fail(MARS_ESTATE, "invalid or freed mars_placer handle");
  return MARS_OK;
}

extern "C" mars_status mars_placer_get_params(const mars_placer* p, float* params) {
  if (mars_status st = check_placer(p)) return st;
  if (!params) return fail(MARS_EINVAL, "params is NULL");
  CK(cudaSetDevice(p->cfg.device));
  CK(cudaStreamSynchronize(p->stream));
  CK(cudaMemcpy(params, p->params, sizeof(float) * p->P, cudaMemcpyDeviceToHost));
  return MARS_OK;
}

extern "C" mars_status mars_placer_set_params(mars_placer* p, const float* params) {
  if (mars_status st = check_placer(p)) return st;
  if (!params) return fail(MARS_EINVAL, "params is NULL");
  CK(cudaSetDevice(p->cfg.device));
  CK(cudaStreamSynchronize(p->stream));
  CK(cudaMemcpy(p->params, params, sizeof(float) * p->P, cudaMemcpyHostToDevice));
  return MARS_OK;
}

static mars_status placer_ensure(mars_placer* p, int64_t N, int64_t S) {
  const int64_t seg = p->cfg.segment;
  if (p->ws_N >= N && p->ws_S >= S && p->ws_seg == seg) return MARS_OK;
  CK(cudaStreamSynchronize(p->stream));
  p->release_ws();
  const PlacerDims& d = p->d;
  const int64_t Hd = d.Hd, Hs = 2 * Hd, nseg = (N + seg - 1) / seg;
  auto al = [&](float** q, size_t n) -> cudaError_t {
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(q), sizeof(float) * (n ? n : 1));
    if (e == cudaSuccess) p->owned.push_back(*q);
    return e;
  };
  PlacerWork& w = p->ws;
  CK(al(&w.xp[0], N * 4 * Hd));
  CK(al(&w.xp[1], N * 4 * Hd));
  CK(al(&w.enc, N * Hs));
  CK(al(&w.keys, N * d.A));
  CK(al(&w.seg_h, nseg * Hs));
  CK(al(&w.seg_c, nseg * Hs));
  CK(al(&w.hbuf, 4 * Hd));
  CK(al(&w.sh, 2 * S * Hs));
  CK(al(&w.sc, S * Hs));
  CK(al(&w.q, S * d.A));
  CK(al(&w.ghh, S * 4 * Hs));
  CK(al(&w.score, S * seg));
  CK(al(&w.ctx, S * Hs));
  CK(al(reinterpret_cast<float**>(&w.bar), 2));
  p->ws_N = N;
  p->ws_S = S;
  p->ws_seg = seg;
  return MARS_OK;
}

// Training workspace for N ops and S samples (saved activations, backward).
static mars_status placer_ensure_train(mars_placer* p, int64_t N, int64_t S) {
  if (p->tr_N >= N && p->tr_S >= S && p->tr_N == N && p->tr_S == S) return MARS_OK;
  CK(cudaStreamSynchronize(p->stream));
  p->release_tr();
  const PlacerDims& d = p->d;
  const int64_t Hd = d.Hd, Hs = 2 * Hd, Hin = Hs + d.De, A = d.A, seg = p->cfg.segment;
  const int64_t SN = S * N, nseg = (N + seg - 1) / seg;
  auto al = [&](void** q, size_t bytes) -> cudaError_t {
    cudaError_t e = cudaMalloc(q, bytes ? bytes : 8);
    if (e == cudaSuccess) p->tr_owned.push_back(*q);
    return e;
  };
  auto alf = [&](float** q, int64_t n) { return al(reinterpret_cast<void**>(q), sizeof(float) * n); };
  PlacerTrain& t = p->tr;
  CK(alf(&t.sv_hprev, SN * Hs));
  CK(alf(&t.sv_cprev, SN * Hs));
  CK(alf(&t.sv_gates, SN * 4 * Hs));
  CK(alf(&t.sv_c, SN * Hs));
  CK(alf(&t.sv_h, SN * Hs));
  CK(alf(&t.sv_q, SN * A));
  CK(alf(&t.sv_alpha, SN * seg));
  CK(alf(&t.sv_ctx, SN * Hs));
  CK(al(reinterpret_cast<void**>(&t.sv_prev), sizeof(int32_t) * SN));
  CK(alf(&t.esv_gates, 2 * N * 4 * Hd));
  CK(alf(&t.esv_c, 2 * N * Hd));
  CK(alf(&t.dz, SN * d.D));
  CK(alf(&t.lterm, SN));
  CK(alf(const_cast<float**>(&t.logp_old), SN));
  CK(alf(const_cast<float**>(&t.adv), S));
  PlacerBwd& b = p->bw;
  CK(alf(&b.dg, SN * 4 * Hs));
  CK(alf(&b.dx, SN * Hin));
  CK(alf(&b.dq, SN * A));
  CK(alf(&b.dvp, SN * A));
  CK(alf(&b.dhr, S * Hs));
  CK(alf(&b.dcr, S * Hs));
  CK(alf(&b.dhr_part, S * Hs));
  CK(al(reinterpret_cast<void**>(&b.dal), sizeof(double) * S * seg));
  CK(alf(&b.de, S * seg));
  CK(alf(&b.dK, N * A));
  CK(alf(&b.denc, N * Hs));
  CK(alf(&b.dinit_h, nseg * Hs));
  CK(alf(&b.dinit_c, nseg * Hs));
  CK(alf(&b.edg, 2 * N * 4 * Hd));
  CK(alf(&b.ehr, 2 * Hd));
  CK(alf(&b.ecr, 2 * Hd));
  CK(alf(&p->grads, p->P + 1));
  // transposes: W_ihᵀ [Hin x 4Hs], W_hhᵀ [Hs x 4Hs], W_qᵀ [Hs x A], enc W_hhᵀ x2 [Hd x 4Hd]
  CK(alf(&p->wT, Hin * 4 * Hs + Hs * 4 * Hs + Hs * A + 2 * Hd * 4 * Hd));
  CK(alf(&p->X, SN * std::max<int64_t>(Hin, Hs)));
  CK(alf(&p->tmpNH, N * std::max<int64_t>(Hs, d.H)));
  CK(alf(&p->Ein, N * d.H));
  CK(alf(&p->ebuf, 2 * N * std::max<int64_t>(Hd, d.H)));
  size_t pt = 0;
  const int64_t shapes[][3] = {{SN, 4 * Hs, Hin}, {SN, 4 * Hs, Hs}, {SN, A, Hs}, {N, A, Hs},
                               {N, 4 * Hd, d.H}, {N, 4 * Hd, Hd}};
  for (auto& sh : shapes) pt = std::max(pt, gemm_tn_partial_floats(sh[0], (int)sh[1], (int)sh[2]));
  CK(al(reinterpret_cast<void**>(&p->part), sizeof(double) * pt));
  CK(al(reinterpret_cast<void**>(&p->order_b), sizeof(int32_t) * N));
  {   // backward-direction op order of the encoder steps (c23)
    std::vector<int32_t> ord((size_t)N);
    for (int64_t t2 = 0; t2 < N; ++t2) {
      const int64_t j0 = (t2 / seg) * seg, j1 = std::min(N, j0 + seg);
      ord[t2] = (int32_t)(j1 - 1 - (t2 - j0));
    }
    CK(cudaMemcpy(p->order_b, ord.data(), sizeof(int32_t) * N, cudaMemcpyHostToDevice));
  }
  b.N = (int32_t)N;
  b.S = (int32_t)S;
  b.seg = (int32_t)seg;
  b.Hd = (int32_t)Hd;
  b.Hs = (int32_t)Hs;
  b.Hin = (int32_t)Hin;
  b.A = (int32_t)A;
  b.D = d.D;
  b.wo = p->w.wo;
  b.v = p->w.v;
  b.keys = p->ws.keys;
  b.enc = p->ws.enc;
  b.wihT = p->wT;
  b.whhT = p->wT + Hin * 4 * Hs;
  b.wqT = b.whhT + Hs * 4 * Hs;
  b.ewhhT[0] = b.wqT + Hs * A;
  b.ewhhT[1] = b.ewhhT[0] + Hd * 4 * Hd;
  b.sv_gates = t.sv_gates;
  b.sv_c = t.sv_c;
  b.sv_cprev = t.sv_cprev;
  b.sv_q = t.sv_q;
  b.sv_alpha = t.sv_alpha;
  b.dz = t.dz;
  b.esv_gates = t.esv_gates;
  b.esv_c = t.esv_c;
  p->tr_N = N;
  p->tr_S = S;
  return MARS_OK;
}

// The backward section of placer_loss_grad (every launch stream-ordered, all
// pointers fixed per training workspace, so it is captured once and replayed):
// transposed weights, the decoder BPTT, the decoder's weight gradients, the
// encoder BPTT and its gradients, dL/dE into p->tmpNH, the loss into
// p->grads[P].  E is p->Ein.
static cudaError_t placer_bwd_section(mars_placer* p, int32_t N, int32_t S, cudaStream_t s,
                                      int* nl) {
  const PlacerDims& d = p->d;
  const int64_t Hd = d.Hd, Hs = 2 * Hd, Hin = Hs + d.De, A = d.A, SN = (int64_t)S * N;
  PlacerTrain& t = p->tr;
  PlacerBwd& b = p->bw;
  const float* E = p->Ein;
  cudaError_t e;
#define RE(x) do { if ((e = (x)) != cudaSuccess) return e; } while (0)
  RE(placer_transpose(p->w.dec_wih, (int)(4 * Hs), (int)Hin, const_cast<float*>(b.wihT), s));
  RE(placer_transpose(p->w.dec_whh, (int)(4 * Hs), (int)Hs, const_cast<float*>(b.whhT), s));
  RE(placer_transpose(p->w.wq, (int)A, (int)Hs, const_cast<float*>(b.wqT), s));
  for (int dir = 0; dir < 2; ++dir)
    RE(placer_transpose(p->w.enc_whh[dir], (int)(4 * Hd), (int)Hd, const_cast<float*>(b.ewhhT[dir]), s));
  RE(cudaMemsetAsync(b.dK, 0, sizeof(float) * N * A, s));
  RE(cudaMemsetAsync(b.denc, 0, sizeof(float) * N * Hs, s));
  RE(placer_bwd_decoder(b, s, nl));
  // decoder weight gradients
  PlacerParams G = placer_views(d, p->grads);
  RE(placer_build_x(t.sv_ctx, t.sv_prev, p->w.emb, SN, (int)Hs, d.De, p->X, s));
  RE(gemm_tn(b.dg, p->X, G.dec_wih, SN, (int)(4 * Hs), (int)Hin, p->part, s, nl));
  RE(gemm_tn(b.dg, t.sv_hprev, G.dec_whh, SN, (int)(4 * Hs), (int)Hs, p->part, s, nl));
  RE(placer_colsum(b.dg, SN, (int)(4 * Hs), G.dec_b, s));
  RE(gemm_tn(b.dq, t.sv_hprev, G.wq, SN, (int)A, (int)Hs, p->part, s, nl));
  RE(placer_colsum(b.dvp, SN, (int)A, G.v, s));
  RE(placer_small_tn(t.dz, t.sv_h, SN, d.D, (int)Hs, G.wo, s));
  RE(placer_colsum(t.dz, SN, d.D, G.bo, s));
  RE(placer_emb_grad(b.dx, t.sv_prev, SN, (int)Hs, (int)Hin, d.De, d.D + 1, G.emb, s));
  RE(gemm_tn(b.dK, p->ws.enc, G.wk, N, (int)A, (int)Hs, p->part, s, nl));
  RE(gemm_nn(b.dK, p->w.wk, p->tmpNH, N, (int)Hs, (int)A, s, nl));     // d(K)/d(enc)
  RE(placer_add(b.denc, p->tmpNH, N * Hs, s));
  // encoder BPTT and its gradients
  RE(placer_bwd_encoder(b, s, nl));
  float* Eb = p->ebuf;                      // E in the backward direction's step order
  RE(placer_gather_rows(E, p->order_b, N, d.H, Eb, 0, s));
  RE(gemm_tn(b.edg, E, G.enc_wih[0], N, (int)(4 * Hd), d.H, p->part, s, nl));
  RE(gemm_tn(b.edg + N * 4 * Hd, Eb, G.enc_wih[1], N, (int)(4 * Hd), d.H, p->part, s, nl));
  for (int dir = 0; dir < 2; ++dir) {
    float* hs = p->ebuf;                    // h of each step of this direction, step order
    RE(placer_gather_cols(p->ws.enc, Hs, dir * (int)Hd, dir ? p->order_b : nullptr, N, (int)Hd, hs, s));
    const float* edg = b.edg + (int64_t)dir * N * 4 * Hd;
    if (N > 1)
      RE(gemm_tn(edg + 4 * Hd, hs, G.enc_whh[dir], N - 1, (int)(4 * Hd), (int)Hd, p->part, s, nl));
    else
      RE(cudaMemsetAsync(G.enc_whh[dir], 0, sizeof(float) * 4 * Hd * Hd, s));
    RE(placer_colsum(edg, N, (int)(4 * Hd), G.enc_b[dir], s));
  }
  // dL/dE: forward direction in op order, backward direction scattered by its order
  RE(gemm_nn(b.edg, p->w.enc_wih[0], p->tmpNH, N, d.H, (int)(4 * Hd), s, nl));
  RE(gemm_nn(b.edg + N * 4 * Hd, p->w.enc_wih[1], p->ebuf, N, d.H, (int)(4 * Hd), s, nl));
  RE(placer_gather_rows(p->ebuf, p->order_b, N, d.H, p->tmpNH, 1, s));
  // the loss: sum of the per-op terms / (S N), fixed order
  RE(placer_colsum(t.lterm, SN, 1, p->grads + p->P, s));
#undef RE
  return cudaSuccess;
}

// The PPO loss (c29) of S teacher-forced placements and its gradient: placer
// forward with activations saved and dL/dlogits, then the backward section
// (captured once per workspace, replayed).  Leaves the gradient [P] and the
// loss sum (at [P]) in p->grads and dL/dE [N x H] in p->tmpNH.
static mars_status placer_loss_grad(mars_placer* p, const float* dE_in, int32_t N, int32_t S,
                                    const int32_t* dplace, float clip_eps, float ent_coef, int* nl) {
  cudaStream_t s = p->stream;
  const PlacerDims& d = p->d;
  const int64_t SN = (int64_t)S * N;
  PlacerTrain& t = p->tr;
  PlacerBwd& b = p->bw;
  b.keys = p->ws.keys;                    // the forward workspace may have been regrown
  b.enc = p->ws.enc;
  b.wo = p->w.wo;
  b.v = p->w.v;
  t.clip_eps = clip_eps;
  t.ent_coef = ent_coef;
  // forward with teacher forcing; place / logp / ent outputs into scratch rows of X
  int32_t* dP = reinterpret_cast<int32_t*>(p->X);
  float* dL = p->X + SN;
  float* dH = p->X + 2 * SN;
  CK(placer_forward(d, p->w, p->ws, dE_in, N, p->cfg.segment, S, 0, dplace, dP, dL, dH, s, nl, &t));
  if (dE_in != p->Ein)
    CK(cudaMemcpyAsync(p->Ein, dE_in, sizeof(float) * (size_t)N * d.H, cudaMemcpyDeviceToDevice, s));
  const void* key[3] = {p->ws.keys, p->ws.enc, b.dg};
  if (p->bwd_exec && (key[0] != p->bwd_key[0] || key[1] != p->bwd_key[1] || key[2] != p->bwd_key[2])) {
    cudaGraphExecDestroy(p->bwd_exec);
    p->bwd_exec = nullptr;
  }
  if (!p->bwd_exec) {
    cudaGraph_t graph;
    CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    int cnl = 0;
    cudaError_t e = placer_bwd_section(p, N, S, s, &cnl);
    cudaError_t e2 = cudaStreamEndCapture(s, &graph);
    if (e != cudaSuccess || e2 != cudaSuccess) {
      if (e2 == cudaSuccess) cudaGraphDestroy(graph);
      cudaGetLastError();
      return fail(MARS_ECUDA, "placer backward capture failed: %s",
                  cudaGetErrorString(e != cudaSuccess ? e : e2));
    }
    cudaError_t e3 = cudaGraphInstantiate(&p->bwd_exec, graph, 0);
    cudaGraphDestroy(graph);
    CK(e3);
    for (int k = 0; k < 3; ++k) p->bwd_key[k] = key[k];
    p->bwd_launches = cnl;
  }
  CK(cudaGraphLaunch(p->bwd_exec, s));
  count_launch(nl, (int)p->bwd_launches);
  return MARS_OK;
}

extern "C" mars_status mars_placer_ppo_grad(mars_placer* p, const float* emb, int32_t N,
                                            int32_t num_samples, const int32_t* placements,
                                            const float* logp_old, const float* adv,
                                            float clip_eps, float ent_coef, float* loss,
                                            float* grads, float* demb) {
  if (mars_status st = check_placer(p)) return st;
  if (!emb || !placements || !logp_old || !adv || N < 1)
    return fail(MARS_EINVAL, "NULL input or N < 1");
  if (num_samples < 1 || num_samples > 32) return fail(MARS_EINVAL, "num_samples in [1, 32]");
  const int64_t SN = (int64_t)num_samples * N;
  for (int64_t e = 0; e < SN; ++e)
    if (placements[e] < 0 || placements[e] >= p->d.D) return fail(MARS_EINVAL, "placement out of range");
  const int H = p->d.H;
  if (!(H == 32 || H == 64 || H % 128 == 0))
    return fail(MARS_EINVAL, "training needs in_dim in {32, 64} or a multiple of 128");
  CK(cudaSetDevice(p->cfg.device));
  if (mars_status st = placer_ensure(p, N, num_samples)) return st;
  if (mars_status st = placer_ensure_train(p, N, num_samples)) return st;
  cudaStream_t s = p->stream;
  float* dE = nullptr;
  int32_t* dPl = nullptr;
  struct FreeAll { std::vector<void*> v; cudaStream_t s; ~FreeAll() { for (void* q : v) cudaFreeAsync(q, s); } } fa{{}, s};
  CK(palloc(&dE, (size_t)N * H, s)); fa.v.push_back(dE);
  CK(palloc(&dPl, (size_t)SN, s)); fa.v.push_back(dPl);
  CK(cudaMemcpyAsync(dE, emb, sizeof(float) * (size_t)N * H, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(dPl, placements, sizeof(int32_t) * SN, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(const_cast<float*>(p->tr.logp_old), logp_old, sizeof(float) * SN,
                     cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(const_cast<float*>(p->tr.adv), adv, sizeof(float) * num_samples,
                     cudaMemcpyHostToDevice, s));
  int nl = 0;
  if (mars_status st = placer_loss_grad(p, dE, N, num_samples, dPl, clip_eps, ent_coef, &nl)) return st;
  float lsum = 0.f;
  CK(cudaMemcpyAsync(&lsum, p->grads + p->P, sizeof(float), cudaMemcpyDeviceToHost, s));
  if (grads) CK(cudaMemcpyAsync(grads, p->grads, sizeof(float) * p->P, cudaMemcpyDeviceToHost, s));
  if (demb) CK(cudaMemcpyAsync(demb, p->tmpNH, sizeof(float) * (size_t)N * H, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (loss) *loss = (float)((double)lsum / (double)SN);
  return MARS_OK;
}

extern "C" mars_status mars_placer_sample(mars_placer* p, const float* emb, int32_t N,
                                          int32_t num_samples, uint64_t sample_seed,
                                          const int32_t* forced, int32_t* placements, float* logp,
                                          float* entropy) {
  if (mars_status st = check_placer(p)) return st;
  if (!emb || N < 1) return fail(MARS_EINVAL, "need N >= 1 embeddings");
  if (num_samples < 1 || num_samples > 32) return fail(MARS_EINVAL, "num_samples in [1, 32]");
  if (forced)
    for (int64_t e = 0; e < (int64_t)num_samples * N; ++e)
      if (forced[e] < 0 || forced[e] >= p->d.D) return fail(MARS_EINVAL, "forced placement out of range");
  CK(cudaSetDevice(p->cfg.device));
  if (mars_status st = placer_ensure(p, N, num_samples)) return st;
  cudaStream_t s = p->stream;
  const int64_t SN = (int64_t)num_samples * N;
  float* dE = nullptr;
  int32_t *dF = nullptr, *dP = nullptr;
  float *dL = nullptr, *dH = nullptr;
  struct FreeAll { std::vector<void*> v; cudaStream_t s; ~FreeAll() { for (void* q : v) cudaFreeAsync(q, s); } } fa{{}, s};
  CK(palloc(&dE, (size_t)N * p->d.H, s)); fa.v.push_back(dE);
  CK(palloc(&dP, (size_t)SN, s)); fa.v.push_back(dP);
  CK(palloc(&dL, (size_t)SN, s)); fa.v.push_back(dL);
  CK(palloc(&dH, (size_t)SN, s)); fa.v.push_back(dH);
  if (forced) {
    CK(palloc(&dF, (size_t)SN, s)); fa.v.push_back(dF);
    CK(cudaMemcpyAsync(dF, forced, sizeof(int32_t) * SN, cudaMemcpyHostToDevice, s));
  }
  CK(cudaMemcpyAsync(dE, emb, sizeof(float) * (size_t)N * p->d.H, cudaMemcpyHostToDevice, s));
  int nl = 0;
  CK(placer_forward(p->d, p->w, p->ws, dE, N, p->cfg.segment, num_samples, sample_seed, dF, dP, dL,
                    dH, s, &nl));
  if (placements) CK(cudaMemcpyAsync(placements, dP, sizeof(int32_t) * SN, cudaMemcpyDeviceToHost, s));
  if (logp) CK(cudaMemcpyAsync(logp, dL, sizeof(float) * SN, cudaMemcpyDeviceToHost, s));
  if (entropy) CK(cudaMemcpyAsync(entropy, dH, sizeof(float) * SN, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  return MARS_OK;
}

extern "C" mars_status mars_dgi_encoder_vjp(mars_dgi* m, const mars_graph* g, const float* dE,
                                            float* grads) {
  if (mars_status st = check_dgi(m)) return st;
  if (mars_status st = check_graph(g)) return st;
  if (!dE || !grads) return fail(MARS_EINVAL, "NULL argument");
  if (g->sharded || g->F != m->F) return fail(MARS_EINVAL, "unsharded graph of the model's F");
  if (m->cfg.precision != MARS_FP32) return fail(MARS_EINVAL, "fp32 models only");
  if (m->sage || m->pool) return fail(MARS_EINVAL, "no encoder VJP for the SAGE encoders");
  CK(cudaSetDevice(m->cfg.device));
  if (mars_status st = ensure_ws(m, g)) return st;
  cudaStream_t s = m->stream;
  float* d = nullptr;
  const size_t n = (size_t)g->dev.Nt * m->H;
  CK(palloc(&d, n, s));
  struct F1 { float* p; cudaStream_t s; ~F1() { cudaFreeAsync(p, s); } } f1{d, s};
  CK(cudaMemcpyAsync(d, dE, sizeof(float) * n, cudaMemcpyHostToDevice, s));
  int nl = 0;
  CK(enqueue_encode(m, g, s, &nl));
  CK(enqueue_encoder_backward(m, g, d, s, &nl));
  CK(cudaMemcpyAsync(grads, m->grads, sizeof(float) * m->P, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  g->note_use(s);
  m->last_Nt = 0;
  return MARS_OK;
}

// ---------------------------------------------------------------- PPO (NEXT-3)
struct mars_ppo {
  uint64_t tag = kTagPpo;
  mars_ppo_config cfg{};
  mars_placer* p = nullptr;
  mars_dgi* enc = nullptr;           // joint update of the GCN encoder (NULL: placer only)
  float *m = nullptr, *v = nullptr;  // Adam state of the placer
  double* guard = nullptr;
  AdamDev* st = nullptr;
  float *em = nullptr, *ev = nullptr;    // Adam state of the encoder (joint training)
  double* eguard = nullptr;
  AdamDev* est = nullptr;
  double baseline = 0.0;             // Eq. 7's B_{t-1}
  bool has_baseline = false;
  int64_t iteration = 0;
  ~mars_ppo() {
    for (void* q : {(void*)m, (void*)v, (void*)guard, (void*)st, (void*)em, (void*)ev,
                    (void*)eguard, (void*)est})
      if (q) cudaFree(q);
  }
};

extern "C" void mars_ppo_config_default(mars_ppo_config* c) {
  if (!c) return;
  memset(c, 0, sizeof *c);
  c->clip_eps = 0.2f;
  c->ent_coef = 0.001f;
  c->lr = 3e-4f;
  c->beta1 = 0.9f;
  c->beta2 = 0.999f;
  c->adam_eps = 1e-8f;
  c->clip_norm = 1.0f;
  c->mu = 0.99f;
  c->samples_per_policy = 10;
  c->policies = 2;
  c->minibatches = 4;
  c->epochs = 3;
  c->capacity_bytes = 12e9f;
}

extern "C" mars_status mars_ppo_create(mars_placer* p, mars_dgi* enc, const mars_ppo_config* cfg,
                                       mars_ppo** out) {
  if (!out) return fail(MARS_EINVAL, "out is NULL");
  *out = nullptr;
  if (mars_status st = check_placer(p)) return st;
  if (enc) {
    if (mars_status st = check_dgi(enc)) return st;
    if (enc->H != p->d.H) return fail(MARS_EINVAL, "encoder hidden_dim != placer in_dim");
    if (enc->sage || enc->pool)
      return fail(MARS_EINVAL, "the joint update needs the GCN encoder (no SAGE VJP)");
    if (enc->cfg.device != p->cfg.device) return fail(MARS_EINVAL, "encoder and placer on different devices");
  }
  if (!cfg) return fail(MARS_EINVAL, "NULL config");
  const int S = cfg->samples_per_policy * cfg->policies;
  if (cfg->samples_per_policy < 1 || cfg->policies < 1 || cfg->minibatches < 1 ||
      cfg->epochs < 1 || S % cfg->minibatches || S / cfg->minibatches > 32 ||
      cfg->samples_per_policy > 32)
    return fail(MARS_EINVAL, "bad PPO schedule (samples / minibatches)");
  if (p->d.D > 16) return fail(MARS_EINVAL, "the step-time model supports <= 16 devices");
  CK(cudaSetDevice(p->cfg.device));
  auto* o = new mars_ppo();
  std::unique_ptr<mars_ppo> guard(o);
  o->cfg = *cfg;
  o->p = p;
  o->enc = enc;
  CK(dalloc(&o->m, (size_t)p->P));
  CK(dalloc(&o->v, (size_t)p->P));
  CK(dalloc(&o->guard, (size_t)adam_guard_doubles()));
  CK(dalloc(&o->st, 1));
  CK(cudaMemset(o->m, 0, sizeof(float) * p->P));
  CK(cudaMemset(o->v, 0, sizeof(float) * p->P));
  CK(cudaMemset(o->st, 0, sizeof(AdamDev)));
  if (enc) {
    if (enc->cfg.precision != MARS_FP32) return fail(MARS_EINVAL, "joint training needs an fp32 encoder");
    if (enc->sh.g || enc->dp.R > 1 || enc->comm)
      return fail(MARS_EINVAL, "joint training needs a single-GPU, unsharded encoder");
    CK(dalloc(&o->em, (size_t)enc->P));
    CK(dalloc(&o->ev, (size_t)enc->P));
    CK(dalloc(&o->eguard, (size_t)adam_guard_doubles()));
    CK(dalloc(&o->est, 1));
    CK(cudaMemset(o->em, 0, sizeof(float) * enc->P));
    CK(cudaMemset(o->ev, 0, sizeof(float) * enc->P));
    CK(cudaMemset(o->est, 0, sizeof(AdamDev)));
  }
  *out = guard.release();
  return MARS_OK;
}

static mars_status check_ppo(const mars_ppo* o) {
  if (!o || o->tag != kTagPpo) return fail(MARS_ESTATE, "invalid or freed mars_ppo handle");
  return check_placer(o->p);
}

// One PPO iteration (readings c29-c32): sample policies x samples
// placements from the current policy, measure them (c30), Eq. 7 advantages in
// sampling order (c31), then `epochs` passes over a seeded shuffle of the
// placements in `minibatches` equal minibatches: per minibatch the PPO loss
// gradient (mars_placer_ppo_grad's path), clipped to clip_norm, and an Adam step.
static mars_status ppo_iteration(mars_ppo* o, const float* emb, const mars_graph* g, int32_t N,
                                 const int64_t* dims, const int64_t* indptr,
                                 const int32_t* indices, int32_t* placements_out,
                                 float* step_times_out, float* adv_out, float* mean_loss) {
  mars_placer* p = o->p;
  mars_dgi* enc = o->enc;
  const mars_ppo_config& c = o->cfg;
  if ((!emb && !g) || !dims || !indptr || N < 1) return fail(MARS_EINVAL, "NULL input or N < 1");
  const int H = p->d.H;
  if (!(H == 32 || H == 64 || H % 128 == 0))
    return fail(MARS_EINVAL, "training needs in_dim in {32, 64} or a multiple of 128");
  const int S = c.samples_per_policy * c.policies, mb = S / c.minibatches;
  const int64_t E = indptr[N];
  CK(cudaSetDevice(p->cfg.device));
  cudaStream_t s = p->stream;
  if (mars_status st = placer_ensure(p, N, std::max(S, c.samples_per_policy))) return st;
  if (mars_status st = placer_ensure_train(p, N, mb)) return st;
  float* dE = nullptr;
  int32_t *dPl = nullptr, *dMb = nullptr, *dIdx = nullptr;
  float *dLp = nullptr, *dEnt = nullptr;
  int64_t *dDims = nullptr, *dIp = nullptr;
  double* dT = nullptr;
  struct FreeAll { std::vector<void*> v; cudaStream_t s; ~FreeAll() { for (void* q : v) cudaFreeAsync(q, s); } } fa{{}, s};
  CK(palloc(&dE, (size_t)N * H, s)); fa.v.push_back(dE);
  CK(palloc(&dPl, (size_t)S * N, s)); fa.v.push_back(dPl);
  CK(palloc(&dMb, (size_t)mb * N, s)); fa.v.push_back(dMb);
  CK(palloc(&dLp, (size_t)S * N, s)); fa.v.push_back(dLp);
  CK(palloc(&dEnt, (size_t)S * N, s)); fa.v.push_back(dEnt);
  CK(palloc(&dDims, (size_t)N * 8, s)); fa.v.push_back(dDims);
  CK(palloc(&dIp, (size_t)N + 1, s)); fa.v.push_back(dIp);
  CK(palloc(&dIdx, (size_t)std::max<int64_t>(E, 1), s)); fa.v.push_back(dIdx);
  CK(palloc(&dT, (size_t)S, s)); fa.v.push_back(dT);
  if (enc) {                        // joint: the embeddings are the GCN encoder's, on the device
    CK(cudaStreamSynchronize(enc->stream));
    if (mars_status st = ensure_ws(enc, g)) return st;
    CK(enqueue_encode(enc, g, s, nullptr));
    CK(cudaMemcpyAsync(dE, enc->ws.dY, sizeof(float) * (size_t)N * H, cudaMemcpyDeviceToDevice, s));
  } else {
    CK(cudaMemcpyAsync(dE, emb, sizeof(float) * (size_t)N * H, cudaMemcpyHostToDevice, s));
  }
  CK(cudaMemcpyAsync(dDims, dims, sizeof(int64_t) * N * 8, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(dIp, indptr, sizeof(int64_t) * (N + 1), cudaMemcpyHostToDevice, s));
  if (E > 0) CK(cudaMemcpyAsync(dIdx, indices, sizeof(int32_t) * E, cudaMemcpyHostToDevice, s));
  int nl = 0;
  // 1. sample: `policies` draws of samples_per_policy placements, each its own seed
  for (int q = 0; q < c.policies; ++q) {
    const uint64_t seed = sm64(sm64(c.seed ^ 0x50504F53ULL) ^ (uint64_t)(o->iteration * c.policies + q));
    const int64_t off = (int64_t)q * c.samples_per_policy * N;
    CK(placer_forward(p->d, p->w, p->ws, dE, N, p->cfg.segment, c.samples_per_policy, seed,
                      nullptr, dPl + off, dLp + off, dEnt + off, s, &nl));
  }
  // 2. the environment (c30) and Eq. 7 (c31) in sampling order
  CK(launch_step_time(dPl, S, N, dDims, dIp, dIdx, p->d.D, (double)c.capacity_bytes, dT, s));
  std::vector<double> times(S);
  std::vector<float> lp_old((size_t)S * N);
  CK(cudaMemcpyAsync(times.data(), dT, sizeof(double) * S, cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(lp_old.data(), dLp, sizeof(float) * S * N, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  std::vector<float> adv(S);
  for (int b = 0; b < S; ++b) {
    const double R = -std::sqrt(times[b]);
    o->baseline = o->has_baseline ? (1.0 - c.mu) * R + c.mu * o->baseline : R;
    o->has_baseline = true;
    adv[b] = (float)(R - o->baseline);
  }
  // 3. epochs x minibatches over a seeded shuffle (c32: Fisher-Yates on splitmix64)
  double loss_sum = 0.0;
  int nsteps = 0;
  std::vector<int32_t> order(S);
  std::vector<float> adv_mb(mb), lp_mb((size_t)mb * N);
  for (int ep = 0; ep < c.epochs; ++ep) {
    for (int b = 0; b < S; ++b) order[b] = b;
    const uint64_t key = sm64(sm64(c.seed ^ 0x53485546ULL) ^ (uint64_t)(o->iteration * c.epochs + ep));
    for (int b = S - 1; b > 0; --b) {
      const int r = (int)(sm64(key ^ (uint64_t)b) % (uint64_t)(b + 1));
      std::swap(order[b], order[r]);
    }
    for (int k = 0; k < c.minibatches; ++k) {
      for (int q = 0; q < mb; ++q) {
        const int b = order[k * mb + q];
        CK(cudaMemcpyAsync(dMb + (int64_t)q * N, dPl + (int64_t)b * N, sizeof(int32_t) * N,
                           cudaMemcpyDeviceToDevice, s));
        adv_mb[q] = adv[b];
        memcpy(lp_mb.data() + (size_t)q * N, lp_old.data() + (size_t)b * N, sizeof(float) * N);
      }
      CK(cudaMemcpyAsync(const_cast<float*>(p->tr.logp_old), lp_mb.data(), sizeof(float) * mb * N,
                         cudaMemcpyHostToDevice, s));
      CK(cudaMemcpyAsync(const_cast<float*>(p->tr.adv), adv_mb.data(), sizeof(float) * mb,
                         cudaMemcpyHostToDevice, s));
      const float* Ecur = dE;
      if (enc) {                     // the encoder's current embeddings
        CK(enqueue_encode(enc, g, s, &nl));
        Ecur = enc->ws.dY;
      }
      if (mars_status st = placer_loss_grad(p, Ecur, N, mb, dMb, c.clip_eps, c.ent_coef, &nl)) return st;
      if (enc) {                     // dL/dE (p->tmpNH) on through the GCN, then its Adam step
        CK(enqueue_encoder_backward(enc, g, p->tmpNH, s, &nl));
        CK(launch_adam(enc->params, o->em, o->ev, enc->grads, enc->P, c.lr, c.beta1, c.beta2,
                       c.adam_eps, c.clip_norm, o->eguard, o->est, s, &nl));
      }
      CK(launch_adam(p->params, o->m, o->v, p->grads, p->P, c.lr, c.beta1, c.beta2, c.adam_eps,
                     c.clip_norm, o->guard, o->st, s, &nl));
      float lsum = 0.f;
      CK(cudaMemcpyAsync(&lsum, p->grads + p->P, sizeof(float), cudaMemcpyDeviceToHost, s));
      CK(cudaStreamSynchronize(s));       // the host-side staging buffers are reused
      loss_sum += (double)lsum / ((double)mb * N);
      ++nsteps;
    }
  }
  if (placements_out)
    CK(cudaMemcpyAsync(placements_out, dPl, sizeof(int32_t) * S * N, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (step_times_out)
    for (int b = 0; b < S; ++b) step_times_out[b] = (float)times[b];
  if (adv_out) memcpy(adv_out, adv.data(), sizeof(float) * S);
  if (mean_loss) *mean_loss = (float)(loss_sum / nsteps);
  o->iteration += 1;
  int32_t skipped = 0, eskipped = 0;
  CK(cudaMemcpy(&skipped, &o->st->skipped, sizeof(int32_t), cudaMemcpyDeviceToHost));
  if (enc) CK(cudaMemcpy(&eskipped, &o->est->skipped, sizeof(int32_t), cudaMemcpyDeviceToHost));
  if (skipped || eskipped)
    return fail(MARS_ENUMERIC, "non-finite PPO gradient: %d update(s) skipped", skipped + eskipped);
  if (enc) g->note_use(s);
  return MARS_OK;
}

extern "C" mars_status mars_ppo_iteration(mars_ppo* o, const float* emb, int32_t N,
                                          const int64_t* dims, const int64_t* indptr,
                                          const int32_t* indices, int32_t* placements_out,
                                          float* step_times_out, float* adv_out, float* mean_loss) {
  if (mars_status st = check_ppo(o)) return st;
  if (o->enc) return fail(MARS_ESTATE, "a joint PPO handle takes mars_ppo_iteration_joint");
  return ppo_iteration(o, emb, nullptr, N, dims, indptr, indices, placements_out, step_times_out,
                       adv_out, mean_loss);
}

extern "C" mars_status mars_ppo_iteration_joint(mars_ppo* o, const mars_graph* g,
                                                const int64_t* dims, const int64_t* indptr,
                                                const int32_t* indices, int32_t* placements_out,
                                                float* step_times_out, float* adv_out,
                                                float* mean_loss) {
  if (mars_status st = check_ppo(o)) return st;
  if (!o->enc) return fail(MARS_ESTATE, "mars_ppo_create was given no encoder");
  if (mars_status st = check_graph(g)) return st;
  if (mars_status st = check_dgi(o->enc)) return st;
  if (g->G != 1 || g->sharded || g->F != o->enc->F)
    return fail(MARS_EINVAL, "joint training takes one unsharded op graph of the encoder's F");
  return ppo_iteration(o, nullptr, g, g->Nt, dims, indptr, indices, placements_out,
                       step_times_out, adv_out, mean_loss);
}

extern "C" void mars_free(void* h) {
  if (!h) return;
  uint64_t tag = *static_cast<uint64_t*>(h);
  if (tag == kTagGraph) {
    auto* g = static_cast<mars_graph*>(h);
    cudaSetDevice(g->device);
    g->tag = kTagDead;
    delete g;
  } else if (tag == kTagDgi) {
    auto* m = static_cast<mars_dgi*>(h);
    cudaSetDevice(m->cfg.device);
    cudaStreamSynchronize(m->stream);
    m->tag = kTagDead;
    delete m;
  } else if (tag == kTagPpo) {
    auto* o = static_cast<mars_ppo*>(h);
    o->tag = kTagDead;
    delete o;
  } else if (tag == kTagPlacer) {
    auto* p = static_cast<mars_placer*>(h);
    cudaSetDevice(p->cfg.device);
    p->tag = kTagDead;
    delete p;
  }
}
