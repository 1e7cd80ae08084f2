// Internal declarations shared by the libmars.so translation units (kernels +
// runtime).  Nothing here is part of the ABI; include/mars.h is.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace mars {

constexpr int kLayers = 3;
constexpr int kMaxShards = 8;     // row shards of one graph (one per GPU of a node)

// Per-step scalars the captured step graph reads from device memory (written
// by one H2D copy before each replay, so a replay never bakes them in).
struct StepParams {
  uint64_t step_index;
  int64_t pair_base;
  float inv_batch;      // 1 / global batch B
  float pad;
};

// Adam's device-resident state (adam.cu): the step count and this step's bias
// corrections, written by the guard kernel only when the loss and every
// gradient are finite (otherwise skip = 1 and skipped counts the step).
struct AdamDev {
  int64_t t;            // completed updates (torch's state['step'])
  int32_t skip;         // this step's update was skipped
  int32_t skipped;      // total skipped updates
  double clip_coef;     // min(1, clip / (||g|| + 1e-6))
  float step_size;      // lr / (1 - beta1^t)
  float bc2_sqrt;       // sqrt(1 - beta2^t)
};

// Device view of a loaded graph set (block-diagonal, global node ids).
struct GraphDev {
  int32_t G;            // graphs
  int32_t Nt;           // total nodes
  int64_t nnz;          // nnz(Â) total
  int32_t F;
  const int32_t* node_off;   // [G+1]
  const int32_t* node_graph; // [Nt] graph id of each node
  const int32_t* rowptr;     // [Nt+1]
  const int32_t* colind;     // [nnz] global ids
  const float* vals;         // [nnz]
  const float* X;            // [Nt*F]
  // deterministic reduction chunks: rows [chunk_row[c], chunk_row[c+1]) all in graph chunk_graph[c]
  int32_t nchunks;
  const int32_t* chunk_row;  // [nchunks+1]
  const int32_t* chunk_graph;// [nchunks]
  const int32_t* graph_chunk;// [G+1] first chunk of each graph
  // permutation buckets
  // long rows (degree > long_min, e.g. weight-read hubs): aggregated by one warp
  // per segment of kLongSeg entries plus an in-order combine (spmm.cu); the
  // main SpMM kernels skip them
  int32_t long_min = 0x7fffffff;       // rows with more entries than this are long
  int32_t nlong = 0;
  int32_t nseg = 0;
  const int32_t* long_rows = nullptr;  // [nlong] row ids (view-local)
  const int32_t* long_seg = nullptr;   // [nlong + 1] first segment of each long row
  const int32_t* seg_row = nullptr;    // [nseg] long-row index of each segment
  float* long_part = nullptr;          // [nseg * 2 * 256] fp32 partial sums (scratch)
  int32_t nbuckets;
  const int32_t* bucket_off; // [G+1]
  const int32_t* bucket_log2;// [G]
  int32_t max_bucket_log2 = 0;  // host copy of max_g bucket_log2[g] (per-graph perm kernel)
  int32_t max_graph_nodes = 0;  // host copy of max_g N_g
  const int32_t* gsize;      // [G] node count N_g of each graph (all shards of a row-sharded graph)
  const int64_t* pair_off;   // [G] pair index of graph g = pair_base + pair_off[g] (c15)
};

// ---------------------------------------------------------------- row sharding
// A row-sharded activation buffer as seen by every shard: shard p holds global
// rows [start[p], start[p+1]) stacked [pos; neg] (2 n_p rows of C) at base[p],
// which is device memory of shard p's GPU (peer-mapped; CUDA IPC across
// processes).  start[q] = INT32_MAX for q > P, so owner(j) = #{q >= 1 : start[q] <= j}.
struct PeerRows {
  const void* base[kMaxShards];
  int32_t start[kMaxShards + 1];
};
// Cross-shard device barrier: shard `me` stores its epoch into slot `me` of
// every shard's arrival array (flags[q], peer-mapped) with release semantics at
// system scope, then spins (acquire) until every slot of its own array reaches
// the epoch.  epoch is a local device counter, so captured replays advance it.
// A wait longer than ~20 s sets *err and returns (no hang).
struct ShardSync {
  int32_t P, me;
  unsigned long long* flags[kMaxShards];
  unsigned long long* epoch;
  int32_t* err;
};
// Peer-visible small buffers read after a barrier (head exchange, gradients).
struct PeerPtrs {
  const void* p[kMaxShards];
};
cudaError_t launch_shard_barrier(const ShardSync& s, cudaStream_t st, int* launches);
// Head exchange: t[c] = Σ_p x_p[c] over shards in rank order (fp64), c < H; the
// loss slot x_p[H] is summed into *loss_g.  mode 0: outd = sig(t / N), outf =
// (float) outd (readout s);  mode 1: outd = t, outf = (float) t (dv).
cudaError_t launch_head_xsum(const PeerPtrs& x, int P, int H, int mode, const int32_t* gsize,
                             double* outd, float* outf, double* loss_g, cudaStream_t st,
                             int* launches);
// out[k] = Σ_p g_p[k] (fp64, rank order) for k outside [keep_b, keep_e) and
// (unless sum_last) k != n - 1; the others (row-sharded graph: dM and the
// loss, already global on every shard) out[k] = g_me[k].
cudaError_t launch_grad_sum(const PeerPtrs& g, int P, int me, int64_t n, int64_t keep_b,
                            int64_t keep_e, int sum_last, float* out, cudaStream_t st,
                            int* launches);

// ---------------------------------------------------------------- builder.cu
// Builds the CSR of Â for the packed set.  d_indptr: [Nt + G] int64 concatenated
// per-graph indptr arrays; d_indices: [Et] local indices; node_off/edge_off
// per graph.  Outputs rowptr [Nt+1], colind (allocated by caller with the
// returned capacity), deg, dinv, vals.  err_flag: set nonzero on malformed input.
struct BuilderIO {
  int32_t G, Nt;
  int64_t Et;
  const int64_t* indptr;     // [Nt+G]
  const int32_t* indices;    // [Et]
  const int32_t* node_off;   // [G+1]
  const int64_t* edge_off;   // [G+1]
  const int32_t* node_graph; // [Nt]
  int32_t* cnt;              // [Nt+1] scratch
  int32_t* off_dup;          // [Nt+1] scratch
  int32_t* cursor;           // [Nt] scratch
  int32_t* buf;              // [Nt+2Et] scratch
  int32_t* buf2;             // [Nt+2Et] scratch
  int32_t* ucnt;             // [Nt+1] scratch
  int32_t* rowptr;           // [Nt+1] out
  int32_t* deg;              // [Nt] out
  float* dinv;               // [Nt] out
  int32_t* err;              // [1]
  void* scan_tmp;            // scratch for scans
  size_t scan_tmp_bytes;
};
size_t scan_tmp_bytes(int64_t n);
cudaError_t scan_exclusive_i32(const int32_t* in, int32_t* out, int64_t n, void* tmp,
                               cudaStream_t s, int* launches);
cudaError_t build_csr_phase1(const BuilderIO& io, cudaStream_t s);  // -> rowptr (host reads nnz)
cudaError_t build_csr_phase2(const BuilderIO& io, int32_t* colind, float* vals,
                             cudaStream_t s);

// ---------------------------------------------------------------- perm.cu
// Corruption permutation (Eq. 2, c12) for every graph of the set; writes
// perm_global[Nt] (global node id of X~ row i).
struct PermWork {
  uint64_t* keys;     // [Nt]
  int32_t* bucket;    // [Nt]
  int32_t* bcnt;      // [nbuckets+1]
  int32_t* bstart;    // [nbuckets+1]
  int32_t* bcur;      // [nbuckets]
  int32_t* members;   // [Nt]
  void* scan_tmp;
};
cudaError_t launch_perm(const GraphDev& g, uint64_t seed, const StepParams* sp,
                        const PermWork& w, int32_t* perm_global, cudaStream_t s, int* launches);
// launch_perm + launch_colperm over the same (unsharded) view in one launch of
// one CTA per graph (buckets and members in shared memory); returns
// cudaErrorNotSupported when a graph is too large for it (the caller then
// runs the two launches above).
cudaError_t launch_perm_graph(const GraphDev& g, uint64_t seed, const StepParams* sp,
                              const PermWork& w, int32_t* perm_global, int32_t* colperm,
                              cudaStream_t s, int* launches);

// ---------------------------------------------------------------- spmm.cu
// A row is long when its serial gather time would exceed about half the row
// kernel's duration: degree > kLongFactor x rows per resident warp slot
// (Nt / (SMs x 32)), clamped to [kLongMin, kLongMax] (graph load, mars_api.cu).
constexpr int kLongFactor = 8;
constexpr int kLongMin = 128;
constexpr int kLongMax = 1024;
constexpr int kLongSeg = 128;   // entries per segment
// Forward aggregate of both branches: Y[i] = Σ_j a_ij act(T[j]), Y[Nt+i] = Σ_j a_ij
// act(T[Nt+j]).  layer1: T = X (pos) and X[pi[j]] (neg), act = identity; `perm`
// is then colperm[k] = pi[colind[k]] (launch_colperm), indexed like colind.
// Otherwise act = PReLU(alpha[act_layer]).  neg_rows = 0 aggregates only the
// positive branch (encode).
// in_bf16 / out_bf16: storage type of T / Y (fp32 or bf16); fp32 accumulation.
// peers != nullptr (row-sharded graph, layers 2-3 only): T is gathered from the
// shards' buffers by global column id (C in {128, 256}, in_bf16 == out_bf16).
cudaError_t launch_spmm_fwd(const GraphDev& g, int C, const void* T, int in_bf16,
                            const int32_t* perm, const float* alpha_dev, int act_layer, void* Y,
                            int out_bf16, int both, cudaStream_t s, int* launches,
                            const PeerRows* peers = nullptr, float* row_scale = nullptr);
// row_scale (fp32 storage only, may be null): per stored row the power-of-two
// scale 2^(14 - e) of its max |value| (operand scaling of gemm_tc3h.cu).
// Backward aggregate dH = Â_n dY (Â_n symmetric) with the PReLU'(Z) epilogue:
// dZ = dH ⊙ (Z > 0 ? 1 : a), dalpha partials Σ dH·min(Z,0) -> slots[gridDim].
// dY, Z, dZ share one storage type (bf16 != 0: bf16).
cudaError_t launch_spmm_bwd(const GraphDev& g, int C, const void* dY, const void* Z, int bf16,
                            const float* alpha_dev, int layer, void* dZ, double* slots,
                            int* nslots, cudaStream_t s, int* launches,
                            const PeerRows* peers = nullptr, float* row_scale = nullptr);
int spmm_bwd_slots(const GraphDev& g);
// Layer 1's corrupted-branch column ids: colperm[k] = pi[colind[k]] over the
// view's entries (launch_spmm_fwd's `perm` argument for act_layer < 0).
cudaError_t launch_max_degree(const int32_t* rowptr, int32_t Nt, int32_t* out, cudaStream_t s);
cudaError_t launch_colperm(const GraphDev& g, const int32_t* perm, int32_t* colperm,
                           cudaStream_t s, int* launches);

// ---------------------------------------------------------------- gemm_simt.cu
// fp32 SIMT GEMMs (parity path).
cudaError_t gemm_nn(const float* A, const float* B, float* C, int64_t M, int N, int K,
                    cudaStream_t s, int* launches);       // C[M×N] = A[M×K] B[K×N]
cudaError_t gemm_nt(const float* A, const float* B, float* C, int64_t M, int N, int K,
                    cudaStream_t s, int* launches);       // C[M×N] = A[M×K] B[N×K]ᵀ
size_t gemm_tn_partial_floats(int64_t R, int M, int N);
cudaError_t gemm_tn(const float* A, const float* B, float* out, int64_t R, int M, int N,
                    double* partial, cudaStream_t s, int* launches);  // out[M×N] = Aᵀ B, A[R×M], B[R×N]

// ---------------------------------------------------------------- gemm_common.cu
// tcgen05 GEMMs are specialised for H in {128, 256} and C_in in {64, 128, 256}.
bool tc_supported(int cin, int h);
bool tc3h_supported(int cin, int h);   // the 3xFP16 fp32 path (also the tiny widths)
size_t tc_dw_partial_floats(int64_t R, int CIN);
// gemm_tc3h.cu: 3xFP16 row GEMMs with power-of-two scaling (fp32 path)
// The same split for up to three layers in one launch (the DGI step's W1..W3).
struct W3Split {
  const float* W[3];
  int cin[3];
  int H;
  float* wsc[3];
  void *bt_hi[3], *bt_lo[3], *b_hi[3], *b_lo[3];   // fp16
};
cudaError_t tc3h_split_weights_all(const W3Split& a, int nl, cudaStream_t s, int* launches);
cudaError_t tc3h_split_weights(const float* W, int CIN, int H, float* wsc, void* Bt_hi,
                               void* Bt_lo, void* B_hi, void* B_lo, cudaStream_t s,
                               int* launches);
cudaError_t tc3h_gemm_rows(const float* A, const float* rs, const void* B_hi, const void* B_lo,
                           const float* inv_tb, float* C, int64_t M, int N, int K, cudaStream_t s,
                           int* launches);
cudaError_t tc3h_gemm_dw(const float* Y, const float* rs_y, const float* dZ, const float* rs_dz,
                         float* dW, int64_t R, int CIN, int H, float* part, cudaStream_t s,
                         int* launches);
int tc_dw_chunks(int64_t R, int CIN);
cudaError_t tc3h_row_scales(const float* A, int64_t M, int K, float* rs, cudaStream_t s,
                            int* launches);
bool tc_tmap(CUtensorMap* m, CUtensorMapDataType dt, int elem_bytes, const void* base,
             int64_t rows, int64_t cols, int box_cols, int box_rows, CUtensorMapSwizzle swz);
int tc_num_sms();
bool tc_tmap_blocks(CUtensorMap* m, CUtensorMapDataType dt, int elem_bytes, const void* base,
                    int64_t rows, int64_t cols, int box_rows, int nblk);

// ---------------------------------------------------------------- gemm_tc16.cu
// bf16 path (MARS_BF16): one kind::f16 MMA per k-step, bf16 operands, fp32
// accumulation in TMEM.  Same support condition as tc_supported.
cudaError_t tc16_weights(const float* W, int CIN, int H, void* Bt16, void* B16, cudaStream_t s,
                         int* launches);   // Bt16 = bf16(Wᵀ) [H×Cin], B16 = bf16(W) [Cin×H]
cudaError_t tc16_gemm_rows(const void* A, const void* B, void* C, int64_t M, int N, int K,
                           cudaStream_t s, int* launches);   // C = A·Bᵀ, all bf16
size_t tc16_dw_partial_floats(int64_t R, int CIN);
cudaError_t tc16_gemm_dw(const void* Y, const void* dZ, float* dW, int64_t R, int CIN, int H,
                         float* part, cudaStream_t s, int* launches);

// ---------------------------------------------------------------- head.cu
struct HeadWork {
  double* colsum_part;  // [nchunks*H]
  double* dv_part;      // [nchunks*nb*H]
  double* loss_part;    // [nchunks*nb]
  float* s;             // [G*H]
  float* v;             // [G*H]
  float* dm;            // [G*H] (already divided by N_g)
  float* dv;            // [G*H]
  double* dvd;          // [G*H]
  double* sd;           // [G*H]
  float* dl;            // [nb*Nt]
  double* loss_g;       // [G] per-graph loss (already / (2 N_g B))
  double* slots;        // [nslots] dalpha3 partials
  float* rs_dz3;        // [nb*Nt] power-of-two row scales of dZ3 (fp32 storage) or null
  // NEXT-4 (c34-c36, c39): nb stacked blocks of Nt rows (even; block 0
  // positive, 1..K corrupted, > K padding), K corruption samples, readout
  // 0 = sig(mean), 1 = mean; loss 0 = BCE (Eq. 6), 1 = InfoNCE.  The default
  // DGI step: nb = 2, K = 1, readout 0, loss 0.
  int32_t nb, K, readout, loss;
};
// Forward head + head backward: writes grads of M (dM) and the loss slot,
// dZ3 into dZ, dalpha3 partials into w.slots.
// Z3 / dZ storage: fp32 or bf16 (bf16 != 0).
// Row-sharded graph: the two per-graph reductions (readout sum, dv + loss) are
// exchanged between shards: chunk sums -> own x buffer, barrier, rank-ordered sum.
struct HeadShard {
  const ShardSync* sync;
  double* x_own[2];          // [H + 1] each, peer-visible
  PeerPtrs x_peers[2];
};
cudaError_t launch_head(const GraphDev& g, int H, const void* Z3, int bf16,
                        const float* params_M, const float* alpha_dev, const StepParams* sp,
                        const HeadWork& w, void* dZ, float* grad_M, float* loss_out, int* nslots,
                        cudaStream_t s, int* launches, const HeadShard* hs = nullptr);
int head_slots(const GraphDev& g, int nb);

// ---------------------------------------------------------------- contrast.cu (NEXT-4)
// out[k*G + g] = pair_off[g]*K + k: the pair index offset of corruption sample
// k of graph g when every graph draws K samples (c34).
cudaError_t launch_pair_off_k(const int64_t* pair_off, int32_t G, int32_t K, int64_t* out,
                              cudaStream_t s, int* launches);
// The stacked layer-1 inputs Xs [nb*Nt x F] fp32: block 0 = X, block k in
// 1..K = the k-th corruption of X (corruption 0: rows X[perms[(k-1)*Nt + i]];
// 1: X ⊙ Bernoulli keep mask, c35), blocks > K = 0.
cudaError_t launch_corrupt(const GraphDev& g, int32_t K, int32_t nb, int32_t corruption,
                           float mask_rate, uint64_t seed, const StepParams* sp,
                           const int64_t* pair_off_k, const int32_t* perms, float* Xs,
                           cudaStream_t s, int* launches);
// SAGE-GCN aggregation (c37): valsR[k] = 1/deg(row), valsC[k] = 1/deg(col) of
// each CSR entry (deg counts the self loop): Â_mean = D^-1 (A + I) and its
// transpose on the same (symmetric) pattern.
cudaError_t launch_sage_vals(const GraphDev& g, float* valsR, float* valsC, cudaStream_t s,
                             int* launches);
// SAGE-mean encoder (c38): the redirected CSR (self entry -> row self_off + i
// of the stacked [U_n; U_s] operand) with forward values (1 self, 1/deg_N(i)
// neighbours), backward values (1, 1/deg_N(j)) and neighbour-only transpose
// values (0, 1/deg_N(j)); vb / vn may be null.
cudaError_t launch_sage_csr(const GraphDev& g, int64_t self_off, int32_t* colS, float* vf,
                            float* vb, float* vn, cudaStream_t s, int* launches);
// SAGE-pool encoder (c40), over the R stacked rows (blocks of Nt rows, each
// aggregating within its block): the element-wise max aggregation of
// ReLU(U + bp) with its argmax, its backward (gradient routed to the argmax,
// masked by ReLU'), z = a + b, and dZ = (d1 + d2) ⊙ PReLU' with dα block
// partials (cdiv(R, 8) slots).  rs (row scales) may be null.
cudaError_t launch_maxagg(const GraphDev& g, const float* U, const float* bp, int64_t R, int H,
                          float* agg, int32_t* idx, float* rs, cudaStream_t s, int* launches);
cudaError_t launch_maxagg_bwd(const GraphDev& g, const float* dagg, const int32_t* idx,
                              const float* U, const float* bp, int64_t R, int H, float* dU,
                              float* rs, cudaStream_t s, int* launches);
cudaError_t launch_add(const float* a, const float* b, float* out, int64_t n, cudaStream_t s,
                       int* launches);
cudaError_t launch_add_prelu_bwd(const float* d1, const float* d2, const float* Z,
                                 const float* alpha, int layer, int64_t R, int H, float* dZ,
                                 float* rs, double* slots, int* nslots, cudaStream_t s,
                                 int* launches);
// out = PReLU_{*slope}(in) row by row (out may be null) + power-of-two row scales (rs may be null).
cudaError_t launch_rowprep(const float* in, int64_t rows, int C, const float* slope, float* out,
                           float* rs, cudaStream_t s, int* launches);
// grad[0] = Σ slots (fixed order, double)
cudaError_t launch_reduce_slots(double* slots, int n, float* grad, cudaStream_t s,
                                int* launches);
// H3 = PReLU(Z3) for the first `rows` rows (encode); Z fp32 or bf16, out fp32
cudaError_t launch_prelu(const void* Z, int bf16, const float* alpha_dev, int layer, float* out,
                         int64_t n, cudaStream_t s, int* launches);
// fp32 copy of a bf16 array (export hooks)
cudaError_t launch_upcast(const void* in, float* out, int64_t n, cudaStream_t s);

// ---------------------------------------------------------------- featurize.cu
// NEXT-1: X [N x F] from op types [N] and shape dims [N x 8] (device buffers);
// dmax: one device u64 of scratch.
cudaError_t launch_featurize(const int32_t* types, const int64_t* dims, int32_t N, int32_t F,
                             unsigned long long* dmax, float* X, cudaStream_t s);

// ---------------------------------------------------------------- placer.cu (NEXT-2)
struct PlacerDims {
  int32_t H;      // op-embedding width (the DGI encoder's H)
  int32_t Hd;     // encoder LSTM size per direction (c22: 256; decoder = 2 Hd)
  int32_t A;      // attention size (c27)
  int32_t De;     // device-embedding size (c25)
  int32_t D;      // devices
};
struct PlacerParams {   // views into the flat parameter vector (c28 layout)
  float *enc_wih[2], *enc_whh[2], *enc_b[2];
  float *wq, *wk, *v;
  float *dec_wih, *dec_whh, *dec_b;
  float *emb, *wo, *bo;
};
struct PlacerWork {     // device scratch sized for N ops and S samples
  float* xp[2];         // [N x 4Hd]
  float* enc;           // [N x 2Hd]
  float* keys;          // [N x A]
  float *seg_h, *seg_c; // [nseg x 2Hd]
  float* hbuf;          // [2 x 2 x Hd]
  float *sh, *sc;       // [2 x S x 2Hd], [S x 2Hd]
  float *q, *ghh, *score, *ctx;   // [S x A], [S x 8Hd], [S x seg], [S x 2Hd]
  unsigned int* bar;    // [2] grid-barrier counters
};
// Training forward: the decoder / encoder activations the backward needs and
// the PPO output gradient (placer.cu, with placer_forward's `train`).
struct PlacerTrain {
  float *sv_hprev, *sv_cprev, *sv_gates, *sv_c, *sv_h, *sv_q, *sv_alpha, *sv_ctx;
  int32_t* sv_prev;
  float *esv_gates, *esv_c;            // encoder [2][N][4Hd], [2][N][Hd]
  const float* logp_old;               // [S x N]
  const float* adv;                    // [S]
  float *dz, *lterm;                   // [S x N x D], [S x N]
  float clip_eps, ent_coef;
};
// Backward pass state (placer_bwd.cu).
struct PlacerBwd {
  int32_t N, S, seg, Hd, Hs, Hin, A, D;
  const float *wo, *v, *keys, *enc;    // weights / forward tensors
  const float *wihT, *whhT, *wqT;      // decoder transposes [Hin x 4Hs], [Hs x 4Hs], [Hs x A]
  const float* ewhhT[2];               // encoder W_hhᵀ [Hd x 4Hd]
  const float *sv_gates, *sv_c, *sv_cprev, *sv_q, *sv_alpha;
  const float* dz;
  float *dg, *dx, *dq, *dvp;           // per (b, i): [SN x 4Hs], [SN x Hin], [SN x A], [SN x A]
  float *dhr, *dcr, *dhr_part;         // [S x Hs]
  double* dal;                         // [S x seg] (double: the softmax backward cancels)
  float* de;                           // [S x seg]
  float *dK, *denc;                    // [N x A], [N x Hs] (accumulated; zeroed first)
  float *dinit_h, *dinit_c;            // [nseg x Hs]
  const float *esv_gates, *esv_c;
  float *edg;                          // [2][N][4Hd]
  float *ehr, *ecr;                    // [2 x Hd]
};
cudaError_t placer_transpose(const float* in, int rows, int cols, float* out, cudaStream_t s);
cudaError_t placer_bwd_decoder(const PlacerBwd& w, cudaStream_t s, int* launches);
cudaError_t placer_bwd_encoder(const PlacerBwd& w, cudaStream_t s, int* launches);
cudaError_t placer_colsum(const float* in, int64_t rows, int cols, float* out, cudaStream_t s);
cudaError_t placer_emb_grad(const float* dx, const int32_t* prev, int64_t SN, int Hs, int Hin,
                            int De, int D1, float* out, cudaStream_t s);
cudaError_t placer_gather_rows(const float* in, const int32_t* order, int64_t rows, int cols,
                               float* out, int scatter_add, cudaStream_t s);
cudaError_t placer_add(float* a, const float* b, int64_t n, cudaStream_t s);
// NEXT-3 environment (c30): out[b] = per-step seconds of placement b (place [S x N]).
cudaError_t launch_step_time(const int32_t* place, int32_t S, int32_t N, const int64_t* dims,
                             const int64_t* indptr, const int32_t* indices, int D,
                             double capacity, double* out, cudaStream_t s);
cudaError_t placer_build_x(const float* ctx, const int32_t* prev, const float* emb, int64_t SN,
                           int Hs, int De, float* X, cudaStream_t s);
cudaError_t placer_gather_cols(const float* in, int64_t ld, int col0, const int32_t* order,
                               int64_t rows, int cols, float* out, cudaStream_t s);
cudaError_t placer_small_tn(const float* dz, const float* h, int64_t R, int D, int Hs, float* out,
                            cudaStream_t s);
int64_t placer_num_params(const PlacerDims& d);
PlacerParams placer_views(const PlacerDims& d, float* base);
cudaError_t placer_init(const PlacerDims& d, float* params, uint64_t seed, cudaStream_t s);
cudaError_t placer_prepare(const PlacerDims& d);
// E [N x H] device; place / logp / ent [S x N] device; forced [S x N] device or null.
cudaError_t placer_forward(const PlacerDims& d, const PlacerParams& w, const PlacerWork& ws,
                           const float* E, int32_t N, int32_t seg, int32_t S, uint64_t sample_seed,
                           const int32_t* forced, int32_t* place, float* logp, float* ent,
                           cudaStream_t s, int* launches, const PlacerTrain* train = nullptr);

// ---------------------------------------------------------------- adam.cu
// grads: [P + 1], the loss at grads[P]; guard_part: adam_guard_doubles() doubles.
int adam_guard_doubles();
cudaError_t launch_adam(float* params, float* m, float* v, const float* grads, int64_t P,
                        double lr, double beta1, double beta2, double eps, double clip_norm,
                        double* guard_part, AdamDev* st, cudaStream_t s, int* launches);

}  // namespace mars
