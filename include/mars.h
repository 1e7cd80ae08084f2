/*
 * include/mars.h -- C ABI of libmars.so, the B200 (sm_100a) implementation of
 * the data-parallel hot path of Mars (Lan, Chen & Li, "Accelerated Device
 * Placement Optimization with Contrastive Learning", ICPP'21): one Deep Graph
 * Infomax (DGI) pre-training step of the 3-layer GCN operation encoder over a
 * DNN op graph (§3.1-§3.2, Eqs. 1-6), its backward pass and Adam.
 *
 * Citations "P:Lnnn" are lines of the paper text; "c<k>" are the readings of
 * silent / garbled passages listed in DESIGN.md §3.
 *
 * Conventions (all calls):
 *  - Every call returns mars_status; nothing throws across the ABI.  On a
 *    non-OK status mars_last_error() returns a thread-local message.
 *  - Inputs are BORROWED: host arrays are copied during the call and may be
 *    freed on return.  Output arrays are allocated by the caller (host memory
 *    unless stated).  Handles belong to the caller until mars_free().
 *  - Handles are not thread-safe; distinct handles are independent.
 *  - There is no CPU fallback: with no usable CUDA device every compute call
 *    returns MARS_ECUDA.
 *  - Flat parameter layout (H = hidden_dim, F = in_dim, P = F*H + 3*H*H + 3):
 *      [ W1 (F×H row-major) | W2 (H×H) | W3 (H×H) | M (H×H) | a1 a2 a3 ]
 *    Z_l = Y_l · W_l, so W_l is C_in×H (Eq. 1's Θ); M is the bilinear matrix of
 *    Eq. 5 (the paper's "W"); a_l is the PReLU slope of layer l (c6).
 */
#ifndef MARS_H_
#define MARS_H_

#include <stdint.h>

#if defined(__GNUC__)
#define MARS_API __attribute__((visibility("default")))
#else
#define MARS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  MARS_OK = 0,
  MARS_EINVAL = 1,      /* invalid argument / malformed graph                    */
  MARS_ENOMEM = 2,      /* device or host allocation failed                      */
  MARS_ECUDA = 3,       /* CUDA runtime / driver error, or no device             */
  MARS_ENCCL = 4,       /* NCCL error (multi-GPU data parallelism)               */
  MARS_ENUMERIC = 5,    /* non-finite loss detected                              */
  MARS_ESTATE = 6       /* wrong / freed handle, or call out of order            */
} mars_status;

typedef enum { MARS_FP32 = 0, MARS_BF16 = 1 } mars_precision;

/* Thread-local text for the last non-OK status of this thread ("" if none). */
MARS_API const char* mars_last_error(void);
/* Library version string, e.g. "mars-b200 0.1 sm_100a". */
MARS_API const char* mars_version(void);
/* P = F*H + 3*H*H + 3 (the flat layout above). */
MARS_API int64_t mars_num_params(int32_t in_dim, int32_t hidden_dim);

typedef struct mars_graph mars_graph;   /* device-resident Â_n of 1..G op graphs */
typedef struct mars_dgi mars_dgi;       /* params, Adam state, workspaces, stream */

/* ------------------------------------------------------------------------ */
/* a1-a3: ingest op graphs and build Â_n = D̂^-1/2 (A ∨ Aᵀ + I) D̂^-1/2.        */
/* ------------------------------------------------------------------------ */
/* One op graph in host memory: N ops, directed data-flow edges
 * u->v ("v requires the output of u") as a CSR whose row u lists the
 * consumers v of u, and the per-op feature matrix X (one-hot op type +
 * normalised input/output shapes).  Duplicate edges and self-loops are
 * allowed (collapsed / dropped, c2). */
typedef struct {
  int32_t num_nodes;          /* N >= 1                                        */
  const int64_t* indptr;      /* [N+1], indptr[0] = 0, non-decreasing          */
  const int32_t* indices;     /* [indptr[N]], each in [0, N)                   */
  int32_t feat_dim;           /* F, identical for every graph of a set         */
  const float* features;      /* [N*F] row-major fp32                          */
} mars_graph_desc;

/* Loads G >= 1 graphs as ONE block-diagonal set on `device` and builds, in
 * device kernels, the symmetrised CSR of Â (colind ascending per row, the
 * diagonal included), integer degrees d_i = |row i| (c3), dinv_i = f32(1/√d_i)
 * and vals_ij = f32(1/√(d_i d_j)) computed in double and rounded once (c4).
 * EINVAL: G < 1, N < 1, malformed indptr, index out of range, F mismatch,
 * F not in {16, 32, 64, 128, 256}, or ΣN + 2·ΣE >= 2^31.  Immutable. */
MARS_API mars_status mars_graph_load(const mars_graph_desc* graphs, int32_t num_graphs, int32_t device,
                            mars_graph** out);

/* Shape queries.  Any output pointer may be NULL. */
MARS_API mars_status mars_graph_info(const mars_graph* g, int32_t* num_graphs, int64_t* total_nodes,
                            int64_t* total_nnz, int32_t* feat_dim);
/* Node count and nnz(Â) of graph `graph_idx` of the set. */
MARS_API mars_status mars_graph_size(const mars_graph* g, int32_t graph_idx, int32_t* num_nodes,
                            int64_t* nnz);
/* Test hook (parity P1): copies graph `graph_idx`'s CSR with LOCAL indices to
 * host arrays rowptr[N+1], colind[nnz], deg[N], dinv[N], vals[nnz] (any may be
 * NULL). */
MARS_API mars_status mars_graph_export_csr(const mars_graph* g, int32_t graph_idx, int32_t* rowptr,
                                  int32_t* colind, int32_t* deg, float* dinv, float* vals);

/* NEXT-1 featuriser ("the operation type is encoded as a one-hot
 * vector ... input and output shapes ... normalised"; reading c16): writes the
 * feature matrix X [N x F] (host, row-major fp32) of one op graph from its op
 * types [N] (>= 0; types >= F - 8 share the last type slot, "other") and shape
 * dims [N x 8] (int64: the first input's 4 dims then the op's 4 output dims;
 * <= 0 = absent / unknown).  Slots [0, F-8): one-hot type; [F-8, F): each dim
 * divided by the largest dim of the graph (f32 of the double quotient), 0 for
 * unknown dims.  Runs on `device`; synchronous; inputs borrowed.  EINVAL on
 * N < 1, an unsupported F, or a negative type. */
MARS_API mars_status mars_featurize(const int32_t* types, const int64_t* dims, int32_t num_nodes,
                                    int32_t feat_dim, int32_t device, float* X);

/* ------------------------------------------------------------------------ */
/* The pre-training model: 3 GCN layers with PReLU (Eq. 1),     */
/* sigmoid-mean readout (Eq. 4), bilinear discriminator (Eq. 5), BCE (Eq. 6), */
/* Adam (c13).                                                               */
/* ------------------------------------------------------------------------ */
typedef struct {
  int32_t in_dim;             /* F in {16, 32, 64, 128, 256}                    */
  int32_t hidden_dim;         /* H in {32, 64, 128, 256} (paper: 256)  */
  int32_t num_layers;         /* L: must be 3 (c10)                     */
  int32_t precision;          /* mars_precision: MARS_FP32 (reference, c18)     */
  double lr, beta1, beta2, eps; /* Adam (c13): defaults 1e-3, 0.9, 0.999, 1e-8  */
  double clip_norm;           /* <= 0: no clipping (default)                    */
  uint64_t seed;              /* Xavier init (c14) and corruption keys (c12)    */
  const float* init_params;   /* optional [P] host; NULL => Xavier-uniform(seed) */
  int32_t device;             /* CUDA device ordinal                           */
  int32_t world_size, rank;   /* data parallelism; 1, 0 for a single GPU       */
  const void* nccl_unique_id; /* 128-byte ncclUniqueId: the gradient exchange is an NCCL
                                 allreduce (optional with world_size 1: a 1-rank
                                 communicator).  NULL with world_size > 1: peer-memory
                                 exchange (mars_dp_export / mars_dp_connect below). */
  int32_t encoder;            /* MARS_ENCODER_GCN (Eq. 1, default), _SAGE or _SAGE_POOL */
} mars_dgi_config;

/* The graph encoder (NEXT-4: "[33] uses GraphSAGE as the graph encoder",
 * P:L222; reading c38).  MARS_ENCODER_SAGE: GraphSAGE with the mean
 * aggregator and a root weight, per layer Z = H W_s + (Â_N H) W_n, Â_N =
 * D_N^-1 (A v Aᵀ) over the neighbours without the node itself (an isolated
 * node aggregates 0), PReLU as in Eq. 1, no bias.  Parameters [W1s F×H |
 * W1n F×H | W2s | W2n | W3s | W3n (H×H each) | M H×H | α1 α2 α3]; default init
 * U(-b, b), b = sqrt(6 / (2 C_in + H)) for both halves of a layer (Xavier on
 * the concatenated [2 C_in × H] map), b = sqrt(6 / 2H) for M, tags 1..7 in
 * layout order (c14's generator), α = 0.25.  MARS_FP32 only; not row-sharded;
 * the contrastive variants apply except the SAGE-GCN aggregator; no
 * mars_dgi_encoder_vjp (so no joint PPO update).  The hooks export, per layer,
 * the GEMM input H_{l-1} (X~ stacked for layer 1) as "Y". */
/* MARS_ENCODER_SAGE_POOL: GraphSAGE with the pooling aggregator (the encoder
 * of [33]; reading c40): per layer P = ReLU(h W_p + b_p), agg_i = element-wise
 * max of P over the neighbours of i without i (0 for an isolated node),
 * h' = PReLU(h W_s + agg W_n).  Parameters per layer [W_s C_in×H | W_n H×H |
 * W_p C_in×H | b_p H], then [M H×H | α1 α2 α3]; default init U(-b, b) with
 * b = sqrt(6 / (C_in + 2H)) for W_s and W_n, sqrt(6 / (C_in + H)) for W_p,
 * b_p = 0, sqrt(6 / 2H) for M, tags 1..10 over the matrices in layout order,
 * α = 0.25.  Same restrictions as MARS_ENCODER_SAGE. */
enum { MARS_ENCODER_GCN = 0, MARS_ENCODER_SAGE = 1, MARS_ENCODER_SAGE_POOL = 2 };

/* Fills cfg with the defaults above (F = 64, H = 256, L = 3, FP32, seed 0,
 * device 0, world 1). */
MARS_API void mars_dgi_config_default(mars_dgi_config* cfg);
/* Allocates params (init per c14 unless init_params), Adam state (m = v = 0,
 * t = 0) and a library stream on cfg->device; with world_size > 1 and an
 * nccl_unique_id joins the NCCL communicator (ncclCommInitRank; every rank
 * must call collectively); with world_size > 1 and no id allocates the
 * peer-visible buffers of the peer-memory exchange (connect before stepping). */
MARS_API mars_status mars_dgi_create(const mars_dgi_config* cfg, mars_dgi** out);
/* Parameter count P of the model (mars_num_params for MARS_ENCODER_GCN). */
MARS_API int64_t mars_dgi_num_params(const mars_dgi* m);
/* Rank 0 only: writes a fresh 128-byte ncclUniqueId to out128. */
MARS_API mars_status mars_nccl_get_unique_id(void* out128);
/* Use `cuda_stream` (a cudaStream_t, e.g. torch.cuda.current_stream()) instead
 * of the library stream.  NULL restores the library stream. */
MARS_API mars_status mars_dgi_set_stream(mars_dgi* m, void* cuda_stream);
/* Dense-transform implementation (a6/a12) of the MARS_FP32 path.
 * MARS_GEMM_AUTO (default): tcgen05 tensor cores at fp32 accuracy for every
 *   supported width -- Z = Y·W, dY = dZ·Wᵀ and dW = Yᵀ·dZ as 3xFP16 with
 *   exact power-of-two row / tensor scaling (kind::f16); the narrow widths of
 *   the tiny configuration (H in {32, 64}, C_in in {16, 32}) run on wider
 *   tiles whose missing rows / columns TMA zero-fills.
 * MARS_GEMM_SIMT: always FFMA (A/B comparisons).
 * (The MARS_BF16 path always uses its bf16 kernels.) */
enum { MARS_GEMM_AUTO = 0, MARS_GEMM_SIMT = 1 };
MARS_API mars_status mars_dgi_set_gemm_impl(mars_dgi* m, int32_t impl);
/* Enables (1) / disables (0) CUDA-Graph capture of the step (default 1). */
MARS_API mars_status mars_dgi_set_graph_capture(mars_dgi* m, int32_t enable);

/* NEXT-4 contrastive variants ("there are many choices of the
 * corruption function, readout function and loss function in contrastive
 * learning ... other contrastive learning methods should also work"; the
 * GraphSAGE encoder of [33]).  Readings c34-c37:
 *   num_neg     K >= 1 corruption samples per graph, all scored against ONE
 *               positive branch (c34): L_g = 1/(2N)[Σ softplus(-l_i) + (1/K)
 *               Σ_k Σ softplus(l~_i^k)]; sample k of graph g draws pair index
 *               pair_base + pair_off(g) K + k (k = 0..K-1), so K samples of a
 *               graph reproduce mars_step on K consecutive copies of it (c20)
 *               while computing the positive branch once.  Activations hold
 *               K + 1 blocks of ΣN rows (rounded up to an even count).
 *   corruption  MARS_CORRUPT_PERMUTE: X~ = X[pi] (DGI, Eq. 2, default);
 *               MARS_CORRUPT_MASK: X~ = X ⊙ Bernoulli keep mask, each feature
 *               zeroed with probability mask_rate (counter-based, c35).
 *   readout     MARS_READOUT_SIGMOID_MEAN: s = sig(mean H3) (Eq. 4, default);
 *               MARS_READOUT_MEAN: s = mean H3 (c36).
 *   aggregator  MARS_AGG_GCN: Â = D^-1/2 (A v Aᵀ + I) D^-1/2 (Eq. 1, default);
 *               MARS_AGG_SAGE_GCN: Â = D^-1 (A v Aᵀ + I), the GraphSAGE mean
 *               aggregator over the node and its neighbours (c37); the
 *               backward uses Âᵀ.  mars_encode / mars_dgi_encoder_vjp follow it.
 *   loss        MARS_LOSS_BCE: Eq. 6 (default); MARS_LOSS_INFONCE: per node, its
 *               positive score against its K corrupted counterparts, L = (1/B)
 *               Σ_g (1/N) Σ_i [log Σ_{k=0..K} e^{l_ik} - l_i0] (k = 0 the
 *               positive, c39).
 * The default {1, PERMUTE, 0, SIGMOID_MEAN, GCN, BCE} is the paper's DGI step. */
enum { MARS_CORRUPT_PERMUTE = 0, MARS_CORRUPT_MASK = 1 };
enum { MARS_READOUT_SIGMOID_MEAN = 0, MARS_READOUT_MEAN = 1 };
enum { MARS_AGG_GCN = 0, MARS_AGG_SAGE_GCN = 1 };
enum { MARS_LOSS_BCE = 0, MARS_LOSS_INFONCE = 1 };
typedef struct {
  int32_t num_neg;            /* K in [1, 64]                                      */
  int32_t corruption;         /* MARS_CORRUPT_*                                    */
  float mask_rate;            /* MARS_CORRUPT_MASK: in [0, 1]                      */
  int32_t readout;            /* MARS_READOUT_*                                    */
  int32_t aggregator;         /* MARS_AGG_*                                        */
  int32_t loss;               /* MARS_LOSS_*                                       */
} mars_contrastive;
/* Sets the variant for later steps / encodes (the workspace and captured steps
 * are rebuilt on the next call).  EINVAL on an out-of-range field; ESTATE on a
 * row-shard-attached model (the sharded step runs the default only). */
MARS_API mars_status mars_dgi_set_contrastive(mars_dgi* m, const mars_contrastive* c);
MARS_API mars_status mars_dgi_get_contrastive(const mars_dgi* m, mars_contrastive* c);

/* Optional outputs of a step (host pointers; NULL = not requested). */
typedef struct {
  float* loss;                /* [1]  L averaged over the GLOBAL batch (c15)    */
  float* grads;               /* [P]  global-batch mean gradient BEFORE Adam    */
  int32_t* perms;             /* [K x ΣN] corruption permutations (sample-major),
                                 LOCAL indices; EINVAL with MARS_CORRUPT_MASK  */
} mars_step_out;

/* One DGI step over every graph of `g` (each graph = one (graph, sample) pair,
 * pair index = global_pair_base + graph index, c15):
 *   a4  pi = argsort_(key,i) sm64 keys (c12), X~ = X[pi] (Eq. 2)
 *   a5-a7 Y_l = Â_n·act(T_{l-1}), Z_l = Y_l·W_l, both branches (Eqs. 1, 3)
 *   a8-a10 s = sig(mean H3), scores h_iᵀ M s, BCE loss (Eqs. 4-6)
 *   a11-a12 full backward; a13 NCCL allreduce(sum) when world_size > 1;
 *   a14 Adam.
 * global_batch = B, the number of pairs over all ranks the loss is averaged
 * over.  Asynchronous on the library stream unless an output is requested. */
MARS_API mars_status mars_dgi_step(mars_dgi* m, const mars_graph* g, uint64_t step_index,
                          int64_t global_pair_base, int64_t global_batch, mars_step_out* out);

/* NEXT-1, the pre-training schedule ("pre-train the graph encoder ...
 * for 1000 iterations and save the parameters corresponding to the lowest
 * loss"): n_steps consecutive mars_dgi_step calls (step indices step0 ..
 * step0 + n_steps - 1) on `g`, tracking on the device, without host syncs,
 * the lowest loss and the parameters that produced it (those before that
 * step's Adam update; ties: the earliest step wins, c17).  Outputs (host,
 * optional): losses [n_steps], best_params [P], best_loss, best_step (0-based
 * within the run).  Synchronous.  The model's live parameters are the final
 * ones (after n_steps updates). */
MARS_API mars_status mars_dgi_pretrain(mars_dgi* m, const mars_graph* g, uint64_t step0,
                                       int32_t n_steps, int64_t global_pair_base,
                                       int64_t global_batch, float* losses, float* best_params,
                                       float* best_loss, int64_t* best_step);

/* a15: node embeddings H3 = encoder(X, A) of the positive branch (P:L132,
 * L153) for every node of the set, [ΣN × H] fp32 row-major HOST array.
 * Synchronous.  Overwrites the activations kept for the export hook. */
MARS_API mars_status mars_encode(mars_dgi* m, const mars_graph* g, float* embeddings);

/* Test hook (parity P3): the last step's saved activations of layer
 * `layer` in 1..3, stacked [pos; neg]: Y [2ΣN × C_in], Z [2ΣN × H] (host,
 * fp32; either may be NULL). */
MARS_API mars_status mars_dgi_export_activations(const mars_dgi* m, int32_t layer, float* Y, float* Z);
/* Rows per branch (ΣN, or the shard's own rows) of the activations the last
 * step saved -- the row count of the export hooks' [pos; neg] arrays is twice
 * this; 0 after mars_encode (which overwrites them). */
MARS_API mars_status mars_dgi_saved_rows(const mars_dgi* m, int64_t* rows_per_branch);
/* Test hook (parity P3 at the bench size): with keep != 0 every later step also
 * copies its backward intermediates -- dZ_l (l = 3, 2, 1) and dY_l = dZ_l W_lᵀ
 * (l = 3, 2), which the step overwrites in place -- into separate device
 * buffers (5 × 2ΣN × H elements, allocated on the next step).  A debugging aid:
 * it adds 5 device-to-device copies per step.  keep = 0 releases them. */
MARS_API mars_status mars_dgi_set_keep_backward(mars_dgi* m, int32_t keep);
/* The last step's kept dZ_layer [2ΣN × H] and, for layer in {2, 3}, dY_layer
 * [2ΣN × H] (host fp32; either may be NULL; dY must be NULL for layer 1).
 * MARS_ESTATE unless keep_backward was on for that step. */
MARS_API mars_status mars_dgi_export_backward(const mars_dgi* m, int32_t layer, float* dY, float* dZ);

/* Checkpoint / resume: params, Adam m and v ([P] each) and step count t. */
MARS_API mars_status mars_dgi_get_state(const mars_dgi* m, float* params, float* adam_m, float* adam_v,
                               int64_t* t);
MARS_API mars_status mars_dgi_set_state(mars_dgi* m, const float* params, const float* adam_m,
                               const float* adam_v, int64_t t);

/* Reporting hook: phases of the step schedule. */
typedef enum {
  MARS_PH_PERM = 0,       /* a4 corruption permutation                       */
  MARS_PH_SPMM_FWD = 1,   /* a5 Y_l = Â_n act(T_{l-1}) (3 per step)          */
  MARS_PH_GEMM_FWD = 2,   /* a6 Z_l = Y_l W_l (3 per step)                    */
  MARS_PH_HEAD = 3,       /* a8-a11 readout, scores, loss, head backward, dZ3 */
  MARS_PH_GEMM_DW = 4,    /* a12 dW_l = Y_lᵀ dZ_l (3 per step)                */
  MARS_PH_GEMM_DY = 5,    /* a12 dY_l = dZ_l W_lᵀ (2 per step)                */
  MARS_PH_SPMM_BWD = 6,   /* a12 dZ_{l-1} = (Â_n dY_l) ⊙ PReLU' (2 per step)  */
  MARS_PH_ALLREDUCE = 7,  /* a13 NCCL gradient allreduce                      */
  MARS_PH_ADAM = 8,       /* a14                                              */
  MARS_PH_REDUCE = 9,     /* dalpha partial reductions                        */
  MARS_PH_EXCHANGE = 10   /* row-sharded graph: barriers, head / grad exchange */
} mars_phase;

/* Reporting hook: runs one step exactly like mars_dgi_step (same kernels,
 * same state update) but eagerly, with a CUDA event recorded on the launching
 * stream after every kernel group; writes up to max_phases (phase id, device
 * milliseconds) pairs in schedule order.  Synchronous. */
MARS_API mars_status mars_dgi_profile_step(mars_dgi* m, const mars_graph* g, uint64_t step_index,
                                           int64_t global_pair_base, int64_t global_batch,
                                           int32_t* phase_ids, float* phase_ms,
                                           int32_t max_phases, int32_t* n_phases);

/* Test / micro-benchmark hook for the dense-transform kernels (a6, a12) in
 * isolation, host buffers in and out, on `device`:
 *   op 0 ("rows"): C[M×N] = A[M×K] · Bᵀ with B [N×K]   (forward / dY shape)
 *   op 1 ("dw")  : C[K×N] = Aᵀ · B with A [M×K], B [M×N] (weight gradient;
 *                  M = R rows reduced over, N must be 256)
 * impl = MARS_GEMM_AUTO or MARS_GEMM_SIMT.  Runs `iters` timed launches after
 * one warm-up and writes the mean device milliseconds per launch to *ms. */
MARS_API mars_status mars_debug_gemm(int32_t device, int32_t op, int32_t impl, const float* A,
                                     const float* B, float* C, int64_t M, int32_t N, int32_t K,
                                     int32_t iters, float* ms);

/* ------------------------------------------------------------------------ */
/* Data parallelism over peer memory (a13): the R ranks of  */
/* a job (one process per GPU, world_size R > 1, no nccl_unique_id) map each */
/* other's gradient buffers (CUDA IPC; NVLink / NVSwitch between GPUs, or     */
/* the same device).  After its backward every rank signals a device-side    */
/* barrier, then sums the R partial gradient vectors (+ loss; each already   */
/* scaled by 1/B_global) in rank order in fp64 -- identical on every rank, so */
/* the replicated Adam keeps identical parameters -- and a second barrier     */
/* releases the buffers for the next step.  One kernel reads the peers'      */
/* partials directly: no staging copies, no host involvement, captured in    */
/* the step's CUDA Graph.  A barrier wait longer than ~20 s sets an error     */
/* flag (MARS_ECUDA from mars_dgi_read_step) instead of hanging.             */
/* Protocol: mars_dgi_create (world_size R, rank r, same seed on every rank) */
/* -> mars_dp_export (mars_dp_blob_bytes() bytes) -> all-gather the blobs in */
/* rank order (e.g. torch.distributed) -> mars_dp_connect -> mars_dgi_step on */
/* every rank with the same step index (steps wait on device for the peers). */
/* ------------------------------------------------------------------------ */
MARS_API int64_t mars_dp_blob_bytes(void);
/* Writes this rank's CUDA IPC handles (gradients, barrier flags) into blob. */
MARS_API mars_status mars_dp_export(const mars_dgi* m, void* blob);
/* blobs: the R ranks' blobs concatenated in rank order.  EINVAL if they do
 * not describe the same job (world size, ranks, parameter count). */
MARS_API mars_status mars_dp_connect(mars_dgi* m, const void* blobs);

/* Reloads a graph set in place (a1-a3): graphs[i] must have the node count
 * and feat_dim of the set's graph i (the edges may differ).  The new edges and
 * features go into the existing device buffers -- no allocation unless more
 * entries of Â are stored than before -- after every step already enqueued
 * on the old contents (waited for on the device, not the host).  Models keep
 * the CUDA Graphs they captured for this handle when the number of stored
 * entries and the long-row structure are unchanged: a data loader that
 * alternates two handles re-captures nothing.  Synchronous with respect to
 * the host for the CSR build (it returns when the set is ready).  EINVAL on
 * mismatched sizes or malformed input (the set's contents are then undefined
 * until a successful reload). */
MARS_API mars_status mars_graph_reload(mars_graph* g, const mars_graph_desc* graphs,
                                       int32_t num_graphs);

/* Global pair indices of the graphs of a set (c15): graph i's corruption
 * seed uses pair index global_pair_base + pair_offsets[i] (default i).  With
 * a balanced (e.g. LPT) assignment of graphs to ranks, passing each graph's
 * global index keeps every graph's corruption independent of the rank count.
 * Host array [num_graphs], each >= 0.  Takes effect from the next step. */
MARS_API mars_status mars_graph_set_pair_offsets(mars_graph* g, const int64_t* pair_offsets);

/* ------------------------------------------------------------------------ */
/* NEXT-2: the segment-level sequence-to-sequence placer, forward (PAPER.md  */
/* §3.3, Fig. 6; sizes P:L234; readings c22-c28 in DESIGN.md).  */
/* The op embeddings (mars_encode's output, in op order) are split into      */
/* segments of s ops; a bidirectional LSTM (enc_hidden per direction) encodes */
/* a segment starting from the previous segment's final states; a            */
/* unidirectional LSTM (2 x enc_hidden) with Bahdanau additive attention     */
/* over the segment's encoder outputs decodes one device per op, feeding the */
/* previous op's device embedding back (start token per segment); devices    */
/* are drawn by Gumbel-max from softmax(W_o s_t + b_o) with counter-based    */
/* splitmix64 noise, so a draw depends only on (sample_seed, sample, op).    */
/* ------------------------------------------------------------------------ */
typedef struct mars_placer mars_placer;
typedef struct {
  int32_t in_dim;             /* H: width of the op embeddings (multiple of 16)   */
  int32_t enc_hidden;         /* encoder LSTM size per direction: 64, 128, 256 (c22: 256) */
  int32_t attn_dim;           /* attention size, multiple of 128 (c27: 512)       */
  int32_t dev_embed;          /* device-embedding size in [1, 256] (c25: 64)       */
  int32_t num_devices;        /* D in [2, 64]                                     */
  int32_t segment;            /* s in [1, 1024] (128)                     */
  uint64_t seed;              /* init (c28)                                       */
  const float* init_params;   /* optional [mars_placer_num_params] host           */
  int32_t device;
} mars_placer_config;
/* Defaults: H 256, enc_hidden 256, attn 512, dev_embed 64, D 4, s 128, seed 0. */
MARS_API void mars_placer_config_default(mars_placer_config* cfg);
MARS_API int64_t mars_placer_num_params(const mars_placer_config* cfg);
MARS_API mars_status mars_placer_create(const mars_placer_config* cfg, mars_placer** out);
/* Flat fp32 parameters (layout: DESIGN.md §12): host buffers, synchronous. */
MARS_API mars_status mars_placer_get_params(const mars_placer* p, float* params);
MARS_API mars_status mars_placer_set_params(mars_placer* p, const float* params);
/* The placer forward for num_samples (1..32) placements of one op graph:
 * embeddings [N x in_dim] (host, op order).  forced [num_samples x N] (host,
 * optional): teacher forcing -- the decoder consumes these devices and
 * log pi / entropy are evaluated for them (PPO's re-evaluation of sampled
 * placements).  Outputs (host, each optional) [num_samples x N]: placements
 * (the drawn or forced device per op), logp = log pi(placement) per op,
 * entropy of pi per op.  Synchronous.  EINVAL on bad sizes or a forced device
 * outside [0, D). */
MARS_API mars_status mars_placer_sample(mars_placer* p, const float* embeddings, int32_t num_ops,
                                        int32_t num_samples, uint64_t sample_seed,
                                        const int32_t* forced, int32_t* placements, float* logp,
                                        float* entropy);

/* The encoder's vector-Jacobian product (NEXT-3's joint update): the gradient
 * [P] (flat layout, host; dM = 0) of sum(dE ⊙ H3) with H3 = mars_encode(m, g)
 * at the current parameters, for an external loss's dL/dH3 = dE [ΣN x H] (host).
 * fp32 models; unsharded graphs; synchronous.  Overwrites the step's saved
 * activations. */
MARS_API mars_status mars_dgi_encoder_vjp(mars_dgi* m, const mars_graph* g, const float* dE,
                                          float* grads);

/* NEXT-3 (§3.4; readings c29-c31): the PPO loss
 * of S placements re-evaluated under the current policy (teacher forcing) --
 *   L = -(1/(S N)) sum_{b,i} min(rho A_b, clip(rho, 1 - eps, 1 + eps) A_b)
 *       - ent_coef (1/(S N)) sum_{b,i} H_bi,   rho = exp(log pi(p_bi) - logp_old_bi)
 * -- and its gradient by backpropagation through time: grads [P] (the flat
 * parameter layout, host, optional) and dL/d embeddings [N x in_dim] (host,
 * optional; continues into the GCN encoder for the joint update).
 * placements / logp_old [S x N], adv [S]: host.  in_dim must be 32, 64 or a
 * multiple of 128.  Synchronous. */
MARS_API mars_status mars_placer_ppo_grad(mars_placer* p, const float* embeddings, int32_t num_ops,
                                          int32_t num_samples, const int32_t* placements,
                                          const float* logp_old, const float* adv,
                                          float clip_eps, float ent_coef, float* loss,
                                          float* grads, float* d_embeddings);

/* NEXT-3: PPO training of the placer (c29-c32).  One
 * iteration: sample policies x samples_per_policy placements from the current
 * policy, measure each with the synthetic per-step-time model (c30: per-device
 * compute + received bytes, out of memory -> 100 s), Eq. 7 advantages over the
 * placements in sampling order with the baseline carried across iterations,
 * then `epochs` passes over a seeded shuffle in `minibatches` minibatches: the
 * PPO loss gradient (mars_placer_ppo_grad) clipped to clip_norm and an Adam
 * step (lr 3e-4).  Defaults are the paper's. */
typedef struct mars_ppo mars_ppo;
typedef struct {
  float clip_eps, ent_coef, lr, beta1, beta2, adam_eps, clip_norm, mu;
  int32_t samples_per_policy, policies, minibatches, epochs;
  uint64_t seed;
  float capacity_bytes;       /* device memory of the step-time model (c30)      */
} mars_ppo_config;
MARS_API void mars_ppo_config_default(mars_ppo_config* cfg);
/* encoder: the DGI-pre-trained GCN to train jointly (NULL: placer only). */
MARS_API mars_status mars_ppo_create(mars_placer* placer, mars_dgi* encoder,
                                     const mars_ppo_config* cfg, mars_ppo** out);
/* One iteration on one op graph: embeddings [N x in_dim] (host), shape dims
 * [N x 8] and the directed data-flow CSR (indptr [N+1], indices) for the
 * step-time model.  Optional host outputs: placements [S x N], step_times [S],
 * advantages [S] (S = policies x samples_per_policy), mean minibatch loss. */
MARS_API mars_status mars_ppo_iteration(mars_ppo* o, const float* embeddings, int32_t num_ops,
                                        const int64_t* dims, const int64_t* indptr,
                                        const int32_t* indices, int32_t* placements,
                                        float* step_times, float* advantages, float* mean_loss);
/* The joint update of Mars ("jointly train the two components ... end
 * to end"): the embeddings are the encoder's (mars_encode on the device, one
 * op graph in g) and every minibatch also back-propagates dL/dE through the
 * three GCN layers (the stacked backward of the DGI step with a zero
 * corrupted half) into an Adam step of the encoder (its own Adam state,
 * the PPO lr / clip).  fp32, single-GPU encoders. */
MARS_API mars_status mars_ppo_iteration_joint(mars_ppo* o, const mars_graph* g, const int64_t* dims,
                                              const int64_t* indptr, const int32_t* indices,
                                              int32_t* placements, float* step_times,
                                              float* advantages, float* mean_loss);

/* Copies the most recent step's loss and global-mean gradient (the values
 * Adam consumed) to host memory (either may be NULL).  Synchronous.  For a
 * row-sharded model, ECUDA if a cross-shard barrier timed out. */
MARS_API mars_status mars_dgi_read_step(mars_dgi* m, float* loss, float* grads);

/* Asynchronous loss read-back for a training loop that reads every step's
 * loss without stalling the device between steps (a10's scalar, the value
 * mars_dgi_read_step returns).  mars_dgi_enqueue_loss enqueues, on the
 * library stream after everything enqueued so far (normally the step just
 * launched), a device-to-host copy of the most recent step's loss into a
 * page-locked slot owned by the model, and returns a ticket (0, 1, 2, ...).
 * mars_dgi_wait_loss blocks until that copy has landed and returns the loss;
 * MARS_ENUMERIC if a step up to that one skipped its Adam update (the check
 * mars_dgi_read_step makes).  The last 16 tickets are valid (EINVAL for
 * older ones); enqueueing a 17th waits for the oldest slot's copy. */
MARS_API mars_status mars_dgi_enqueue_loss(mars_dgi* m, int64_t* ticket);
MARS_API mars_status mars_dgi_wait_loss(mars_dgi* m, int64_t ticket, float* loss);

/* ------------------------------------------------------------------------ */
/* Row-sharded single graph: one op graph too large for   */
/* one GPU (config 5: ~1M ops) split into P <= 8 contiguous row blocks, one   */
/* per GPU.  Eq. 1's aggregation Â_n·act(T) on shard p needs the     */
/* rows of T owned by other shards wherever its rows have columns outside the */
/* block (the halo).  Every shard's activation buffers are mapped into every  */
/* other shard's address space (CUDA IPC across processes, or peer access in  */
/* one process) and the SpMM kernels gather halo rows directly by global      */
/* column id over NVLink -- the exchange is fused into the aggregation.       */
/* Device-side barriers order the reads; the readout sum (Eq. 4) and dv/loss  */
/* (Eqs. 5-6) are exchanged after the shard-local reductions; W / alpha       */
/* gradients are summed over shards in rank order, so every shard holds       */
/* identical parameters.  One step of the P shards equals one step of the     */
/* unsharded graph (one (graph, sample) pair, global_batch 1) up to fp32      */
/* reduction order.  Every shard computes the whole corruption permutation   */
/* and keeps the whole X (a few hundred MB at 1M ops).                        */
/* Protocol: every shard (one process per GPU, or all in one process):       */
/*   mars_graph_load_shard -> mars_dgi_create (same seed) -> mars_shard_attach */
/*   -> mars_shard_export (blob, mars_shard_blob_bytes() bytes) -> all-gather */
/*   the P blobs in rank order (e.g. torch.distributed) -> mars_shard_connect */
/*   (or mars_shard_connect_local for models of one process) -> mars_dgi_step */
/*   on every shard with the same step index.  A shard's step waits on device */
/*   for its peers, so steps of the P shards must be enqueued without waiting */
/*   for each other (out = NULL, then mars_dgi_read_step).  The graph must     */
/*   outlive the model.  Needs hidden_dim in {128, 256}, the tcgen05 GEMMs and */
/*   world_size 1 (no data parallelism on top).                               */
/* ------------------------------------------------------------------------ */
/* Loads shard `shard` of `num_shards` (<= 8) of one op graph: builds Â_n of
 * the whole graph on `device` (as mars_graph_load), splits the rows into
 * contiguous blocks balanced by nnz (start_p = first row whose rowptr >=
 * p·nnz/P, each block >= 1 row).  EINVAL as mars_graph_load, or bad shard
 * indices, or fewer nodes than shards. */
MARS_API mars_status mars_graph_load_shard(const mars_graph_desc* graph, int32_t num_shards,
                                           int32_t shard, int32_t device, mars_graph** out);
/* Host-only (no device needed): the row split mars_graph_load_shard uses.
 * rowptr [N+1] of Â (nnz offsets); writes starts[P+1]: start_0 = 0,
 * start_p = max(start_{p-1} + 1, min(N - (P - p), first row r with
 * rowptr[r] >= floor(p·nnz / P))), start_P = N. */
MARS_API mars_status mars_shard_partition(const int32_t* rowptr, int32_t num_nodes,
                                          int32_t num_shards, int32_t* starts);
/* Shard geometry (any pointer may be NULL): shard count, index, the owned
 * global rows [row_begin, row_end), their nnz, and the halo (distinct
 * columns of the owned rows owned by other shards).  Unsharded graphs report
 * 1, 0, [0, N), nnz, 0. */
MARS_API mars_status mars_graph_shard_info(const mars_graph* g, int32_t* num_shards, int32_t* shard,
                                           int32_t* row_begin, int32_t* row_end,
                                           int64_t* local_nnz, int64_t* halo_rows);
/* Binds model m to shard graph g for its lifetime: allocates the fixed
 * workspace and the peer-visible exchange buffers. */
MARS_API mars_status mars_shard_attach(mars_dgi* m, const mars_graph* g);
/* Size of the blob mars_shard_export writes. */
MARS_API int64_t mars_shard_blob_bytes(void);
/* Writes this shard's CUDA IPC handles (+ geometry check) into blob. */
MARS_API mars_status mars_shard_export(const mars_dgi* m, void* blob);
/* blobs: the P shards' blobs concatenated in rank order.  Opens the peers'
 * buffers; after this, mars_dgi_step(m, g, ...) runs the sharded step. */
MARS_API mars_status mars_shard_connect(mars_dgi* m, const void* blobs);
/* Same for P models of this process (models[q] attached to shard q); enables
 * peer access between distinct devices. */
MARS_API mars_status mars_shard_connect_local(mars_dgi* const* models, int32_t num_shards);

/* Kernel launches enqueued by the most recent mars_dgi_step (for reporting). */
MARS_API int64_t mars_dgi_last_launches(const mars_dgi* m);

/* Frees a mars_graph*, mars_dgi*, mars_placer* or mars_ppo* (tag-checked; NULL is a no-op). */
MARS_API void mars_free(void* handle);

#ifdef __cplusplus
}
#endif
#endif /* MARS_H_ */
