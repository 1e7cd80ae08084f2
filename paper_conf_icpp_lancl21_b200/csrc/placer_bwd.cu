// NEXT-3: the backward of the placer (§3.3-§3.4; readings c22-c29),
// i.e. the gradient of the PPO loss with respect to every placer parameter and
// to the op embeddings, from the activations the training forward saved
// (placer.cu, sv_*) and dL/dlogits (dz, written by the forward).
//
// Backpropagation through time runs the recurrences in reverse, op by op, as a
// short chain of small kernels per op (stream order is the barrier):
//   decoder (per op i, last to first; segments are independent, c24):
//     kb_cell   dh = W_oᵀ dz_i + dh_rec, dc, dgates (saved), dc_rec     [S x Hs]
//     kb_xt     dx = W_ihᵀ dgates -> dctx, dE_emb;  W_hhᵀ dgates          [S x (Hin + Hs)]
//     kb_dalpha dalpha_k = dctx . enc_k                                     [S x len]
//     kb_datt   de_k = alpha_k (dalpha_k - sum alpha dalpha);  dq, dv terms [S x A]
//     kb_keys   dK_k += sum_b de_bk v (1 - u²);  denc_k += sum_b alpha_bk dctx_b
//     kb_rec    dh_rec = W_hhᵀ dgates + W_qᵀ dq  (segment start: -> d_init)
//   encoder (per forward step t, last to first, both directions together):
//     ke_cell   dh = denc + dh_rec (+ d_init at a segment's end), dgates (saved)
//     ke_rec    dh_rec = W_hhᵀ dgates
// Weight gradients are GEMMs / fixed-order column sums over the saved per-op
// vectors afterwards (mars_api.cu), so every reduction is deterministic.
// Transposed weight copies (W_ihᵀ, W_hhᵀ, W_qᵀ) make every matrix-vector
// product a row-contiguous dot product: one warp per output, lanes over K.
#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

constexpr int kT = 256;

__global__ void k_transpose(const float* __restrict__ in, int rows, int cols, float* __restrict__ out) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= (int64_t)rows * cols) return;
  const int r = (int)(e / cols), c = (int)(e % cols);
  out[(int64_t)c * rows + r] = in[e];
}

// ---- decoder
// grid (cdiv(S * Hs, kT)): thread (b, u)
__global__ void kb_cell(PlacerBwd w, int i, int first, int last) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int Hs = w.Hs;
  if (e >= (int64_t)w.S * Hs) return;
  const int b = (int)(e / Hs), u = (int)(e % Hs);
  const int64_t bi = (int64_t)b * w.N + i;
  float dh = last ? 0.f : w.dhr[e];
  float dcr = last ? 0.f : w.dcr[e];
  for (int d = 0; d < w.D; ++d) dh = fmaf(w.wo[(int64_t)d * Hs + u], w.dz[bi * w.D + d], dh);
  const float* g = w.sv_gates + bi * 4 * Hs;
  const float ig = g[u], fg = g[Hs + u], gg = g[2 * Hs + u], og = g[3 * Hs + u];
  const float c = w.sv_c[bi * Hs + u], tc = tanhf(c);
  const float dc = dcr + dh * og * (1.f - tc * tc);
  float* dg = w.dg + bi * 4 * Hs;
  dg[u] = dc * gg * ig * (1.f - ig);
  dg[Hs + u] = dc * w.sv_cprev[bi * Hs + u] * fg * (1.f - fg);
  dg[2 * Hs + u] = dc * ig * (1.f - gg * gg);
  dg[3 * Hs + u] = dh * tc * og * (1.f - og);
  w.dcr[e] = dc * fg;                       // into the state entering op i
  (void)first;
}

// grid (S * (Hin + Hs)) warps: output o < Hin: dx[b][o] = W_ih[:, o] . dg;
// o >= Hin: dhr_part[b][o - Hin] = W_hh[:, o - Hin] . dg
__global__ void kb_xt(PlacerBwd w, int i) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  const int Hs = w.Hs, Hin = w.Hin, R = 4 * Hs;
  if (warp >= w.S * (Hin + Hs)) return;
  const int b = warp / (Hin + Hs), o = warp % (Hin + Hs);
  const float* dg = w.dg + ((int64_t)b * w.N + i) * R;
  const float* wt = o < Hin ? w.wihT + (int64_t)o * R : w.whhT + (int64_t)(o - Hin) * R;
  double acc = 0.0;                 // dctx feeds the attention backward's cancellation
  for (int r = lane; r < R; r += 32) acc += (double)wt[r] * (double)dg[r];
  acc = warp_sum(acc);
  if (lane == 0) {
    if (o < Hin) w.dx[((int64_t)b * w.N + i) * Hin + o] = (float)acc;
    else w.dhr_part[(int64_t)b * Hs + (o - Hin)] = (float)acc;
  }
}

// grid (S * len) warps: dalpha[b][k] = dctx_b . enc_{j0 + k}
__global__ void kb_dalpha(PlacerBwd w, int i, int j0, int len) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= w.S * len) return;
  const int b = warp / len, k = warp % len;
  const float* dctx = w.dx + ((int64_t)b * w.N + i) * w.Hin;
  const float* en = w.enc + (int64_t)(j0 + k) * w.Hs;
  double acc = 0.0;
  for (int c = lane; c < w.Hs; c += 32) acc += (double)dctx[c] * (double)en[c];
  acc = warp_sum(acc);
  if (lane == 0) w.dal[(int64_t)b * w.seg + k] = acc;   // kept in double: it cancels next
}

// grid (S, cdiv(A, kT)): de_k (every block, redundant), then per a:
// dq[b][a] = sum_k de_k v_a (1 - u_ka²), dvp[b][i][a] = sum_k de_k u_ka,
// u_ka = tanh(q_a + K_{j0+k, a}); block (b, 0) also stores de.
__global__ void kb_datt(PlacerBwd w, int i, int j0, int len) {
  // the softmax backward cancels (dalpha_k - sum alpha dalpha): double for the
  // sums and de, so the query gradient keeps fp32-level relative accuracy
  __shared__ double de[1024];
  __shared__ double red[kT / 32];
  const int b = blockIdx.x;
  const int64_t bi = (int64_t)b * w.N + i;
  const float* al = w.sv_alpha + bi * w.seg;
  double part = 0.0;
  for (int k = threadIdx.x; k < len; k += kT) part += (double)al[k] * w.dal[(int64_t)b * w.seg + k];
  part = warp_sum(part);                        // fixed-order block reduction
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = part;
  __syncthreads();
  double sum = 0.0;
  for (int q = 0; q < kT / 32; ++q) sum += red[q];
  for (int k = threadIdx.x; k < len; k += kT) {
    const double d = (double)al[k] * (w.dal[(int64_t)b * w.seg + k] - sum);
    de[k] = d;
    if (blockIdx.y == 0) w.de[(int64_t)b * w.seg + k] = (float)d;
  }
  __syncthreads();
  const int a = blockIdx.y * kT + threadIdx.x;
  if (a >= w.A) return;
  const float qa = w.sv_q[bi * w.A + a], va = w.v[a];
  double dq = 0.0, dv = 0.0;
  for (int k = 0; k < len; ++k) {
    const float u = tanhf(qa + w.keys[(int64_t)(j0 + k) * w.A + a]);
    dq += de[k] * (double)(va * (1.f - u * u));
    dv += de[k] * (double)u;
  }
  w.dq[bi * w.A + a] = (float)dq;
  w.dvp[bi * w.A + a] = (float)dv;
}

// grid (cdiv(len * (A + Hs), kT)): e < len * A: dK[j0 + k][a] += sum_b de_bk v_a (1 - u²);
// else denc[j0 + k][c] += sum_b alpha_bk dctx_b[c]   (b in order: deterministic)
__global__ void kb_keys(PlacerBwd w, int i, int j0, int len) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nA = (int64_t)len * w.A;
  if (e < nA) {
    const int k = (int)(e / w.A), a = (int)(e % w.A);
    const float kv = w.keys[(int64_t)(j0 + k) * w.A + a];
    float acc = 0.f;
    for (int b = 0; b < w.S; ++b) {
      const float u = tanhf(w.sv_q[((int64_t)b * w.N + i) * w.A + a] + kv);
      acc = fmaf(w.de[(int64_t)b * w.seg + k] * w.v[a], 1.f - u * u, acc);
    }
    w.dK[(int64_t)(j0 + k) * w.A + a] += acc;
    return;
  }
  const int64_t f = e - nA;
  if (f >= (int64_t)len * w.Hs) return;
  const int k = (int)(f / w.Hs), c = (int)(f % w.Hs);
  float acc = 0.f;
  for (int b = 0; b < w.S; ++b) {
    const int64_t bi = (int64_t)b * w.N + i;
    acc = fmaf(w.sv_alpha[bi * w.seg + k], w.dx[bi * w.Hin + c], acc);
  }
  w.denc[(int64_t)(j0 + k) * w.Hs + c] += acc;
}

// grid (S * Hs) warps: dh_rec[b][u] = dhr_part[b][u] + W_q[:, u] . dq_b.  At a
// segment's first op the state entering it is the encoder's (c24): its
// gradient goes to d_init (summed over samples by kb_init) and the recurrence
// restarts at zero for the previous segment's last op.
__global__ void kb_rec(PlacerBwd w, int i) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= w.S * w.Hs) return;
  const int b = warp / w.Hs, u = warp % w.Hs;
  const float* dq = w.dq + ((int64_t)b * w.N + i) * w.A;
  const float* wt = w.wqT + (int64_t)u * w.A;
  float acc = 0.f;
  for (int a = lane; a < w.A; a += 32) acc = fmaf(wt[a], dq[a], acc);
  acc = warp_sum(acc);
  if (lane == 0) w.dhr[(int64_t)b * w.Hs + u] = w.dhr_part[(int64_t)b * w.Hs + u] + acc;
}

// grid (cdiv(Hs, kT)): d_init_{h,c}[j][u] = sum_b dh_rec / dc_rec (fixed order)
__global__ void kb_init(PlacerBwd w, int j) {
  const int u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= w.Hs) return;
  float h = 0.f, c = 0.f;
  for (int b = 0; b < w.S; ++b) {
    h += w.dhr[(int64_t)b * w.Hs + u];
    c += w.dcr[(int64_t)b * w.Hs + u];
  }
  w.dinit_h[(int64_t)j * w.Hs + u] = h;
  w.dinit_c[(int64_t)j * w.Hs + u] = c;
}

// ---- encoder (both directions; step t of the forward order)
// grid (cdiv(2 * Hd, kT)): thread (dir, u)
__global__ void ke_cell(PlacerBwd w, int t, int j, int seg_end) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  const int Hd = w.Hd;
  if (e >= 2 * Hd) return;
  const int dir = e / Hd, u = e % Hd;
  const int j0 = j * w.seg, j1 = min(w.N, j0 + w.seg);
  const int op = dir == 0 ? t : j1 - 1 - (t - j0);
  float dh = w.denc[(int64_t)op * w.Hs + dir * Hd + u] + (t == w.N - 1 ? 0.f : w.ehr[e]);
  float dcr = t == w.N - 1 ? 0.f : w.ecr[e];
  if (seg_end) {                                      // this step's state seeds the decoder
    dh += w.dinit_h[(int64_t)j * w.Hs + dir * Hd + u];
    dcr += w.dinit_c[(int64_t)j * w.Hs + dir * Hd + u];
  }
  const int64_t st = (int64_t)dir * w.N + t;
  const float* g = w.esv_gates + st * 4 * Hd;
  const float ig = g[u], fg = g[Hd + u], gg = g[2 * Hd + u], og = g[3 * Hd + u];
  const float c = w.esv_c[st * Hd + u], tc = tanhf(c);
  const float cprev = t == 0 ? 0.f : w.esv_c[(st - 1) * Hd + u];
  const float dc = dcr + dh * og * (1.f - tc * tc);
  float* dg = w.edg + st * 4 * Hd;
  dg[u] = dc * gg * ig * (1.f - ig);
  dg[Hd + u] = dc * cprev * fg * (1.f - fg);
  dg[2 * Hd + u] = dc * ig * (1.f - gg * gg);
  dg[3 * Hd + u] = dh * tc * og * (1.f - og);
  w.ecr[e] = dc * fg;
}

// grid (2 * Hd) warps: ehr[dir][u] = W_hh_dir[:, u] . dg_dir
__global__ void ke_rec(PlacerBwd w, int t) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  const int Hd = w.Hd;
  if (warp >= 2 * Hd) return;
  const int dir = warp / Hd, u = warp % Hd;
  const float* dg = w.edg + ((int64_t)dir * w.N + t) * 4 * Hd;
  const float* wt = w.ewhhT[dir] + (int64_t)u * 4 * Hd;
  float acc = 0.f;
  for (int r = lane; r < 4 * Hd; r += 32) acc = fmaf(wt[r], dg[r], acc);
  acc = warp_sum(acc);
  if (lane == 0) w.ehr[warp] = acc;
}

// Column sums in fixed order: out[c] = sum_r in[r][c] (r ascending), double.
__global__ void k_colsum_fixed(const float* __restrict__ in, int64_t rows, int cols,
                               float* __restrict__ out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= cols) return;
  double t = 0.0;
  for (int64_t r = 0; r < rows; ++r) t += (double)in[r * cols + c];
  out[c] = (float)t;
}

// demb[d][c] = sum over (b, i) with prev_bi = d of dx[b][i][Hs + c] (order of bi).
__global__ void k_emb_grad(const float* __restrict__ dx, const int32_t* __restrict__ prev,
                           int64_t SN, int Hs, int Hin, int De, int D1, float* __restrict__ out) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= D1 * De) return;
  const int d = e / De, c = e % De;
  double t = 0.0;
  for (int64_t bi = 0; bi < SN; ++bi)
    if (prev[bi] == d) t += (double)dx[bi * Hin + Hs + c];
  out[e] = (float)t;
}

// Row gather with an op order: out[t] = in[op(t)] (encoder backward direction).
__global__ void k_gather_rows(const float* __restrict__ in, const int32_t* __restrict__ order,
                              int64_t rows, int cols, float* __restrict__ out, int scatter_add) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= rows * cols) return;
  const int64_t r = e / cols;
  const int c = (int)(e % cols);
  if (scatter_add) out[(int64_t)order[r] * cols + c] += in[e];
  else out[e] = in[(int64_t)order[r] * cols + c];
}

// X [SN x Hin] = [ctx ; emb[prev]] per (b, i): the decoder LSTM inputs.
__global__ void k_build_x(const float* __restrict__ ctx, const int32_t* __restrict__ prev,
                          const float* __restrict__ emb, int64_t SN, int Hs, int De,
                          float* __restrict__ X) {
  const int Hin = Hs + De;
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= SN * Hin) return;
  const int64_t bi = e / Hin;
  const int c = (int)(e % Hin);
  X[e] = c < Hs ? ctx[bi * Hs + c] : emb[(int64_t)prev[bi] * De + (c - Hs)];
}

// out [rows x cols] = columns [col0, col0 + cols) of in (row stride ld), rows
// in[order[r]] (order null: r).
__global__ void k_gather_cols(const float* __restrict__ in, int64_t ld, int col0,
                              const int32_t* __restrict__ order, int64_t rows, int cols,
                              float* __restrict__ out) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= rows * cols) return;
  const int64_t r = e / cols;
  const int c = (int)(e % cols);
  out[e] = in[(order ? (int64_t)order[r] : r) * ld + col0 + c];
}

// out[d][c] = sum_r dz[r][d] h[r][c] (r ascending, double): dW_o for small D.
__global__ void k_small_tn(const float* __restrict__ dz, const float* __restrict__ h, int64_t R,
                           int D, int Hs, float* __restrict__ out) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= D * Hs) return;
  const int d = e / Hs, c = e % Hs;
  double t = 0.0;
  for (int64_t r = 0; r < R; ++r) t += (double)dz[r * D + d] * (double)h[r * Hs + c];
  out[e] = (float)t;
}

__global__ void k_add(float* __restrict__ a, const float* __restrict__ b, int64_t n) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < n) a[e] += b[e];
}

}  // namespace

cudaError_t placer_transpose(const float* in, int rows, int cols, float* out, cudaStream_t s) {
  k_transpose<<<cdiv((int64_t)rows * cols, kT), kT, 0, s>>>(in, rows, cols, out);
  return cudaGetLastError();
}

cudaError_t placer_bwd_decoder(const PlacerBwd& w, cudaStream_t s, int* launches) {
  const int Hs = w.Hs;
  for (int i = w.N - 1; i >= 0; --i) {
    const int j = i / w.seg, j0 = j * w.seg, j1 = min(w.N, j0 + w.seg), len = j1 - j0;
    const int first = i == j0, last = i == j1 - 1;
    kb_cell<<<cdiv((int64_t)w.S * Hs, kT), kT, 0, s>>>(w, i, first, last);
    kb_xt<<<cdiv((int64_t)w.S * (w.Hin + Hs) * 32, kT), kT, 0, s>>>(w, i);
    kb_dalpha<<<cdiv((int64_t)w.S * len * 32, kT), kT, 0, s>>>(w, i, j0, len);
    kb_datt<<<dim3(w.S, cdiv(w.A, kT)), kT, 0, s>>>(w, i, j0, len);
    kb_keys<<<cdiv((int64_t)len * (w.A + Hs), kT), kT, 0, s>>>(w, i, j0, len);
    kb_rec<<<cdiv((int64_t)w.S * Hs * 32, kT), kT, 0, s>>>(w, i);
    count_launch(launches, 6);
    if (first) {
      kb_init<<<cdiv(Hs, kT), kT, 0, s>>>(w, j);
      count_launch(launches);
    }
  }
  return cudaGetLastError();
}

cudaError_t placer_bwd_encoder(const PlacerBwd& w, cudaStream_t s, int* launches) {
  for (int t = w.N - 1; t >= 0; --t) {
    const int j = t / w.seg, j1 = min(w.N, j * w.seg + w.seg);
    ke_cell<<<cdiv(2 * w.Hd, kT), kT, 0, s>>>(w, t, j, t == j1 - 1);
    ke_rec<<<cdiv((int64_t)2 * w.Hd * 32, kT), kT, 0, s>>>(w, t);
    count_launch(launches, 2);
  }
  return cudaGetLastError();
}

cudaError_t placer_colsum(const float* in, int64_t rows, int cols, float* out, cudaStream_t s) {
  k_colsum_fixed<<<cdiv(cols, 128), 128, 0, s>>>(in, rows, cols, out);
  return cudaGetLastError();
}

cudaError_t placer_emb_grad(const float* dx, const int32_t* prev, int64_t SN, int Hs, int Hin,
                            int De, int D1, float* out, cudaStream_t s) {
  k_emb_grad<<<cdiv((int64_t)D1 * De, 64), 64, 0, s>>>(dx, prev, SN, Hs, Hin, De, D1, out);
  return cudaGetLastError();
}

cudaError_t placer_gather_rows(const float* in, const int32_t* order, int64_t rows, int cols,
                               float* out, int scatter_add, cudaStream_t s) {
  k_gather_rows<<<cdiv(rows * cols, kT), kT, 0, s>>>(in, order, rows, cols, out, scatter_add);
  return cudaGetLastError();
}

cudaError_t placer_build_x(const float* ctx, const int32_t* prev, const float* emb, int64_t SN,
                           int Hs, int De, float* X, cudaStream_t s) {
  k_build_x<<<cdiv(SN * (Hs + De), kT), kT, 0, s>>>(ctx, prev, emb, SN, Hs, De, X);
  return cudaGetLastError();
}

cudaError_t placer_gather_cols(const float* in, int64_t ld, int col0, const int32_t* order,
                               int64_t rows, int cols, float* out, cudaStream_t s) {
  k_gather_cols<<<cdiv(rows * cols, kT), kT, 0, s>>>(in, ld, col0, order, rows, cols, out);
  return cudaGetLastError();
}

cudaError_t placer_small_tn(const float* dz, const float* h, int64_t R, int D, int Hs, float* out,
                            cudaStream_t s) {
  k_small_tn<<<cdiv((int64_t)D * Hs, 128), 128, 0, s>>>(dz, h, R, D, Hs, out);
  return cudaGetLastError();
}

cudaError_t placer_add(float* a, const float* b, int64_t n, cudaStream_t s) {
  k_add<<<cdiv(n, kT), kT, 0, s>>>(a, b, n);
  return cudaGetLastError();
}

}  // namespace mars

namespace mars {
namespace {

// NEXT-3's environment (reading c30): per-step seconds of each placement under a
// synthetic cost model.  One block per placement; thread t sums a fixed
// contiguous range of ops into per-device compute / resident bytes / received
// bytes, then the block combines the threads in order (deterministic, double).
__global__ void __launch_bounds__(256)
k_step_time(const int32_t* __restrict__ place, int32_t N, const int64_t* __restrict__ dims,
            const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices, int D,
            double capacity, double* __restrict__ out) {
  extern __shared__ double sh[];                 // [256][3 D]
  const int b = blockIdx.x, t = threadIdx.x;
  const int32_t* p = place + (int64_t)b * N;
  double* mine = sh + (int64_t)t * 3 * D;
  for (int k = 0; k < 3 * D; ++k) mine[k] = 0.0;
  const int64_t per = (N + 255) / 256;
  const int64_t u0 = t * per, u1 = min((int64_t)N, u0 + per);
  for (int64_t u = u0; u < u1; ++u) {
    double sz = 1.0;
    for (int j = 4; j < 8; ++j) {
      const int64_t dd = dims[u * 8 + j];
      if (dd > 0) sz *= (double)dd;
    }
    const int du = p[u];
    mine[du] += sz * 1e-12;                      // compute
    mine[D + du] += sz * 4.0;                    // resident bytes
    for (int64_t e = indptr[u]; e < indptr[u + 1]; ++e) {
      const int dv = p[indices[e]];
      if (dv != du) mine[2 * D + dv] += sz * 4.0 / 12e9;   // received by the consumer's device
    }
  }
  __syncthreads();
  if (t == 0) {
    double worst = 0.0;
    bool oom = false;
    for (int dv = 0; dv < D; ++dv) {
      double c = 0.0, m = 0.0, r = 0.0;
      for (int q = 0; q < 256; ++q) {
        c += sh[(int64_t)q * 3 * D + dv];
        m += sh[(int64_t)q * 3 * D + D + dv];
        r += sh[(int64_t)q * 3 * D + 2 * D + dv];
      }
      if (m > capacity) oom = true;
      worst = fmax(worst, c + r);
    }
    out[b] = oom ? 100.0 : worst;
  }
}

}  // namespace

cudaError_t launch_step_time(const int32_t* place, int32_t S, int32_t N, const int64_t* dims,
                             const int64_t* indptr, const int32_t* indices, int D,
                             double capacity, double* out, cudaStream_t s) {
  const size_t smem = sizeof(double) * 256 * 3 * D;
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(k_step_time, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return e;
  }
  k_step_time<<<S, 256, smem, s>>>(place, N, dims, indptr, indices, D, capacity, out);
  return cudaGetLastError();
}

}  // namespace mars
