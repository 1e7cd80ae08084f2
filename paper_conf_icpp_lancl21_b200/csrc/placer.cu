// NEXT-2: the segment-level sequence-to-sequence placer's forward pass (PAPER.md
// §3.3, Fig. 6; sizes P:L234), readings c22-c28 (DESIGN.md
// §3).  Input: the op embeddings E [N x H] from the DGI-trained encoder (a15);
// output: S sampled placements p [S x N] over D devices with log pi(p) and the
// policy entropy per op (what PPO consumes), or -- with forced
// placements -- log pi / entropy re-evaluated for given placements.
//
// The placer is recurrent: N sequential LSTM steps for the encoder and N for
// the decoder, each a few matrix-vector products (latency-bound, batch S).
// Layout of the work on the GPU:
//   1. encoder input projections XP_dir = E W_ih_dirᵀ (one FFMA GEMM per
//      direction, [N x 4Hd]) -- the only dense contraction of the encoder;
//   2. k_enc: one persistent grid (cooperative launch) runs both directions'
//      recurrences in lock step: CTA c owns 8 hidden units of one direction
//      (32 gate rows of W_hh resident in shared memory), per step it reads
//      h_{t-1} of its direction, computes its gate rows, updates its units'
//      (h, c) and publishes h_t; one grid barrier per step.  The backward
//      direction walks each segment last op first (c23); both directions'
//      states at a segment's end are the decoder's initial state (c24);
//   3. attention keys K = enc W_kᵀ for all ops (FFMA GEMM, [N x A]);
//   4. k_dec: one persistent grid runs the S decoders in lock step, four grid
//      barriers per op: (A) every CTA evaluates the logits of the previous op
//      redundantly and draws its placement (Gumbel-max, c26; identical in all
//      CTAs), then computes its rows of q = W_q s and W_hh s; (B) attention
//      scores, one key per CTA; (C) softmax + context, 4 columns per CTA;
//      (D) decoder gates of 4 units per CTA + their cell update.
// Every reduction has a fixed order (deterministic); fp32 storage and FMA
// accumulation, double for the Gumbel draw / log-sum-exp.
#include <cooperative_groups.h>

#include "common.cuh"
#include "internal.cuh"

namespace mars {
namespace {

constexpr int kThreads = 256;
constexpr int kEncUnits = 8;                  // hidden units per encoder CTA

__device__ __forceinline__ float sigm(float x) { return 1.f / (1.f + expf(-x)); }

// Grid barrier over gridDim.x CTAs (co-resident: cooperative launch).  bar[0]
// counts arrivals; every CTA's epoch advances by one per call.
__device__ __forceinline__ void grid_bar(unsigned int* bar, unsigned int& epoch) {
  __syncthreads();
  epoch += 1;
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(bar, 1u);
    const unsigned int target = epoch * gridDim.x;
    unsigned int v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
    } while (v < target);
  }
  __syncthreads();
}

// ---------------------------------------------------------------- encoder
struct EncArgs {
  const float* xp[2];          // [N x 4Hd] input projections (no bias)
  const float* whh[2];         // [4Hd x Hd]
  const float* b[2];           // [4Hd]
  float* hbuf;                 // [2 (parity)][2 (dir)][Hd]
  float* enc;                  // [N x 2Hd]
  float* seg_h;                // [nseg x 2Hd]
  float* seg_c;                // [nseg x 2Hd]
  float* sv_gates;             // training: [2][N (step)][4Hd] post-activation i, f, g, o
  float* sv_c;                 // training: [2][N (step)][Hd] cell state after the step
  unsigned int* bar;
  int32_t N, s, Hd;
};

// grid = 2 * Hd / kEncUnits CTAs; CTA c: direction c / (Hd / 8), units u0 .. u0 + 7.
__global__ void __launch_bounds__(kThreads) k_enc(EncArgs a) {
  extern __shared__ float sm[];
  const int Hd = a.Hd;
  const int per_dir = Hd / kEncUnits;
  const int dir = blockIdx.x / per_dir;
  const int u0 = (blockIdx.x % per_dir) * kEncUnits;
  constexpr int ROWS = 4 * kEncUnits;                 // gate rows of this CTA
  float* W = sm;                                      // [ROWS][Hd]
  float* h = sm + ROWS * Hd;                          // [Hd]
  float* g = h + Hd;                                  // [ROWS]
  // row r = gate q * 8 + k  <->  W_hh row q * Hd + u0 + k
  for (int e = threadIdx.x; e < ROWS * Hd; e += kThreads) {
    const int r = e / Hd, col = e % Hd;
    const int q = r / kEncUnits, k = r % kEncUnits;
    W[e] = a.whh[dir][(int64_t)(q * Hd + u0 + k) * Hd + col];
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float c_state = 0.f;                                // thread t < 8 owns unit u0 + t
  unsigned int epoch = 0;
  for (int t = 0; t < a.N; ++t) {
    const int j0 = (t / a.s) * a.s;
    const int j1 = min(a.N, j0 + a.s);
    const int op = dir == 0 ? t : j1 - 1 - (t - j0);
    const float* hp = a.hbuf + ((t & 1) * 2 + dir) * Hd;
    for (int e = threadIdx.x; e < Hd; e += kThreads) h[e] = t == 0 ? 0.f : hp[e];
    __syncthreads();
    // 8 warps x 4 rows: lanes split the Hd-long dot product, fixed-order tree
    for (int r = warp; r < ROWS; r += kThreads / 32) {
      float acc = 0.f;
      for (int col = lane; col < Hd; col += 32) acc = fmaf(W[r * Hd + col], h[col], acc);
      acc = warp_sum(acc);
      if (lane == 0) {
        const int q = r / kEncUnits, k = r % kEncUnits;
        const int row = q * Hd + u0 + k;
        g[r] = acc + a.xp[dir][(int64_t)op * 4 * Hd + row] + a.b[dir][row];
      }
    }
    __syncthreads();
    if (threadIdx.x < kEncUnits) {
      const int k = threadIdx.x;
      const float ig = sigm(g[k]), fg = sigm(g[kEncUnits + k]);
      const float gg = tanhf(g[2 * kEncUnits + k]), og = sigm(g[3 * kEncUnits + k]);
      c_state = fg * c_state + ig * gg;
      const float hn = og * tanhf(c_state);
      if (a.sv_gates) {
        float* sg = a.sv_gates + ((int64_t)dir * a.N + t) * 4 * Hd;
        sg[u0 + k] = ig;
        sg[Hd + u0 + k] = fg;
        sg[2 * Hd + u0 + k] = gg;
        sg[3 * Hd + u0 + k] = og;
        a.sv_c[((int64_t)dir * a.N + t) * Hd + u0 + k] = c_state;
      }
      a.hbuf[(((t + 1) & 1) * 2 + dir) * Hd + u0 + k] = hn;
      a.enc[(int64_t)op * 2 * Hd + dir * Hd + u0 + k] = hn;
      if (t == j1 - 1) {                              // segment end: decoder init (c24)
        const int j = t / a.s;
        a.seg_h[(int64_t)j * 2 * Hd + dir * Hd + u0 + k] = hn;
        a.seg_c[(int64_t)j * 2 * Hd + dir * Hd + u0 + k] = c_state;
      }
    }
    grid_bar(a.bar, epoch);
  }
}

// ---------------------------------------------------------------- decoder
struct DecArgs {
  const float* enc;            // [N x 2Hd]
  const float* keys;           // [N x A]  W_k enc
  const float* seg_h;          // [nseg x Hs]
  const float* seg_c;
  const float* wq;             // [A x Hs]
  const float* v;              // [A]
  const float* wih;            // [4Hs x (2Hd + De)]
  const float* whh;            // [4Hs x Hs]
  const float* b;              // [4Hs]
  const float* emb;            // [(D + 1) x De]
  const float* wo;             // [D x Hs]
  const float* bo;             // [D]
  const int32_t* forced;       // [S x N] or null
  float* sh;                   // [2 (parity)][S x Hs] decoder h
  float* sc;                   // [S x Hs] decoder c (owned units, in place)
  float* q;                    // [S x A]
  float* ghh;                  // [S x 4Hs]
  float* score;                // [S x s]
  float* ctx;                  // [S x 2Hd]
  int32_t* place;              // [S x N]
  float* logp;                 // [S x N]
  float* ent;                  // [S x N]
  // training (NEXT-3): activations for the backward, per (sample b, op i)
  float* sv_hprev;             // [S x N x Hs] decoder state entering op i
  float* sv_cprev;             // [S x N x Hs]
  float* sv_gates;             // [S x N x 4Hs] post-activation i, f, g, o
  float* sv_c;                 // [S x N x Hs]
  float* sv_h;                 // [S x N x Hs]
  float* sv_q;                 // [S x N x A]
  float* sv_alpha;             // [S x N x s]
  float* sv_ctx;               // [S x N x Hs]
  int32_t* sv_prev;            // [S x N] input device index of op i (D = start)
  // PPO (c29): with logp_old / adv, dz [S x N x D] = dL/dlogits and the loss
  // terms lterm [S x N] (-min(rho A, clip(rho) A) - c_ent H, before / (S N))
  const float* logp_old;       // [S x N]
  const float* adv;            // [S]
  float* dz;
  float* lterm;
  float clip_eps, ent_coef;
  unsigned int* bar;
  uint64_t seed_key;           // sm64(sample_seed)
  int32_t N, s, S, Hs, A, De, D, nrows_a;   // nrows_a = A + 4 Hs
};

// Logits of op i from h_s [S x Hs] (every CTA, identical), the draw (c26) and,
// by CTA 0, the outputs.  prev[b] receives the placement.
__device__ void finish_op(const DecArgs& a, const float* hs, int i, int32_t* prev, float* lg) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nd = a.S * a.D;
  for (int e = warp; e < nd; e += kThreads / 32) {
    const int b = e / a.D, d = e % a.D;
    float acc = 0.f;
    for (int c = lane; c < a.Hs; c += 32) acc = fmaf(a.wo[(int64_t)d * a.Hs + c], hs[b * a.Hs + c], acc);
    acc = warp_sum(acc);
    if (lane == 0) lg[e] = acc + a.bo[d];
  }
  __syncthreads();
  if (threadIdx.x < a.S) {
    const int b = threadIdx.x;
    const float* z = lg + b * a.D;
    int p = 0;
    if (a.forced) {
      p = a.forced[(int64_t)b * a.N + i];
    } else {
      double best = -INFINITY;
      for (int d = 0; d < a.D; ++d) {
        const uint64_t r = sm64(a.seed_key ^ (((uint64_t)b * a.N + i) * a.D + d));
        const double u = ((double)(r >> 11) + 0.5) * 0x1p-53;
        const double gsc = (double)z[d] - log(-log(u));
        if (gsc > best) { best = gsc; p = d; }
      }
    }
    double m = -INFINITY;
    for (int d = 0; d < a.D; ++d) m = fmax(m, (double)z[d]);
    double se = 0.0;
    for (int d = 0; d < a.D; ++d) se += exp((double)z[d] - m);
    const double lse = m + log(se);
    double en = 0.0;
    for (int d = 0; d < a.D; ++d) {
      const double lp = (double)z[d] - lse;
      en -= exp(lp) * lp;
    }
    prev[b] = p;
    if (blockIdx.x == 0) {
      const int64_t bi = (int64_t)b * a.N + i;
      a.place[bi] = p;
      a.logp[bi] = (float)((double)z[p] - lse);
      a.ent[bi] = (float)en;
      if (a.dz) {
        // L = -(1/n) sum min(rho A, clip(rho, 1-eps, 1+eps) A) - (c/n) sum H, n = S N;
        // dL/dz_d = g (1[d = p] - pi_d) + (c/n) pi_d (log pi_d + H), g = dL/dlog pi(p)
        const double n = (double)a.S * a.N;
        const double A = a.adv[b];
        const double lpn = (double)z[p] - lse;
        const double rho = exp(lpn - (double)a.logp_old[bi]);
        const double rc = fmin(fmax(rho, 1.0 - a.clip_eps), 1.0 + a.clip_eps);
        const double un = rho * A, cl = rc * A;
        const double g = un <= cl ? -rho * A / n : 0.0;   // the min picks the unclipped term
        a.lterm[bi] = (float)(-fmin(un, cl) - (double)a.ent_coef * en);
        for (int d = 0; d < a.D; ++d) {
          const double lp = (double)z[d] - lse, pd = exp(lp);
          a.dz[bi * a.D + d] = (float)(g * ((d == p ? 1.0 : 0.0) - pd) +
                                       (double)a.ent_coef / n * pd * (lp + en));
        }
      }
    }
  }
  __syncthreads();
}

// Persistent decoder; grid = G CTAs (cooperative).  Per op i of segment j:
//   A: [i > 0] finish op i-1;  rows of q = W_q s and W_hh s  (s = seg init at a
//      segment's first op, else h of op i-1)
//   B: score[b][k] = v . tanh(q[b] + K[j0 + k]), key k = CTA index (k < len)
//   C: softmax over k (per CTA, redundant) and ctx columns of this CTA
//   D: gates of this CTA's units from [ctx; emb(prev)], cell update
__global__ void __launch_bounds__(kThreads) k_dec(DecArgs a) {
  extern __shared__ float sm[];
  const int S = a.S, Hs = a.Hs, A = a.A, De = a.De;
  const int Hin = Hs + De;                     // decoder input = [ctx (2Hd = Hs); emb]
  float* hs = sm;                              // [S x Hs]  decoder state s_{t-1}
  float* lg = hs + S * Hs;                     // [S x D]
  float* xin = lg + S * a.D;                   // [S x Hin] decoder input
  float* al = xin + S * Hin;                   // [S x s]   attention weights
  float* gt = al + S * a.s;                    // [S x 16]  gate values of this CTA's units
  int32_t* prev = reinterpret_cast<int32_t*>(gt + S * 16);   // [S]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int G = gridDim.x;
  unsigned int epoch = 0;
  const int units = Hs / G;                    // decoder units per CTA (4 at G = 128)
  for (int i = 0; i <= a.N; ++i) {
    const int j = i / a.s, j0 = j * a.s, len = min(a.s, a.N - j0);
    const bool first = i == j0;
    // ---- A
    {
      const float* hcur = a.sh + ((i & 1) ^ 1) * S * Hs;   // h after op i-1
      for (int e = threadIdx.x; e < S * Hs; e += kThreads) hs[e] = hcur[e];
      __syncthreads();
      if (i > 0) finish_op(a, hs, i - 1, prev, lg);
      if (i == a.N) break;
      if (first) {
        for (int e = threadIdx.x; e < S * Hs; e += kThreads)
          hs[e] = a.seg_h[(int64_t)j * Hs + e % Hs];
        if (threadIdx.x < S) prev[threadIdx.x] = a.D;      // start token
        __syncthreads();
      }
      if (a.sv_hprev && blockIdx.x == 0) {
        for (int e = threadIdx.x; e < S * Hs; e += kThreads)
          a.sv_hprev[((int64_t)(e / Hs) * a.N + i) * Hs + e % Hs] = hs[e];
        if (threadIdx.x < S) a.sv_prev[(int64_t)threadIdx.x * a.N + i] = prev[threadIdx.x];
      }
      // rows r in [0, A): q;  [A, A + 4Hs): W_hh s
      for (int r = blockIdx.x * (kThreads / 32) + warp; r < a.nrows_a; r += G * (kThreads / 32)) {
        const float* w = r < A ? a.wq + (int64_t)r * Hs : a.whh + (int64_t)(r - A) * Hs;
        for (int b = 0; b < S; ++b) {
          float acc = 0.f;
          for (int c = lane; c < Hs; c += 32) acc = fmaf(w[c], hs[b * Hs + c], acc);
          acc = warp_sum(acc);
          if (lane == 0) {
            if (r < A) {
              a.q[b * A + r] = acc;
              if (a.sv_q) a.sv_q[((int64_t)b * a.N + i) * A + r] = acc;
            } else {
              a.ghh[(int64_t)b * 4 * Hs + (r - A)] = acc;
            }
          }
        }
      }
    }
    grid_bar(a.bar, epoch);
    // ---- B: one key per CTA (keys k = blockIdx.x, blockIdx.x + G, ...)
    for (int k = blockIdx.x; k < len; k += G) {
      const float* K = a.keys + (int64_t)(j0 + k) * A;
      for (int b = warp; b < S; b += kThreads / 32) {
        float acc = 0.f;
        for (int c = lane; c < A; c += 32) acc = fmaf(a.v[c], tanhf(a.q[b * A + c] + K[c]), acc);
        acc = warp_sum(acc);
        if (lane == 0) a.score[b * a.s + k] = acc;
      }
    }
    grid_bar(a.bar, epoch);
    // ---- C: softmax (every CTA) + this CTA's context columns
    for (int b = warp; b < S; b += kThreads / 32) {
      float m = -INFINITY;
      for (int k = lane; k < len; k += 32) m = fmaxf(m, a.score[b * a.s + k]);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(kFull, m, o));
      float sum = 0.f;
      for (int k = lane; k < len; k += 32) {
        const float e = expf(a.score[b * a.s + k] - m);
        al[b * a.s + k] = e;
        sum += e;
      }
      sum = warp_sum(sum);
      const float inv = 1.f / sum;
      for (int k = lane; k < len; k += 32) al[b * a.s + k] *= inv;
    }
    __syncthreads();
    if (a.sv_alpha && blockIdx.x == 0)
      for (int e = threadIdx.x; e < S * len; e += kThreads)
        a.sv_alpha[((int64_t)(e / len) * a.N + i) * a.s + e % len] = al[(e / len) * a.s + e % len];
    {
      const int ncols = Hs / G > 0 ? Hs / G : 1;          // ctx columns of this CTA
      for (int e = threadIdx.x; e < S * ncols; e += kThreads) {
        const int b = e / ncols, col = blockIdx.x * ncols + e % ncols;
        if (col >= Hs) continue;
        float acc = 0.f;
        for (int k = 0; k < len; ++k) acc = fmaf(al[b * a.s + k], a.enc[(int64_t)(j0 + k) * Hs + col], acc);
        a.ctx[b * Hs + col] = acc;
        if (a.sv_ctx) a.sv_ctx[((int64_t)b * a.N + i) * Hs + col] = acc;
      }
    }
    grid_bar(a.bar, epoch);
    // ---- D: gates of units [u0, u0 + units) and their cell update
    {
      for (int e = threadIdx.x; e < S * Hin; e += kThreads) {
        const int b = e / Hin, c = e % Hin;
        xin[e] = c < Hs ? a.ctx[b * Hs + c] : a.emb[prev[b] * De + (c - Hs)];
      }
      __syncthreads();
      const int u0 = blockIdx.x * units;
      const int nrow = 4 * units;
      for (int r = warp; r < nrow; r += kThreads / 32) {
        const int q = r / units, k = r % units;
        const int row = q * Hs + u0 + k;
        const float* w = a.wih + (int64_t)row * Hin;
        for (int b = 0; b < S; ++b) {
          float acc = 0.f;
          for (int c = lane; c < Hin; c += 32) acc = fmaf(w[c], xin[b * Hin + c], acc);
          acc = warp_sum(acc);
          if (lane == 0) gt[b * 16 + r] = acc + a.ghh[(int64_t)b * 4 * Hs + row] + a.b[row];
        }
      }
      __syncthreads();
      for (int e = threadIdx.x; e < S * units; e += kThreads) {
        const int b = e / units, k = e % units, u = u0 + k;
        const float* gg = gt + b * 16;
        const float ig = sigm(gg[k]), fg = sigm(gg[units + k]);
        const float g2 = tanhf(gg[2 * units + k]), og = sigm(gg[3 * units + k]);
        const float cp = first ? a.seg_c[(int64_t)j * Hs + u] : a.sc[b * Hs + u];
        const float cn = fg * cp + ig * g2;
        const float hn = og * tanhf(cn);
        a.sc[b * Hs + u] = cn;
        a.sh[(i & 1) * S * Hs + b * Hs + u] = hn;
        if (a.sv_gates) {
          const int64_t bi = (int64_t)b * a.N + i;
          float* sg = a.sv_gates + bi * 4 * Hs;
          sg[u] = ig;
          sg[Hs + u] = fg;
          sg[2 * Hs + u] = g2;
          sg[3 * Hs + u] = og;
          a.sv_cprev[bi * Hs + u] = cp;
          a.sv_c[bi * Hs + u] = cn;
          a.sv_h[bi * Hs + u] = hn;
        }
      }
    }
    grid_bar(a.bar, epoch);
  }
}

// c28 init: w = f32((2u - 1) k), u = (sm64(sm64(seed ^ tag) ^ idx) >> 40) 2^-24.
__global__ void k_placer_init(float* __restrict__ p, int64_t n, uint64_t seed, uint64_t tag,
                              float k) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double u = (double)(sm64(sm64(seed ^ tag) ^ (uint64_t)i) >> 40) * (1.0 / 16777216.0);
  p[i] = __double2float_rn(__dmul_rn(__dsub_rn(__dmul_rn(2.0, u), 1.0), (double)k));
}

}  // namespace

// ---------------------------------------------------------------- host side
int64_t placer_num_params(const PlacerDims& d) {
  const int64_t Hs = 2LL * d.Hd;
  return 2 * (4LL * d.Hd * d.H + 4LL * d.Hd * d.Hd + 4LL * d.Hd) + (int64_t)d.A * Hs +
         (int64_t)d.A * 2 * d.Hd + d.A + 4 * Hs * (2LL * d.Hd + d.De) + 4 * Hs * Hs + 4 * Hs +
         (int64_t)(d.D + 1) * d.De + (int64_t)d.D * Hs + d.D;
}

PlacerParams placer_views(const PlacerDims& d, float* base) {
  PlacerParams v{};
  const int64_t Hs = 2LL * d.Hd;
  float* p = base;
  auto take = [&](int64_t n) { float* r = p; p += n; return r; };
  for (int dir = 0; dir < 2; ++dir) {
    v.enc_wih[dir] = take(4LL * d.Hd * d.H);
    v.enc_whh[dir] = take(4LL * d.Hd * d.Hd);
    v.enc_b[dir] = take(4LL * d.Hd);
  }
  v.wq = take((int64_t)d.A * Hs);
  v.wk = take((int64_t)d.A * 2 * d.Hd);
  v.v = take(d.A);
  v.dec_wih = take(4 * Hs * (2LL * d.Hd + d.De));
  v.dec_whh = take(4 * Hs * Hs);
  v.dec_b = take(4 * Hs);
  v.emb = take((int64_t)(d.D + 1) * d.De);
  v.wo = take((int64_t)d.D * Hs);
  v.bo = take(d.D);
  return v;
}

cudaError_t placer_init(const PlacerDims& d, float* params, uint64_t seed, cudaStream_t s) {
  // tensors in layout order with their fan (c28)
  const int64_t Hs = 2LL * d.Hd;
  struct T { int64_t n; double fan; } ts[] = {
      {4LL * d.Hd * d.H, (double)d.Hd}, {4LL * d.Hd * d.Hd, (double)d.Hd}, {4LL * d.Hd, (double)d.Hd},
      {4LL * d.Hd * d.H, (double)d.Hd}, {4LL * d.Hd * d.Hd, (double)d.Hd}, {4LL * d.Hd, (double)d.Hd},
      {(int64_t)d.A * Hs, (double)Hs}, {(int64_t)d.A * 2 * d.Hd, 2.0 * d.Hd}, {d.A, (double)d.A},
      {4 * Hs * (2LL * d.Hd + d.De), (double)Hs}, {4 * Hs * Hs, (double)Hs}, {4 * Hs, (double)Hs},
      {(int64_t)(d.D + 1) * d.De, 1.0}, {(int64_t)d.D * Hs, (double)Hs}, {d.D, (double)Hs}};
  int64_t off = 0;
  for (int t = 0; t < 15; ++t) {
    const float k = (float)(1.0 / sqrt(ts[t].fan));
    k_placer_init<<<cdiv(ts[t].n, 256), 256, 0, s>>>(params + off, ts[t].n, seed,
                                                     (uint64_t)(101 + t), k);
    off += ts[t].n;
  }
  return cudaGetLastError();
}

size_t placer_enc_smem(const PlacerDims& d) {
  return sizeof(float) * (4 * kEncUnits * (size_t)d.Hd + d.Hd + 4 * kEncUnits);
}
size_t placer_dec_smem(const PlacerDims& d, int S, int seg) {
  const int Hs = 2 * d.Hd;
  return sizeof(float) * ((size_t)S * Hs + (size_t)S * d.D + (size_t)S * (Hs + d.De) +
                          (size_t)S * seg + (size_t)S * 16) + sizeof(int32_t) * S;
}

int placer_dec_grid(const PlacerDims& d) { return 2 * d.Hd / 4; }   // 4 decoder units per CTA

cudaError_t placer_forward(const PlacerDims& d, const PlacerParams& w, const PlacerWork& ws,
                           const float* E, int32_t N, int32_t seg, int32_t S, uint64_t sample_seed,
                           const int32_t* forced, int32_t* place, float* logp, float* ent,
                           cudaStream_t s, int* launches, const PlacerTrain* train) {
  const int Hs = 2 * d.Hd;
  cudaError_t e;
  // 1. encoder input projections (FFMA GEMMs)
  for (int dir = 0; dir < 2; ++dir)
    if ((e = gemm_nt(E, w.enc_wih[dir], ws.xp[dir], N, 4 * d.Hd, d.H, s, launches))) return e;
  // 2. encoder recurrence
  if ((e = cudaMemsetAsync(ws.bar, 0, sizeof(unsigned int) * 2, s))) return e;
  {
    EncArgs a{};
    for (int dir = 0; dir < 2; ++dir) {
      a.xp[dir] = ws.xp[dir];
      a.whh[dir] = w.enc_whh[dir];
      a.b[dir] = w.enc_b[dir];
    }
    a.hbuf = ws.hbuf;
    a.enc = ws.enc;
    a.seg_h = ws.seg_h;
    a.seg_c = ws.seg_c;
    a.bar = ws.bar;
    a.N = N;
    a.s = seg;
    a.Hd = d.Hd;
    if (train) {
      a.sv_gates = train->esv_gates;
      a.sv_c = train->esv_c;
    }
    void* args[] = {&a};
    const int grid = 2 * d.Hd / kEncUnits;
    const size_t smem = placer_enc_smem(d);
    if ((e = cudaLaunchCooperativeKernel((void*)k_enc, grid, kThreads, args, smem, s))) return e;
    count_launch(launches);
  }
  // 3. attention keys
  if ((e = gemm_nt(ws.enc, w.wk, ws.keys, N, d.A, 2 * d.Hd, s, launches))) return e;
  // 4. decoder
  {
    DecArgs a{};
    a.enc = ws.enc;
    a.keys = ws.keys;
    a.seg_h = ws.seg_h;
    a.seg_c = ws.seg_c;
    a.wq = w.wq;
    a.v = w.v;
    a.wih = w.dec_wih;
    a.whh = w.dec_whh;
    a.b = w.dec_b;
    a.emb = w.emb;
    a.wo = w.wo;
    a.bo = w.bo;
    a.forced = forced;
    a.sh = ws.sh;
    a.sc = ws.sc;
    a.q = ws.q;
    a.ghh = ws.ghh;
    a.score = ws.score;
    a.ctx = ws.ctx;
    a.place = place;
    a.logp = logp;
    a.ent = ent;
    a.bar = ws.bar + 1;
    a.seed_key = sm64(sample_seed);
    if (train) {
      a.sv_hprev = train->sv_hprev;
      a.sv_cprev = train->sv_cprev;
      a.sv_gates = train->sv_gates;
      a.sv_c = train->sv_c;
      a.sv_h = train->sv_h;
      a.sv_q = train->sv_q;
      a.sv_alpha = train->sv_alpha;
      a.sv_ctx = train->sv_ctx;
      a.sv_prev = train->sv_prev;
      a.logp_old = train->logp_old;
      a.adv = train->adv;
      a.dz = train->dz;
      a.lterm = train->lterm;
      a.clip_eps = train->clip_eps;
      a.ent_coef = train->ent_coef;
    }
    a.N = N;
    a.s = seg;
    a.S = S;
    a.Hs = Hs;
    a.A = d.A;
    a.De = d.De;
    a.D = d.D;
    a.nrows_a = d.A + 4 * Hs;
    void* args[] = {&a};
    const int grid = placer_dec_grid(d);
    const size_t smem = placer_dec_smem(d, S, seg);
    if (smem > 48 * 1024 &&
        (e = cudaFuncSetAttribute(k_dec, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)))
      return e;
    if ((e = cudaLaunchCooperativeKernel((void*)k_dec, grid, kThreads, args, smem, s))) return e;
    count_launch(launches);
  }
  return cudaGetLastError();
}

cudaError_t placer_prepare(const PlacerDims& d) {
  const size_t smem = placer_enc_smem(d);
  if (smem > 48 * 1024)
    return cudaFuncSetAttribute(k_enc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  return cudaSuccess;
}

}  // namespace mars
