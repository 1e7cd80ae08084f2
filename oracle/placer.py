"""CPU oracle of the segment-level sequence-to-sequence placer's forward pass
(NEXT-2; §3.3, Fig. 6; sizes P:L234) -- TEST
INFRASTRUCTURE ONLY, like the rest of oracle/: only tests/ may import it.

Plain numpy in float64, step by step in the paper's order; the readings of
what the paper leaves open are c22-c28 in DESIGN.md §3:

  c22  "Both hidden LSTM layers have a size of 512": the bi-LSTM layer's output
       is 512 = 2 x 256 (forward ++ backward, 256 each); the decoder LSTM has 512.
  c23  "it will take the encoded hidden states of the previous segment as the
       initial hidden state": each direction starts a segment from its own final
       (h, c) of the previous segment (zeros for the first).  The forward
       direction is thus one LSTM over all ops; the backward one runs each
       segment last-op-first, continuing from the previous segment's state.
  c24  decoder initial state of segment j: ([h_f; h_b], [c_f; c_b]) of segment
       j's encoder (forward final at the segment's last op, backward final at
       its first op) -- the usual seq2seq bridge, sizes 256 + 256 = 512.
  c25  Bahdanau "context-based input attention" [2]: at decode step t the query
       is the previous decoder state s_{t-1}; e_k = v . tanh(W_q s_{t-1} +
       W_k enc_k) over the segment's encoder outputs, alpha = softmax(e),
       ctx = sum alpha_k enc_k; the decoder input is [ctx ; E[p_{t-1}]], E a
       learned device embedding (64) with a start token (index D) at the first
       op of every segment.
  c26  logits = W_o s_t + b_o over D devices; p_t ~ softmax(logits) drawn by
       Gumbel-max with counter-based noise: u = ((sm64(sm64(seed) ^ ((b N + i) D
       + d)) >> 11) + 0.5) 2^-53, g = -log(-log u), p = argmax_d(logit_d + g_d)
       (lowest d on ties); log pi(p) and the entropy of softmax(logits) per op.
  c27  attention size A = 512, no biases in the attention.
  c28  LSTM cells as torch.nn.LSTM (gates i, f, g, o; one bias per cell = b_ih
       + b_hh); init U(-k, k) with k = 1/sqrt(fan) (LSTM: its hidden size,
       linear maps: in_features, embedding: 1), from splitmix64 as c14.

Parity pins (tests/test_oracle_placer.py): the LSTM against torch.nn.LSTM
(float64, bidirectional, one segment = the whole sequence), the segment carry
invariants, attention against a hand-evaluated case, the Gumbel-max draw
against softmax probabilities (chi-square), and log pi / entropy against
torch.distributions.Categorical.
"""
from __future__ import annotations

import math

import numpy as np

from . import sm64

M64 = (1 << 64) - 1


def shapes(H: int = 256, Hd: int = 256, A: int = 512, De: int = 64, D: int = 4):
    """Flat parameter layout, in order: name -> shape (c22-c28)."""
    Hs = 2 * Hd
    return [("enc_f.W_ih", (4 * Hd, H)), ("enc_f.W_hh", (4 * Hd, Hd)), ("enc_f.b", (4 * Hd,)),
            ("enc_b.W_ih", (4 * Hd, H)), ("enc_b.W_hh", (4 * Hd, Hd)), ("enc_b.b", (4 * Hd,)),
            ("att.W_q", (A, Hs)), ("att.W_k", (A, 2 * Hd)), ("att.v", (A,)),
            ("dec.W_ih", (4 * Hs, 2 * Hd + De)), ("dec.W_hh", (4 * Hs, Hs)), ("dec.b", (4 * Hs,)),
            ("emb", (D + 1, De)), ("out.W", (D, Hs)), ("out.b", (D,))]


def num_params(**kw) -> int:
    return int(sum(np.prod(s) for _, s in shapes(**kw)))


def unpack(flat, **kw):
    out, o = {}, 0
    flat = np.asarray(flat, np.float64)
    for name, shp in shapes(**kw):
        n = int(np.prod(shp))
        out[name] = flat[o:o + n].reshape(shp)
        o += n
    return out


def _sm64_np(z):
    """splitmix64 mixer on a uint64 array (numpy wraps mod 2^64)."""
    z = (z + np.uint64(0x9E3779B97F4A7C15)).astype(np.uint64)
    z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)).astype(np.uint64)
    z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)).astype(np.uint64)
    return z ^ (z >> np.uint64(31))


def init_params(seed: int, H: int = 256, Hd: int = 256, A: int = 512, De: int = 64, D: int = 4):
    """c28: U(-k, k), u from splitmix64 per tensor (tag = tensor index + 101):
    w = f32((2u - 1) k), u = (sm64(sm64(seed ^ tag) ^ idx) >> 40) 2^-24, k = f32(1/sqrt(fan))."""
    Hs = 2 * Hd
    fan = {"enc_f": Hd, "enc_b": Hd, "dec.W": Hs, "dec.b": Hs, "att.W_q": Hs, "att.W_k": 2 * Hd,
           "att.v": A, "emb": 1, "out": Hs}
    res = []
    for t, (name, shp) in enumerate(shapes(H, Hd, A, De, D)):
        key = next(k for k in fan if name.startswith(k))
        k = np.float32(1.0 / math.sqrt(fan[key]))
        base = np.uint64(sm64((seed ^ (101 + t)) & M64))
        n = int(np.prod(shp))
        z = _sm64_np(base ^ np.arange(n, dtype=np.uint64))
        u = (z >> np.uint64(40)).astype(np.float64) * (1.0 / 16777216.0)
        res.append(((2.0 * u - 1.0) * float(k)).astype(np.float32))
    return np.concatenate(res)


def _sig(x):
    return 1.0 / (1.0 + np.exp(-x))


def lstm_cell(x, h, c, W_ih, W_hh, b):
    """torch.nn.LSTMCell (c28): gates = W_ih x + W_hh h + b, order i, f, g, o."""
    g = W_ih @ x + W_hh @ h + b
    n = h.shape[0]
    i, f, gg, o = _sig(g[:n]), _sig(g[n:2 * n]), np.tanh(g[2 * n:3 * n]), _sig(g[3 * n:])
    c2 = f * c + i * gg
    return o * np.tanh(c2), c2


def encoder(E, P, s: int):
    """The bi-LSTM over segments (c22, c23).  E [N x H].  Returns enc [N x 2Hd] and
    per segment the decoder's initial state (c24)."""
    N = E.shape[0]
    Hd = P["enc_f.W_hh"].shape[1]
    enc = np.zeros((N, 2 * Hd))
    hf, cf = np.zeros(Hd), np.zeros(Hd)
    hb, cb = np.zeros(Hd), np.zeros(Hd)
    init = []
    for j0 in range(0, N, s):
        j1 = min(N, j0 + s)
        for t in range(j0, j1):
            hf, cf = lstm_cell(E[t], hf, cf, P["enc_f.W_ih"], P["enc_f.W_hh"], P["enc_f.b"])
            enc[t, :Hd] = hf
        for t in range(j1 - 1, j0 - 1, -1):
            hb, cb = lstm_cell(E[t], hb, cb, P["enc_b.W_ih"], P["enc_b.W_hh"], P["enc_b.b"])
            enc[t, Hd:] = hb
        init.append((np.concatenate([hf, hb]), np.concatenate([cf, cb])))
    return enc, init


def gumbel(sample_seed: int, b: int, N: int, i: int, D: int):
    """c26: the Gumbel noise of sample b, op i, devices 0..D-1."""
    k = sm64(sample_seed & M64)
    g = np.zeros(D)
    for d in range(D):
        z = sm64(k ^ ((((b * N + i) * D + d)) & M64))
        u = ((z >> 11) + 0.5) * (2.0 ** -53)
        g[d] = -math.log(-math.log(u))
    return g


def attention(s_prev, enc_seg, P, keys=None):
    """c25: Bahdanau additive attention over the segment's encoder outputs:
    e_k = v . tanh(W_q s_prev + W_k enc_k); keys (optional) = the W_k enc_k of
    the segment, [s x A], which do not depend on the decode step."""
    q = P["att.W_q"] @ s_prev
    if keys is None:
        keys = enc_seg @ P["att.W_k"].T
    e = np.tanh(q[None, :] + keys) @ P["att.v"]
    a = np.exp(e - e.max())
    a /= a.sum()
    return a @ enc_seg, a


def decode(E, P, s: int, D: int, num_samples: int, sample_seed: int, forced=None):
    """The placer forward (c22-c26) for num_samples placements.  forced [S x N]
    (optional): teacher forcing -- the decoder consumes these placements and
    log pi / entropy are evaluated for them (PPO's re-evaluation).
    Returns placements [S x N] int32, logp [S x N], entropy [S x N], logits
    [S x N x D]."""
    N = E.shape[0]
    enc, init = encoder(E, P, s)
    S = num_samples
    place = np.zeros((S, N), np.int32)
    logp = np.zeros((S, N))
    ent = np.zeros((S, N))
    logits_all = np.zeros((S, N, D))
    for b in range(S):
        for j, j0 in enumerate(range(0, N, s)):
            j1 = min(N, j0 + s)
            h, c = init[j][0].copy(), init[j][1].copy()
            keys = enc[j0:j1] @ P["att.W_k"].T
            prev = D                                  # start token
            for i in range(j0, j1):
                ctx, _ = attention(h, enc[j0:j1], P, keys)
                x = np.concatenate([ctx, P["emb"][prev]])
                h, c = lstm_cell(x, h, c, P["dec.W_ih"], P["dec.W_hh"], P["dec.b"])
                z = P["out.W"] @ h + P["out.b"]
                logits_all[b, i] = z
                if forced is not None:
                    p = int(forced[b][i])
                else:
                    p = int(np.argmax(z + gumbel(sample_seed, b, N, i, D)))
                m = z.max()
                lse = m + math.log(np.exp(z - m).sum())
                lp = z - lse
                place[b, i] = p
                logp[b, i] = lp[p]
                ent[b, i] = -float(np.sum(np.exp(lp) * lp))
                prev = p
    return place, logp, ent, logits_all
