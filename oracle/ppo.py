"""CPU oracle of the joint PPO update (NEXT-3; §3.4, Eq. 7 P:L188-L196,
hyper-parameters P:L237) -- TEST INFRASTRUCTURE ONLY, like the rest of oracle/.

Plain PyTorch CPU ops in float64 with autograd (a library primitive for the
chain rule), step by step in the paper's order.  Readings:

  c29  PPO's probability ratio is taken per op decision: rho_bi = exp(log pi_new
       (p_bi) - log pi_old(p_bi)), every op of placement b sharing its advantage
       A_b; L = -(1/(S N)) sum_b,i min(rho A, clip(rho, 1 - eps, 1 + eps) A)
       - c_ent (1/(S N)) sum_b,i H_bi (eps 0.2, c_ent 0.001).
  c30  The environment is a synthetic per-step-time model of a placed training
       graph (not the paper's TF measurement): op i costs w_i = prod of its
       output dims x 1e-12 s on its device; an edge u -> v across devices costs
       the bytes of u's output (prod of dims x 4) / 12e9 B/s, charged to v's
       device; a device whose resident bytes (sum of its ops' output bytes x 4)
       exceed its capacity is out of memory and the placement costs 100 s
       ("an extremely long per-step time ... such as 100 seconds");
       r = max_d (compute_d + comm_in_d).
  c31  Eq. 7: R_t = -sqrt(r_t); B_t = (1 - mu) R_t + mu B_{t-1}, B_1 = R_1, mu =
       0.99; A_t = R_t - B_t, over the placements in the order they were sampled.

The placer forward is oracle/placer.py's, re-expressed in torch so autograd
gives the gradients of L with respect to every placer parameter and to the
op embeddings (which continue into the GCN encoder's backward).
"""
from __future__ import annotations

import math

import numpy as np
import torch

from . import placer as PL


def step_time(place, dims, indptr, indices, num_devices: int, capacity: float):
    """c30: per-step seconds of one placement.  place [N]; dims [N x 8] int64
    (output dims in [:, 4:8], <= 0 absent); directed CSR (u -> v)."""
    place = np.asarray(place)
    out = np.where(np.asarray(dims)[:, 4:] > 0, np.asarray(dims)[:, 4:], 1).astype(np.float64)
    size = np.prod(out, axis=1)                       # elements of each op's output
    comp = np.zeros(num_devices)
    comm = np.zeros(num_devices)
    mem = np.zeros(num_devices)
    N = place.shape[0]
    for u in range(N):
        comp[place[u]] += size[u] * 1e-12
        mem[place[u]] += size[u] * 4.0
        for e in range(int(indptr[u]), int(indptr[u + 1])):
            v = int(indices[e])
            if place[v] != place[u]:
                comm[place[v]] += size[u] * 4.0 / 12e9
    if np.any(mem > capacity):
        return 100.0
    return float(np.max(comp + comm))


def advantages(times, mu: float = 0.99, B_prev=None):
    """c31 / Eq. 7 over placements in sampling order; returns (A, B_last)."""
    A = np.zeros(len(times))
    B = B_prev
    for t, r in enumerate(times):
        R = -math.sqrt(r)
        B = R if B is None else (1.0 - mu) * R + mu * B
        A[t] = R - B
    return A, B


def _lstm(x, h, c, W_ih, W_hh, b):
    g = W_ih @ x + W_hh @ h + b
    n = h.shape[0]
    i, f, gg, o = torch.sigmoid(g[:n]), torch.sigmoid(g[n:2 * n]), torch.tanh(g[2 * n:3 * n]), \
        torch.sigmoid(g[3 * n:])
    c2 = f * c + i * gg
    return o * torch.tanh(c2), c2


def placer_logp(E, params, dims: dict, s: int, placements):
    """Teacher-forced placer forward in torch (the same steps as
    oracle/placer.decode): returns (log pi [S x N], entropy [S x N]) as
    differentiable tensors; E and params are torch float64 leaves."""
    o, P = 0, {}
    for name, shp in PL.shapes(**dims):
        n = int(np.prod(shp))
        P[name] = params[o:o + n].view(*shp)
        o += n
    N = E.shape[0]
    Hd, D = dims["Hd"], dims["D"]
    enc_rows = [None] * N
    hf = torch.zeros(Hd, dtype=E.dtype); cf = torch.zeros(Hd, dtype=E.dtype)
    hb = torch.zeros(Hd, dtype=E.dtype); cb = torch.zeros(Hd, dtype=E.dtype)
    fwd, bwd, init = [None] * N, [None] * N, []
    for j0 in range(0, N, s):
        j1 = min(N, j0 + s)
        for t in range(j0, j1):
            hf, cf = _lstm(E[t], hf, cf, P["enc_f.W_ih"], P["enc_f.W_hh"], P["enc_f.b"])
            fwd[t] = hf
        for t in range(j1 - 1, j0 - 1, -1):
            hb, cb = _lstm(E[t], hb, cb, P["enc_b.W_ih"], P["enc_b.W_hh"], P["enc_b.b"])
            bwd[t] = hb
        init.append((torch.cat([hf, hb]), torch.cat([cf, cb])))
    enc = torch.stack([torch.cat([fwd[t], bwd[t]]) for t in range(N)])
    S = len(placements)
    logp = [[None] * N for _ in range(S)]
    ent = [[None] * N for _ in range(S)]
    for b in range(S):
        for j, j0 in enumerate(range(0, N, s)):
            j1 = min(N, j0 + s)
            h, c = init[j]
            keys = enc[j0:j1] @ P["att.W_k"].T
            prev = D
            for i in range(j0, j1):
                e = torch.tanh(P["att.W_q"] @ h + keys) @ P["att.v"]
                ctx = torch.softmax(e, 0) @ enc[j0:j1]
                h, c = _lstm(torch.cat([ctx, P["emb"][prev]]), h, c, P["dec.W_ih"], P["dec.W_hh"],
                             P["dec.b"])
                z = P["out.W"] @ h + P["out.b"]
                lp = torch.log_softmax(z, 0)
                p = int(placements[b][i])
                logp[b][i] = lp[p]
                ent[b][i] = -(lp.exp() * lp).sum()
                prev = p
    return (torch.stack([torch.stack(r) for r in logp]), torch.stack([torch.stack(r) for r in ent]))


def ppo_loss(logp_new, logp_old, ent, adv, eps: float = 0.2, c_ent: float = 0.001):
    """c29: the clipped surrogate with per-op ratios and the entropy bonus."""
    adv = torch.as_tensor(np.asarray(adv, np.float64))[:, None]
    rho = torch.exp(logp_new - torch.as_tensor(np.asarray(logp_old, np.float64)))
    surr = torch.minimum(rho * adv, torch.clamp(rho, 1.0 - eps, 1.0 + eps) * adv)
    n = logp_new.numel()
    return -surr.sum() / n - c_ent * ent.sum() / n


def ppo_grads(E, params, dims, s, placements, logp_old, adv, eps=0.2, c_ent=0.001,
              dtype=torch.float64):
    """(loss, dL/dparams, dL/dE).  dtype float64 is the oracle; float32 runs the
    same formulation in single precision -- a second fp32 implementation that
    measures how much fp32 rounding alone moves each gradient block (its
    conditioning), against which the GPU's error is judged (reading c33)."""
    Et = torch.tensor(np.asarray(E, np.float64), dtype=dtype, requires_grad=True)
    pt = torch.tensor(np.asarray(params, np.float64), dtype=dtype, requires_grad=True)
    lp, ent = placer_logp(Et, pt, dims, s, placements)
    L = ppo_loss(lp.double(), logp_old, ent.double(), adv, eps, c_ent)
    L.backward()
    return (float(L.detach()), pt.grad.double().numpy().copy(), Et.grad.double().numpy().copy())
