"""CPU oracle of the NEXT-4 contrastive variants ("there
are many choices of the corruption function, readout function and loss
function ... other contrastive learning methods should also work"; GraphSAGE
in [33]) -- TEST INFRASTRUCTURE ONLY, like the rest of oracle/: only
tests/ may import it.

Plain PyTorch CPU ops in float64 with autograd (the chain rule as a library
primitive, as in oracle/ppo.py), one graph at a time, step by step in the
paper's order -- Eq. 1 encoder, Eq. 2 corruption, Eq. 4 readout, Eq. 5
discriminator, Eq. 6 loss -- with the variant's choices.  Readings
(DESIGN.md §3):

  c34  K corruption samples share one positive branch: L_g = 1/(2N)[Σ_i
       softplus(-l_i) + (1/K) Σ_k Σ_i softplus(l~_i^k)], L = (1/B) Σ_g L_g;
       sample k of graph g uses pair index pair_base + pair_off[g] K + k.
  c35  feature masking: X~ = X ⊙ keep, keep[i][f] iff u >= rate with u =
       (sm64(sm64(key ^ 0x6D61736B) ^ (i F + f)) >> 40) 2^-24 and key =
       sm64(sm64(sm64(seed) ^ step) ^ pair) (the c12 sample key).
  c36  mean readout: s = (1/N) Σ_i h_i (no sigmoid).
  c37  SAGE-GCN aggregation: Â = D^-1 (A v Aᵀ + I), D the row sums (the
       GraphSAGE mean aggregator over the node and its neighbours).
  c38  SAGE-mean encoder (GraphSAGE, mean aggregator with a root weight, no
       bias): h' = PReLU(h W_s + (Â_N h) W_n), Â_N = D_N^-1 (A v Aᵀ) without
       self loops (an isolated node aggregates 0); parameters [W1s | W1n | W2s |
       W2n | W3s | W3n | M | α], init U(-b, b) with b = f32(sqrt(6 / (2 C_in +
       H))) per layer (sqrt(6 / 2H) for M), tags 1..7 in layout order (c14's
       generator), α = 0.25.
  c40  SAGE-pool encoder (GraphSAGE's pooling aggregator, the encoder of
       [33]): P = ReLU(h W_p + b_p); agg_i = max_{j in N(i)} P_j element-wise
       over the neighbours without the node (0 for an isolated node);
       h' = PReLU(h W_s + agg W_n).  Parameters per layer [W_s C x H | W_n H x H
       | W_p C x H | b_p H], then M and α; init U(-b, b) with b =
       f32(sqrt(6 / (C + 2H))) for W_s and W_n, f32(sqrt(6 / (C + H))) for W_p,
       b_p = 0, f32(sqrt(6 / 2H)) for M, tags 1..10 over the matrices in layout
       order (c14's generator), α = 0.25.
  c39  InfoNCE loss: per node i, softmax over its K + 1 logits (k = 0 the
       positive, k = 1..K its corrupted counterparts, same node index);
       L = (1/B) Σ_g (1/N_g) Σ_i [log Σ_k e^{l_ik} - l_i0].

The corruption permutations are oracle.perm's (the C oracle, c12).  Parity
pins: tests/test_oracle_variants.py (the default variant against the C
oracle's step; K samples against the C oracle on K copies; masking rates 0 and
1 in closed form; the readouts and aggregators against the C oracle's encoder
plus a hand-written numpy head, brute-force loops, and finite differences).
"""
from __future__ import annotations

import numpy as np
import torch

from . import perm as _perm

M64 = (1 << 64) - 1


def _sm64(z: int) -> int:
    z = (z + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def _sm64_np(z):
    z = (z + np.uint64(0x9E3779B97F4A7C15)).astype(np.uint64)
    z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)).astype(np.uint64)
    z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)).astype(np.uint64)
    return z ^ (z >> np.uint64(31))


def mask_keep(seed: int, step: int, pair: int, N: int, F: int, rate: float) -> np.ndarray:
    """c35: the [N x F] keep mask of one (graph, sample) pair.  rate is taken as
    the float32 the ABI stores, compared in double."""
    key = _sm64(_sm64(_sm64(seed & M64) ^ (step & M64)) ^ (pair & M64))
    km = np.uint64(_sm64(key ^ 0x6D61736B))
    e = np.arange(N * F, dtype=np.uint64)
    u = (_sm64_np(km ^ e) >> np.uint64(40)).astype(np.float64) * (1.0 / 16777216.0)
    return (u >= float(np.float32(rate))).reshape(N, F)


def adjacency(g) -> np.ndarray:
    """Â = A v Aᵀ + I, binary (Eq. 1; readings c1-c3)."""
    N = g.num_nodes
    A = np.zeros((N, N))
    for u in range(N):
        for e in range(int(g.indptr[u]), int(g.indptr[u + 1])):
            v = int(g.indices[e])
            A[u, v] = A[v, u] = 1.0
    np.fill_diagonal(A, 1.0)
    return A


def normalise(A: np.ndarray, aggregator: str) -> np.ndarray:
    d = A.sum(1)
    if aggregator == "gcn":          # D^-1/2 Â D^-1/2 (Eq. 1)
        r = 1.0 / np.sqrt(d)
        return r[:, None] * A * r[None, :]
    if aggregator == "sage_gcn":     # D^-1 Â (c37)
        return A / d[:, None]
    raise ValueError(aggregator)


def num_params(F: int, H: int, encoder: str = "gcn") -> int:
    if encoder == "sage_pool":
        return 2 * F * H + 8 * H * H + 3 * H + 3
    return F * H + 3 * H * H + 3 + (F * H + 2 * H * H if encoder == "sage" else 0)


def _xavier_block(seed: int, tag: int, n: int, fan: float):
    b = float(np.float32(np.sqrt(6.0 / fan)))
    base = np.uint64(_sm64((seed ^ tag) & M64))
    z = _sm64_np(base ^ np.arange(n, dtype=np.uint64))
    u = (z >> np.uint64(40)).astype(np.float64) * (1.0 / 16777216.0)
    return ((2.0 * u - 1.0) * b).astype(np.float32)


def sage_pool_init(seed: int, F: int, H: int) -> np.ndarray:
    """c40: per layer W_s, W_n, W_p (tags 3l+1..3l+3), b_p = 0; M tag 10; α."""
    out = []
    for l in range(3):
        C = F if l == 0 else H
        out.append(_xavier_block(seed, 3 * l + 1, C * H, C + 2 * H))
        out.append(_xavier_block(seed, 3 * l + 2, H * H, C + 2 * H))
        out.append(_xavier_block(seed, 3 * l + 3, C * H, C + H))
        out.append(np.zeros(H, np.float32))
    out.append(_xavier_block(seed, 10, H * H, 2 * H))
    out.append(np.full(3, 0.25, np.float32))
    return np.concatenate(out)


def unpack_sage_pool(p, F: int, H: int):
    """[(W_s, W_n, W_p, b_p) per layer], M, alpha (c40 layout)."""
    o, layers = 0, []
    for l in range(3):
        C = F if l == 0 else H
        Ws = p[o:o + C * H].view(C, H); o += C * H
        Wn = p[o:o + H * H].view(H, H); o += H * H
        Wp = p[o:o + C * H].view(C, H); o += C * H
        bp = p[o:o + H]; o += H
        layers.append((Ws, Wn, Wp, bp))
    M = p[o:o + H * H].view(H, H); o += H * H
    return layers, M, p[o:o + 3]


def neighbour_lists(g):
    """N(i) of A v Aᵀ without self loops, ascending."""
    A = adjacency(g)
    np.fill_diagonal(A, 0.0)
    return [np.nonzero(A[i])[0] for i in range(g.num_nodes)]


def encoder_sage_pool(nbrs, X, layers, alpha):
    """c40 x 3 (torch, autograd through the element-wise max)."""
    h = X
    for l in range(3):
        Ws, Wn, Wp, bp = layers[l]
        P = torch.relu(h @ Wp + bp)
        zero = torch.zeros(P.shape[1], dtype=P.dtype)
        agg = torch.stack([P[torch.from_numpy(nb)].max(0).values if len(nb) else zero
                           for nb in nbrs])
        h = torch.nn.functional.prelu(h @ Ws + agg @ Wn, alpha[l:l + 1])
    return h


def sage_init(seed: int, F: int, H: int) -> np.ndarray:
    """c38: W1s W1n W2s W2n W3s W3n M with c14's generator, tags 1..7."""
    out = []
    for t in range(1, 8):
        fin = F if t <= 2 else H
        fan = 2 * H if t == 7 else 2 * fin + H
        b = float(np.float32(np.sqrt(6.0 / fan)))
        base = np.uint64(_sm64((seed ^ t) & M64))
        z = _sm64_np(base ^ np.arange(fin * H, dtype=np.uint64))
        u = (z >> np.uint64(40)).astype(np.float64) * (1.0 / 16777216.0)
        out.append(((2.0 * u - 1.0) * b).astype(np.float32))
    out.append(np.full(3, 0.25, np.float32))
    return np.concatenate(out)


def unpack_sage(p, F: int, H: int):
    """((W1s, W1n), (W2s, W2n), (W3s, W3n)), M, alpha (c38 layout)."""
    o, mats = 0, []
    for fin in (F, F, H, H, H, H, H):
        mats.append(p[o:o + fin * H].view(fin, H))
        o += fin * H
    return ((mats[0], mats[1]), (mats[2], mats[3]), (mats[4], mats[5])), mats[6], p[o:o + 3]


def neighbour_mean(g) -> np.ndarray:
    """Â_N = D_N^-1 (A v Aᵀ), no self loops; rows of isolated nodes are 0 (c38)."""
    A = adjacency(g)
    np.fill_diagonal(A, 0.0)
    d = A.sum(1)
    return A / np.where(d > 0, d, 1.0)[:, None]


def encoder_sage(AN, X, Wp, alpha):
    """c38 x 3: h' = PReLU(h W_s + (Â_N h) W_n)."""
    h = X
    for l in range(3):
        Ws, Wn = Wp[l]
        h = torch.nn.functional.prelu(h @ Ws + AN @ (h @ Wn), alpha[l:l + 1])
    return h


def unpack(p, F: int, H: int):
    o = 0
    out = []
    for n, shp in ((F * H, (F, H)), (H * H, (H, H)), (H * H, (H, H)), (H * H, (H, H))):
        out.append(p[o:o + n].view(*shp))
        o += n
    out.append(p[o:o + 3])
    return out          # W1, W2, W3, M, alpha


def encoder(An, X, W, alpha):
    """Eq. 1 x 3 with PReLU (c10)."""
    h = X
    for l in range(3):
        h = torch.nn.functional.prelu(An @ (h @ W[l]), alpha[l:l + 1])
    return h


_encoder_gcn = encoder        # (step_grads' `encoder` argument shadows the name)


def corrupted(g, X, seed, step, pair, corruption, mask_rate):
    N, F = X.shape
    if corruption == "permute":      # Eq. 2, c12
        pi = _perm(seed, step, pair, N).astype(np.int64)
        return X[torch.from_numpy(pi)]
    if corruption == "mask":         # c35
        return X * torch.from_numpy(mask_keep(seed, step, pair, N, F, mask_rate)).to(X.dtype)
    raise ValueError(corruption)


def step_grads(graphs, params, F: int, H: int, seed: int, step: int, pair_base: int = 0,
               B: float | None = None, num_neg: int = 1, corruption: str = "permute",
               mask_rate: float = 0.0, readout: str = "sigmoid_mean", aggregator: str = "gcn",
               pair_off=None, sparse: bool = False, encoder: str = "gcn", loss: str = "bce",
               dtype=torch.float64):
    """(loss, dL/dparams) of one step over a graph set (c34-c38).  B = number of
    graphs the loss is averaged over (default: len(graphs)); pair_off[g]
    defaults to g.  sparse: Â as a torch sparse matrix (larger graphs).
    encoder "sage": the c38 encoder (aggregator unused).  dtype float64 is the
    oracle; float32 runs the same formulation in single precision -- a second
    fp32 implementation that measures how much fp32 rounding alone moves the
    result (the conditioning), as oracle/ppo.py does (reading c33)."""
    p = torch.tensor(np.asarray(params, np.float64), dtype=dtype, requires_grad=True)
    if encoder == "sage":
        Wp, M, al = unpack_sage(p, F, H)
        enc = lambda A_, X_: encoder_sage(A_, X_, Wp, al)   # noqa: E731
    elif encoder == "sage_pool":
        layers, M, al = unpack_sage_pool(p, F, H)
        enc = lambda A_, X_: encoder_sage_pool(A_, X_, layers, al)   # noqa: E731
    else:
        W1, W2, W3, M, al = unpack(p, F, H)
        enc = lambda A_, X_: _encoder_gcn(A_, X_, (W1, W2, W3), al)   # noqa: E731
    B = float(len(graphs) if B is None else B)
    K = int(num_neg)
    sp = torch.nn.functional.softplus
    total = torch.zeros((), dtype=dtype)
    for gi, g in enumerate(graphs):
        if encoder == "sage_pool":
            An = neighbour_lists(g)                      # the encoder takes neighbour lists
        else:
            An_np = neighbour_mean(g) if encoder == "sage" else normalise(adjacency(g), aggregator)
            An = torch.from_numpy(An_np).to(dtype)
        if sparse and encoder != "sage_pool":
            An = An.to_sparse()
        X = torch.tensor(np.asarray(g.features, np.float64), dtype=dtype)
        N = g.num_nodes
        Hp = enc(An, X)
        m = Hp.mean(0)                                   # Eq. 4
        s = torch.sigmoid(m) if readout == "sigmoid_mean" else m
        if readout not in ("sigmoid_mean", "mean"):
            raise ValueError(readout)
        v = M @ s                                        # Eq. 5: l_i = h_iᵀ M s
        po = gi if pair_off is None else int(pair_off[gi])
        if loss == "infonce":                            # c39
            logits = [Hp @ v]
            for k in range(K):
                Xt = corrupted(g, X, seed, step, pair_base + po * K + k, corruption, mask_rate)
                logits.append(enc(An, Xt) @ v)
            Lg = torch.stack(logits)                     # [K + 1, N]
            total = total + (torch.logsumexp(Lg, 0) - Lg[0]).sum() / N / B
            continue
        if loss != "bce":
            raise ValueError(loss)
        pos = sp(-(Hp @ v)).sum()
        neg = torch.zeros((), dtype=torch.float64)
        for k in range(K):
            Xt = corrupted(g, X, seed, step, pair_base + po * K + k, corruption, mask_rate)
            neg = neg + sp(enc(An, Xt) @ v).sum()
        total = total + (pos + neg / K) / (2.0 * N) / B  # Eq. 6 with c34
    total.backward()
    return float(total.detach()), p.grad.double().numpy().copy()


def encode(graphs, params, F: int, H: int, aggregator: str = "gcn", encoder_: str = "gcn"):
    """a15 under the variant's aggregator / encoder: H3 of every node, stacked."""
    p = torch.tensor(np.asarray(params, np.float64))
    out = []
    for g in graphs:
        X = torch.tensor(np.asarray(g.features, np.float64))
        if encoder_ == "sage":
            Wp, _, al = unpack_sage(p, F, H)
            out.append(encoder_sage(torch.from_numpy(neighbour_mean(g)), X, Wp, al))
        elif encoder_ == "sage_pool":
            layers, _, al = unpack_sage_pool(p, F, H)
            out.append(encoder_sage_pool(neighbour_lists(g), X, layers, al))
        else:
            W1, W2, W3, _, al = unpack(p, F, H)
            An = torch.from_numpy(normalise(adjacency(g), aggregator))
            out.append(encoder(An, X, (W1, W2, W3), al))
    return torch.cat(out).numpy()
