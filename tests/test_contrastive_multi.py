"""K corruption samples per graph (reading c20):
L_g = 1/(2N) [Σ_i softplus(-l_i) + (1/K) Σ_k Σ_i softplus(l~_i^k)] -- the DGI
objective of Eq. 6 with the expectation over corruptions (Eq. 2,
P:L126-L130) estimated from K samples instead of one.  It equals the mean over
K (graph, sample) pairs of the same graph, which is how the batch API runs it
(`corruption_samples`).  Pinned here against an independent PyTorch float64
autograd formulation with one shared positive branch and K negative branches;
the GPU path is checked against the same formulation."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG
from tests.util import scaled_err


def _torch_dgi_k(g, perms, params, F, H):
    """Shared positive branch, K corrupted branches X[pi_k], autograd."""
    p = torch.tensor(params, dtype=torch.float64, requires_grad=True)
    o = 0
    W1 = p[o:o + F * H].view(F, H); o += F * H
    W2 = p[o:o + H * H].view(H, H); o += H * H
    W3 = p[o:o + H * H].view(H, H); o += H * H
    M = p[o:o + H * H].view(H, H); o += H * H
    al = p[o:o + 3]
    N = g.num_nodes
    A = torch.zeros(N, N, dtype=torch.float64)
    for u in range(N):
        for e in range(g.indptr[u], g.indptr[u + 1]):
            v = int(g.indices[e])
            if u != v:
                A[u, v] = 1.0
                A[v, u] = 1.0
    A = A + torch.eye(N, dtype=torch.float64)
    d = A.sum(1).rsqrt()
    An = d[:, None] * A * d[None, :]
    X = torch.tensor(g.features, dtype=torch.float64)

    def enc(h):
        for l, W in enumerate((W1, W2, W3)):
            h = torch.nn.functional.prelu(An @ h @ W, al[l:l + 1])
        return h
    Hp = enc(X)
    s = torch.sigmoid(Hp.mean(0))
    v = M @ s
    sp = torch.nn.functional.softplus
    pos = sp(-(Hp @ v)).sum()
    neg = sum(sp(enc(X[torch.tensor(pi.astype(np.int64))]) @ v).sum() for pi in perms)
    loss = (pos + neg / len(perms)) / (2 * N)
    loss.backward()
    return float(loss), p.grad.numpy()


@pytest.mark.parametrize("K", [1, 2, 4])
def test_k_samples_equal_k_pairs_oracle(K):
    g = SG.tiny(3)
    F, H, seed, step = 16, 32, 5, 7
    p = oracle.xavier(seed, F, H).astype(np.float64)
    b = oracle.Batch(mars.corruption_samples([g], K))
    perms = b.perms(seed, step, 0)
    loss, grads, *_ = oracle.step_grads(b, H, p, perms)
    N = g.num_nodes
    tl, tg = _torch_dgi_k(g, [perms[k * N:(k + 1) * N] for k in range(K)], p, F, H)
    assert abs(loss - tl) < 1e-13
    assert scaled_err(grads, tg) < 1e-12
    # the K samples are distinct permutations
    if K > 1:
        assert not np.array_equal(perms[:N], perms[N:2 * N])


def test_corruption_samples_layout():
    gs = [SG.tiny(0), SG.tiny(1)]
    out = mars.corruption_samples(gs, 3)
    assert [id(x) for x in out] == [id(gs[0])] * 3 + [id(gs[1])] * 3
    with pytest.raises(ValueError):
        mars.corruption_samples(gs, 0)


@pytest.mark.gpu
@pytest.mark.parametrize("K", [2, 3])
def test_k_samples_gpu(K):
    g = SG.tiny(2)
    F, H, seed, step = 16, 32, 11, 4
    gg = mars.graph_load(mars.corruption_samples([g], K))
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(gg, step, 0, global_batch=K, want_loss=True, want_grads=True, want_perms=True)
    N = g.num_nodes
    perms = out["perms"]
    b = oracle.Batch(mars.corruption_samples([g], K))
    assert np.array_equal(perms, b.perms(seed, step, 0))
    tl, tg = _torch_dgi_k(g, [perms[k * N:(k + 1) * N] for k in range(K)], p0, F, H)
    assert abs(out["loss"] - tl) / abs(tl) <= 1e-5
    assert scaled_err(out["grads"], tg) <= 1e-5
    m.free()
    gg.free()
