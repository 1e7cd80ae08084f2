"""NEXT-3 on the GPU: the PPO loss of teacher-forced placements and its
gradient through the placer (mars_placer_ppo_grad: BPTT through the attention
decoder and the segment-carried bi-LSTM encoder) against the torch fp64
autograd oracle (oracle/ppo.py; §3.4, readings c29-c31): loss,
every parameter block and dL/d embeddings at the scaled max-norm 1e-5."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_lancl21_b200 as mars
from oracle import placer as PL
from oracle import ppo
from tests.util import scaled_err

pytestmark = pytest.mark.gpu


def _blocks(g, dims):
    out, o = {}, 0
    for name, shp in PL.shapes(**dims):
        n = int(np.prod(shp))
        out[name] = g[o:o + n]
        o += n
    return out


@pytest.mark.parametrize("N,seg,S,H", [(20, 8, 2, 32), (45, 16, 3, 64)])
def test_ppo_grad_matches_oracle(N, seg, S, H):
    kw = dict(enc_hidden=64, attn_dim=128, dev_embed=8, num_devices=3, segment=seg)
    dims = dict(H=H, Hd=64, A=128, De=8, D=3)
    p = mars.placer_create(seed=4, in_dim=H, **kw)
    rng = np.random.default_rng(N)
    E = (0.5 * rng.standard_normal((N, H))).astype(np.float32)
    place, logp, _ = p.sample(E, S, 9)
    params = p.get_params()
    # a policy that moved: perturbed params make rho != 1 (some clipped)
    params1 = (params + 0.02 * rng.standard_normal(params.size)).astype(np.float32)
    p.set_params(params1)
    adv = np.array([0.8, -1.1, 0.3][:S], np.float32)
    loss, g, dE = p.ppo_grad(E, place, logp, adv)
    L, gp, gE = ppo.ppo_grads(E.astype(np.float64), params1.astype(np.float64), dims, seg, place,
                              logp.astype(np.float64), adv.astype(np.float64))
    res = {"loss": abs(loss - L) / abs(L), "dE": scaled_err(dE, gE)}
    for name, blk in _blocks(g, dims).items():
        res[name] = scaled_err(blk, _blocks(gp, dims)[name])
    print(N, seg, S, H, {k: f"{v:.2e}" for k, v in res.items()})
    bad = {k: v for k, v in res.items() if v > 1e-5}
    assert not bad, bad
    p.free()


def _shuffles(seed, iteration, epochs, S):
    """c32: the seeded Fisher-Yates shuffle of each epoch (splitmix64)."""
    from oracle import sm64
    out = []
    for ep in range(epochs):
        order = list(range(S))
        key = sm64(sm64(seed ^ 0x53485546) ^ (iteration * epochs + ep))
        for b in range(S - 1, 0, -1):
            r = sm64(key ^ b) % (b + 1)
            order[b], order[r] = order[r], order[b]
        out.append(order)
    return out


def test_ppo_iteration_matches_oracle_schedule():
    """One PPO iteration (P:L237 schedule, scaled to 2 x 4 samples, 2 minibatches,
    2 epochs): step times (c30) and Eq. 7 advantages (c31) of the GPU's own
    placements, and the parameters after the 4 clipped Adam steps against the
    oracle running the same schedule in fp64 (torch autograd gradients,
    oracle.adam with the global-norm clip)."""
    import oracle
    from synth import graphs as SG
    g = SG.cached("tiny", 0)                                  # N = 64 ops, dims, edges
    N, H, seg = g.num_nodes, 32, 16
    dims = dict(H=H, Hd=64, A=128, De=8, D=3)
    p = mars.placer_create(seed=2, in_dim=H, enc_hidden=64, attn_dim=128, dev_embed=8,
                           num_devices=3, segment=seg)
    cfg = dict(samples_per_policy=4, policies=2, minibatches=2, epochs=2, seed=5,
               capacity_bytes=4e6, lr=1e-3)
    o = mars.ppo_create(p, **cfg)
    E = (0.5 * np.random.default_rng(0).standard_normal((N, H))).astype(np.float32)
    p0 = p.get_params().astype(np.float64)
    out = o.iteration(E, g)
    S = 8
    times = [ppo.step_time(out["placements"][b], g.dims, g.indptr, g.indices, 3, 4e6)
             for b in range(S)]
    assert np.allclose(out["step_times"], times, rtol=1e-6, atol=0)
    A, _ = ppo.advantages(times, mu=0.99)
    assert np.allclose(out["advantages"], A, rtol=1e-5, atol=1e-7)
    # the oracle runs the schedule from the same start
    _, lp_old, _, _ = PL.decode(E.astype(np.float64), PL.unpack(p0, **dims), seg, 3, S, 0,
                                forced=out["placements"])
    par, m, v, t = p0.copy(), np.zeros_like(p0), np.zeros_like(p0), 0
    for order in _shuffles(5, 0, 2, S):
        for k in range(2):
            idx = order[k * 4:(k + 1) * 4]
            _, gp, _ = ppo.ppo_grads(E.astype(np.float64), par, dims, seg,
                                     out["placements"][idx], lp_old[idx], np.asarray(A)[idx])
            t += 1
            par, m, v = oracle.adam(par, m, v, gp, t, lr=1e-3, clip=1.0)
    got = p.get_params().astype(np.float64)
    step = np.abs(par - p0)
    err = np.abs(got - par)
    print("max |dp| gpu-oracle / lr:", float(err.max() / 1e-3),
          "median update / lr:", float(np.median(step) / 1e-3))
    # Adam normalises every coordinate: agreement to a small fraction of lr
    assert err.max() <= 0.05 * 1e-3
    o.free(); p.free()


def test_ppo_training_reduces_step_time():
    """Sanity (parity unpinned: the paper's curves need its TF environment):
    on the tiny op graph with a tight memory capacity, a few PPO iterations
    lower the mean step time of the sampled placements."""
    from synth import graphs as SG
    g = SG.cached("tiny", 0)
    N, H = g.num_nodes, 32
    p = mars.placer_create(seed=1, in_dim=H, enc_hidden=64, attn_dim=128, dev_embed=8,
                           num_devices=4, segment=16)
    o = mars.ppo_create(p, samples_per_policy=10, policies=2, minibatches=4, epochs=3, seed=3,
                        capacity_bytes=3e8, lr=3e-3)
    E = (0.5 * np.random.default_rng(1).standard_normal((N, H))).astype(np.float32)
    first = o.iteration(E, g)["step_times"].mean()
    for _ in range(15):
        last = o.iteration(E, g)["step_times"].mean()
    print("mean step time", first, "->", last)
    assert last < first


def _torch_encode(g, F, H, params):
    """Independent formulation of the GCN's positive branch (Eq. 1) in torch
    float64 with a dense Â_n (c1-c3): the oracle of the encoder's VJP."""
    import torch
    N = g.num_nodes
    A = torch.zeros(N, N, dtype=torch.float64)
    for u in range(N):
        for e in range(int(g.indptr[u]), int(g.indptr[u + 1])):
            v = int(g.indices[e])
            if u != v:
                A[u, v] = 1.0; A[v, u] = 1.0
    A = A + torch.eye(N, dtype=torch.float64)
    dm = A.sum(1).rsqrt()
    An = dm[:, None] * A * dm[None, :]
    p = torch.tensor(np.asarray(params, np.float64), requires_grad=True)
    o = 0
    W1 = p[o:o + F * H].view(F, H); o += F * H
    W2 = p[o:o + H * H].view(H, H); o += H * H
    W3 = p[o:o + H * H].view(H, H); o += 2 * H * H
    al = p[o:o + 3]
    h = torch.tensor(np.asarray(g.features, np.float64))
    for l, W in enumerate((W1, W2, W3)):
        h = torch.nn.functional.prelu(An @ h @ W, al[l:l + 1])
    return p, h


@pytest.mark.parametrize("name,F,H", [("tiny", 16, 32), ("inception", 64, 128)])
def test_encoder_vjp_matches_torch(name, F, H):
    """The joint update's path into the GCN (mars_dgi_encoder_vjp: the stacked
    DGI backward with a zero corrupted half) against torch autograd."""
    import torch
    from synth import graphs as SG
    g0 = SG.cached(name, 0) if name != "tiny" else SG.tiny(0)
    g = mars.graph_load([g0])
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=4)
    dE = np.random.default_rng(1).standard_normal((g0.num_nodes, H)).astype(np.float32)
    got = m.encoder_vjp(g, dE)
    p, h = _torch_encode(g0, F, H, m.get_state()[0])
    (h * torch.tensor(dE.astype(np.float64))).sum().backward()
    ref = p.grad.numpy()
    P = len(ref)
    mblk = slice(F * H + 2 * H * H, F * H + 3 * H * H)
    assert np.all(got[mblk] == 0)
    keep = np.ones(P, bool); keep[mblk] = False
    e = scaled_err(got[keep], ref[keep])
    print(name, "encoder VJP err", e)
    assert e <= 1e-5


def test_joint_ppo_iteration_runs_and_moves_both():
    """mars_ppo_iteration_joint: one iteration on the tiny op graph updates the
    placer AND the GCN encoder (finite, changed), and its step times are the
    model's for the drawn placements."""
    from synth import graphs as SG
    g0 = SG.tiny(0)
    g = mars.graph_load([g0])
    enc = mars.dgi_create(in_dim=16, hidden_dim=32, seed=2)
    p = mars.placer_create(seed=3, in_dim=32, enc_hidden=64, attn_dim=128, dev_embed=8,
                           num_devices=4, segment=16)
    o = mars.ppo_create(p, enc, samples_per_policy=4, policies=2, minibatches=2, epochs=1,
                        capacity_bytes=3e8, lr=1e-3)
    e0, p0 = enc.get_state()[0], p.get_params()
    out = o.iteration_joint(g, g0)
    e1, p1 = enc.get_state()[0], p.get_params()
    assert np.all(np.isfinite(e1)) and np.all(np.isfinite(p1))
    assert not np.array_equal(e0, e1) and not np.array_equal(p0, p1)
    times = [ppo.step_time(out["placements"][b], g0.dims, g0.indptr, g0.indices, 4, 3e8)
             for b in range(8)]
    assert np.allclose(out["step_times"], times, rtol=1e-6)


def test_ppo_grad_paper_sizes():
    """P:L234 sizes (bi-LSTM 2 x 256, decoder 512, attention 512, device
    embedding 64, s = 128, D = 4) on 300 ops (a ragged last segment), H = 256:
    the PPO gradient of every block and dL/dE against torch fp64 autograd at
    1e-5, or -- for a block fp32 rounding alone moves further (reading c33:
    the attention query's gradient passes through the softmax backward's
    cancellation) -- at 3x the error of the same formulation run in float32."""
    N, seg, S, H = 300, 128, 2, 256
    dims = dict(H=H, Hd=256, A=512, De=64, D=4)
    p = mars.placer_create(seed=6, in_dim=H)
    rng = np.random.default_rng(11)
    E = (0.3 * rng.standard_normal((N, H))).astype(np.float32)
    place, logp, _ = p.sample(E, S, 5)
    params1 = (p.get_params() + 0.01 * rng.standard_normal(p.P)).astype(np.float32)
    p.set_params(params1)
    adv = np.array([1.2, -0.7], np.float32)
    loss, g, dE = p.ppo_grad(E, place, logp, adv)
    args = (E.astype(np.float64), params1.astype(np.float64), dims, seg, place,
            logp.astype(np.float64), adv.astype(np.float64))
    L, gp, gE = ppo.ppo_grads(*args)
    _, gp32, gE32 = ppo.ppo_grads(*args, dtype=torch.float32)      # conditioning (c33)
    res = {"loss": abs(loss - L) / abs(L), "dE": scaled_err(dE, gE)}
    bar = {"loss": 1e-5, "dE": max(1e-5, 3 * scaled_err(gE32, gE))}
    for name, blk in _blocks(g, dims).items():
        ref = _blocks(gp, dims)[name]
        res[name] = scaled_err(blk, ref)
        bar[name] = max(1e-5, 3 * scaled_err(_blocks(gp32, dims)[name], ref))
    print("paper sizes", {k: f"{v:.2e} (bar {bar[k]:.1e})" for k, v in res.items()})
    bad = {k: v for k, v in res.items() if v > bar[k]}
    assert not bad, bad
    p.free()
