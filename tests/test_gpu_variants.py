"""GPU parity of the NEXT-4 contrastive variants (mars_dgi_set_contrastive;
readings c34-c39) against the variant oracle (oracle/variants.py, float64
autograd), through the C ABI: K corruption samples sharing one positive
branch, feature-masking corruption, the mean readout, the SAGE-GCN
aggregator and the InfoNCE loss, alone and combined, and the SAGE-mean encoder, fp32 (<= 1e-5 scaled) and bf16
(2e-2).  At the GNMT bench size, where the fp64 oracle is too slow end to end,
the shared-positive step is checked against the same K samples run as K
copies of the graph (c20) -- a property that holds at any size."""
import numpy as np
import pytest
import torch

import oracle
from oracle import variants as V
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG
from tests.util import scaled_err

pytestmark = pytest.mark.gpu
TOL = 1e-5


def _graphs(F):
    # several chunks (<= 256 rows) per graph and a ragged tail
    return [SG.tiny(0, N=300, F=F), SG.tiny(1, N=77, F=F), SG.tiny(2, N=517, F=F)]


def _run(gs, F, H, variant, seed=5, step=3, pair_base=0, precision=mars.MARS_FP32, impl="auto"):
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed, precision=precision)
    m.set_gemm_impl(impl)
    m.set_contrastive(**variant)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(g, step, pair_base, want_loss=True, want_grads=True,
                 want_perms=variant.get("corruption", "permute") == "permute")
    m.free(); g.free()
    return p0, out


VARIANTS = [
    dict(num_neg=2),
    dict(num_neg=3),
    dict(num_neg=4),
    dict(corruption="mask", mask_rate=0.25),
    dict(num_neg=3, corruption="mask", mask_rate=0.5),
    dict(readout="mean"),
    dict(aggregator="sage_gcn"),
    dict(num_neg=2, readout="mean", aggregator="sage_gcn"),
    dict(loss="infonce"),
    dict(num_neg=3, loss="infonce"),
    dict(num_neg=2, corruption="mask", mask_rate=0.2, readout="mean", loss="infonce"),
]


# End to end against fp64, the bar is 1e-5 where the forward's rounding flips
# no PReLU branch (c19).  At H = 256 the 3xFP16 forward (~1e-6)
# flips a few of the ~10^6 pre-activations of these graphs and each flip moves
# dW1 / dW2 by ~1e-4 -- the default step behaves the same (its H = 256 gate is
# stage-wise, tests/stagewise.py: every stage <= 1.4e-6 on these graphs) -- so
# the H = 256 variant logic is checked end to end on the FFMA GEMMs.
SIZES = [(16, 32, "auto"), (16, 32, "simt"), (64, 128, "auto"), (64, 256, "simt")]


def _noise_spread(gs, p0, F, H, seed, step, pb, variant, encoder="gcn", eps=1e-6, seeds=3):
    """Conditioning probe for the tcgen05 (3xFP16) path: the largest change of
    the fp64 oracle's gradient when every pre-activation Z of the encoder is
    perturbed by relative noise eps (the 3xFP16 rounding scale), over a few
    draws.  A PReLU kink within that noise of zero flips the branch."""
    kw = dict(pair_base=pb, encoder=encoder, sparse=encoder != "sage_pool", **variant)
    _, g0 = V.step_grads(gs, p0, F, H, seed, step, **kw)
    worst = 0.0
    for sd in range(seeds):
        gen = torch.Generator().manual_seed(sd)
        noise = lambda z: z * (1 + eps * torch.randn(z.shape, generator=gen, dtype=z.dtype))  # noqa

        def gcn(An, X, W, alpha):
            h = X
            for l in range(3):
                h = torch.nn.functional.prelu(noise(An @ (h @ W[l])), alpha[l:l + 1])
            return h

        def sage(AN, X, Wp, alpha):
            h = X
            for l in range(3):
                Ws, Wn = Wp[l]
                h = torch.nn.functional.prelu(noise(h @ Ws + AN @ (h @ Wn)), alpha[l:l + 1])
            return h
        saved = (V._encoder_gcn, V.encoder_sage)
        V._encoder_gcn, V.encoder_sage = gcn, sage
        try:
            _, g1 = V.step_grads(gs, p0, F, H, seed, step, **kw)
        finally:
            V._encoder_gcn, V.encoder_sage = saved
        worst = max(worst, scaled_err(g1, g0))
    return worst


def _grad_bar(impl, gs, p0, F, H, seed, step, pb, variant, encoder="gcn"):
    """1e-5, or on the tcgen05 path 3 x the conditioning probe if larger (the
    c33 rule): the FFMA GEMMs' ~1e-7 rounding flips no kink on
    these graphs, 3xFP16's ~1e-6 can."""
    if impl != "auto":
        return TOL
    return max(TOL, 3 * _noise_spread(gs, p0, F, H, seed, step, pb, variant, encoder))


@pytest.mark.parametrize("F,H,impl", SIZES)
@pytest.mark.parametrize("variant", VARIANTS, ids=lambda v: "-".join(f"{k}={x}" for k, x in v.items()))
def test_variant_step_vs_oracle(variant, F, H, impl):
    gs = _graphs(F)
    seed, step, pb = 5, 3, 11
    p0, out = _run(gs, F, H, variant, seed, step, pb, impl=impl)
    loss, grads = V.step_grads(gs, p0, F, H, seed, step, pair_base=pb, sparse=True, **variant)
    assert abs(out["loss"] - loss) / abs(loss) <= TOL
    err = scaled_err(out["grads"], grads)
    if err > TOL:                       # only then is the (slower) conditioning probe needed
        bar = _grad_bar(impl, gs, p0, F, H, seed, step, pb, variant)
        print(f"{variant} F={F} H={H} {impl}: grads err {err:.2e}, conditioning bar {bar:.2e}")
        assert err <= bar, (err, bar)
    if "perms" in out:
        K = variant.get("num_neg", 1)
        Nt = sum(g.num_nodes for g in gs)
        perms = out["perms"].reshape(K, Nt)
        off = 0
        for gi, g in enumerate(gs):
            for k in range(K):
                ref = oracle.perm(seed, step, pb + gi * K + k, g.num_nodes)
                assert np.array_equal(perms[k, off:off + g.num_nodes], ref)
            off += g.num_nodes


def _cancellation(gs, p, F, H, seed, step, num_neg=1, corruption="permute", mask_rate=0.0,
                  readout="sigmoid_mean", aggregator="gcn"):
    """max over graphs of (|Σ_pos dl h| + (1/K) Σ_k |Σ dl~ h~|) / |dv| (max-norms):
    how much dv = Σ dl h -- the sum every gradient flows through -- cancels."""
    pt = torch.tensor(p)
    W1, W2, W3, M, al = V.unpack(pt, F, H)
    worst = 0.0
    for gi, g in enumerate(gs):
        An = torch.from_numpy(V.normalise(V.adjacency(g), aggregator))
        X = torch.tensor(np.asarray(g.features, np.float64))
        Hp = V.encoder(An, X, (W1, W2, W3), al)
        s = torch.sigmoid(Hp.mean(0)) if readout == "sigmoid_mean" else Hp.mean(0)
        v = M @ s
        a = ((torch.sigmoid(Hp @ v) - 1)[:, None] * Hp).sum(0)
        parts, tot = [a.abs().max()], a.clone()
        for k in range(num_neg):
            Hn = V.encoder(An, V.corrupted(g, X, seed, step, gi * num_neg + k, corruption,
                                           mask_rate), (W1, W2, W3), al)
            b = (torch.sigmoid(Hn @ v)[:, None] * Hn).sum(0) / num_neg
            parts.append(b.abs().max())
            tot = tot + b
        worst = max(worst, float(sum(parts) / tot.abs().max()))
    return worst


@pytest.mark.parametrize("variant", [dict(num_neg=3), dict(num_neg=3, readout="mean"),
                                     dict(corruption="mask", mask_rate=0.25, aggregator="sage_gcn")],
                         ids=lambda v: "-".join(f"{k}={x}" for k, x in v.items()))
def test_variant_bf16(variant):
    """bf16 storage + bf16 MMAs end to end against fp64.  The 2e-2 bar of
    DESIGN.md §6 is a stage-wise bar; end to end, bf16 rounding of H3 enters
    every gradient through dv = Σ dl_i h_i, a difference of positive and
    corrupted sums that cancels more or less depending on the variant (the
    plain-mean readout gives scores near 0, dl near -1/2 and +1/2, and several
    times the cancellation of sig(mean)).  So the variant is held to 2e-2 or to
    1.5 x the default step's own end-to-end bf16 error scaled by the ratio of
    the two cancellation factors, whichever is larger (the c33 rule: the bar
    follows the conditioning)."""
    gs = _graphs(64)
    errs, canc = {}, {}
    for name, v in (("default", {}), ("variant", variant)):
        p0, out = _run(gs, 64, 128, v, precision=mars.MARS_BF16)
        loss, grads = V.step_grads(gs, p0, 64, 128, 5, 3, sparse=True, **v)
        errs[name] = (abs(out["loss"] - loss) / abs(loss), scaled_err(out["grads"], grads))
        canc[name] = _cancellation(gs, p0, 64, 128, 5, 3, **v)
    bar = max(2e-2, 1.5 * errs["default"][1] * max(1.0, canc["variant"] / canc["default"]))
    print("bf16 end to end (loss, grads):", errs, "cancellation:", canc, "bar:", bar)
    assert errs["variant"][0] <= 2e-2
    assert errs["variant"][1] <= bar


def test_default_variant_is_the_dgi_step():
    """set_contrastive() with the defaults gives the same step, bit for bit."""
    gs = _graphs(64)
    _, a = _run(gs, 64, 256, {})
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=64, hidden_dim=256, seed=5)
    b = m.step(g, 3, 0, want_loss=True, want_grads=True)
    assert a["loss"] == b["loss"] and np.array_equal(a["grads"], b["grads"])
    m.free(); g.free()


@pytest.mark.parametrize("K", [2, 4])
def test_shared_positive_equals_k_copies_at_gnmt_size(K):
    """c34 = c20 at the bench's graph size (H = 256, tcgen05 GEMMs): one
    positive branch + K samples vs the K-copies batch, same permutations."""
    gs = [SG.cached("gnmt", 0)]
    F, H, seed, step = 64, 256, 7, 2
    _, a = _run(gs, F, H, dict(num_neg=K), seed, step)
    gc = mars.graph_load(mars.corruption_samples(gs, K))
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed)
    b = m.step(gc, step, 0, global_batch=K, want_loss=True, want_grads=True, want_perms=True)
    m.free(); gc.free()
    N = gs[0].num_nodes
    assert np.array_equal(a["perms"], b["perms"])          # sample k = copy k, pair k
    assert abs(a["loss"] - b["loss"]) / abs(b["loss"]) <= 1e-6
    err = scaled_err(a["grads"], b["grads"])
    print(f"K={K} N={N}: shared vs copies grads scaled err {err:.2e}")
    assert err <= 1e-5


def test_captured_replay_matches_eager():
    """The captured step (second step on a set) replays the variant schedule."""
    gs = _graphs(64)
    variant = dict(num_neg=3, corruption="mask", mask_rate=0.3, aggregator="sage_gcn")
    res = []
    for cap in (True, False):
        g = mars.graph_load(gs)
        m = mars.dgi_create(in_dim=64, hidden_dim=128, seed=2)
        m.set_graph_capture(cap)
        m.set_contrastive(**variant)
        losses = [m.step(g, s, 0, want_loss=True)["loss"] for s in range(4)]
        res.append((losses, m.get_state()[0]))
        m.free(); g.free()
    assert res[0][0] == res[1][0]
    assert np.array_equal(res[0][1], res[1][1])


def test_sage_encode_and_vjp():
    gs = _graphs(64)
    F, H = 64, 128
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=4)
    m.set_contrastive(aggregator="sage_gcn")
    p0 = m.get_state()[0].astype(np.float64)
    emb = m.encode(g)
    ref = V.encode(gs, p0, F, H, aggregator="sage_gcn")
    assert scaled_err(emb, ref) <= TOL
    dE = np.random.default_rng(0).standard_normal(emb.shape).astype(np.float32)
    got = m.encoder_vjp(g, dE)
    p = torch.tensor(p0, requires_grad=True)
    W1, W2, W3, _, al = V.unpack(p, F, H)
    out, o = [], 0
    for gr in gs:
        An = torch.from_numpy(V.normalise(V.adjacency(gr), "sage_gcn"))
        out.append(V.encoder(An, torch.tensor(np.asarray(gr.features, np.float64)), (W1, W2, W3), al))
    (torch.cat(out) * torch.tensor(dE, dtype=torch.float64)).sum().backward()
    assert scaled_err(got, p.grad.numpy()) <= TOL
    m.free(); g.free()


def test_variant_errors():
    m = mars.dgi_create(in_dim=16, hidden_dim=32)
    for bad in (dict(num_neg=0), dict(num_neg=65), dict(mask_rate=1.5, corruption="mask")):
        with pytest.raises(mars.MarsError):
            m.set_contrastive(**bad)
    m.set_contrastive(corruption="mask", mask_rate=0.1)
    g = mars.graph_load([SG.tiny(0)])
    with pytest.raises(mars.MarsError):
        m.step(g, 0, 0, want_perms=True)       # masking has no permutations
    assert m.get_contrastive()["corruption"] == "mask"
    m.free(); g.free()


# ----------------------------------------------------------------- SAGE-mean encoder (c38)
def _run_sage(gs, F, H, variant, seed=6, step=2, pair_base=0, capture=True, impl="auto"):
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed, encoder="sage")
    m.set_gemm_impl(impl)
    m.set_graph_capture(capture)
    m.set_contrastive(**variant)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(g, step, pair_base, want_loss=True, want_grads=True)
    m.free(); g.free()
    return p0, out


def test_sage_init_bit_exact():
    for F, H in ((16, 32), (64, 256)):
        m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=13, encoder="sage")
        assert m.P == V.num_params(F, H, "sage")
        assert m.get_state()[0].tobytes() == V.sage_init(13, F, H).tobytes()
        m.free()


@pytest.mark.parametrize("F,H,impl", SIZES)
@pytest.mark.parametrize("variant", [dict(), dict(num_neg=3), dict(num_neg=2, corruption="mask",
                                                                   mask_rate=0.3),
                                     dict(readout="mean"), dict(num_neg=2, loss="infonce")],
                         ids=lambda v: "-".join(f"{k}={x}" for k, x in v.items()) or "default")
def test_sage_step_vs_oracle(variant, F, H, impl):
    gs = _graphs(F)
    p0, out = _run_sage(gs, F, H, variant, pair_base=4, impl=impl)
    loss, grads = V.step_grads(gs, p0, F, H, 6, 2, pair_base=4, sparse=True, encoder="sage",
                               **variant)
    assert abs(out["loss"] - loss) / abs(loss) <= TOL
    err = scaled_err(out["grads"], grads)
    if err > TOL:
        bar = _grad_bar(impl, gs, p0, F, H, 6, 2, 4, variant, encoder="sage")
        print(f"sage {variant} F={F} H={H} {impl}: grads err {err:.2e}, conditioning bar {bar:.2e}")
        assert err <= bar, (err, bar)


def test_sage_encode_vs_oracle_and_hooks():
    gs = _graphs(64)
    F, H = 64, 256
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=3, encoder="sage")
    p0 = m.get_state()[0].astype(np.float64)
    emb = m.encode(g)
    assert scaled_err(emb, V.encode(gs, p0, F, H, encoder_="sage")) <= TOL
    with pytest.raises(mars.MarsError):
        m.encoder_vjp(g, np.zeros_like(emb))
    with pytest.raises(mars.MarsError):
        m.set_contrastive(aggregator="sage_gcn")
    m.step(g, 0, 0)
    Y1, Z1 = m.export_activations(1)          # layer 1's GEMM input is X~ stacked
    Nt = sum(x.num_nodes for x in gs)
    X = np.concatenate([np.asarray(x.features) for x in gs])
    assert np.array_equal(Y1[:Nt], X)
    m.free(); g.free()


def test_sage_captured_replay_matches_eager():
    gs = _graphs(64)
    res = []
    for cap in (True, False):
        g = mars.graph_load(gs)
        m = mars.dgi_create(in_dim=64, hidden_dim=128, seed=2, encoder="sage")
        m.set_graph_capture(cap)
        m.set_contrastive(num_neg=2)
        losses = [m.step(g, s, 0, want_loss=True)["loss"] for s in range(4)]
        res.append((losses, m.get_state()[0]))
        m.free(); g.free()
    assert res[0][0] == res[1][0]
    assert np.array_equal(res[0][1], res[1][1])


def test_sage_config_errors():
    with pytest.raises(mars.MarsError):
        mars.dgi_create(in_dim=64, hidden_dim=128, encoder="sage", precision=mars.MARS_BF16)


def _edge_graphs(F):
    """A one-node graph, a graph with isolated nodes (no edges at all for some
    ops) and a small DAG -- degenerate neighbourhoods for every aggregator."""
    rng = np.random.default_rng(7)

    class G:
        pass
    one = G()
    one.num_nodes, one.indptr, one.indices = 1, np.zeros(2, np.int64), np.zeros(0, np.int32)
    one.features = rng.random((1, F), dtype=np.float32)
    iso = G()
    N = 40
    src = np.array([3, 3, 7, 10, 10, 11, 20], np.int64)
    dst = np.array([4, 5, 8, 11, 12, 12, 21], np.int32)
    indptr = np.zeros(N + 1, np.int64)
    np.add.at(indptr, src + 1, 1)
    iso.num_nodes, iso.indptr, iso.indices = N, np.cumsum(indptr), dst
    iso.features = rng.random((N, F), dtype=np.float32)
    return [one, iso, SG.tiny(3, N=61, F=F)]


@pytest.mark.parametrize("encoder,variant", [("gcn", dict(num_neg=2, loss="infonce")),
                                             ("gcn", dict(num_neg=3, aggregator="sage_gcn",
                                                          readout="mean")),
                                             ("sage", dict(num_neg=2, corruption="mask",
                                                           mask_rate=0.4)),
                                             ("sage", dict(loss="infonce"))])
def test_variants_degenerate_graphs(encoder, variant):
    gs = _edge_graphs(16)
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=16, hidden_dim=32, seed=9, encoder=encoder)
    m.set_contrastive(**variant)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(g, 1, 2, want_loss=True, want_grads=True)
    emb = m.encode(g)
    p1 = m.get_state()[0].astype(np.float64)          # after the step's Adam update
    m.free(); g.free()
    loss, grads = V.step_grads(gs, p0, 16, 32, 9, 1, pair_base=2, encoder=encoder, **variant)
    assert np.isfinite(out["loss"]) and np.all(np.isfinite(out["grads"]))
    assert abs(out["loss"] - loss) / abs(loss) <= TOL
    err = scaled_err(out["grads"], grads)
    if err > TOL:
        bar = _grad_bar("auto", gs, p0, 16, 32, 9, 1, 2, variant, encoder)
        print(f"degenerate {encoder} {variant}: grads err {err:.2e}, conditioning bar {bar:.2e}")
        assert err <= bar, (err, bar)
    assert scaled_err(emb, V.encode(gs, p1, 16, 32, aggregator=variant.get("aggregator", "gcn"),
                                    encoder_=encoder)) <= TOL


# ----------------------------------------------------------------- SAGE-pool encoder (c40)
def test_sage_pool_init_bit_exact():
    for F, H in ((16, 32), (64, 256)):
        m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=13, encoder="sage_pool")
        assert m.P == V.num_params(F, H, "sage_pool")
        assert m.get_state()[0].tobytes() == V.sage_pool_init(13, F, H).tobytes()
        m.free()


def _run_pool(gs, F, H, variant, impl="auto", capture=True, seed=6, step=2, pair_base=4):
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed, encoder="sage_pool")
    m.set_gemm_impl(impl)
    m.set_graph_capture(capture)
    m.set_contrastive(**variant)
    # non-zero pool biases so the ReLU masks matter
    p = m.get_state()[0].copy()
    rng = np.random.default_rng(3)
    o = 0
    for l in range(3):
        C = F if l == 0 else H
        o += 2 * C * H + H * H
        p[o:o + H] = rng.standard_normal(H).astype(np.float32) * 0.1
        o += H
    m.set_state(p, np.zeros_like(p), np.zeros_like(p), 0)
    out = m.step(g, step, pair_base, want_loss=True, want_grads=True)
    p1 = m.get_state()[0]
    emb = m.encode(g)
    m.free(); g.free()
    return p.astype(np.float64), out, p1.astype(np.float64), emb


POOL_VARIANTS = [dict(), dict(num_neg=2, corruption="mask", mask_rate=0.3),
                 dict(num_neg=3, loss="infonce", readout="mean")]


def _pool_noise_spread(gs, p0, F, H, variant, eps=1e-6, seeds=5):
    """Conditioning probe: the largest change of the fp64 oracle's gradient
    when every pool pre-activation U = h W_p + b_p is perturbed by relative
    noise eps (the 3xFP16 rounding scale), over a few noise draws."""
    orig = V.encoder_sage_pool
    kw = dict(pair_base=4, encoder="sage_pool", **variant)
    _, g0 = V.step_grads(gs, p0, F, H, 6, 2, **kw)
    worst = 0.0
    for sd in range(seeds):
        gen = torch.Generator().manual_seed(sd)

        def noisy(nbrs, X, layers, alpha):
            h = X
            for l in range(3):
                Ws, Wn, Wp, bp = layers[l]
                U = h @ Wp + bp
                U = U * (1 + eps * torch.randn(U.shape, generator=gen, dtype=U.dtype))
                P = torch.relu(U)
                zero = torch.zeros(P.shape[1], dtype=P.dtype)
                agg = torch.stack([P[torch.from_numpy(nb)].max(0).values if len(nb) else zero
                                   for nb in nbrs])
                h = torch.nn.functional.prelu(h @ Ws + agg @ Wn, alpha[l:l + 1])
            return h
        V.encoder_sage_pool = noisy
        try:
            _, g1 = V.step_grads(gs, p0, F, H, 6, 2, **kw)
        finally:
            V.encoder_sage_pool = orig
        worst = max(worst, scaled_err(g1, g0))
    return worst


@pytest.mark.parametrize("F,H,impl", SIZES)
@pytest.mark.parametrize("variant", POOL_VARIANTS,
                         ids=lambda v: "-".join(f"{k}={x}" for k, x in v.items()) or "default")
def test_sage_pool_step_vs_oracle(variant, F, H, impl):
    """The element-wise max routes each gradient to one neighbour, so two
    neighbours within rounding of each other (near ties: tens to hundreds on
    these graphs) can swap the route -- a conditioning effect like c19's PReLU
    flips.  The gradient bar is therefore c33's: 1e-5 or 3 x the error of the
    same formulation run at the path's rounding, whichever is larger -- torch
    float32 for the FFMA GEMMs (which take exactly torch's routes: equal errors,
    measured), and for the tcgen05 path (3xFP16, ~1e-6 relative) the fp64
    oracle with 1e-6 relative noise on the pool pre-activations (measured:
    that noise alone moves the oracle's gradient by up to 5e-3 on these
    graphs).  The loss and the embeddings, which do not route, stay at 1e-5."""
    gs = _graphs(F)
    p0, out, p1, emb = _run_pool(gs, F, H, variant, impl)
    kw = dict(pair_base=4, encoder="sage_pool", **variant)
    loss, grads = V.step_grads(gs, p0, F, H, 6, 2, **kw)
    _, g32 = V.step_grads(gs, p0, F, H, 6, 2, dtype=torch.float32, **kw)
    cond = scaled_err(g32, grads)
    if impl == "auto":                                  # tcgen05 3xFP16 GEMMs
        cond = max(cond, _pool_noise_spread(gs, p0, F, H, variant))
    err = scaled_err(out["grads"], grads)
    print(f"sage_pool {variant} F={F} H={H} {impl}: grads err {err:.2e}, conditioning {cond:.2e}")
    assert abs(out["loss"] - loss) / abs(loss) <= TOL
    assert err <= max(TOL, 3 * cond), (err, cond)
    assert scaled_err(emb, V.encode(gs, p1, F, H, encoder_="sage_pool")) <= TOL


def test_sage_pool_degenerate_graphs_and_capture():
    gs = _edge_graphs(16)
    p0, out, p1, emb = _run_pool(gs, 16, 32, dict(num_neg=2))
    loss, grads = V.step_grads(gs, p0, 16, 32, 6, 2, pair_base=4, encoder="sage_pool", num_neg=2)
    assert abs(out["loss"] - loss) / abs(loss) <= TOL
    assert scaled_err(out["grads"], grads) <= TOL
    assert scaled_err(emb, V.encode(gs, p1, 16, 32, encoder_="sage_pool")) <= TOL
    # captured replay = eager, bitwise
    gs = _graphs(64)
    res = []
    for cap in (True, False):
        g = mars.graph_load(gs)
        m = mars.dgi_create(in_dim=64, hidden_dim=128, seed=2, encoder="sage_pool")
        m.set_graph_capture(cap)
        losses = [m.step(g, s, 0, want_loss=True)["loss"] for s in range(4)]
        res.append((losses, m.get_state()[0]))
        m.free(); g.free()
    assert res[0][0] == res[1][0] and np.array_equal(res[0][1], res[1][1])
