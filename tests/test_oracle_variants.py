"""Pins for the NEXT-4 variant oracle (oracle/variants.py; readings c34-c39):
the default variant against the C oracle's step, K shared-positive samples
against the C oracle on K copies of each graph (c20), feature masking at rates
0 and 1 in closed form, the readouts against the C oracle's encoder plus a
hand-written numpy head, the SAGE-GCN encoder against brute-force loops and
its constant-feature special case, the SAGE-mean encoder (c38) against
brute-force loops, its W_n = 0 and constant-feature special cases and its
init layout, and every variant's gradient against central finite
differences."""
import math
from types import SimpleNamespace

import numpy as np
import pytest

import oracle
from oracle import variants as V
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG
from tests.util import scaled_err

F, H, SEED, STEP = 16, 32, 5, 7


def _graphs():
    return [SG.tiny(0, N=40), SG.tiny(1, N=29)]


def _params(seed=SEED):
    return oracle.xavier(seed, F, H).astype(np.float64)


def _with_features(g, X):
    return SimpleNamespace(num_nodes=g.num_nodes, indptr=g.indptr, indices=g.indices,
                           features=np.ascontiguousarray(X, np.float32))


def _softplus(x):
    return np.maximum(x, 0) + np.log1p(np.exp(-np.abs(x)))


def _head_loss(Hp, Hn_list, p, readout):
    """Eqs. 4-6 by hand in numpy from given positive / corrupted embeddings."""
    M = p[F * H + 2 * H * H:F * H + 3 * H * H].reshape(H, H)
    m = Hp.mean(0)
    s = 1 / (1 + np.exp(-m)) if readout == "sigmoid_mean" else m
    v = M @ s
    N = Hp.shape[0]
    neg = sum(_softplus(Hn @ v).sum() for Hn in Hn_list) / len(Hn_list)
    return (_softplus(-(Hp @ v)).sum() + neg) / (2 * N)


def _c_encode(g, p):
    return oracle.encode(oracle.Batch([g]), H, p)


def test_default_variant_is_the_c_oracle_step():
    gs, p = _graphs(), _params()
    b = oracle.Batch(gs)
    loss, grads, *_ = oracle.step_grads(b, H, p, b.perms(SEED, STEP, 3))
    vl, vg = V.step_grads(gs, p, F, H, SEED, STEP, pair_base=3)
    assert abs(vl - loss) < 1e-13
    assert scaled_err(vg, grads) < 1e-12


@pytest.mark.parametrize("K", [2, 3])
def test_k_shared_samples_equal_c_oracle_on_copies(K):
    """c34 = c20: the shared positive branch with K samples is the C oracle's
    step on K consecutive copies of every graph (pair g K + k), B = K G."""
    gs, p = _graphs(), _params()
    copies = mars.corruption_samples(gs, K)
    b = oracle.Batch(copies)
    loss, grads, *_ = oracle.step_grads(b, H, p, b.perms(SEED, STEP, 0))
    vl, vg = V.step_grads(gs, p, F, H, SEED, STEP, num_neg=K)
    assert abs(vl - loss) < 1e-13
    assert scaled_err(vg, grads) < 1e-12


@pytest.mark.parametrize("rate", [0.0, 1.0])
def test_mask_rates_zero_and_one_closed_form(rate):
    """rate 0: X~ = X, so l~ = l and L_g = (1/2N) Σ [softplus(-l) + softplus(l)];
    rate 1: X~ = 0, so H~ = 0, l~ = 0 and every corrupted term is log 2."""
    gs, p = _graphs(), _params()
    vl, _ = V.step_grads(gs, p, F, H, SEED, STEP, num_neg=2, corruption="mask", mask_rate=rate)
    want = 0.0
    for g in gs:
        Hp = _c_encode(g, p)
        Hn = Hp if rate == 0.0 else np.zeros_like(Hp)
        want += _head_loss(Hp, [Hn], p, "sigmoid_mean") / len(gs)
        if rate == 1.0:
            N = g.num_nodes
            M = p[F * H + 2 * H * H:F * H + 3 * H * H].reshape(H, H)
            v = M @ (1 / (1 + np.exp(-Hp.mean(0))))
            assert abs(_head_loss(Hp, [Hn], p, "sigmoid_mean")
                       - (_softplus(-(Hp @ v)).sum() + N * math.log(2)) / (2 * N)) < 1e-13
    assert abs(vl - want) < 1e-12


def test_mask_statistics_and_keys():
    N, Fm, rate = 200, 64, 0.3
    k = V.mask_keep(SEED, STEP, 4, N, Fm, rate)
    n = N * Fm
    zeroed = n - int(k.sum())
    assert abs(zeroed - rate * n) < 4 * math.sqrt(n * rate * (1 - rate))
    assert np.array_equal(k, V.mask_keep(SEED, STEP, 4, N, Fm, rate))
    assert not np.array_equal(k, V.mask_keep(SEED, STEP, 5, N, Fm, rate))
    assert not np.array_equal(k, V.mask_keep(SEED, STEP + 1, 4, N, Fm, rate))
    # monotone in the rate: a feature kept at 0.5 is kept at 0.3
    k5 = V.mask_keep(SEED, STEP, 4, N, Fm, 0.5)
    assert np.all(k[k5])


@pytest.mark.parametrize("readout", ["sigmoid_mean", "mean"])
def test_readouts_against_c_encoder_and_numpy_head(readout):
    """Forward loss: the C oracle encodes the positive graph and each permuted
    copy (features X[pi_k], same structure); the head is written out in numpy."""
    gs, p = _graphs(), _params()
    K = 2
    want = 0.0
    for gi, g in enumerate(gs):
        Hp = _c_encode(g, p)
        Hn = []
        for k in range(K):
            pi = oracle.perm(SEED, STEP, gi * K + k, g.num_nodes)
            Hn.append(_c_encode(_with_features(g, np.asarray(g.features)[pi]), p))
        want += _head_loss(Hp, Hn, p, readout) / len(gs)
    vl, _ = V.step_grads(gs, p, F, H, SEED, STEP, num_neg=K, readout=readout)
    assert abs(vl - want) < 1e-12


def _prelu(x, a):
    return np.where(x > 0, x, a * x)


def test_sage_encoder_brute_force_loops():
    """c37 written as per-node loops: h_i' = PReLU((1/|N(i)|+1) Σ_{j in N(i) ∪ {i}} h_j W)."""
    g, p = SG.tiny(2, N=23), _params(9)
    W = [p[:F * H].reshape(F, H), p[F * H:F * H + H * H].reshape(H, H),
         p[F * H + H * H:F * H + 2 * H * H].reshape(H, H)]
    al = p[-3:]
    nb = [set([i]) for i in range(g.num_nodes)]
    for u in range(g.num_nodes):
        for e in range(int(g.indptr[u]), int(g.indptr[u + 1])):
            v = int(g.indices[e])
            nb[u].add(v)
            nb[v].add(u)
    h = np.asarray(g.features, np.float64)
    for l in range(3):
        out = np.zeros((g.num_nodes, H))
        for i in range(g.num_nodes):
            agg = sum(h[j] for j in sorted(nb[i])) / len(nb[i])
            out[i] = _prelu(agg @ W[l], al[l])
        h = out
    got = V.encode([g], p, F, H, aggregator="sage_gcn")
    assert np.max(np.abs(got - h)) < 1e-12 * max(1.0, np.max(np.abs(h)))


def test_sage_constant_features_reduce_to_an_mlp():
    """Rows of D^-1 Â sum to 1: constant feature rows stay constant, and every
    embedding equals the 3-layer PReLU MLP of the feature row."""
    g, p = SG.tiny(3, N=31), _params(11)
    x = np.random.default_rng(0).standard_normal(F)
    gc = _with_features(g, np.tile(x, (g.num_nodes, 1)))
    got = V.encode([gc], p, F, H, aggregator="sage_gcn")
    h = x.astype(np.float32).astype(np.float64)
    for l, (o, n) in enumerate(((0, F * H), (F * H, H * H), (F * H + H * H, H * H))):
        h = _prelu(h @ p[o:o + n].reshape(-1, H), p[-3 + l])
    assert np.max(np.abs(got - h[None, :])) < 1e-12 * max(1.0, np.max(np.abs(h)))
    # the symmetric GCN normalisation does not have this property
    gcn = V.encode([gc], p, F, H, aggregator="gcn")
    assert np.max(np.abs(gcn - h[None, :])) > 1e-6


@pytest.mark.parametrize("kw", [dict(readout="mean"), dict(aggregator="sage_gcn"),
                                dict(corruption="mask", mask_rate=0.3, num_neg=2),
                                dict(num_neg=3, readout="mean", aggregator="sage_gcn")])
def test_variant_gradients_finite_differences(kw):
    gs, p = [SG.tiny(4, N=18)], _params(13)
    _, grads = V.step_grads(gs, p, F, H, SEED, STEP, **kw)
    rng = np.random.default_rng(1)
    idx = list(rng.choice(p.size - 3, 5, replace=False)) + [p.size - 3, p.size - 1]
    for i in idx:
        h = 1e-5
        pp, pm = p.copy(), p.copy()
        pp[i] += h
        pm[i] -= h
        fd = (V.step_grads(gs, pp, F, H, SEED, STEP, **kw)[0]
              - V.step_grads(gs, pm, F, H, SEED, STEP, **kw)[0]) / (2 * h)
        assert abs(fd - grads[i]) <= 1e-7 + 1e-5 * abs(grads[i]), (i, fd, grads[i])


# ----------------------------------------------------------------- SAGE-mean (c38)
def _sage_params(seed=21):
    return V.sage_init(seed, F, H).astype(np.float64)


def _sage_blocks(p):
    o, mats = 0, []
    for fin in (F, F, H, H, H, H):
        mats.append(p[o:o + fin * H].reshape(fin, H))
        o += fin * H
    return [(mats[0], mats[1]), (mats[2], mats[3]), (mats[4], mats[5])], p[-3:]


def test_sage_init_layout_and_bounds():
    p = V.sage_init(3, F, H)
    assert p.size == V.num_params(F, H, "sage") == F * H + 3 * H * H + 3 + F * H + 2 * H * H
    o = 0
    for t, fin in enumerate((F, F, H, H, H, H, H), start=1):
        blk = p[o:o + fin * H]
        b = np.float32(np.sqrt(6.0 / (2 * H if t == 7 else 2 * fin + H)))
        assert np.all(np.abs(blk) <= b) and np.std(blk) > 0.5 * b / np.sqrt(3)
        o += fin * H
    assert np.array_equal(p[-3:], np.full(3, 0.25, np.float32))
    # W_s and W_n of a layer are different draws
    assert not np.array_equal(p[:F * H], p[F * H:2 * F * H])


def test_sage_mean_encoder_brute_force_loops():
    """c38 as per-node loops: h_i' = PReLU(h_i W_s + mean_{j in N(i)} h_j W_n),
    N(i) the neighbours without i; a node without neighbours aggregates 0."""
    g = SG.tiny(5, N=26)
    p = _sage_params()
    Wp, al = _sage_blocks(p)
    nb = [set() for _ in range(g.num_nodes)]
    for u in range(g.num_nodes):
        for e in range(int(g.indptr[u]), int(g.indptr[u + 1])):
            v = int(g.indices[e])
            if v != u:
                nb[u].add(v)
                nb[v].add(u)
    h = np.asarray(g.features, np.float64)
    for l in range(3):
        out = np.zeros((g.num_nodes, H))
        for i in range(g.num_nodes):
            agg = sum(h[j] for j in sorted(nb[i])) / len(nb[i]) if nb[i] else np.zeros(h.shape[1])
            out[i] = _prelu(h[i] @ Wp[l][0] + agg @ Wp[l][1], al[l])
        h = out
    got = V.encode([g], p, F, H, encoder_="sage")
    assert np.max(np.abs(got - h)) < 1e-12 * max(1.0, np.max(np.abs(h)))


def test_sage_special_cases():
    """W_n = 0: the graph drops out (a per-node 3-layer PReLU MLP with W_s).
    Constant feature rows: the neighbour mean is the row itself, so a node with
    neighbours is the MLP with W_s + W_n and an isolated node the MLP with W_s."""
    g = SG.tiny(6, N=30)
    p = _sage_params(4)
    Wp, al = _sage_blocks(p)

    def mlp(x, mats):
        h = x
        for l, Wl in enumerate(mats):
            h = _prelu(h @ Wl, al[l])
        return h
    X = np.asarray(g.features, np.float64)
    q = p.copy()                             # zero the W_n blocks
    offs, o = [], 0
    for fin in (F, F, H, H, H, H):
        offs.append((o, fin))
        o += fin * H
    for k in (1, 3, 5):
        q[offs[k][0]:offs[k][0] + offs[k][1] * H] = 0.0
    got = V.encode([g], q, F, H, encoder_="sage")
    want = mlp(X.astype(np.float32).astype(np.float64), [w[0] for w in Wp])
    assert np.max(np.abs(got - want)) < 1e-12 * max(1.0, np.max(np.abs(want)))
    # constant rows; node 0 made isolated by removing its edges
    x = np.random.default_rng(2).standard_normal(F).astype(np.float32)
    N = g.num_nodes
    keep = [(u, int(g.indices[e])) for u in range(N)
            for e in range(int(g.indptr[u]), int(g.indptr[u + 1]))
            if u != 0 and int(g.indices[e]) != 0]
    indptr = np.zeros(N + 1, np.int64)
    for u, _ in keep:
        indptr[u + 1] += 1
    gi = SimpleNamespace(num_nodes=N, indptr=np.cumsum(indptr),
                         indices=np.array([v for _, v in keep], np.int32),
                         features=np.tile(x, (N, 1)))
    got = V.encode([gi], p, F, H, encoder_="sage")
    both = mlp(x.astype(np.float64), [w[0] + w[1] for w in Wp])
    root = mlp(x.astype(np.float64), [w[0] for w in Wp])
    deg = V.neighbour_mean(gi).sum(1)
    for i in range(N):
        want = both if deg[i] > 0 else root
        assert np.max(np.abs(got[i] - want)) < 1e-12 * max(1.0, np.max(np.abs(want)))
    assert deg[0] == 0


@pytest.mark.parametrize("kw", [dict(), dict(num_neg=2, corruption="mask", mask_rate=0.3),
                                dict(readout="mean", num_neg=3)])
def test_sage_gradients_finite_differences(kw):
    gs, p = [SG.tiny(7, N=17)], _sage_params(8)
    _, grads = V.step_grads(gs, p, F, H, SEED, STEP, encoder="sage", **kw)
    rng = np.random.default_rng(3)
    idx = list(rng.choice(p.size - 3, 6, replace=False)) + [F * H + 5, p.size - 2]
    for i in idx:
        h = 1e-5
        pp, pm = p.copy(), p.copy()
        pp[i] += h
        pm[i] -= h
        fd = (V.step_grads(gs, pp, F, H, SEED, STEP, encoder="sage", **kw)[0]
              - V.step_grads(gs, pm, F, H, SEED, STEP, encoder="sage", **kw)[0]) / (2 * h)
        assert abs(fd - grads[i]) <= 1e-7 + 1e-5 * abs(grads[i]), (i, fd, grads[i])


# ----------------------------------------------------------------- InfoNCE (c39)
@pytest.mark.parametrize("K", [1, 3])
def test_infonce_against_c_encoder_and_numpy(K):
    """Forward loss from the C oracle's embeddings with the softmax written out
    in numpy; K = 1 is also checked against its closed form softplus(l~ - l)."""
    gs, p = _graphs(), _params()
    M = p[F * H + 2 * H * H:F * H + 3 * H * H].reshape(H, H)
    want = 0.0
    for gi, g in enumerate(gs):
        Hp = _c_encode(g, p)
        v = M @ (1 / (1 + np.exp(-Hp.mean(0))))
        L = [Hp @ v]
        for k in range(K):
            pi = oracle.perm(SEED, STEP, gi * K + k, g.num_nodes)
            L.append(_c_encode(_with_features(g, np.asarray(g.features)[pi]), p) @ v)
        L = np.array(L)
        m = L.max(0)
        lse = m + np.log(np.exp(L - m).sum(0))
        per = lse - L[0]
        if K == 1:
            assert np.max(np.abs(per - _softplus(L[1] - L[0]))) < 1e-13
        want += per.mean() / len(gs)
    vl, _ = V.step_grads(gs, p, F, H, SEED, STEP, num_neg=K, loss="infonce")
    assert abs(vl - want) < 1e-12


@pytest.mark.parametrize("kw", [dict(num_neg=1), dict(num_neg=3, readout="mean"),
                                dict(num_neg=2, encoder="sage")])
def test_infonce_gradients_finite_differences(kw):
    gs = [SG.tiny(8, N=19)]
    p = _sage_params(5) if kw.get("encoder") == "sage" else _params(6)
    _, grads = V.step_grads(gs, p, F, H, SEED, STEP, loss="infonce", **kw)
    rng = np.random.default_rng(4)
    for i in list(rng.choice(p.size - 3, 6, replace=False)) + [p.size - 1]:
        h = 1e-5
        pp, pm = p.copy(), p.copy()
        pp[i] += h
        pm[i] -= h
        fd = (V.step_grads(gs, pp, F, H, SEED, STEP, loss="infonce", **kw)[0]
              - V.step_grads(gs, pm, F, H, SEED, STEP, loss="infonce", **kw)[0]) / (2 * h)
        assert abs(fd - grads[i]) <= 1e-7 + 1e-5 * abs(grads[i]), (i, fd, grads[i])


# ----------------------------------------------------------------- SAGE-pool (c40)
def _pool_blocks(p):
    o, layers = 0, []
    for l in range(3):
        C = F if l == 0 else H
        Ws = p[o:o + C * H].reshape(C, H); o += C * H
        Wn = p[o:o + H * H].reshape(H, H); o += H * H
        Wp = p[o:o + C * H].reshape(C, H); o += C * H
        bp = p[o:o + H]; o += H
        layers.append((Ws, Wn, Wp, bp))
    return layers, p[-3:]


def test_sage_pool_init_layout():
    p = V.sage_pool_init(3, F, H)
    assert p.size == V.num_params(F, H, "sage_pool")
    layers, al = _pool_blocks(p.astype(np.float64))
    for l, (Ws, Wn, Wp, bp) in enumerate(layers):
        C = F if l == 0 else H
        assert np.all(np.abs(Ws) <= np.float32(np.sqrt(6.0 / (C + 2 * H))))
        assert np.all(np.abs(Wp) <= np.float32(np.sqrt(6.0 / (C + H))))
        assert np.all(bp == 0)
    assert np.array_equal(al, np.full(3, 0.25))


def test_sage_pool_encoder_brute_force_loops():
    """c40 as per-node loops: P = ReLU(h W_p + b); agg_i = element-wise max over
    the neighbours (0 when there are none); h' = PReLU(h W_s + agg W_n)."""
    g = SG.tiny(5, N=26)
    p = V.sage_pool_init(21, F, H).astype(np.float64)
    rng = np.random.default_rng(0)
    layers, al = _pool_blocks(p)
    layers = [(Ws, Wn, Wp, rng.standard_normal(H) * 0.1) for Ws, Wn, Wp, _ in layers]
    q = p.copy()                                     # non-zero biases
    o = 0
    for l in range(3):
        C = F if l == 0 else H
        o += 2 * C * H + H * H
        q[o:o + H] = layers[l][3]
        o += H
    nb = [set() for _ in range(g.num_nodes)]
    for u in range(g.num_nodes):
        for e in range(int(g.indptr[u]), int(g.indptr[u + 1])):
            v = int(g.indices[e])
            if v != u:
                nb[u].add(v); nb[v].add(u)
    h = np.asarray(g.features, np.float64)
    for l in range(3):
        Ws, Wn, Wp, bp = layers[l]
        P = np.maximum(h @ Wp + bp, 0.0)
        out = np.zeros((g.num_nodes, H))
        for i in range(g.num_nodes):
            agg = np.max(P[sorted(nb[i])], axis=0) if nb[i] else np.zeros(H)
            out[i] = _prelu(h[i] @ Ws + agg @ Wn, al[l])
        h = out
    got = V.encode([g], q, F, H, encoder_="sage_pool")
    assert np.max(np.abs(got - h)) < 1e-12 * max(1.0, np.max(np.abs(h)))


def test_sage_pool_wn_zero_is_an_mlp():
    g = SG.tiny(6, N=30)
    p = V.sage_pool_init(4, F, H).astype(np.float64)
    layers, al = _pool_blocks(p)
    q = p.copy()
    o = 0
    for l in range(3):
        C = F if l == 0 else H
        q[o + C * H:o + C * H + H * H] = 0.0         # W_n = 0
        o += 2 * C * H + H * H + H
    h = np.asarray(g.features, np.float64)
    for l in range(3):
        h = _prelu(h @ layers[l][0], al[l])
    got = V.encode([g], q, F, H, encoder_="sage_pool")
    assert np.max(np.abs(got - h)) < 1e-12 * max(1.0, np.max(np.abs(h)))


@pytest.mark.parametrize("kw", [dict(), dict(num_neg=2, corruption="mask", mask_rate=0.3),
                                dict(num_neg=2, loss="infonce")])
def test_sage_pool_gradients_finite_differences(kw):
    gs = [SG.tiny(7, N=17)]
    p = V.sage_pool_init(8, F, H).astype(np.float64)
    _, grads = V.step_grads(gs, p, F, H, SEED, STEP, encoder="sage_pool", **kw)
    rng = np.random.default_rng(5)
    # weights of every block incl. W_p and the pool bias b_p of layer 1
    idx = list(rng.choice(p.size - 3, 6, replace=False)) + [2 * F * H + H * H + 3, p.size - 1]
    for i in idx:
        h = 1e-6
        pp, pm = p.copy(), p.copy()
        pp[i] += h
        pm[i] -= h
        fd = (V.step_grads(gs, pp, F, H, SEED, STEP, encoder="sage_pool", **kw)[0]
              - V.step_grads(gs, pm, F, H, SEED, STEP, encoder="sage_pool", **kw)[0]) / (2 * h)
        assert abs(fd - grads[i]) <= 1e-7 + 1e-5 * abs(grads[i]), (i, fd, grads[i])
