"""GPU parity of the aggregation (spmm.cu) on graphs outside the op-graph
generators' shape, fp32 (1e-5) and bf16 (2e-2) against the fp64 oracle
(DESIGN.md §6, §7):

  * uniform random edges: no locality, neighbours spread over the whole graph;
  * a star hub whose row has thousands of entries (far beyond the kEll = 8
    entries of the ELL copy and the 32-entry chunks), plus a chain;
  * a long local graph (N = 20011, ragged against every block size) mixed with
    long-range edges.
"""
import numpy as np
import pytest

import oracle
import paper_conf_icpp_lancl21_b200 as mars
from synth.graphs import OpGraph
from tests.test_gpu_parity import _forward_backward_case
from tests.util import scaled_err, split_params

pytestmark = pytest.mark.gpu


def _graph(name, N, src, dst, F=64, seed=0):
    src = np.asarray(src, np.int64)
    dst = np.asarray(dst, np.int64)
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    indptr = np.zeros(N + 1, np.int64)
    np.add.at(indptr, src + 1, 1)
    indptr = np.cumsum(indptr)
    rng = np.random.default_rng(seed)
    X = rng.uniform(-1.0, 1.0, (N, F)).astype(np.float32)
    return OpGraph(name, N, indptr, dst.astype(np.int32), X)


def random_graph(N=3000, E=6000, seed=1):
    rng = np.random.default_rng(seed)
    return _graph("random", N, rng.integers(0, N, E), rng.integers(0, N, E), seed=seed)


def star_graph(N=2600, seed=2):
    rng = np.random.default_rng(seed)
    hub = 1500
    leaves = np.setdiff1d(np.arange(N), [hub])
    src = np.concatenate([np.full(leaves.size, hub), np.arange(N - 1)])
    dst = np.concatenate([leaves, np.arange(1, N)])
    extra = rng.integers(0, N, 400)
    src = np.concatenate([src, extra])
    dst = np.concatenate([dst, rng.integers(0, N, 400)])
    return _graph("star", N, src, dst, seed=seed)


def long_graph(N=20011, seed=3):
    rng = np.random.default_rng(seed)
    src = np.arange(N)
    dst = np.clip(src + rng.integers(1, 24, N), 0, N - 1)
    far = rng.integers(0, N, N // 10)
    return _graph("long", N, np.concatenate([src, far]),
                  np.concatenate([dst, rng.integers(0, N, far.size)]), seed=seed)


CASES = {"random": random_graph, "star": star_graph, "long": long_graph}


@pytest.mark.parametrize("name", list(CASES))
@pytest.mark.parametrize("H", [128, 256])
def test_edge_spmm_fp32(name, H):
    _forward_backward_case([CASES[name]()], 64, H, 5, e2e_grads=False)


@pytest.mark.parametrize("name,alpha", [("random", None), ("star", None), ("long", None),
                                        ("long", (1.5, -0.3, 0.7)), ("random", (0.0, 1.0, 2.0))])
def test_edge_spmm_bf16(name, alpha):
    """bf16 path; `alpha` overrides the PReLU slopes: the forward aggregation
    applies PReLU on packed bf16 pairs only for 0 <= a <= 1 and widens first
    otherwise (spmm.cu), both branches are checked."""
    gs = [CASES[name]()]
    F, H, seed = 64, 256, 6
    init = None
    if alpha is not None:
        init = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed).get_state()[0].copy()
        init[-3:] = alpha
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed, precision=mars.MARS_BF16,
                        init_params=init)
    b = oracle.Batch(gs)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(g, 0, 0, want_loss=True, want_grads=True, want_perms=True)
    perms = b.perms(seed, 0, 0)
    assert np.array_equal(out["perms"], perms)
    acts = {}
    for l in (1, 2, 3):
        acts[f"Y{l}"], acts[f"Z{l}"] = m.export_activations(l)
    # Y_l stage-wise: the oracle's aggregation of the GPU's own Z_{l-1}
    P = split_params(p0, F, H)
    rows = np.arange(2 * b.Nt)
    for l in (2, 3):
        y = oracle.spmm_rows(b, acts[f"Z{l - 1}"], rows, P["alpha"][l - 2])
        e = scaled_err(acts[f"Y{l}"], y)
        assert e <= 2e-2, (l, e)
    loss_sw, grads_sw, _ = oracle.backward(b, H, p0, acts)
    assert abs(out["loss"] - loss_sw) / abs(loss_sw) <= 1e-4
    for nm, blk in split_params(out["grads"], F, H).items():
        e = scaled_err(blk, split_params(grads_sw, F, H)[nm])
        assert e <= 2e-2, (nm, e)
    m.free()
    g.free()
