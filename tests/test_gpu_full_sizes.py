"""GPU parity at BASELINE.json's full sizes, in the launch configurations
`bench.py --workload ...` times: the Inception-V3 set (16
graphs, H = 128), the BERT-large set (8 graphs, H = 256) and the 1.1M-op
stress graph (one graph, H = 256), each through the fp32 and the bf16 path.
Too large for the oracle end to end, so stage by stage at the GPU's own stage
inputs: Inception x16 and BERT x8 through every stage of the step
(tests/stagewise.py); the 1.1M-op graph (20+ GB of host arrays for the full
chain) through sampled Y_l / Z_l rows, the head (loss, dM) and dW3.  (The
GNMT bench set is `test_gpu_parity.py::test_bench_config_stagewise` and
`test_gpu_bf16.py::test_bf16_bench_config_stagewise`.)
"""
import numpy as np
import pytest

import oracle
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG
from tests import stagewise
from tests.util import scaled_err, split_params

pytestmark = pytest.mark.gpu


def _bf16_round(W):
    w = np.asarray(W, np.float32).view(np.uint32).astype(np.uint64)
    w = ((w + 0x7FFF + ((w >> 16) & 1)) & 0xFFFF0000).astype(np.uint32)
    return w.view(np.float32).astype(np.float64)


def _graphs(name, count):
    if name == "1m":
        return [SG.make("1m", 0)]
    return [SG.cached(name, i) for i in range(count)]


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
@pytest.mark.parametrize("name,count,H", [("inception", 16, 128), ("bert", 8, 256)])
def test_full_size_stagewise(name, count, H, precision):
    """Inception x16 and BERT x8 (long hub rows: the segmented SpMM path):
    every stage of the step against the oracle (tests/stagewise.py)."""
    gs = _graphs(name, count)
    F, seed = 64, 9
    bf = precision == "bf16"
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed,
                        precision=mars.MARS_BF16 if bf else mars.MARS_FP32)
    stagewise.step_stagewise(m, g, gs, F, H, seed, step=2, base=0, B=len(gs), bf16=bf,
                             tol=2e-2 if bf else 1e-5, nrows=400, rng_seed=3)
    m.free()
    g.free()


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
@pytest.mark.parametrize("name,count,H", [("1m", 1, 256)])
def test_full_size_sampled(name, count, H, precision):
    gs = _graphs(name, count)
    F, seed, B = 64, 9, len(gs)
    bf = precision == "bf16"
    tol = 2e-2 if bf else 1e-5
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed,
                        precision=mars.MARS_BF16 if bf else mars.MARS_FP32)
    b = oracle.Batch(gs)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(g, 2, 0, global_batch=B, want_loss=True, want_grads=True, want_perms=True)
    perms = b.perms(seed, 2, 0)
    assert np.array_equal(out["perms"], perms)
    P = split_params(p0, F, H)
    rng = np.random.default_rng(3)
    rows = np.unique(np.concatenate([rng.integers(0, 2 * b.Nt, 400),
                                     [0, b.Nt - 1, b.Nt, 2 * b.Nt - 1]]))
    prev = oracle.layer1_input(b, perms)
    res = {}
    for l in (1, 2, 3):
        Y, Z = m.export_activations(l)
        W = P[f"W{l}"].reshape(-1, H)
        y = oracle.spmm_rows(b, prev, rows, None if l == 1 else P["alpha"][l - 2])
        res[f"Y{l}"] = scaled_err(Y[rows], y)
        Wm = _bf16_round(W) if bf else W
        res[f"Z{l}"] = scaled_err(Z[rows], Y[rows].astype(np.float64) @ Wm)
        assert res[f"Y{l}"] <= tol and res[f"Z{l}"] <= tol, res
        prev = Z
    loss, s, dM, dZ3, da3 = oracle.head(b, H, p0, prev, B=B)
    res["loss"] = abs(out["loss"] - loss) / loss
    assert res["loss"] <= (1e-4 if bf else 1e-5)
    G = split_params(out["grads"].astype(np.float64), F, H)
    res["dM"] = scaled_err(G["M"].reshape(H, H), dM)
    assert res["dM"] <= tol
    res["dalpha3"] = abs(G["alpha"][2] - da3) / max(abs(da3), 1e-30)
    assert res["dalpha3"] <= tol
    Y3, _ = m.export_activations(3)
    res["dW3"] = scaled_err(G["W3"].reshape(H, H), Y3.astype(np.float64).T @ dZ3)
    assert res["dW3"] <= tol
    print(name, precision, res)
    m.free()
    g.free()
