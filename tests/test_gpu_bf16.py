"""bf16 path (MARS_BF16: bf16 activation storage, bf16 tcgen05 MMAs, fp32
accumulation / fp32 master params) vs the fp64 oracle at BASELINE.json's bf16
bar, 2e-2 scaled max-norm:
  P1 permutations bit-exact;
  P2 forward end to end (Z_l, embeddings);
  P3 backward stage-wise at the GPU's own (bf16) activations; loss stage-wise.
"""
import numpy as np
import pytest

import oracle
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG
from tests import stagewise
from tests.util import scaled_err, split_params

pytestmark = pytest.mark.gpu
TOL = 2e-2


def _run(gs, F, H, seed, B=None):
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed, precision=mars.MARS_BF16)
    b = oracle.Batch(gs)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(g, 0, 0, global_batch=B or len(gs), want_loss=True, want_grads=True,
                 want_perms=True)
    return g, m, b, p0, out


def test_bf16_config_validation():
    with pytest.raises(mars.MarsError):
        mars.dgi_create(in_dim=16, hidden_dim=32, precision=mars.MARS_BF16)


@pytest.mark.parametrize("name,H", [("gnmt", 256), ("bert", 256), ("inception", 128)])
def test_bf16_step(name, H):
    gs = [SG.cached(name, 0)]
    F = 64
    g, m, b, p0, out = _run(gs, F, H, 2)
    perms = b.perms(2, 0, 0)
    assert np.array_equal(out["perms"], perms)
    acts = {}
    for l in (1, 2, 3):
        acts[f"Y{l}"], acts[f"Z{l}"] = m.export_activations(l)
    ref = oracle.forward(b, H, p0, perms)
    res = {}
    for k in ("Y1", "Z1", "Z2", "Z3"):
        res[k] = scaled_err(acts[k], ref[k])
        assert res[k] <= TOL, (k, res[k])
    loss_sw, grads_sw, _ = oracle.backward(b, H, p0, acts)
    res["loss"] = abs(out["loss"] - loss_sw) / abs(loss_sw)
    assert res["loss"] <= 1e-4
    for nm, blk in split_params(out["grads"], F, H).items():
        e = scaled_err(blk, split_params(grads_sw, F, H)[nm])
        res["P3_" + nm] = e
        assert e <= TOL, (nm, e)
    emb = m.encode(g)
    res["encode"] = scaled_err(emb, oracle.encode(b, H, m.get_state()[0].astype(np.float64)))
    assert res["encode"] <= TOL
    print("bf16", name, res)


def test_bf16_bench_config_stagewise():
    """The bench workload on the bf16 path: every stage of the step (forward
    rows, head, dZ / dY / dW / dalpha of all three layers) against the oracle
    at the GPU's own bf16 stage inputs, 2e-2 (tests/stagewise.py)."""
    gs = [SG.cached("gnmt", i) for i in range(16)]
    F, H = 64, 256
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=0, precision=mars.MARS_BF16)
    stagewise.step_stagewise(m, g, gs, F, H, 0, step=0, base=0, B=16, bf16=True, tol=TOL,
                             rng_seed=1)
    m.free(); g.free()


def test_bf16_training_decreases_loss():
    gs = [SG.cached("gnmt", 1)]
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=64, hidden_dim=256, seed=1, precision=mars.MARS_BF16)
    first = m.step(g, 0, 0, want_loss=True)["loss"]
    for s in range(1, 100):
        m.step(g, s, 0)
    last = m.step(g, 100, 0, want_loss=True)["loss"]
    assert np.isfinite(last) and last < first
