"""NEXT-3 on the GPU: the PPO loss of teacher-forced placements and its
gradient through the placer (mars_placer_ppo_grad: BPTT through the attention
decoder and the segment-carried bi-LSTM encoder) against the torch fp64
autograd oracle (oracle/ppo.py; §3.4, readings c29-c31): loss,
every parameter block and dL/d embeddings at the scaled max-norm 1e-5."""
import numpy as np
import pytest

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
