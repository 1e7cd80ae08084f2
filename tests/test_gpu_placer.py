"""NEXT-2 on the GPU: the segment-level seq2seq placer forward (mars_placer_*)
against the numpy fp64 oracle (oracle/placer.py; §3.3, readings
c22-c28):
  * parameter init bit-exact (c28);
  * teacher-forced: log pi and entropy of every op at 1e-5 (scaled max-norm);
  * sampled: every drawn device is the Gumbel-max choice of the ORACLE's logits
    for that op (the oracle evaluated along the GPU's own draws), except where
    the two best scores are within the logits' rounding (counted, must be 0 on
    these cases); log pi / entropy of the draws at 1e-5;
  * ragged last segment, one-op segments, one op, small and paper sizes;
  * the embeddings are the DGI encoder's own output (mars_encode)."""
import numpy as np
import pytest

import paper_conf_icpp_lancl21_b200 as mars
from oracle import placer as PL
from synth import graphs as SG
from tests.util import scaled_err

pytestmark = pytest.mark.gpu


def _embeddings(name="inception", H=256, idx=0):
    g = mars.graph_load([SG.cached(name, idx)])
    m = mars.dgi_create(in_dim=64, hidden_dim=H, seed=3)
    E = m.encode(g)
    m.free(); g.free()
    return E


@pytest.mark.parametrize("kw", [dict(in_dim=64, enc_hidden=64, attn_dim=128, dev_embed=8,
                                     num_devices=3, segment=16),
                                dict()])
def test_placer_init_bit_exact(kw):
    p = mars.placer_create(seed=11, **kw)
    dims = dict(H=kw.get("in_dim", 256), Hd=kw.get("enc_hidden", 256), A=kw.get("attn_dim", 512),
                De=kw.get("dev_embed", 64), D=kw.get("num_devices", 4))
    assert p.P == PL.num_params(**dims)
    assert p.get_params().tobytes() == PL.init_params(11, **dims).tobytes()


def _check(E, S, seed, sample_seed, **kw):
    p = mars.placer_create(seed=seed, in_dim=E.shape[1], **kw)
    dims = dict(H=E.shape[1], Hd=kw.get("enc_hidden", 256), A=kw.get("attn_dim", 512),
                De=kw.get("dev_embed", 64), D=kw.get("num_devices", 4))
    s = kw.get("segment", 128)
    P = PL.unpack(p.get_params(), **dims)
    place, logp, ent = p.sample(E, S, sample_seed)
    # the oracle along the GPU's own draws
    o_place, o_logp, o_ent, o_logits = PL.decode(E.astype(np.float64), P, s, dims["D"], S,
                                                 sample_seed, forced=place)
    res = {"logp": scaled_err(logp, o_logp), "entropy": scaled_err(ent, o_ent)}
    N = E.shape[0]
    ties = flips = 0
    for b in range(S):
        for i in range(N):
            sc = o_logits[b, i] + PL.gumbel(sample_seed, b, N, i, dims["D"])
            o = np.argsort(sc)[::-1]
            if sc[o[0]] - sc[o[1]] < 1e-4:
                ties += 1
            elif place[b, i] != o[0]:
                flips += 1
    res["flips"], res["ties"] = flips, ties
    # teacher forcing with fresh random devices: log pi / entropy of forced placements
    forced = np.random.default_rng(seed).integers(0, dims["D"], (S, N)).astype(np.int32)
    f_place, f_logp, f_ent = p.sample(E, S, sample_seed, forced=forced)
    assert np.array_equal(f_place, forced)
    _, of_logp, of_ent, _ = PL.decode(E.astype(np.float64), P, s, dims["D"], S, 0, forced=forced)
    res["forced_logp"] = scaled_err(f_logp, of_logp)
    res["forced_entropy"] = scaled_err(f_ent, of_ent)
    print(res)
    assert flips == 0 and res["logp"] <= 1e-5 and res["entropy"] <= 1e-5
    assert res["forced_logp"] <= 1e-5 and res["forced_entropy"] <= 1e-5
    # deterministic; the draw depends on the sample seed
    again = p.sample(E, S, sample_seed)[0]
    assert np.array_equal(again, place)
    if N * S > 20:
        assert not np.array_equal(p.sample(E, S, sample_seed + 1)[0], place)
    p.free()
    return res


def test_placer_small_ragged_segments():
    E = np.random.default_rng(0).standard_normal((150, 64)).astype(np.float32) * 0.5
    _check(E, 3, 5, 17, enc_hidden=64, attn_dim=128, dev_embed=8, num_devices=3, segment=16)


def test_placer_edge_shapes():
    rng = np.random.default_rng(1)
    for N, seg in ((1, 128), (7, 1), (33, 32)):
        E = rng.standard_normal((N, 32)).astype(np.float32)
        _check(E, 2, 6, 3, enc_hidden=64, attn_dim=128, dev_embed=4, num_devices=5, segment=seg)


def test_placer_paper_sizes_on_encoder_output():
    """P:L234 sizes (bi-LSTM 2 x 256 = 512, decoder 512, attention 512, s = 128),
    D = 4 devices, S = 4 samples, on an Inception-V3 op graph's embeddings."""
    E = _embeddings()
    _check(E, 4, 7, 99)


def test_placer_gnmt_graph():
    """A GNMT-4 op graph (~12k ops, 93 segments) at paper sizes, S = 2."""
    E = _embeddings("gnmt")
    _check(E, 2, 8, 41)


def test_placer_and_ppo_argument_validation():
    with pytest.raises(mars.MarsError):
        mars.placer_create(enc_hidden=48)                 # 64, 128 or 256 only
    with pytest.raises(mars.MarsError):
        mars.placer_create(num_devices=1)
    p = mars.placer_create(in_dim=32, enc_hidden=64, attn_dim=128, dev_embed=8, num_devices=3,
                           segment=8)
    E = np.zeros((10, 32), np.float32)
    with pytest.raises(mars.MarsError):
        p.sample(E, 33, 0)                                # 1..32 samples
    with pytest.raises(mars.MarsError):
        p.sample(E, 2, 0, forced=np.full((2, 10), 3))     # device outside [0, D)
    with pytest.raises(mars.MarsError):
        mars.ppo_create(p, samples_per_policy=3, policies=1, minibatches=2)   # 3 % 2 != 0
    enc = mars.dgi_create(in_dim=16, hidden_dim=64, seed=1)
    with pytest.raises(mars.MarsError):
        mars.ppo_create(p, enc)                           # encoder H != placer in_dim
    o = mars.ppo_create(p, samples_per_policy=2, policies=1, minibatches=1, epochs=1)
    g = mars.graph_load([SG.tiny(0)])
    with pytest.raises(mars.MarsError):
        o.iteration_joint(g, SG.tiny(0))                  # created without an encoder
    assert mars.mars.lib().mars_placer_get_params(None, None) == mars.mars.MARS_ESTATE
    p.free()
