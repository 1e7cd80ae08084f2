"""Pins for the placer oracle (NEXT-2, oracle/placer.py; §3.3 P:L161-L172,
P:L234; readings c22-c28): torch.nn.LSTM / LSTMCell as independent LSTM
formulations, the segment-carry invariants, a hand-evaluated attention case,
the Gumbel-max draw against the softmax probabilities, and log pi / entropy
against torch.distributions.Categorical."""
import math

import numpy as np
import pytest
import torch

from oracle import placer as PL

SMALL = dict(H=16, Hd=8, A=12, De=4, D=3)


def _params(seed=1, **kw):
    kw = {**SMALL, **kw}
    return PL.unpack(PL.init_params(seed, **kw), **kw), kw


def test_init_bounds_and_layout():
    P, kw = _params()
    assert PL.num_params(**kw) == sum(v.size for v in P.values())
    assert np.all(np.abs(P["enc_f.W_hh"]) <= 1 / math.sqrt(kw["Hd"]))
    assert np.all(np.abs(P["dec.W_ih"]) <= 1 / math.sqrt(2 * kw["Hd"]))
    assert np.all(np.abs(P["emb"]) <= 1.0)
    assert abs(P["dec.W_hh"].std() - (1 / math.sqrt(2 * kw["Hd"])) / math.sqrt(3)) < 0.01


def test_encoder_one_segment_is_torch_bilstm():
    """With s >= N there is one segment: the encoder is a plain bidirectional LSTM
    (c22, c28), so it must equal torch.nn.LSTM(bidirectional=True) in float64."""
    P, kw = _params(seed=2)
    N = 37
    E = np.random.default_rng(0).standard_normal((N, kw["H"]))
    enc, init = PL.encoder(E, P, s=64)
    lstm = torch.nn.LSTM(kw["H"], kw["Hd"], bidirectional=True).double()
    with torch.no_grad():
        for sfx, d in (("", "enc_f"), ("_reverse", "enc_b")):
            getattr(lstm, "weight_ih_l0" + sfx).copy_(torch.tensor(P[d + ".W_ih"]))
            getattr(lstm, "weight_hh_l0" + sfx).copy_(torch.tensor(P[d + ".W_hh"]))
            getattr(lstm, "bias_ih_l0" + sfx).copy_(torch.tensor(P[d + ".b"]))
            getattr(lstm, "bias_hh_l0" + sfx).zero_()
        out, (hn, cn) = lstm(torch.tensor(E)[:, None, :])
    assert np.max(np.abs(enc - out[:, 0, :].numpy())) < 1e-13
    h0, c0 = init[0]
    assert np.max(np.abs(h0 - hn[:, 0, :].reshape(-1).numpy())) < 1e-13      # c24 bridge
    assert np.max(np.abs(c0 - cn[:, 0, :].reshape(-1).numpy())) < 1e-13


def test_segment_carry_invariants():
    """c23: the forward direction is one LSTM over all ops whatever the segment
    size; the backward direction of the LAST segment starts from the previous
    segment's final backward state, so it differs from a fresh start."""
    P, kw = _params(seed=3)
    N = 50
    E = np.random.default_rng(1).standard_normal((N, kw["H"]))
    Hd = kw["Hd"]
    enc1, _ = PL.encoder(E, P, s=N)
    enc2, init2 = PL.encoder(E, P, s=16)
    assert np.array_equal(enc1[:, :Hd], enc2[:, :Hd])
    assert len(init2) == 4
    # the last segment [48, 50) run from a zero backward state differs
    fresh, _ = PL.encoder(E[48:], P, s=16)
    assert not np.allclose(fresh[:, Hd:], enc2[48:, Hd:])
    # the first segment equals an independent run of its ops
    first, _ = PL.encoder(E[:16], P, s=16)
    assert np.array_equal(first, enc2[:16])


def test_attention_hand_case():
    """c25 with A = 1, two keys: e_k = v tanh(q + w_k . enc_k), softmax, ctx."""
    P = {"att.W_q": np.array([[0.5, -1.0]]), "att.W_k": np.array([[1.0, 2.0]]),
         "att.v": np.array([2.0])}
    enc = np.array([[0.1, 0.2], [-0.3, 0.4]])
    s_prev = np.array([1.0, 0.25])
    ctx, a = PL.attention(s_prev, enc, P)
    q = 0.5 * 1.0 - 1.0 * 0.25                         # 0.25
    e = [2.0 * math.tanh(q + 0.1 + 0.4), 2.0 * math.tanh(q - 0.3 + 0.8)]
    w = np.exp(np.array(e) - max(e))
    w /= w.sum()
    assert np.allclose(a, w, rtol=0, atol=1e-15)
    assert np.allclose(ctx, w @ enc, rtol=0, atol=1e-15)


def test_gumbel_max_follows_softmax():
    """c26: argmax(logit + g) over the counter-based Gumbel noise draws device d
    with probability softmax(logits)_d (chi-square over 20000 draws)."""
    z = np.array([0.3, -1.0, 1.2])
    p = np.exp(z - z.max()); p /= p.sum()
    n = 20000
    cnt = np.zeros(3)
    for i in range(n):
        cnt[int(np.argmax(z + PL.gumbel(99, 0, n, i, 3)))] += 1
    chi2 = float(np.sum((cnt - n * p) ** 2 / (n * p)))
    assert chi2 < 13.8                                 # p = 0.001 at 2 dof


def test_decoder_against_torch_formulation():
    """The teacher-forced decoder (c24-c26) written independently with
    torch.nn.LSTMCell and torch ops: logits, log pi and entropy agree."""
    P, kw = _params(seed=4)
    N, s, D, S = 21, 8, kw["D"], 2
    E = np.random.default_rng(2).standard_normal((N, kw["H"]))
    forced = np.random.default_rng(3).integers(0, D, (S, N))
    place, logp, ent, logits = PL.decode(E, P, s, D, S, 5, forced=forced)
    assert np.array_equal(place, forced)
    enc, init = PL.encoder(E, P, s)
    T = {k: torch.tensor(v) for k, v in P.items()}
    cell = torch.nn.LSTMCell(2 * kw["Hd"] + kw["De"], 2 * kw["Hd"]).double()
    with torch.no_grad():
        cell.weight_ih.copy_(T["dec.W_ih"]); cell.weight_hh.copy_(T["dec.W_hh"])
        cell.bias_ih.copy_(T["dec.b"]); cell.bias_hh.zero_()
        encT = torch.tensor(enc)
        for b in range(S):
            for j, j0 in enumerate(range(0, N, s)):
                j1 = min(N, j0 + s)
                h = torch.tensor(init[j][0])[None]; c = torch.tensor(init[j][1])[None]
                prev = D
                for i in range(j0, j1):
                    scores = torch.tanh(h @ T["att.W_q"].T + encT[j0:j1] @ T["att.W_k"].T) @ T["att.v"]
                    ctx = torch.softmax(scores, 0) @ encT[j0:j1]
                    h, c = cell(torch.cat([ctx, T["emb"][prev]])[None], (h, c))
                    z = (h @ T["out.W"].T + T["out.b"])[0]
                    dist = torch.distributions.Categorical(logits=z)
                    assert np.max(np.abs(z.numpy() - logits[b, i])) < 1e-13
                    assert abs(float(dist.log_prob(torch.tensor(forced[b, i]))) - logp[b, i]) < 1e-13
                    assert abs(float(dist.entropy()) - ent[b, i]) < 1e-13
                    prev = int(forced[b, i])


def test_sampled_placements_are_gumbel_argmax_of_own_logits():
    P, kw = _params(seed=6)
    N, D = 30, kw["D"]
    E = np.random.default_rng(4).standard_normal((N, kw["H"]))
    place, logp, ent, logits = PL.decode(E, P, 10, D, 3, 77)
    for b in range(3):
        for i in range(N):
            assert place[b, i] == int(np.argmax(logits[b, i] + PL.gumbel(77, b, N, i, D)))
    # teacher forcing with the sampled placements reproduces everything
    p2, lp2, e2, l2 = PL.decode(E, P, 10, D, 3, 123, forced=place)
    assert np.array_equal(p2, place) and np.array_equal(lp2, logp) and np.array_equal(l2, logits)
