"""Pins for the PPO oracle (NEXT-3, oracle/ppo.py; §3.4 Eq. 7, P:L237;
readings c29-c31): Eq. 7 on a hand-evaluated sequence, the step-time model on
a hand-evaluated graph, the torch placer equal to the numpy placer, the
surrogate's special cases, and finite differences of the loss."""
import math

import numpy as np
import torch

from oracle import placer as PL
from oracle import ppo

SMALL = dict(H=8, Hd=4, A=6, De=3, D=3)


def test_eq7_hand_sequence():
    A, B = ppo.advantages([1.0, 4.0, 9.0], mu=0.99)
    # R = -1, -2, -3; B1 = R1; B2 = .01 R2 + .99 B1; B3 = .01 R3 + .99 B2
    B2 = 0.01 * -2 + 0.99 * -1
    B3 = 0.01 * -3 + 0.99 * B2
    assert A[0] == 0.0
    assert abs(A[1] - (-2 - B2)) < 1e-15 and abs(A[2] - (-3 - B3)) < 1e-15
    assert abs(B - B3) < 1e-15
    A2, _ = ppo.advantages([16.0], B_prev=B)           # the baseline carries over steps
    assert abs(A2[0] - (-4 - (0.01 * -4 + 0.99 * B3))) < 1e-15


def test_step_time_hand_case():
    """3 ops 0 -> 1 -> 2; outputs of 1000, 2000, 3000 elements."""
    dims = np.zeros((3, 8), np.int64)
    dims[:, 4] = [1000, 2000, 3000]
    indptr = np.array([0, 1, 2, 2]); indices = np.array([1, 2])
    # all on device 0: compute only
    assert abs(ppo.step_time([0, 0, 0], dims, indptr, indices, 2, 1e9) - 6000e-12) < 1e-24
    # op 2 on device 1: it receives op 1's 8000 bytes
    t = ppo.step_time([0, 0, 1], dims, indptr, indices, 2, 1e9)
    assert abs(t - max(3000e-12, 3000e-12 + 8000 / 12e9)) < 1e-24
    # capacity below one device's resident bytes: out of memory, 100 s
    assert ppo.step_time([0, 0, 0], dims, indptr, indices, 2, 20000.0) == 100.0


def _case(N=9, s=4, S=2, seed=3):
    params = PL.init_params(seed, **SMALL).astype(np.float64)
    E = np.random.default_rng(seed).standard_normal((N, SMALL["H"]))
    forced = np.random.default_rng(seed + 1).integers(0, SMALL["D"], (S, N))
    return params, E, forced, s


def test_torch_placer_equals_numpy_placer():
    params, E, forced, s = _case()
    _, logp, ent, _ = PL.decode(E, PL.unpack(params, **SMALL), s, SMALL["D"], 2, 0, forced=forced)
    lp, en = ppo.placer_logp(torch.tensor(E), torch.tensor(params), SMALL, s, forced)
    assert np.max(np.abs(lp.detach().numpy() - logp)) < 1e-13
    assert np.max(np.abs(en.detach().numpy() - ent)) < 1e-13


def test_surrogate_special_cases():
    """rho = 1 (new = old): L = -mean(A) - c mean(H), and dL/dlog pi = -A / n."""
    lp = torch.tensor([[-1.0, -2.0], [-0.5, -1.5]], dtype=torch.float64, requires_grad=True)
    ent = torch.tensor([[1.0, 1.1], [0.9, 1.2]], dtype=torch.float64)
    adv = [0.5, -2.0]
    L = ppo.ppo_loss(lp, lp.detach().numpy(), ent, adv, c_ent=0.001)
    assert abs(float(L) - (-(0.5 * 2 - 2.0 * 2) / 4 - 0.001 * 4.2 / 4)) < 1e-15
    L.backward()
    assert np.allclose(lp.grad.numpy(), -np.array([[0.5, 0.5], [-2.0, -2.0]]) / 4, atol=1e-15)
    # clipped: rho = e^0.5 > 1.2 with A > 0 -> no gradient through that op
    lp2 = torch.tensor([[0.5]], dtype=torch.float64, requires_grad=True)
    ppo.ppo_loss(lp2, np.zeros((1, 1)), torch.zeros(1, 1, dtype=torch.float64), [1.0]).backward()
    assert float(lp2.grad[0, 0]) == 0.0


def test_ppo_gradients_finite_differences():
    params, E, forced, s = _case()
    _, logp_old, _, _ = PL.decode(E, PL.unpack(params, **SMALL), s, SMALL["D"], 2, 0, forced=forced)
    rng = np.random.default_rng(7)
    p1 = params + 0.05 * rng.standard_normal(params.size)       # ratios != 1, some clipped
    adv = [0.7, -1.3]
    L, gp, gE = ppo.ppo_grads(E, p1, SMALL, s, forced, logp_old, adv)
    h = 1e-6
    for i in rng.choice(params.size, 25, replace=False):
        q = p1.copy(); q[i] += h
        lp_ = ppo.ppo_grads(E, q, SMALL, s, forced, logp_old, adv)[0]
        q[i] -= 2 * h
        lm_ = ppo.ppo_grads(E, q, SMALL, s, forced, logp_old, adv)[0]
        assert abs((lp_ - lm_) / (2 * h) - gp[i]) < 1e-6 * max(1.0, abs(gp[i])), i
    for (r, c) in [(0, 0), (4, 3), (8, 7)]:
        Q = E.copy(); Q[r, c] += h
        lp_ = ppo.ppo_grads(Q, p1, SMALL, s, forced, logp_old, adv)[0]
        Q[r, c] -= 2 * h
        lm_ = ppo.ppo_grads(Q, p1, SMALL, s, forced, logp_old, adv)[0]
        assert abs((lp_ - lm_) / (2 * h) - gE[r, c]) < 1e-6 * max(1.0, abs(gE[r, c]))
