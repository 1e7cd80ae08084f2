"""Pins for the corruption permutation (Eq. 2; reading c12)."""
import json
import os

import numpy as np
import pytest

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
M64 = (1 << 64) - 1


def test_splitmix64_reference_vectors():
    with open(os.path.join(GOLDEN, "splitmix64.json")) as f:
        gold = json.load(f)
    x = gold["seed"]
    for want in gold["outputs"]:
        assert oracle.sm64(x) == want
        x = (x + 0x9E3779B97F4A7C15) & M64


@pytest.mark.parametrize("N", [1, 2, 7, 64, 1000, 12345])
def test_perm_is_bijection(N):
    for step in range(3):
        p = oracle.perm(0, step, 5, N)
        assert sorted(p.tolist()) == list(range(N))


def test_perm_sorted_by_key_then_index():
    """pi lists node indices in ascending (key_i, i) order, key_i = sm64(k ^ i)."""
    seed, step, pair, N = 42, 7, 3, 500
    k = oracle.sm64(oracle.sm64(oracle.sm64(seed) ^ step) ^ pair)
    keys = [oracle.sm64(k ^ i) for i in range(N)]
    p = oracle.perm(seed, step, pair, N)
    seq = [(keys[i], i) for i in p]
    assert seq == sorted(seq)


def test_perm_depends_on_seed_step_pair():
    a = oracle.perm(1, 2, 3, 100)
    assert not np.array_equal(a, oracle.perm(1, 2, 4, 100))
    assert not np.array_equal(a, oracle.perm(1, 3, 3, 100))
    assert not np.array_equal(a, oracle.perm(2, 2, 3, 100))
    assert np.array_equal(a, oracle.perm(1, 2, 3, 100))


def test_perm_uniformity_chi2():
    """pi[0] and pi[N-1] are uniform over [0, N) across steps (statistical pin of
    'shuffles the features between nodes').  chi^2 with 7 dof, p < 1e-4
    threshold 29.9."""
    N, T = 8, 4000
    c0 = np.zeros(N); cl = np.zeros(N)
    for s in range(T):
        p = oracle.perm(99, s, 0, N)
        c0[p[0]] += 1; cl[p[-1]] += 1
    e = T / N
    assert ((c0 - e) ** 2 / e).sum() < 29.9
    assert ((cl - e) ** 2 / e).sum() < 29.9
