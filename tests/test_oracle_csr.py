"""Pins for the oracle's Â_n builder (Eq. 1; Â = A + I, D̂; c1-c4).

Each check is fixed by something other than the oracle itself: a brute-force
set construction, a hand-derived golden fixture, or a property of the
mathematics (symmetry, the sqrt(d) eigenvector, spectral radius 1).
"""
import json
import os

import numpy as np
import pytest

import oracle
from synth import graphs as SG

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _brute(N, indptr, indices):
    """Brute force from the definition: S = {(u,v),(v,u): u->v, u != v} ∪ {(i,i)}."""
    S = set((i, i) for i in range(N))
    for u in range(N):
        for e in range(indptr[u], indptr[u + 1]):
            v = int(indices[e])
            if u != v:
                S.add((u, v)); S.add((v, u))
    rows = [[] for _ in range(N)]
    for (u, v) in sorted(S):
        rows[u].append(v)
    return rows


def _random_digraph(rng, N, E, self_loops=True, dups=True):
    src = rng.integers(0, N, E)
    dst = rng.integers(0, N, E)
    if not self_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
    if dups and len(src):
        k = min(len(src), 5)
        src = np.concatenate([src, src[:k]]); dst = np.concatenate([dst, dst[:k]])
    o = np.argsort(src, kind="stable")
    src, dst = src[o], dst[o]
    indptr = np.zeros(N + 1, np.int64)
    np.add.at(indptr, src + 1, 1)
    return np.cumsum(indptr), dst.astype(np.int32)


CASES = [("tiny", SG.tiny(0)), ("tiny1", SG.tiny(1))]


@pytest.mark.parametrize("name,g", CASES)
def test_csr_matches_bruteforce(name, g):
    c = oracle.csr(g.num_nodes, g.indptr, g.indices)
    rows = _brute(g.num_nodes, g.indptr, g.indices)
    assert c.rowptr[0] == 0
    for i in range(g.num_nodes):
        assert list(c.colind[c.rowptr[i]:c.rowptr[i + 1]]) == rows[i]
        assert c.deg[i] == len(rows[i])
        assert c.dinv[i] == np.float32(1.0 / np.sqrt(np.float64(len(rows[i]))))
    for i in range(g.num_nodes):
        for k in range(c.rowptr[i], c.rowptr[i + 1]):
            j = c.colind[k]
            assert c.vals[k] == np.float32(1.0 / np.sqrt(np.float64(c.deg[i]) * np.float64(c.deg[j])))


@pytest.mark.parametrize("seed", range(8))
def test_csr_fuzz(seed):
    rng = np.random.default_rng(seed)
    N = int(rng.integers(1, 60))
    E = int(rng.integers(0, 4 * N))
    indptr, indices = _random_digraph(rng, N, E)
    c = oracle.csr(N, indptr, indices)
    rows = _brute(N, indptr, indices)
    got = [list(c.colind[c.rowptr[i]:c.rowptr[i + 1]]) for i in range(N)]
    assert got == rows


def test_csr_golden_path3():
    """Hand-derived fixture tests/golden/path3_csr.json (Eq. 1 on the path 0->1->2)."""
    with open(os.path.join(GOLDEN, "path3_csr.json")) as f:
        gold = json.load(f)
    c = oracle.csr(3, np.array(gold["indptr"]), np.array(gold["indices"], np.int32))
    assert list(c.rowptr) == gold["rowptr"]
    assert list(c.colind) == gold["colind"]
    assert list(c.deg) == gold["deg"]
    np.testing.assert_array_equal(c.vals, np.array(gold["vals_f32"], np.float32))


def test_no_edges_is_identity():
    c = oracle.csr(5, np.zeros(6, np.int64), np.zeros(0, np.int32))
    assert list(c.rowptr) == [0, 1, 2, 3, 4, 5]
    assert list(c.colind) == [0, 1, 2, 3, 4]
    assert np.all(c.vals == 1.0)


def test_single_node_self_loop_only():
    c = oracle.csr(1, np.array([0, 3], np.int64), np.array([0, 0, 0], np.int32))
    assert list(c.rowptr) == [0, 1] and list(c.colind) == [0] and c.deg[0] == 1


@pytest.mark.parametrize("name", ["tiny", "inception"])
def test_invariants(name):
    g = SG.make(name, 0)
    c = oracle.csr(g.num_nodes, g.indptr, g.indices)
    N = g.num_nodes
    assert np.all(np.diff(c.rowptr) >= 1)
    assert c.rowptr[-1] == c.deg.sum()
    for i in range(N):
        row = c.colind[c.rowptr[i]:c.rowptr[i + 1]]
        assert np.all(np.diff(row) > 0)                # strictly increasing
        assert i in set(row.tolist())                  # diagonal present
    # val_ij == val_ji bitwise (the formula is symmetric)
    pos = {}
    for i in range(N):
        for k in range(c.rowptr[i], c.rowptr[i + 1]):
            pos[(i, int(c.colind[k]))] = c.vals[k]
    for (i, j), v in pos.items():
        assert pos[(j, i)].tobytes() == v.tobytes()


def test_sqrt_degree_eigenvector_and_spectral_radius():
    """Â_n · sqrt(d) = sqrt(d) and rho(Â_n) = 1 (Â_n = D^-1/2 Â D^-1/2 is similar to
    the random-walk matrix D^-1 Â, whose rows sum to 1)."""
    g = SG.tiny(0)
    An = oracle.dense_anorm(oracle.dense_adjacency(g.num_nodes, g.indptr, g.indices))
    d = np.sum(An > 0, axis=1).astype(np.float64)
    sd = np.sqrt(d)
    np.testing.assert_allclose(An @ sd, sd, rtol=1e-14)
    ev = np.linalg.eigvalsh(An)
    assert abs(ev.max() - 1.0) < 1e-12 and ev.min() >= -1.0 - 1e-12


def test_dense_anorm_vs_csr():
    g = SG.tiny(2)
    An = oracle.dense_anorm(oracle.dense_adjacency(g.num_nodes, g.indptr, g.indices))
    c = oracle.csr(g.num_nodes, g.indptr, g.indices)
    D = np.zeros_like(An)
    for i in range(g.num_nodes):
        for k in range(c.rowptr[i], c.rowptr[i + 1]):
            D[i, c.colind[k]] = 1.0 / np.sqrt(float(c.deg[i]) * float(c.deg[c.colind[k]]))
    np.testing.assert_allclose(An, D, rtol=1e-15, atol=0)
