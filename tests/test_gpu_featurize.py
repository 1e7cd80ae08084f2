"""NEXT-1 featuriser on the GPU (mars_featurize) vs the oracle (P:L106,
reading c16): bit-exact on the hand-derived examples, on every generator's op
lists, and on edge cases (one op, no known dim, type overflow, huge dims)."""
import json
import os

import numpy as np
import pytest

import oracle
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_featurize_golden():
    with open(os.path.join(GOLDEN, "featurize_example.json")) as f:
        gold = json.load(f)
    for case in gold["cases"]:
        X = mars.featurize(case["types"], case["dims"], case["F"])
        assert X.tobytes() == np.array(case["X"], np.float32).tobytes(), case["note"]


@pytest.mark.parametrize("name", ["tiny", "inception", "gnmt", "bert"])
def test_featurize_matches_oracle(name):
    g = SG.cached(name, 0)
    F = g.feat_dim
    for FF in sorted({F, 64, 256}):
        got = mars.featurize(g.types, g.dims, FF)
        assert got.tobytes() == oracle.featurize(g.types, g.dims, FF).tobytes()


def test_featurize_edge_cases():
    rng = np.random.default_rng(0)
    cases = [([5], np.zeros((1, 8))),                                    # one op, no dims
             ([0, 100, 7], rng.integers(-3, 5, (3, 8))),                 # overflow type, unknowns
             (rng.integers(0, 60, 5000), rng.integers(1, 2 ** 40, (5000, 8)))]   # large dims
    for types, dims in cases:
        for F in (16, 32, 128):
            got = mars.featurize(types, dims, F)
            assert got.tobytes() == oracle.featurize(types, dims, F).tobytes()
    with pytest.raises(mars.MarsError):
        mars.featurize([0, -1], np.zeros((2, 8)), 16)
    with pytest.raises(mars.MarsError):
        mars.featurize([0], np.zeros((1, 8)), 24)
