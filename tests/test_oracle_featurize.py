"""Pins for the oracle's featuriser (NEXT-1, reading c16): the
hand-derived worked examples of tests/golden/featurize_example.json, and the
invariants every X must satisfy (one 1 per row in the type slots, shape slots
in [0, 1] with the graph's largest dim mapping to exactly 1)."""
import json
import os

import numpy as np
import pytest

import oracle
from synth import graphs as SG

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_featurize_golden():
    with open(os.path.join(GOLDEN, "featurize_example.json")) as f:
        gold = json.load(f)
    for case in gold["cases"]:
        X = oracle.featurize(case["types"], case["dims"], case["F"])
        assert X.tobytes() == np.array(case["X"], np.float32).tobytes(), case["note"]


@pytest.mark.parametrize("name", ["tiny", "inception", "gnmt", "bert"])
def test_featurize_invariants_and_generator_agreement(name):
    g = SG.cached(name, 0)
    F = g.feat_dim
    X = oracle.featurize(g.types, g.dims, F)
    assert np.all(X[:, :F - 8].sum(1) == 1.0)
    assert np.all((X[:, F - 8:] >= 0) & (X[:, F - 8:] <= 1))
    assert np.any(X[:, F - 8:] == 1.0)                  # the largest dim maps to 1
    # the input generator synthesises the paper's X with the same reading (c16)
    assert X.tobytes() == np.ascontiguousarray(g.features, np.float32).tobytes()


def test_featurize_rejects_negative_type():
    with pytest.raises(ValueError):
        oracle.featurize([0, -1], np.zeros((2, 8)), 16)
