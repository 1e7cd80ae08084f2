"""Shared test helpers (comparison metric of DESIGN.md §6)."""
import numpy as np


def scaled_err(got, ref) -> float:
    """max|got - ref| / max(max|ref|, 1e-30): the scaled max-norm of DESIGN.md §6."""
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    if ref.size == 0:
        return 0.0
    return float(np.max(np.abs(got - ref)) / max(float(np.max(np.abs(ref))), 1e-30))


def split_params(p, F, H):
    p = np.asarray(p)
    o = 0
    out = {}
    for name, n in (("W1", F * H), ("W2", H * H), ("W3", H * H), ("M", H * H), ("alpha", 3)):
        out[name] = p[o:o + n]
        o += n
    return out
