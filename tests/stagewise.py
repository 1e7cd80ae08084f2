"""Stage-wise parity of one whole DGI step at sizes too large for the oracle
end to end (protocol P2/P3), shared by the bench-configuration
and full-size GPU tests.

Every stage is compared against the oracle evaluated at the GPU's own inputs
of that stage (exported through the test hooks), so one rounding-level
difference upstream cannot flip a PReLU branch downstream (reading c19):

  forward  Y_l rows      oracle.spmm_rows(GPU act(Z_{l-1}))        sampled rows
           Z_l rows      Y_l(GPU) · W_l                            sampled rows
  head     loss, dM      oracle.head(GPU Z3)
           dZ3           oracle.head(GPU Z3)                       all rows
           dalpha3       oracle.head(GPU Z3)
  layer l  dW_l          Y_l(GPU)ᵀ · dZ_l(GPU)                     all rows
           dY_l          dZ_l(GPU) · W_lᵀ                          all rows (l = 3, 2)
           dZ_{l-1}      oracle.prelu_backward(oracle.spmm_rows(dY_l(GPU)), Z_{l-1}(GPU))
           dalpha_{l-1}  the same call's sum                       all rows

Matrices use the scaled max-norm max|gpu - ref| / max|ref|; the scalars
(loss, dalpha_l) their relative error |gpu - ref| / |ref| (key "dalpha<l>").
The dalpha_l are sums over 2ΣN·H terms of both signs, so their error is also
reported against Σ|dH·min(Z,0)|, the sum's own scale ("dalpha<l>_cond",
diagnostic only).
"""
import numpy as np

import oracle
from tests.util import split_params

CHUNK = 1 << 16


def bf16_round(W):
    """Round-to-nearest-even to bf16, returned as float64 (the bf16 path's weights)."""
    w = np.ascontiguousarray(W, np.float32).view(np.uint32).astype(np.uint64)
    w = ((w + 0x7FFF + ((w >> 16) & 1)) & 0xFFFF0000).astype(np.uint32)
    return w.view(np.float32).astype(np.float64)


class _MaxErr:
    """Scaled max-norm accumulated over row chunks."""

    def __init__(self):
        self.num = 0.0
        self.den = 0.0

    def add(self, got, ref):
        self.num = max(self.num, float(np.max(np.abs(np.asarray(got, np.float64) - ref))))
        self.den = max(self.den, float(np.max(np.abs(ref))))

    @property
    def err(self):
        return self.num / max(self.den, 1e-30)


def _scaled(got, ref):
    e = _MaxErr()
    e.add(got, ref)
    return e.err


def step_stagewise(m, g, gs, F, H, seed, step, base, B, bf16, tol, nrows=300, rng_seed=0):
    """Runs one step of model m (fresh: parameters = its init) on graph set g
    (= the graphs gs) with the backward intermediates kept, and checks every
    stage.  Returns the dict of measured errors."""
    b = oracle.Batch(gs)
    m.set_keep_backward(True)
    p0 = m.get_state()[0].astype(np.float64)
    out = m.step(g, step, base, global_batch=B, want_loss=True, want_grads=True, want_perms=True)
    perms = b.perms(seed, step, base)
    assert np.array_equal(out["perms"], perms)
    P = split_params(p0, F, H)
    Wm = {l: P[f"W{l}"].reshape(-1, H) for l in (1, 2, 3)}
    if bf16:                                   # the bf16 GEMMs consume bf16(W)
        Wm = {l: bf16_round(w) for l, w in Wm.items()}
    alpha = P["alpha"]
    Nt = b.Nt
    R = 2 * Nt
    rng = np.random.default_rng(rng_seed)
    rows = np.unique(np.concatenate([rng.integers(0, R, nrows), [0, Nt - 1, Nt, R - 1]]))
    res = {}

    # ---- forward, sampled rows (P2 stage-wise)
    prev = oracle.layer1_input(b, perms)
    for l in (1, 2, 3):
        Y, Z = m.export_activations(l)
        y = oracle.spmm_rows(b, prev, rows, None if l == 1 else alpha[l - 2])
        res[f"Y{l}"] = _scaled(Y[rows], y)
        res[f"Z{l}"] = _scaled(Z[rows], Y[rows].astype(np.float64) @ Wm[l])
        prev = Z
    del prev, Y, Z

    # ---- head from the GPU's Z3
    _, Z3 = m.export_activations(3)
    loss, s, dM, dZ3_ref, da3 = oracle.head(b, H, p0, Z3, B=B)
    G = split_params(out["grads"].astype(np.float64), F, H)   # fp64: no float32 promotion below
    res["loss"] = abs(out["loss"] - loss) / abs(loss)
    res["dM"] = _scaled(G["M"].reshape(H, H), dM)
    _, dZ = m.export_backward(3)
    res["dZ3"] = _scaled(dZ, dZ3_ref)
    terms = np.abs(np.minimum(Z3.astype(np.float64), 0.0) * (dZ3_ref / np.where(Z3 > 0, 1.0, alpha[2])))
    res["dalpha3"] = abs(G["alpha"][2] - da3) / max(abs(da3), 1e-30)
    res["dalpha3_cond"] = abs(G["alpha"][2] - da3) / max(float(terms.sum()), 1e-30)
    del dZ3_ref, terms, Z3

    # ---- layers 3, 2, 1: dW, dY, aggregation + PReLU' (all rows, chunked)
    all_rows = np.arange(R, dtype=np.int64)
    for l in (3, 2, 1):
        Y, _ = m.export_activations(l)
        dw = np.zeros((Y.shape[1], H))
        for r0 in range(0, R, CHUNK):
            dw += Y[r0:r0 + CHUNK].astype(np.float64).T @ dZ[r0:r0 + CHUNK].astype(np.float64)
        res[f"dW{l}"] = _scaled(G[f"W{l}"].reshape(-1, H), dw)
        del Y
        if l == 1:
            break
        dY, _ = m.export_backward(l)
        e = _MaxErr()
        for r0 in range(0, R, CHUNK):
            e.add(dY[r0:r0 + CHUNK], dZ[r0:r0 + CHUNK].astype(np.float64) @ Wm[l].T)
        res[f"dY{l}"] = e.err
        dY64 = dY.astype(np.float64)
        del dY
        _, dZn = m.export_backward(l - 1)
        _, Zp = m.export_activations(l - 1)
        e = _MaxErr()
        da, mag = 0.0, 0.0
        for r0 in range(0, R, CHUNK):
            rr = all_rows[r0:r0 + CHUNK]
            dH = oracle.spmm_rows(b, dY64, rr)
            z = Zp[r0:r0 + CHUNK].astype(np.float64)
            dz_ref, part = oracle.prelu_backward(dH, z, alpha[l - 2])
            e.add(dZn[r0:r0 + CHUNK], dz_ref)
            da += part
            mag += float(np.sum(np.abs(dH * np.minimum(z, 0.0))))
        res[f"dZ{l - 1}"] = e.err
        res[f"dalpha{l - 1}"] = abs(G["alpha"][l - 2] - da) / max(abs(da), 1e-30)
        res[f"dalpha{l - 1}_cond"] = abs(G["alpha"][l - 2] - da) / max(mag, 1e-30)
        del dY64, Zp
        dZ = dZn
    m.set_keep_backward(False)
    print({k: f"{v:.2e}" for k, v in res.items()})
    loss_tol = 1e-4 if bf16 else tol
    for k, v in res.items():
        if k.endswith("_cond"):
            continue
        assert v <= (loss_tol if k == "loss" else tol), (k, v, res)
    return res
