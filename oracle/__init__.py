"""CPU oracle for the Mars DGI pre-training step -- TEST INFRASTRUCTURE ONLY.

Plain double-precision C (``mars_oracle.c``) behind a numpy/ctypes wrapper.  It
is the parity authority for the CUDA library and shares no code with it.  Only
``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package; the product package
``paper_conf_icpp_lancl21_b200`` never does.

Every function cites the passage of the paper (``P:Lnnn`` = line of PAPER.md)
it follows; readings of silent / garbled passages are ``c<k>`` in DESIGN.md §3.
Parity pins live in ``tests/test_oracle_*.py``.  Parity unpinned: the
end-to-end learning curve (the paper prints no DGI loss values).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mars_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")
_lock = threading.Lock()
_libs = {}
_variant = "serial"

i32p = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
i64p = np.ctypeslib.ndpointer(dtype=np.int64, flags="C_CONTIGUOUS")
f32p = np.ctypeslib.ndpointer(dtype=np.float32, flags="C_CONTIGUOUS")
f64p = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")


def build(force: bool = False, variant: str = "serial") -> str:
    """Compile liboracle.so with gcc -O2 (no fast-math: IEEE double throughout);
    variant "omp": the same source with -fopenmp (liboracle_omp.so, for the
    multi-core CPU baseline; bitwise identical results)."""
    out = _LIB_OMP if variant == "omp" else _LIB
    if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(_SRC):
        tmp = out + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fno-fast-math",
                               "-ffp-contract=off"] + (["-fopenmp"] if variant == "omp" else []) +
                              ["-o", tmp, _SRC, "-lm"])
        os.replace(tmp, out)
    return out


def set_variant(variant: str) -> str:
    """Select the build every later call uses: "serial" (default) or "omp"
    (OpenMP over the outer loops; OMP_NUM_THREADS threads).  Returns the old one."""
    global _variant
    if variant not in ("serial", "omp"):
        raise ValueError(variant)
    old, _variant = _variant, variant
    return old


def lib():
    with _lock:
        if _variant not in _libs:
            L = ctypes.CDLL(build(variant=_variant))
            L.oracle_sm64.restype = ctypes.c_uint64
            L.oracle_sm64.argtypes = [ctypes.c_uint64]
            L.oracle_csr.restype = ctypes.c_int64
            L.oracle_csr.argtypes = [ctypes.c_int32, i64p, i32p, i32p, i32p, i32p, f32p, f32p]
            L.oracle_perm.restype = None
            L.oracle_perm.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                      ctypes.c_int32, i32p]
            L.oracle_xavier.restype = None
            L.oracle_xavier.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int32, f32p]
            L.oracle_forward.restype = None
            L.oracle_forward.argtypes = [ctypes.c_int32, i32p, i32p, i32p, ctypes.c_int32,
                                         ctypes.c_int32, f64p, i32p, f64p] + [f64p] * 6
            L.oracle_backward.restype = ctypes.c_double
            L.oracle_backward.argtypes = [ctypes.c_int32, i32p, i32p, i32p, ctypes.c_int32,
                                          ctypes.c_int32, ctypes.c_double, f64p] + [f64p] * 6 + \
                                         [f64p, ctypes.c_void_p]
            L.oracle_encode.restype = None
            L.oracle_encode.argtypes = [ctypes.c_int32, i32p, i32p, i32p, ctypes.c_int32,
                                        ctypes.c_int32, f64p, f64p, f64p]
            L.oracle_adam.restype = None
            L.oracle_adam.argtypes = [ctypes.c_int64, f64p, f64p, f64p, f64p, ctypes.c_int64,
                                      ctypes.c_double, ctypes.c_double, ctypes.c_double,
                                      ctypes.c_double, ctypes.c_double]
            L.oracle_head.restype = ctypes.c_double
            L.oracle_head.argtypes = [ctypes.c_int32, i32p, ctypes.c_int32, ctypes.c_double, f64p,
                                      ctypes.c_double, f64p, f64p, f64p, f64p, f64p]
            L.oracle_spmm_rows.restype = None
            L.oracle_spmm_rows.argtypes = [ctypes.c_int32, i32p, i32p, ctypes.c_int32, f64p,
                                           ctypes.c_double, ctypes.c_int64, i64p, f64p]
            L.oracle_prelu_backward.restype = ctypes.c_double
            L.oracle_prelu_backward.argtypes = [ctypes.c_int64, f64p, f64p, ctypes.c_double, f64p]
            L.oracle_featurize.restype = ctypes.c_int
            L.oracle_featurize.argtypes = [ctypes.c_int32, ctypes.c_int32, i32p, i64p, f32p]
            L.oracle_dense_anorm.restype = None
            L.oracle_dense_anorm.argtypes = [ctypes.c_int32, i32p, f64p]
            L.oracle_dense_step.restype = ctypes.c_double
            L.oracle_dense_step.argtypes = [ctypes.c_int32, i32p, ctypes.c_int32, ctypes.c_int32,
                                            f64p, i32p, f64p, f64p, ctypes.c_void_p]
            _libs[_variant] = L
    return _libs[_variant]


def num_params(F: int, H: int) -> int:
    """Flat layout [W1 F×H | W2 H×H | W3 H×H | M H×H | a1 a2 a3]."""
    return F * H + 3 * H * H + 3


def sm64(z: int) -> int:
    return int(lib().oracle_sm64(ctypes.c_uint64(z & 0xFFFFFFFFFFFFFFFF)))


# --------------------------------------------------------------------------- a2/a3
class CSR:
    """Â = A ∨ Aᵀ + I (binary) in CSR with degrees and the f32 normalisation values
    (Eq. 1; readings c1-c4)."""

    def __init__(self, rowptr, colind, deg, dinv, vals):
        self.rowptr, self.colind, self.deg, self.dinv, self.vals = rowptr, colind, deg, dinv, vals

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])


def csr(num_nodes: int, indptr, indices) -> CSR:
    N = int(num_nodes)
    indptr = np.ascontiguousarray(indptr, dtype=np.int64)
    indices = np.ascontiguousarray(indices, dtype=np.int32)
    cap = N + 2 * int(indptr[N]) + 1
    rowptr = np.zeros(N + 1, np.int32)
    colind = np.zeros(cap, np.int32)
    deg = np.zeros(N, np.int32)
    dinv = np.zeros(N, np.float32)
    vals = np.zeros(cap, np.float32)
    z = lib().oracle_csr(N, indptr, indices, rowptr, colind, deg, dinv, vals)
    return CSR(rowptr, colind[:z].copy(), deg, dinv, vals[:z].copy())


# --------------------------------------------------------------------------- a4
def perm(seed: int, step: int, pair: int, num_nodes: int) -> np.ndarray:
    """π for one (graph, sample) pair (Eq. 2; reading c12)."""
    out = np.zeros(max(int(num_nodes), 1), np.int32)
    lib().oracle_perm(ctypes.c_uint64(seed & (2**64 - 1)), ctypes.c_uint64(step & (2**64 - 1)),
                      ctypes.c_uint64(pair & (2**64 - 1)), int(num_nodes), out)
    return out[:num_nodes]


def featurize(types, dims, F: int) -> np.ndarray:
    """NEXT-1 featuriser (reading c16): X [N x F] from op types [N] and
    shape dims [N x 8] (first input's 4, output's 4; <= 0 unknown)."""
    types = np.ascontiguousarray(types, np.int32)
    dims = np.ascontiguousarray(dims, np.int64).reshape(-1, 8)
    X = np.zeros((types.size, F), np.float32)
    if lib().oracle_featurize(types.size, F, types, dims, X) != 0:
        raise ValueError("negative op type")
    return X


def xavier(seed: int, F: int, H: int) -> np.ndarray:
    """Default parameter init (reading c14)."""
    out = np.zeros(num_params(F, H), np.float32)
    lib().oracle_xavier(ctypes.c_uint64(seed & (2**64 - 1)), F, H, out)
    return out


# --------------------------------------------------------------------------- batch packing
class Batch:
    """G graphs packed block-diagonally (reading c15): node offsets, global CSR."""

    def __init__(self, graphs):
        """graphs: iterable of objects with num_nodes, indptr, indices, features."""
        self.graphs = list(graphs)
        self.G = len(self.graphs)
        self.node_off = np.zeros(self.G + 1, np.int32)
        rp, ci, Xs = [np.zeros(1, np.int32)], [], []
        self.csrs = []
        for g, gr in enumerate(self.graphs):
            c = csr(gr.num_nodes, gr.indptr, gr.indices)
            self.csrs.append(c)
            off = int(self.node_off[g])
            self.node_off[g + 1] = off + gr.num_nodes
            rp.append(c.rowptr[1:] + int(rp[-1][-1]))
            ci.append(c.colind + off)
            Xs.append(np.asarray(gr.features, np.float64).reshape(gr.num_nodes, -1))
        self.rowptr = np.ascontiguousarray(np.concatenate(rp), np.int32)
        self.colind = np.ascontiguousarray(np.concatenate(ci), np.int32)
        self.X = np.ascontiguousarray(np.concatenate(Xs, 0), np.float64)
        self.F = self.X.shape[1]
        self.Nt = int(self.node_off[-1])

    def perms(self, seed: int, step: int, pair_base: int) -> np.ndarray:
        """Concatenated local permutations; pair index = pair_base + g (c15)."""
        return np.ascontiguousarray(np.concatenate(
            [perm(seed, step, pair_base + g, gr.num_nodes) for g, gr in enumerate(self.graphs)]),
            np.int32)


# --------------------------------------------------------------------------- a5-a12
def forward(batch: Batch, H: int, params, perms):
    """Y_l, Z_l (l = 1..3) of both branches, stacked [pos; neg] (Eqs. 1-3)."""
    F, Nt = batch.F, batch.Nt
    R = 2 * Nt
    p = np.ascontiguousarray(params, np.float64)
    Y1 = np.zeros((R, F)); Z1 = np.zeros((R, H))
    Y2 = np.zeros((R, H)); Z2 = np.zeros((R, H))
    Y3 = np.zeros((R, H)); Z3 = np.zeros((R, H))
    lib().oracle_forward(batch.G, batch.node_off, batch.rowptr, batch.colind, F, H, batch.X,
                         np.ascontiguousarray(perms, np.int32), p, Y1, Z1, Y2, Z2, Y3, Z3)
    return dict(Y1=Y1, Z1=Z1, Y2=Y2, Z2=Z2, Y3=Y3, Z3=Z3)


def backward(batch: Batch, H: int, params, acts, B: float | None = None):
    """Loss (Eq. 6 as c8), s_g (Eq. 4) and gradients at the given activations."""
    F = batch.F
    p = np.ascontiguousarray(params, np.float64)
    grads = np.zeros(num_params(F, H))
    s = np.zeros((batch.G, H))
    a = {k: np.ascontiguousarray(v, np.float64) for k, v in acts.items()}
    loss = lib().oracle_backward(batch.G, batch.node_off, batch.rowptr, batch.colind, F, H,
                                 float(batch.G if B is None else B), p, a["Y1"], a["Z1"], a["Y2"],
                                 a["Z2"], a["Y3"], a["Z3"], grads, s.ctypes.data)
    return loss, grads, s


def step_grads(batch: Batch, H: int, params, perms, B: float | None = None):
    acts = forward(batch, H, params, perms)
    loss, grads, s = backward(batch, H, params, acts, B)
    return loss, grads, s, acts


def head(batch: Batch, H: int, params, Z3, B: float | None = None):
    """Head only (a8-a11) at the given Z3: loss, s [G×H], dM [H×H], dZ3, dalpha3."""
    F = batch.F
    p = np.ascontiguousarray(params, np.float64)
    M = np.ascontiguousarray(p[F * H + 2 * H * H:F * H + 3 * H * H])
    a3 = float(p[-1])
    Z3 = np.ascontiguousarray(Z3, np.float64)
    s = np.zeros((batch.G, H)); dM = np.zeros((H, H)); dZ3 = np.zeros_like(Z3)
    da = np.zeros(1)
    loss = lib().oracle_head(batch.G, batch.node_off, H, float(batch.G if B is None else B), M, a3,
                             Z3, s, dM, dZ3, da)
    return loss, s, dM, dZ3, float(da[0])


def layer1_input(batch: Batch, perms) -> np.ndarray:
    """T0 = [X; X~] with X~[i] = X[off_g + pi[i]] (Eq. 2), stacked as the GPU does."""
    perms = np.asarray(perms, np.int64)
    gid = np.repeat(np.arange(batch.G), np.diff(batch.node_off))
    src = batch.node_off[gid].astype(np.int64) + perms
    return np.ascontiguousarray(np.concatenate([batch.X, batch.X[src]], 0))


def spmm_rows(batch: Batch, T, rows, alpha=None) -> np.ndarray:
    """Rows `rows` (stacked ids) of Â_n · act(T), act = PReLU_alpha or identity."""
    T = np.ascontiguousarray(T, np.float64)
    rows = np.ascontiguousarray(rows, np.int64)
    out = np.zeros((rows.size, T.shape[1]))
    lib().oracle_spmm_rows(batch.Nt, batch.rowptr, batch.colind, T.shape[1], T,
                           float("nan") if alpha is None else float(alpha), rows.size, rows, out)
    return out


def prelu_backward(dH, Z, alpha: float):
    """Row a12's PReLU stage (c6): (dZ = dH ⊙ PReLU'(Z), Σ_{Z<=0} dH·Z)."""
    dH = np.ascontiguousarray(dH, np.float64)
    Z = np.ascontiguousarray(Z, np.float64)
    assert dH.shape == Z.shape
    dZ = np.zeros_like(dH)
    da = lib().oracle_prelu_backward(dH.size, dH, Z, float(alpha), dZ)
    return dZ, float(da)


def encode(batch: Batch, H: int, params) -> np.ndarray:
    out = np.zeros((batch.Nt, H))
    lib().oracle_encode(batch.G, batch.node_off, batch.rowptr, batch.colind, batch.F, H, batch.X,
                        np.ascontiguousarray(params, np.float64), out)
    return out


def adam(params, m, v, grads, t, lr=1e-3, b1=0.9, b2=0.999, eps=1e-8, clip=0.0):
    """In-place torch.optim.Adam step (a14, reading c13).  Returns (params, m, v)."""
    p = np.ascontiguousarray(params, np.float64).copy()
    m = np.ascontiguousarray(m, np.float64).copy()
    v = np.ascontiguousarray(v, np.float64).copy()
    g = np.ascontiguousarray(grads, np.float64)
    lib().oracle_adam(p.size, p, m, v, g, int(t), lr, b1, b2, eps, clip)
    return p, m, v


# --------------------------------------------------------------------------- dense mode
def dense_adjacency(num_nodes: int, indptr, indices) -> np.ndarray:
    A = np.zeros((num_nodes, num_nodes), np.int32)
    for u in range(num_nodes):
        for e in range(int(indptr[u]), int(indptr[u + 1])):
            A[u, int(indices[e])] += 1
    return A


def dense_anorm(adj: np.ndarray) -> np.ndarray:
    N = adj.shape[0]
    out = np.zeros((N, N))
    lib().oracle_dense_anorm(N, np.ascontiguousarray(adj, np.int32), out)
    return out


def dense_step(adj, X, perm_, params, H):
    """Single-graph step with dense Â_n (tiny graphs only).  Returns loss, grads, emb."""
    adj = np.ascontiguousarray(adj, np.int32)
    X = np.ascontiguousarray(X, np.float64)
    N, F = X.shape
    grads = np.zeros(num_params(F, H))
    emb = np.zeros((N, H))
    loss = lib().oracle_dense_step(N, adj, F, H, X, np.ascontiguousarray(perm_, np.int32),
                                   np.ascontiguousarray(params, np.float64), grads, emb.ctypes.data)
    return loss, grads, emb
