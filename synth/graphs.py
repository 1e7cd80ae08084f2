"""Seeded synthetic DNN op graphs shaped like the paper's workloads.

This module is the ONE input source shared by the CPU oracle (tests) and the
CUDA path; it holds none of the method's arithmetic (no normalisation, no
permutation, no GCN).  It emits, per graph, the directed data-flow CSR
(row u lists the consumers v of u's output) and the per-op feature
matrix X (one-hot op type + input/output shapes normalised by the graph's
largest dimension; reading c16).

Construction (DESIGN.md §5 "input recipe"): a forward template per model, a
mechanical ``tf.gradients``-style backward (one gradient op per differentiable
input, AddN where a tensor has several consumers), then optimizer ops, ordered
by (locality key, phase, creation index) so that id ranges are local.
Workloads: Inception-V3 at batch 1, 299x299; GNMT-4 with 256
hidden units, T ~ U[20, 50], batch 256; BERT (24 layers, hidden 1024 per
BASELINE.json's "BERT-large-shaped", seq 384, batch 24).
"""
from __future__ import annotations

import os
from dataclasses import dataclass, field

import numpy as np

MASK64 = (1 << 64) - 1

# Fixed op-type table (<= 56 entries).  Types not listed fold into the last slot.
TYPE_TABLE = [
    "VariableV2", "Identity", "Const", "Placeholder", "StridedSlice", "GatherV2", "ConcatV2",
    "MatMul", "BiasAdd", "Split", "Sigmoid", "Tanh", "Add", "Mul", "Sub", "Conv2D",
    "FusedBatchNorm", "Relu", "MaxPool", "AvgPool", "Softmax", "BatchMatMul", "Reshape",
    "Transpose", "Mean", "SquaredDifference", "Rsqrt", "Pow", "RealDiv", "Sqrt", "Square", "Cast",
    "GreaterEqual", "RandomUniform", "SparseSoftmaxCrossEntropyWithLogits", "Squeeze", "Pack",
    "Fill", "AddN", "OnesLike", "AssignSub", "Assign", "ApplyAdam", "ApplyRMSProp",
    "Conv2DBackpropInput", "Conv2DBackpropFilter", "FusedBatchNormGrad", "ReluGrad",
    "SigmoidGrad", "TanhGrad", "BiasAddGrad", "MaxPoolGrad", "AvgPoolGrad", "SoftmaxGrad",
    "UnsortedSegmentSum", "Other",
]
TYPE_INDEX = {t: i for i, t in enumerate(TYPE_TABLE)}

# Gradient op type emitted for (forward type, input slot).
_GRAD_TYPE = {
    "Conv2D": ("Conv2DBackpropInput", "Conv2DBackpropFilter"),
    "FusedBatchNorm": "FusedBatchNormGrad", "Relu": "ReluGrad", "Sigmoid": "SigmoidGrad",
    "Tanh": "TanhGrad", "MaxPool": "MaxPoolGrad", "AvgPool": "AvgPoolGrad",
    "Softmax": "SoftmaxGrad", "BiasAdd": ("Identity", "BiasAddGrad"),
    "GatherV2": ("UnsortedSegmentSum", None), "Identity": "Identity", "Squeeze": "Reshape",
    "Pack": "StridedSlice", "ConcatV2": "StridedSlice", "Split": "ConcatV2", "Mean": "RealDiv",
    "SparseSoftmaxCrossEntropyWithLogits": "Mul", "Rsqrt": "Mul", "Pow": "Mul", "Square": "Mul",
    "SquaredDifference": "Mul", "RealDiv": "RealDiv", "Sqrt": "RealDiv",
}
# What a gradient op reads besides the incoming gradient.
_NEEDS_INPUTS = {"MatMul", "BatchMatMul", "Mul", "Conv2D", "FusedBatchNorm", "RealDiv", "Pow",
                 "Square", "SquaredDifference", "MaxPool", "GatherV2"}
_NEEDS_OUTPUT = {"Sigmoid", "Tanh", "Relu", "Softmax", "Rsqrt", "Sqrt", "MaxPool",
                 "SparseSoftmaxCrossEntropyWithLogits"}
_NO_GRAD = {"Const", "Placeholder", "Fill", "RandomUniform", "GreaterEqual", "Cast",
            "OnesLike", "AssignSub", "Assign", "ApplyAdam", "ApplyRMSProp", "VariableV2"}


def sm64(z: int) -> int:
    """splitmix64, used only to derive per-graph seeds (Appendix A.7 of SURVEY.md)."""
    z = (z + 0x9E3779B97F4A7C15) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def graph_seed(global_index: int) -> int:
    return sm64(0x6D617273 ^ int(global_index))


@dataclass
class OpGraph:
    name: str
    num_nodes: int
    indptr: np.ndarray          # int64 [N+1], directed data-flow CSR (u -> consumers)
    indices: np.ndarray         # int32 [E]
    features: np.ndarray        # float32 [N, F]
    types: np.ndarray = field(default=None)   # int32 [N] op-type index
    dims: np.ndarray = field(default=None)    # int64 [N, 8]: first input's 4 dims, own
                                              # output's 4 dims, 0 = unknown / absent

    @property
    def num_edges(self) -> int:
        return int(self.indptr[-1])

    @property
    def feat_dim(self) -> int:
        return int(self.features.shape[1])


class _Builder:
    """Accumulates ops: type, inputs (op ids), output shape, locality key, phase."""

    def __init__(self):
        self.type, self.inputs, self.shape, self.key, self.phase = [], [], [], [], []
        self.trainable = set()
        self.rg = []            # requires-grad flag per op

    def op(self, t, inputs=(), shape=(), key=(0, 0), phase=0):
        i = len(self.type)
        inputs = [int(x) for x in inputs]
        self.type.append(t)
        self.inputs.append(inputs)
        self.shape.append(tuple(int(s) for s in shape))
        self.key.append(tuple(key))
        self.phase.append(phase)
        rg = False
        if phase == 0 and t not in _NO_GRAD:
            if t == "Identity" and len(inputs) == 1 and inputs[0] in self.trainable:
                rg = True
            else:
                rg = any(self.rg[x] for x in inputs)
        self.rg.append(rg)
        return i

    def var(self, shape, key=(-1, 0), trainable=True):
        v = self.op("VariableV2", (), shape, key)
        if trainable:
            self.trainable.add(v)
        r = self.op("Identity", (v,), shape, key)
        return v, r

    def const(self, key, shape=()):
        return self.op("Const", (), shape, key)

    # -------------------------------------------------------------- backward
    def backward(self, loss):
        """Mechanical reverse pass: one gradient op per differentiable input of
        each forward op, AddN when a tensor has several consumers."""
        nf = len(self.type)
        contrib = [[] for _ in range(nf)]
        grad_of = {}
        for o in range(nf - 1, -1, -1):
            if not self.rg[o]:
                continue
            t = self.type[o]
            if o == loss:
                g = self.op("OnesLike", (o,), self.shape[o], self.key[o], 1)
            elif not contrib[o]:
                continue
            elif len(contrib[o]) == 1:
                g = contrib[o][0]
            else:
                g = self.op("AddN", contrib[o], self.shape[o], self.key[o], 1)
            grad_of[o] = g
            ins = self.inputs[o]
            for k, x in enumerate(ins):
                if not self.rg[x]:
                    continue
                gt = _GRAD_TYPE.get(t, t)
                if isinstance(gt, tuple):
                    gt = gt[min(k, len(gt) - 1)]
                    if gt is None:
                        continue
                reads = [g]
                if t in _NEEDS_INPUTS:
                    reads += [y for j, y in enumerate(ins) if j != k]
                if t in _NEEDS_OUTPUT:
                    reads.append(o)
                gid = self.op(gt, reads, self.shape[x], self.key[o], 1)
                contrib[x].append(gid)
        return grad_of

    # -------------------------------------------------------------- finish
    def finish(self, name, F, rng_types=None) -> OpGraph:
        N = len(self.type)
        order = sorted(range(N), key=lambda i: (self.key[i], self.phase[i], i))
        new_id = np.empty(N, np.int64)
        new_id[np.asarray(order, np.int64)] = np.arange(N)
        src, dst = [], []
        for v in range(N):
            for u in self.inputs[v]:
                src.append(new_id[u])
                dst.append(new_id[v])
        src = np.asarray(src, np.int64)
        dst = np.asarray(dst, np.int64)
        o = np.lexsort((dst, src))
        src, dst = src[o], dst[o]
        indptr = np.zeros(N + 1, np.int64)
        np.add.at(indptr, src + 1, 1)
        indptr = np.cumsum(indptr)
        types = np.array([TYPE_INDEX.get(self.type[i], len(TYPE_TABLE) - 1) for i in order], np.int32)
        in_shapes = [self.shape[self.inputs[i][0]] if self.inputs[i] else () for i in order]
        out_shapes = [self.shape[i] for i in order]
        X = featurize(types, in_shapes, out_shapes, F)
        return OpGraph(name, N, indptr, dst.astype(np.int32), X, types,
                       shape_dims(in_shapes, out_shapes))


def shape_dims(in_shapes, out_shapes):
    """[N, 8] int64: the first input's and the output's first 4 dims (0 = absent)."""
    N = len(in_shapes)
    dims = np.zeros((N, 8), np.int64)
    for i in range(N):
        for j, d in enumerate(tuple(in_shapes[i])[:4]):
            dims[i, j] = d
        for j, d in enumerate(tuple(out_shapes[i])[:4]):
            dims[i, 4 + j] = d
    return dims


def featurize(types, in_shapes, out_shapes, F):
    """One-hot op type in slots [0, F-8) (types beyond fold into the last slot),
    then 4 input dims and 4 output dims divided by the graph-wide largest
    dimension (reading c16).  Unknown dims are 0."""
    N = len(types)
    X = np.zeros((N, F), np.float32)
    nt = F - 8
    X[np.arange(N), np.minimum(np.asarray(types), nt - 1)] = 1.0
    dims = np.zeros((N, 8), np.float64)
    for i in range(N):
        for j, d in enumerate(tuple(in_shapes[i])[:4]):
            dims[i, j] = d
        for j, d in enumerate(tuple(out_shapes[i])[:4]):
            dims[i, 4 + j] = d
    mx = dims.max() if dims.size else 0.0
    if mx > 0:
        dims = dims / mx
    X[:, nt:] = dims.astype(np.float32)
    return X


# =========================================================================== tiny
def tiny(seed_index: int = 0, N: int = 64, F: int = 16) -> OpGraph:
    """Config 1: random layered DAG.  Node j picks k_j in {1,2,3} (p=.3/.4/.3)
    distinct predecessors from [max(0, j-8), j); op types uniform over 8; shapes
    random powers of two <= 256."""
    rng = np.random.default_rng(graph_seed(seed_index))
    types = rng.integers(0, 8, N).astype(np.int32)
    out_shapes = [tuple(int(2 ** rng.integers(0, 9)) for _ in range(int(rng.integers(1, 5))))
                  for _ in range(N)]
    src, dst, first_in = [], [], [None] * N
    for j in range(1, N):
        k = int(rng.choice([1, 2, 3], p=[0.3, 0.4, 0.3]))
        lo = max(0, j - 8)
        k = min(k, j - lo)
        preds = np.sort(rng.choice(np.arange(lo, j), size=k, replace=False))
        for p in preds:
            src.append(int(p)); dst.append(j)
        first_in[j] = int(preds[0])
    in_shapes = [out_shapes[first_in[j]] if first_in[j] is not None else () for j in range(N)]
    src = np.asarray(src, np.int64); dst = np.asarray(dst, np.int64)
    o = np.lexsort((dst, src))
    indptr = np.zeros(N + 1, np.int64)
    np.add.at(indptr, src[o] + 1, 1)
    X = featurize(types, in_shapes, out_shapes, F)
    return OpGraph("tiny", N, np.cumsum(indptr), dst[o].astype(np.int32), X, types,
                   shape_dims(in_shapes, out_shapes))


# =========================================================================== GNMT
def _lstm_cell(b, x, h, c, Wr, br, key, B, Hd):
    ax = b.const(key)
    cat = b.op("ConcatV2", (x, h, ax), (B, 2 * Hd), key)
    mm = b.op("MatMul", (cat, Wr), (B, 4 * Hd), key)
    ba = b.op("BiasAdd", (mm, br), (B, 4 * Hd), key)
    sd = b.const(key)
    sp = b.op("Split", (sd, ba), (B, Hd), key)
    i = b.op("Sigmoid", (sp,), (B, Hd), key)
    fb = b.const(key)
    fa = b.op("Add", (sp, fb), (B, Hd), key)
    f = b.op("Sigmoid", (fa,), (B, Hd), key)
    o = b.op("Sigmoid", (sp,), (B, Hd), key)
    g = b.op("Tanh", (sp,), (B, Hd), key)
    fc = b.op("Mul", (f, c), (B, Hd), key)
    ig = b.op("Mul", (i, g), (B, Hd), key)
    c2 = b.op("Add", (fc, ig), (B, Hd), key)
    tc = b.op("Tanh", (c2,), (B, Hd), key)
    h2 = b.op("Mul", (o, tc), (B, Hd), key)
    return h2, c2


def gnmt(seed_index: int = 0, F: int = 64, T: int | None = None, layers: int = 4,
         hidden: int = 256, batch: int = 256, vocab: int = 32000) -> OpGraph:
    """Config 3: GNMT-4 (4-layer LSTM encoder + 4-layer decoder with attention)
    unrolled over T ~ U[20, 50] steps, training graph with Adam."""
    rng = np.random.default_rng(graph_seed(seed_index))
    if T is None:
        T = int(rng.integers(20, 51))
    B, Hd = batch, hidden
    b = _Builder()
    g0 = (-1, 0)
    emb_e = b.var((vocab, Hd), g0)[1]
    emb_d = b.var((vocab, Hd), g0)[1]
    enc = [(b.var((2 * Hd, 4 * Hd), g0)[1], b.var((4 * Hd,), g0)[1]) for _ in range(layers)]
    dec = [(b.var((2 * Hd, 4 * Hd), g0)[1], b.var((4 * Hd,), g0)[1]) for _ in range(layers)]
    memW = b.var((Hd, Hd), g0)[1]
    attW = b.var((2 * Hd, Hd), g0)[1]
    projW = b.var((Hd, vocab), g0)[1]
    src_ids = b.op("Placeholder", (), (B, T), g0)
    tgt_ids = b.op("Placeholder", (), (B, T), g0)
    labels = b.op("Placeholder", (), (B, T), g0)
    zero = b.op("Fill", (), (B, Hd), g0)
    hs = [zero] * layers
    cs = [zero] * layers
    enc_out = []
    for t in range(T):
        key = (t, 0)
        ids = b.op("StridedSlice", (src_ids,), (B,), key)
        x = b.op("GatherV2", (emb_e, ids), (B, Hd), key)
        for L in range(layers):
            kL = (t, L)
            h2, c2 = _lstm_cell(b, x, hs[L], cs[L], enc[L][0], enc[L][1], kL, B, Hd)
            if L >= 2:
                h2r = b.op("Add", (h2, x), (B, Hd), kL)      # residual connection
            else:
                h2r = h2
            hs[L], cs[L] = h2, c2
            x = h2r
        enc_out.append(x)
    mem = b.op("Pack", enc_out, (B, T, Hd), (T, 0))                 # fan-in T hub
    keys = b.op("MatMul", (mem, memW), (B, T, Hd), (T, 0))
    hd = list(hs)
    cd = list(cs)
    att = zero
    losses = []
    for t in range(T):
        key = (T + 1 + t, 0)
        ids = b.op("StridedSlice", (tgt_ids,), (B,), key)
        e = b.op("GatherV2", (emb_d, ids), (B, Hd), key)
        ax = b.const(key)
        x = b.op("ConcatV2", (e, att, ax), (B, 2 * Hd), key)     # input feeding
        xin = b.op("MatMul", (x, dec[0][0]), (B, Hd), key) if False else x
        for L in range(layers):
            kL = (T + 1 + t, 1 + L)
            h2, c2 = _lstm_cell(b, xin if L else e, hd[L], cd[L], dec[L][0], dec[L][1], kL, B, Hd)
            h2r = b.op("Add", (h2, xin), (B, Hd), kL) if L >= 2 else h2
            hd[L], cd[L] = h2, c2
            xin = h2r
        kA = (T + 1 + t, 9)
        sc = b.op("BatchMatMul", (keys, xin), (B, T), kA)
        al = b.op("Softmax", (sc,), (B, T), kA)
        ctx = b.op("BatchMatMul", (al, mem), (B, Hd), kA)
        ax2 = b.const(kA)
        ch = b.op("ConcatV2", (ctx, xin, ax2), (B, 2 * Hd), kA)
        am = b.op("MatMul", (ch, attW), (B, Hd), kA)
        att = b.op("Tanh", (am,), (B, Hd), kA)
        lg = b.op("MatMul", (att, projW), (B, vocab), kA)
        lb = b.op("StridedSlice", (labels,), (B,), kA)
        ce = b.op("SparseSoftmaxCrossEntropyWithLogits", (lg, lb), (B,), kA)
        losses.append(ce)
    kl = (2 * T + 2, 0)
    tot = b.op("AddN", losses, (B,), kl)
    loss = b.op("Mean", (tot,), (), kl)
    grads = b.backward(loss)
    _adam_ops(b, grads, (2 * T + 3, 0))
    return b.finish("gnmt", F)


def _adam_ops(b, grads, key):
    """ApplyAdam per trainable variable: reads var, slots m and v, the shared
    lr / beta-power scalars (hubs) and the variable's gradient."""
    lr = b.op("Const", (), (), key)
    b1p = b.op("VariableV2", (), (), key)
    b2p = b.op("VariableV2", (), (), key)
    for v in sorted(b.trainable):
        read = v + 1                                           # var() emits the read next
        if read not in grads:
            continue
        m = b.op("VariableV2", (), b.shape[v], key)
        s = b.op("VariableV2", (), b.shape[v], key)
        b.op("ApplyAdam", (v, m, s, b1p, b2p, lr, grads[read]), b.shape[v], key, 2)
    b.op("Mul", (b1p,), (), key, 2)
    b.op("Mul", (b2p,), (), key, 2)


# =========================================================================== Inception-V3
def inception(seed_index: int = 0, F: int = 64) -> OpGraph:
    """Config 2: Inception-V3 training graph at batch 1, 299x299: stem,
    3x module A, B, 4x C, D, 2x E, aux head; 97 conv blocks; RMSProp."""
    rng = np.random.default_rng(graph_seed(seed_index))
    b = _Builder()
    blk = [0]

    def conv(x, cin, cout, k, hw, stride=1):
        key = (blk[0], 0)
        blk[0] += 1
        kh, kw = k
        w = b.var((kh, kw, cin, cout), key)[1]
        hw2 = (hw[0] // stride, hw[1] // stride)
        cv = b.op("Conv2D", (x, w), (1, hw2[0], hw2[1], cout), key)
        beta = b.var((cout,), key)[1]
        mmv, mmr = b.var((cout,), key, trainable=False)
        mvv, mvr = b.var((cout,), key, trainable=False)
        bn = b.op("FusedBatchNorm", (cv, beta, mmr, mvr), (1, hw2[0], hw2[1], cout), key)
        for var, rd in ((mmv, mmr), (mvv, mvr)):                # moving-average updates
            sub = b.op("Sub", (rd, bn), (cout,), key)
            dc = b.const(key)
            mu = b.op("Mul", (sub, dc), (cout,), key)
            b.op("AssignSub", (var, mu), (cout,), key)
        return b.op("Relu", (bn,), (1, hw2[0], hw2[1], cout), key), hw2

    def pool(x, kind, c, hw, stride):
        key = (blk[0], 1)
        hw2 = (hw[0] // stride, hw[1] // stride)
        return b.op(kind, (x,), (1, hw2[0], hw2[1], c), key), hw2

    def concat(xs, c, hw):
        key = (blk[0], 2)
        ax = b.const(key)
        return b.op("ConcatV2", list(xs) + [ax], (1, hw[0], hw[1], c), key)

    img = b.op("Placeholder", (), (1, 299, 299, 3), (-1, 0))
    hw = (299, 299)
    x, hw = conv(img, 3, 32, (3, 3), hw, 2)
    x, hw = conv(x, 32, 32, (3, 3), hw)
    x, hw = conv(x, 32, 64, (3, 3), hw)
    x, hw = pool(x, "MaxPool", 64, hw, 2)
    x, hw = conv(x, 64, 80, (1, 1), hw)
    x, hw = conv(x, 80, 192, (3, 3), hw)
    x, hw = pool(x, "MaxPool", 192, hw, 2)
    c = 192
    for pf in (32, 64, 64):                                        # module A x3
        b1, _ = conv(x, c, 64, (1, 1), hw)
        b2, _ = conv(x, c, 48, (1, 1), hw); b2, _ = conv(b2, 48, 64, (5, 5), hw)
        b3, _ = conv(x, c, 64, (1, 1), hw); b3, _ = conv(b3, 64, 96, (3, 3), hw)
        b3, _ = conv(b3, 96, 96, (3, 3), hw)
        b4, _ = pool(x, "AvgPool", c, hw, 1); b4, _ = conv(b4, c, pf, (1, 1), hw)
        c = 64 + 64 + 96 + pf
        x = concat((b1, b2, b3, b4), c, hw)
    b1, hw2 = conv(x, c, 384, (3, 3), hw, 2)                        # module B
    b2, _ = conv(x, c, 64, (1, 1), hw); b2, _ = conv(b2, 64, 96, (3, 3), hw)
    b2, _ = conv(b2, 96, 96, (3, 3), hw, 2)
    b3, _ = pool(x, "MaxPool", c, hw, 2)
    hw = hw2; c = 384 + 96 + c
    x = concat((b1, b2, b3), c, hw)
    aux_in = None
    for mid in (128, 160, 160, 192):                               # module C x4
        b1, _ = conv(x, c, 192, (1, 1), hw)
        b2, _ = conv(x, c, mid, (1, 1), hw); b2, _ = conv(b2, mid, mid, (1, 7), hw)
        b2, _ = conv(b2, mid, 192, (7, 1), hw)
        b3, _ = conv(x, c, mid, (1, 1), hw)
        for kk, co in (((7, 1), mid), ((1, 7), mid), ((7, 1), mid), ((1, 7), 192)):
            b3, _ = conv(b3, mid, co, kk, hw)
        b4, _ = pool(x, "AvgPool", c, hw, 1); b4, _ = conv(b4, c, 192, (1, 1), hw)
        c = 768
        x = concat((b1, b2, b3, b4), c, hw)
        aux_in = x
    a, ahw = pool(aux_in, "AvgPool", c, hw, 3)                      # aux head
    a, ahw = conv(a, c, 128, (1, 1), ahw)
    a, ahw = conv(a, 128, 768, (5, 5), ahw, 5)
    a, _ = conv(a, 768, 1001, (1, 1), ahw)
    b1, hw2 = conv(x, c, 192, (1, 1), hw); b1, _ = conv(b1, 192, 320, (3, 3), hw, 2)  # module D
    b2, _ = conv(x, c, 192, (1, 1), hw); b2, _ = conv(b2, 192, 192, (1, 7), hw)
    b2, _ = conv(b2, 192, 192, (7, 1), hw); b2, _ = conv(b2, 192, 192, (3, 3), hw, 2)
    b3, _ = pool(x, "MaxPool", c, hw, 2)
    hw = (hw[0] // 2, hw[1] // 2); c = 320 + 192 + c
    x = concat((b1, b2, b3), c, hw)
    for _ in range(2):                                             # module E x2
        b1, _ = conv(x, c, 320, (1, 1), hw)
        b2, _ = conv(x, c, 384, (1, 1), hw)
        b2a, _ = conv(b2, 384, 384, (1, 3), hw); b2b, _ = conv(b2, 384, 384, (3, 1), hw)
        b2 = concat((b2a, b2b), 768, hw)
        b3, _ = conv(x, c, 448, (1, 1), hw); b3, _ = conv(b3, 448, 384, (3, 3), hw)
        b3a, _ = conv(b3, 384, 384, (1, 3), hw); b3b, _ = conv(b3, 384, 384, (3, 1), hw)
        b3 = concat((b3a, b3b), 768, hw)
        b4, _ = pool(x, "AvgPool", c, hw, 1); b4, _ = conv(b4, c, 192, (1, 1), hw)
        c = 2048
        x = concat((b1, b2, b3, b4), c, hw)
    key = (blk[0], 3)
    x = b.op("AvgPool", (x,), (1, 1, 1, c), key)
    rnd = b.op("RandomUniform", (), (1, 1, 1, c), key)
    ge = b.op("GreaterEqual", (rnd,), (1, 1, 1, c), key)
    cst = b.op("Cast", (ge,), (1, 1, 1, c), key)
    x = b.op("Mul", (x, cst), (1, 1, 1, c), key)
    lw = b.var((1, 1, c, 1001), key)[1]
    lb = b.var((1001,), key)[1]
    lg = b.op("Conv2D", (x, lw), (1, 1, 1, 1001), key)
    lg = b.op("BiasAdd", (lg, lb), (1, 1, 1, 1001), key)
    lg = b.op("Squeeze", (lg,), (1, 1001), key)
    al = b.op("Squeeze", (a,), (1, 1001), key)
    lab = b.op("Placeholder", (), (1,), (-1, 0))
    l1 = b.op("SparseSoftmaxCrossEntropyWithLogits", (lg, lab), (1,), key)
    l2 = b.op("SparseSoftmaxCrossEntropyWithLogits", (al, lab), (1,), key)
    tot = b.op("AddN", (l1, l2), (1,), key)
    loss = b.op("Mean", (tot,), (), key)
    grads = b.backward(loss)
    okey = (blk[0] + 1, 0)
    lr = b.op("Const", (), (), okey)
    for v in sorted(b.trainable):                                  # RMSProp with slots
        if v + 1 not in grads:
            continue
        ms = b.op("VariableV2", (), b.shape[v], b.key[v])
        mom = b.op("VariableV2", (), b.shape[v], b.key[v])
        b.op("ApplyRMSProp", (v, ms, mom, lr, grads[v + 1]), b.shape[v], b.key[v], 2)
    del rng
    return b.finish("inception", F)


# =========================================================================== BERT
def bert(seed_index: int = 0, F: int = 64, layers: int = 24, hidden: int = 1024,
         seq: int = 384, batch: int = 24, heads: int = 16) -> OpGraph:
    """Config 4: BERT-large-shaped training graph (24 layers, hidden 1024, seq
    384, batch 24) with in-graph AdamWeightDecay (~12 ops per var)."""
    b = _Builder()
    Bs, S, Hd = batch, seq, hidden
    g0 = (-1, 0)
    ids = b.op("Placeholder", (), (Bs, S), g0)
    mask = b.op("Placeholder", (), (Bs, 1, 1, S), g0)
    emb = b.var((30522, Hd), g0)[1]
    pos = b.var((512, Hd), g0)[1]
    x = b.op("GatherV2", (emb, ids), (Bs * S, Hd), (0, 0))
    x = b.op("Add", (x, pos), (Bs * S, Hd), (0, 0))

    def dense(x, cin, cout, key):
        w = b.var((cin, cout), key)[1]
        bb = b.var((cout,), key)[1]
        m = b.op("MatMul", (x, w), (Bs * S, cout), key)
        return b.op("BiasAdd", (m, bb), (Bs * S, cout), key)

    def dropout(x, shp, key):
        r = b.op("RandomUniform", (), shp, key)
        ge = b.op("GreaterEqual", (r,), shp, key)
        c = b.op("Cast", (ge,), shp, key)
        sc = b.op("Mul", (x, b.const(key)), shp, key)
        return b.op("Mul", (sc, c), shp, key)

    def layernorm(x, key):
        shp = (Bs * S, Hd)
        g = b.var((Hd,), key)[1]
        be = b.var((Hd,), key)[1]
        mu = b.op("Mean", (x,), (Bs * S, 1), key)
        sd = b.op("SquaredDifference", (x, mu), shp, key)
        var = b.op("Mean", (sd,), (Bs * S, 1), key)
        ve = b.op("Add", (var, b.const(key)), (Bs * S, 1), key)
        rs = b.op("Rsqrt", (ve,), (Bs * S, 1), key)
        sc = b.op("Mul", (rs, g), shp, key)
        xm = b.op("Mul", (x, sc), shp, key)
        mm = b.op("Mul", (mu, sc), shp, key)
        sb = b.op("Sub", (be, mm), shp, key)
        return b.op("Add", (xm, sb), shp, key)

    x = layernorm(x, (0, 1))
    for L in range(layers):
        key = (L + 1, 0)
        dh = Hd // heads
        qkv = []
        for _ in range(3):
            d = dense(x, Hd, Hd, key)
            r = b.op("Reshape", (d,), (Bs, S, heads, dh), key)
            qkv.append(b.op("Transpose", (r,), (Bs, heads, S, dh), key))
        sc = b.op("BatchMatMul", (qkv[0], qkv[1]), (Bs, heads, S, S), key)
        sc = b.op("Mul", (sc, b.const(key)), (Bs, heads, S, S), key)
        sc = b.op("Add", (sc, mask), (Bs, heads, S, S), key)
        p = b.op("Softmax", (sc,), (Bs, heads, S, S), key)
        p = dropout(p, (Bs, heads, S, S), key)
        ctx = b.op("BatchMatMul", (p, qkv[2]), (Bs, heads, S, dh), key)
        ctx = b.op("Transpose", (ctx,), (Bs, S, heads, dh), key)
        ctx = b.op("Reshape", (ctx,), (Bs * S, Hd), key)
        ao = dense(ctx, Hd, Hd, key)
        ao = dropout(ao, (Bs * S, Hd), key)
        ao = b.op("Add", (ao, x), (Bs * S, Hd), key)
        x1 = layernorm(ao, key)
        key2 = (L + 1, 1)
        h = dense(x1, Hd, 4 * Hd, key2)
        shp = (Bs * S, 4 * Hd)
        p3 = b.op("Pow", (h, b.const(key2)), shp, key2)             # tanh-GELU
        m1 = b.op("Mul", (p3, b.const(key2)), shp, key2)
        a1 = b.op("Add", (h, m1), shp, key2)
        m2 = b.op("Mul", (a1, b.const(key2)), shp, key2)
        th = b.op("Tanh", (m2,), shp, key2)
        a2 = b.op("Add", (th, b.const(key2)), shp, key2)
        m3 = b.op("Mul", (h, b.const(key2)), shp, key2)
        h = b.op("Mul", (m3, a2), shp, key2)
        o = dense(h, 4 * Hd, Hd, key2)
        o = dropout(o, (Bs * S, Hd), key2)
        o = b.op("Add", (o, x1), (Bs * S, Hd), key2)
        x = layernorm(o, key2)
    kf = (layers + 1, 0)
    pooled = b.op("StridedSlice", (x,), (Bs, Hd), kf)
    pooled = dense(pooled, Hd, Hd, kf)
    pooled = b.op("Tanh", (pooled,), (Bs, Hd), kf)
    lg = dense(pooled, Hd, 2, kf)
    lab = b.op("Placeholder", (), (Bs,), g0)
    ce = b.op("SparseSoftmaxCrossEntropyWithLogits", (lg, lab), (Bs,), kf)
    loss = b.op("Mean", (ce,), (), kf)
    grads = b.backward(loss)
    lr = b.op("Const", (), (), (layers + 2, 0))
    for v in sorted(b.trainable):                       # in-graph AdamWeightDecay
        if v + 1 not in grads:
            continue
        key = b.key[v]
        shp = b.shape[v]
        g = grads[v + 1]
        m = b.op("VariableV2", (), shp, key)
        s = b.op("VariableV2", (), shp, key)
        m1 = b.op("Mul", (m, b.const(key)), shp, key, 2)
        m2 = b.op("Mul", (g, b.const(key)), shp, key, 2)
        mn = b.op("Add", (m1, m2), shp, key, 2)
        sq = b.op("Square", (g,), shp, key, 2)
        v1 = b.op("Mul", (s, b.const(key)), shp, key, 2)
        v2 = b.op("Mul", (sq, b.const(key)), shp, key, 2)
        vn = b.op("Add", (v1, v2), shp, key, 2)
        sr = b.op("Sqrt", (vn,), shp, key, 2)
        de = b.op("Add", (sr, b.const(key)), shp, key, 2)
        up = b.op("RealDiv", (mn, de), shp, key, 2)
        wd = b.op("Mul", (v, b.const(key)), shp, key, 2)
        up = b.op("Add", (up, wd), shp, key, 2)
        st = b.op("Mul", (up, lr), shp, key, 2)
        nv = b.op("Sub", (v, st), shp, key, 2)
        b.op("Assign", (v, nv), shp, key, 2)
        b.op("Assign", (m, mn), shp, key, 2)
        b.op("Assign", (s, vn), shp, key, 2)
    return b.finish("bert", F)


# =========================================================================== registry / cache
def make(name: str, index: int = 0, **kw) -> OpGraph:
    if name == "tiny":
        return tiny(index, **kw)
    if name == "inception":
        return inception(index, **kw)
    if name == "gnmt":
        return gnmt(index, **kw)
    if name == "bert":
        return bert(index, **kw)
    if name == "1m":
        return gnmt(index, T=kw.pop("T", 3000), **kw)
    raise ValueError(name)


def cached(name: str, index: int = 0, cache_dir: str | None = None, **kw) -> OpGraph:
    """make() with an .npz cache under build/graphs/ (same bytes for every consumer)."""
    if cache_dir is None:
        cache_dir = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                 "build", "graphs")
    tag = "_".join(f"{k}{v}" for k, v in sorted(kw.items()))
    path = os.path.join(cache_dir, f"{name}_{index}{'_' + tag if tag else ''}.npz")
    if os.path.exists(path):
        z = np.load(path)
        if "dims" in z.files:
            return OpGraph(name, int(z["N"]), z["indptr"], z["indices"], z["X"], z["types"],
                           z["dims"])
    g = make(name, index, **kw)
    try:
        os.makedirs(cache_dir, exist_ok=True)
        tmp = path + f".tmp{os.getpid()}.npz"
        np.savez(tmp, N=g.num_nodes, indptr=g.indptr, indices=g.indices, X=g.features,
                 types=g.types, dims=g.dims)
        os.replace(tmp, path)
    except OSError:
        pass
    return g


def batch(name: str, count: int, base_index: int = 0, **kw):
    return [cached(name, base_index + i, **kw) for i in range(count)]
