"""Thin ctypes binding of libmars.so (include/mars.h) -- argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels; there is no
CPU fallback.  If libmars.so is missing this module raises on import-time use
(``lib()``), and every compute call raises ``MarsError`` with the library's
status when no CUDA device is usable.

Names follow the C ABI: ``graph_load``, ``dgi_create``, ``dgi_step``,
``encode``, ``free`` (+ the test hooks ``graph_export_csr`` and
``dgi_export_activations``).  ``Graph`` / ``DGI`` wrap the handles.
"""
from __future__ import annotations

import ctypes
import os
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmars.so")

MARS_OK, MARS_EINVAL, MARS_ENOMEM, MARS_ECUDA, MARS_ENCCL, MARS_ENUMERIC, MARS_ESTATE = range(7)
MARS_FP32, MARS_BF16 = 0, 1
_STATUS = {0: "OK", 1: "EINVAL", 2: "ENOMEM", 3: "ECUDA", 4: "ENCCL", 5: "ENUMERIC", 6: "ESTATE"}
PHASES = ["perm", "spmm_fwd", "gemm_fwd", "head", "gemm_dw", "gemm_dy", "spmm_bwd", "allreduce",
          "adam", "reduce", "exchange"]


class MarsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"MARS_{_STATUS.get(status, status)}: {msg}")
        self.status = status


class GraphDesc(ctypes.Structure):
    _fields_ = [("num_nodes", ctypes.c_int32), ("indptr", ctypes.c_void_p),
                ("indices", ctypes.c_void_p), ("feat_dim", ctypes.c_int32),
                ("features", ctypes.c_void_p)]


class DgiConfig(ctypes.Structure):
    _fields_ = [("in_dim", ctypes.c_int32), ("hidden_dim", ctypes.c_int32),
                ("num_layers", ctypes.c_int32), ("precision", ctypes.c_int32),
                ("lr", ctypes.c_double), ("beta1", ctypes.c_double), ("beta2", ctypes.c_double),
                ("eps", ctypes.c_double), ("clip_norm", ctypes.c_double),
                ("seed", ctypes.c_uint64), ("init_params", ctypes.c_void_p),
                ("device", ctypes.c_int32), ("world_size", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("nccl_unique_id", ctypes.c_void_p),
                ("encoder", ctypes.c_int32)]


class PlacerConfig(ctypes.Structure):
    _fields_ = [("in_dim", ctypes.c_int32), ("enc_hidden", ctypes.c_int32),
                ("attn_dim", ctypes.c_int32), ("dev_embed", ctypes.c_int32),
                ("num_devices", ctypes.c_int32), ("segment", ctypes.c_int32),
                ("seed", ctypes.c_uint64), ("init_params", ctypes.c_void_p),
                ("device", ctypes.c_int32)]


class PpoConfig(ctypes.Structure):
    _fields_ = [("clip_eps", ctypes.c_float), ("ent_coef", ctypes.c_float), ("lr", ctypes.c_float),
                ("beta1", ctypes.c_float), ("beta2", ctypes.c_float), ("adam_eps", ctypes.c_float),
                ("clip_norm", ctypes.c_float), ("mu", ctypes.c_float),
                ("samples_per_policy", ctypes.c_int32), ("policies", ctypes.c_int32),
                ("minibatches", ctypes.c_int32), ("epochs", ctypes.c_int32),
                ("seed", ctypes.c_uint64), ("capacity_bytes", ctypes.c_float)]


class Contrastive(ctypes.Structure):
    """mars_contrastive (NEXT-4, readings c34-c37)."""
    _fields_ = [("num_neg", ctypes.c_int32), ("corruption", ctypes.c_int32),
                ("mask_rate", ctypes.c_float), ("readout", ctypes.c_int32),
                ("aggregator", ctypes.c_int32), ("loss", ctypes.c_int32)]


CORRUPTIONS = {"permute": 0, "mask": 1}
READOUTS = {"sigmoid_mean": 0, "mean": 1}
AGGREGATORS = {"gcn": 0, "sage_gcn": 1}
LOSSES = {"bce": 0, "infonce": 1}
ENCODERS = {"gcn": 0, "sage": 1, "sage_pool": 2}


class StepOut(ctypes.Structure):
    _fields_ = [("loss", ctypes.c_void_p), ("grads", ctypes.c_void_p), ("perms", ctypes.c_void_p)]


# symbol -> (restype, argtypes); every symbol include/mars.h declares
SIGNATURES = {
    "mars_last_error": (ctypes.c_char_p, []),
    "mars_version": (ctypes.c_char_p, []),
    "mars_num_params": (ctypes.c_int64, [ctypes.c_int32, ctypes.c_int32]),
    "mars_graph_load": (ctypes.c_int, [ctypes.POINTER(GraphDesc), ctypes.c_int32, ctypes.c_int32,
                                       ctypes.POINTER(ctypes.c_void_p)]),
    "mars_graph_info": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                       ctypes.c_void_p, ctypes.c_void_p]),
    "mars_graph_size": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p,
                                       ctypes.c_void_p]),
    "mars_graph_export_csr": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32] + [ctypes.c_void_p] * 5),
    "mars_dgi_config_default": (None, [ctypes.POINTER(DgiConfig)]),
    "mars_dgi_create": (ctypes.c_int, [ctypes.POINTER(DgiConfig), ctypes.POINTER(ctypes.c_void_p)]),
    "mars_dgi_num_params": (ctypes.c_int64, [ctypes.c_void_p]),
    "mars_nccl_get_unique_id": (ctypes.c_int, [ctypes.c_void_p]),
    "mars_dgi_set_stream": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dgi_set_graph_capture": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32]),
    "mars_dgi_set_gemm_impl": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32]),
    "mars_dgi_set_contrastive": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(Contrastive)]),
    "mars_dgi_get_contrastive": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(Contrastive)]),
    "mars_dgi_step": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                     ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(StepOut)]),
    "mars_encode": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dgi_pretrain": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                         ctypes.c_int32, ctypes.c_int64, ctypes.c_int64,
                                         ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                         ctypes.c_void_p]),
    "mars_dgi_export_activations": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32,
                                                   ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dgi_saved_rows": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dgi_set_keep_backward": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32]),
    "mars_dgi_export_backward": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32,
                                                ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dgi_get_state": (ctypes.c_int, [ctypes.c_void_p] * 4 + [ctypes.c_void_p]),
    "mars_dgi_set_state": (ctypes.c_int, [ctypes.c_void_p] * 4 + [ctypes.c_int64]),
    "mars_dgi_profile_step": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                             ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p,
                                             ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p]),
    "mars_dgi_last_launches": (ctypes.c_int64, [ctypes.c_void_p]),
    "mars_debug_gemm": (ctypes.c_int, [ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                       ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                       ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                       ctypes.c_int32, ctypes.c_void_p]),
    "mars_dgi_read_step": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dgi_enqueue_loss": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dgi_wait_loss": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]),
    "mars_graph_load_shard": (ctypes.c_int, [ctypes.POINTER(GraphDesc), ctypes.c_int32,
                                             ctypes.c_int32, ctypes.c_int32,
                                             ctypes.POINTER(ctypes.c_void_p)]),
    "mars_graph_shard_info": (ctypes.c_int, [ctypes.c_void_p] + [ctypes.c_void_p] * 6),
    "mars_shard_partition": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                            ctypes.c_void_p]),
    "mars_shard_attach": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_shard_blob_bytes": (ctypes.c_int64, []),
    "mars_shard_export": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_shard_connect": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_shard_connect_local": (ctypes.c_int, [ctypes.POINTER(ctypes.c_void_p), ctypes.c_int32]),
    "mars_dp_blob_bytes": (ctypes.c_int64, []),
    "mars_dp_export": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_dp_connect": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_graph_set_pair_offsets": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_graph_reload": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(GraphDesc), ctypes.c_int32]),
    "mars_featurize": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                                      ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p]),
    "mars_placer_config_default": (None, [ctypes.POINTER(PlacerConfig)]),
    "mars_placer_num_params": (ctypes.c_int64, [ctypes.POINTER(PlacerConfig)]),
    "mars_placer_create": (ctypes.c_int, [ctypes.POINTER(PlacerConfig),
                                          ctypes.POINTER(ctypes.c_void_p)]),
    "mars_placer_get_params": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_placer_set_params": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "mars_placer_sample": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                                          ctypes.c_int32, ctypes.c_uint64, ctypes.c_void_p,
                                          ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "mars_placer_ppo_grad": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                                            ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p,
                                            ctypes.c_void_p, ctypes.c_float, ctypes.c_float,
                                            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "mars_ppo_config_default": (None, [ctypes.POINTER(PpoConfig)]),
    "mars_ppo_create": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.POINTER(PpoConfig),
                                       ctypes.POINTER(ctypes.c_void_p)]),
    "mars_ppo_iteration": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                                          ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                          ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                          ctypes.c_void_p]),
    "mars_dgi_encoder_vjp": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                            ctypes.c_void_p]),
    "mars_ppo_iteration_joint": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                                ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                                ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]),
    "mars_free": (None, [ctypes.c_void_p]),
}

_lib = None
_lock = threading.Lock()


def lib():
    """Load libmars.so (fails loudly when the CUDA extension was not built)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(f"{LIB_PATH} not built (run `make` or __graft_entry__.build())")
            L = ctypes.CDLL(LIB_PATH)
            lenient = os.environ.get("MARS_BINDING_LENIENT") == "1"   # A/B of older builds
            for name, (res, args) in SIGNATURES.items():
                if lenient and not hasattr(L, name):
                    continue
                fn = getattr(L, name)
                fn.restype = res
                fn.argtypes = args
            _lib = L
    return _lib


def _check(st: int):
    if st != MARS_OK:
        raise MarsError(st, lib().mars_last_error().decode(errors="replace"))


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def version() -> str:
    return lib().mars_version().decode()


def num_params(F: int, H: int) -> int:
    return int(lib().mars_num_params(F, H))


# ------------------------------------------------------------------ graph sets
class Graph:
    """A device-resident set of op graphs (mars_graph*)."""

    def __init__(self, handle, sizes, F):
        self.handle = handle
        self.sizes = list(sizes)
        self.F = F

    @property
    def num_graphs(self):
        return len(self.sizes)

    @property
    def total_nodes(self):
        return int(sum(self.sizes))

    def info(self):
        G = ctypes.c_int32(); Nt = ctypes.c_int64(); Z = ctypes.c_int64(); F = ctypes.c_int32()
        _check(lib().mars_graph_info(self.handle, ctypes.byref(G), ctypes.byref(Nt),
                                     ctypes.byref(Z), ctypes.byref(F)))
        return dict(num_graphs=G.value, total_nodes=Nt.value, nnz=Z.value, feat_dim=F.value)

    def size(self, idx):
        N = ctypes.c_int32(); Z = ctypes.c_int64()
        _check(lib().mars_graph_size(self.handle, idx, ctypes.byref(N), ctypes.byref(Z)))
        return N.value, Z.value

    def export_csr(self, idx):
        return graph_export_csr(self, idx)

    def reload(self, graphs):
        """mars_graph_reload: new contents (same node counts / F) in place."""
        graphs = list(graphs)
        descs = (GraphDesc * len(graphs))()
        keep = []
        for i, g in enumerate(graphs):
            d, k = _desc(g)
            descs[i] = d
            keep.append(k)
        _check(lib().mars_graph_reload(self.handle, descs, len(graphs)))

    def set_pair_offsets(self, offsets):
        """mars_graph_set_pair_offsets: graph i uses pair index pair_base + offsets[i] (c15)."""
        off = np.ascontiguousarray(offsets, np.int64)
        if off.size != self.num_graphs:
            raise ValueError("one offset per graph")
        _check(lib().mars_graph_set_pair_offsets(self.handle, _ptr(off)))

    def free(self):
        if self.handle:
            lib().mars_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def corruption_samples(graphs, K: int):
    """K corruption samples per graph (DESIGN.md reading
    c20): each graph repeated K times consecutively, so with global_batch =
    K·len(graphs) pair g·K + k draws its own permutation and the step's loss is
    1/(2N)[Σ softplus(-l_i) + (1/K) Σ_k Σ_i softplus(l~_i^k)] per graph -- the
    positive branch weighted once, each corruption sample 1/K (the positive
    branch is recomputed per sample)."""
    if K < 1:
        raise ValueError("K >= 1")
    return [g for g in graphs for _ in range(K)]


def featurize(types, dims, feat_dim: int, device: int = 0) -> np.ndarray:
    """mars_featurize (NEXT-1): X [N x F] from op types [N] and shape dims [N x 8]."""
    t = np.ascontiguousarray(types, np.int32)
    d = np.ascontiguousarray(dims, np.int64).reshape(-1, 8)
    if d.shape[0] != t.size:
        raise ValueError("one dims row per op")
    X = np.zeros((t.size, feat_dim), np.float32)
    _check(lib().mars_featurize(_ptr(t), _ptr(d), t.size, int(feat_dim), device, _ptr(X)))
    return X


def graph_load(graphs, device: int = 0) -> Graph:
    """mars_graph_load: graphs = iterable of objects with num_nodes, indptr (int64
    [N+1]), indices (int32), features (float32 [N, F])."""
    graphs = list(graphs)
    keep = []
    descs = (GraphDesc * len(graphs))()
    F = None
    for i, g in enumerate(graphs):
        ip = np.ascontiguousarray(g.indptr, np.int64)
        ix = np.ascontiguousarray(g.indices, np.int32)
        X = np.ascontiguousarray(g.features, np.float32)
        keep += [ip, ix, X]
        F = X.shape[1] if X.ndim == 2 else int(getattr(g, "feat_dim"))
        descs[i] = GraphDesc(int(g.num_nodes), ip.ctypes.data, ix.ctypes.data if ix.size else None,
                             int(F), X.ctypes.data)
    h = ctypes.c_void_p()
    _check(lib().mars_graph_load(descs, len(graphs), device, ctypes.byref(h)))
    return Graph(h, [int(g.num_nodes) for g in graphs], F)


def _desc(g):
    ip = np.ascontiguousarray(g.indptr, np.int64)
    ix = np.ascontiguousarray(g.indices, np.int32)
    X = np.ascontiguousarray(g.features, np.float32)
    d = GraphDesc(int(g.num_nodes), ip.ctypes.data, ix.ctypes.data if ix.size else None,
                  int(X.shape[1]), X.ctypes.data)
    return d, (ip, ix, X)


def graph_load_shard(graph, num_shards: int, shard: int, device: int = 0) -> Graph:
    """mars_graph_load_shard: shard `shard` of `num_shards` row blocks of one op graph
    (SURVEY §8(e)(ii)).  The Graph's sizes are the WHOLE graph's (the permutation
    covers it); shard_info() gives the owned rows."""
    d, keep = _desc(graph)
    h = ctypes.c_void_p()
    _check(lib().mars_graph_load_shard(ctypes.byref(d), int(num_shards), int(shard), device,
                                       ctypes.byref(h)))
    del keep
    g = Graph(h, [int(graph.num_nodes)], d.feat_dim)
    g.sharded = True
    return g


def shard_partition(rowptr, num_shards: int) -> np.ndarray:
    """mars_shard_partition (host only): row starts [P+1] of the nnz-balanced split."""
    rp = np.ascontiguousarray(rowptr, np.int32)
    out = np.zeros(num_shards + 1, np.int32)
    _check(lib().mars_shard_partition(_ptr(rp), rp.size - 1, int(num_shards), _ptr(out)))
    return out


def graph_shard_info(g: Graph):
    P = ctypes.c_int32(); me = ctypes.c_int32(); r0 = ctypes.c_int32(); r1 = ctypes.c_int32()
    z = ctypes.c_int64(); h = ctypes.c_int64()
    _check(lib().mars_graph_shard_info(g.handle, ctypes.byref(P), ctypes.byref(me), ctypes.byref(r0),
                                       ctypes.byref(r1), ctypes.byref(z), ctypes.byref(h)))
    return dict(num_shards=P.value, shard=me.value, row_begin=r0.value, row_end=r1.value,
                local_nnz=z.value, halo_rows=h.value)


def shard_attach(m: "DGI", g: Graph):
    _check(lib().mars_shard_attach(m.handle, g.handle))


def shard_export(m: "DGI") -> bytes:
    buf = ctypes.create_string_buffer(int(lib().mars_shard_blob_bytes()))
    _check(lib().mars_shard_export(m.handle, buf))
    return buf.raw


def shard_connect(m: "DGI", blobs):
    """blobs: the P shards' export blobs in rank order (bytes each)."""
    data = b"".join(blobs)
    buf = ctypes.create_string_buffer(data, len(data))
    _check(lib().mars_shard_connect(m.handle, buf))


def shard_connect_local(models):
    arr = (ctypes.c_void_p * len(models))(*[m.handle for m in models])
    _check(lib().mars_shard_connect_local(arr, len(models)))


def dp_export(m: "DGI") -> bytes:
    """mars_dp_export: this rank's blob for the peer-memory gradient exchange."""
    buf = ctypes.create_string_buffer(int(lib().mars_dp_blob_bytes()))
    _check(lib().mars_dp_export(m.handle, buf))
    return buf.raw


def dp_connect(m: "DGI", blobs):
    """mars_dp_connect: blobs = every rank's dp_export() in rank order."""
    data = b"".join(blobs)
    buf = ctypes.create_string_buffer(data, len(data))
    _check(lib().mars_dp_connect(m.handle, buf))


def graph_export_csr(g: Graph, idx: int):
    N, Z = g.size(idx)
    rowptr = np.zeros(N + 1, np.int32); colind = np.zeros(max(Z, 1), np.int32)
    deg = np.zeros(N, np.int32); dinv = np.zeros(N, np.float32); vals = np.zeros(max(Z, 1), np.float32)
    _check(lib().mars_graph_export_csr(g.handle, idx, _ptr(rowptr), _ptr(colind), _ptr(deg),
                                       _ptr(dinv), _ptr(vals)))
    return dict(rowptr=rowptr, colind=colind[:Z], deg=deg, dinv=dinv, vals=vals[:Z])


# ------------------------------------------------------------------ model
def config_default() -> DgiConfig:
    c = DgiConfig()
    lib().mars_dgi_config_default(ctypes.byref(c))
    return c


def nccl_get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().mars_nccl_get_unique_id(buf))
    return buf.raw


class DGI:
    """A DGI pre-training model instance (mars_dgi*)."""

    def __init__(self, handle, F, H):
        self.handle = handle
        self.F, self.H = F, H
        self.P = int(lib().mars_dgi_num_params(handle))
        self.num_neg = 1
        self.corruption = "permute"

    def set_contrastive(self, num_neg: int = 1, corruption: str = "permute",
                        mask_rate: float = 0.0, readout: str = "sigmoid_mean",
                        aggregator: str = "gcn", loss: str = "bce"):
        """mars_dgi_set_contrastive (NEXT-4): K corruption samples sharing one
        positive branch, permutation or feature-mask corruption, sig(mean) or
        mean readout, GCN or SAGE-GCN aggregation.  The defaults are the paper's
        DGI step."""
        c = Contrastive(int(num_neg), CORRUPTIONS[corruption], float(mask_rate),
                        READOUTS[readout], AGGREGATORS[aggregator], LOSSES[loss])
        _check(lib().mars_dgi_set_contrastive(self.handle, ctypes.byref(c)))
        self.num_neg, self.corruption = int(num_neg), corruption

    def get_contrastive(self) -> dict:
        c = Contrastive()
        _check(lib().mars_dgi_get_contrastive(self.handle, ctypes.byref(c)))
        inv = lambda d, v: next(k for k, x in d.items() if x == v)
        return dict(num_neg=c.num_neg, corruption=inv(CORRUPTIONS, c.corruption),
                    mask_rate=c.mask_rate, readout=inv(READOUTS, c.readout),
                    aggregator=inv(AGGREGATORS, c.aggregator), loss=inv(LOSSES, c.loss))

    def step(self, g: Graph, step_index: int, pair_base: int = 0, global_batch: int | None = None,
             want_loss=False, want_grads=False, want_perms=False):
        return dgi_step(self, g, step_index, pair_base, global_batch, want_loss, want_grads,
                        want_perms)

    def encode(self, g: Graph):
        return encode(self, g)

    def pretrain(self, g: Graph, n_steps: int, step0: int = 0, pair_base: int = 0,
                 global_batch: int | None = None):
        """mars_dgi_pretrain: returns dict(losses, best_params, best_loss,
        best_step)."""
        B = g.num_graphs if global_batch is None else int(global_batch)
        losses = np.zeros(n_steps, np.float32)
        best = np.zeros(self.P, np.float32)
        bl = ctypes.c_float(); bs = ctypes.c_int64()
        _check(lib().mars_dgi_pretrain(self.handle, g.handle, step0 & (2 ** 64 - 1), int(n_steps),
                                       int(pair_base), B, _ptr(losses), _ptr(best),
                                       ctypes.byref(bl), ctypes.byref(bs)))
        return dict(losses=losses, best_params=best, best_loss=bl.value, best_step=bs.value)

    def export_activations(self, layer: int):
        return dgi_export_activations(self, layer)

    def encoder_vjp(self, g: Graph, dE):
        """mars_dgi_encoder_vjp: gradient [P] of sum(dE * encode(g))."""
        d = np.ascontiguousarray(dE, np.float32)
        out = np.zeros(self.P, np.float32)
        _check(lib().mars_dgi_encoder_vjp(self.handle, g.handle, _ptr(d), _ptr(out)))
        return out

    def saved_rows(self) -> int:
        """Rows per branch of the last step's saved activations (0 after encode)."""
        r = ctypes.c_int64()
        _check(lib().mars_dgi_saved_rows(self.handle, ctypes.byref(r)))
        return r.value

    def set_keep_backward(self, keep: bool):
        """Test hook: keep dZ_3..1 and dY_3, dY_2 of every later step."""
        _check(lib().mars_dgi_set_keep_backward(self.handle, 1 if keep else 0))

    def export_backward(self, layer: int):
        """Test hook: (dY_layer or None for layer 1, dZ_layer) of the last step,
        stacked [pos; neg], fp32."""
        R = 2 * self.saved_rows()
        dZ = np.zeros((R, self.H), np.float32)
        dY = np.zeros((R, self.H), np.float32) if layer > 1 else None
        _check(lib().mars_dgi_export_backward(self.handle, layer,
                                              None if dY is None else _ptr(dY), _ptr(dZ)))
        return dY, dZ

    def get_state(self):
        p = np.zeros(self.P, np.float32); m = np.zeros(self.P, np.float32)
        v = np.zeros(self.P, np.float32); t = ctypes.c_int64()
        _check(lib().mars_dgi_get_state(self.handle, _ptr(p), _ptr(m), _ptr(v), ctypes.byref(t)))
        return p, m, v, t.value

    def set_state(self, params=None, m=None, v=None, t=0):
        arrs = [None if a is None else np.ascontiguousarray(a, np.float32) for a in (params, m, v)]
        _check(lib().mars_dgi_set_state(self.handle, *[None if a is None else _ptr(a) for a in arrs],
                                        int(t)))

    def set_stream(self, stream_ptr):
        _check(lib().mars_dgi_set_stream(self.handle, stream_ptr))

    def set_gemm_impl(self, impl: str):
        """'auto' (tcgen05 3xFP16 GEMMs where the widths are supported) or
        'simt' (FFMA everywhere)."""
        _check(lib().mars_dgi_set_gemm_impl(self.handle, GEMM_IMPLS[impl]))

    def set_graph_capture(self, enable: bool):
        _check(lib().mars_dgi_set_graph_capture(self.handle, 1 if enable else 0))

    def profile_step(self, g: Graph, step_index: int, pair_base: int = 0,
                     global_batch: int | None = None):
        """mars_dgi_profile_step: [(phase name, device ms)] in schedule order."""
        B = g.num_graphs if global_batch is None else int(global_batch)
        ids = np.zeros(256, np.int32); ms = np.zeros(256, np.float32); n = ctypes.c_int32()
        _check(lib().mars_dgi_profile_step(self.handle, g.handle, step_index & (2 ** 64 - 1),
                                           int(pair_base), B, _ptr(ids), _ptr(ms), 256,
                                           ctypes.byref(n)))
        return [(PHASES[int(i)], float(t)) for i, t in zip(ids[:n.value], ms[:n.value])]

    def read_step(self, want_grads=True):
        """mars_dgi_read_step: (loss, grads or None) of the most recent step."""
        loss = ctypes.c_float()
        grads = np.zeros(self.P, np.float32) if want_grads else None
        _check(lib().mars_dgi_read_step(self.handle, ctypes.byref(loss),
                                        None if grads is None else _ptr(grads)))
        return loss.value, grads

    def enqueue_loss(self) -> int:
        """mars_dgi_enqueue_loss: ticket of an asynchronous D2H copy of the
        most recent step's loss (see mars.h)."""
        t = ctypes.c_int64()
        _check(lib().mars_dgi_enqueue_loss(self.handle, ctypes.byref(t)))
        return t.value

    def wait_loss(self, ticket: int) -> float:
        """mars_dgi_wait_loss: the loss of an enqueued read-back (blocks)."""
        loss = ctypes.c_float()
        _check(lib().mars_dgi_wait_loss(self.handle, ctypes.c_int64(ticket), ctypes.byref(loss)))
        return loss.value

    def last_launches(self) -> int:
        return int(lib().mars_dgi_last_launches(self.handle))

    def free(self):
        if self.handle:
            lib().mars_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def dgi_create(in_dim=64, hidden_dim=256, precision=MARS_FP32, lr=1e-3, beta1=0.9, beta2=0.999,
               eps=1e-8, clip_norm=0.0, seed=0, init_params=None, device=0, world_size=1, rank=0,
               nccl_unique_id: bytes | None = None, encoder: str = "gcn") -> DGI:
    c = config_default()
    c.encoder = ENCODERS[encoder]
    c.in_dim, c.hidden_dim, c.num_layers, c.precision = in_dim, hidden_dim, 3, precision
    c.lr, c.beta1, c.beta2, c.eps, c.clip_norm = lr, beta1, beta2, eps, clip_norm
    c.seed = seed & (2 ** 64 - 1)
    keep = None
    if init_params is not None:
        keep = np.ascontiguousarray(init_params, np.float32)
        c.init_params = keep.ctypes.data
    c.device, c.world_size, c.rank = device, world_size, rank
    uid = None
    if nccl_unique_id is not None:
        uid = ctypes.create_string_buffer(nccl_unique_id, 128)
        c.nccl_unique_id = ctypes.cast(uid, ctypes.c_void_p)
    h = ctypes.c_void_p()
    _check(lib().mars_dgi_create(ctypes.byref(c), ctypes.byref(h)))
    del keep, uid
    return DGI(h, in_dim, hidden_dim)


def dgi_step(m: DGI, g: Graph, step_index: int, pair_base: int = 0, global_batch: int | None = None,
             want_loss=False, want_grads=False, want_perms=False):
    """mars_dgi_step.  Returns dict with the requested host outputs."""
    B = g.num_graphs if global_batch is None else int(global_batch)
    res = {}
    out = StepOut()
    if want_loss:
        res["loss"] = np.zeros(1, np.float32); out.loss = res["loss"].ctypes.data
    if want_grads:
        res["grads"] = np.zeros(m.P, np.float32); out.grads = res["grads"].ctypes.data
    if want_perms:
        res["perms"] = np.zeros(g.total_nodes * m.num_neg, np.int32)
        out.perms = res["perms"].ctypes.data
    _check(lib().mars_dgi_step(m.handle, g.handle, step_index & (2 ** 64 - 1), int(pair_base), B,
                               ctypes.byref(out)))
    if want_loss:
        res["loss"] = float(res["loss"][0])
    return res


def encode(m: DGI, g: Graph) -> np.ndarray:
    out = np.zeros((g.total_nodes, m.H), np.float32)
    _check(lib().mars_encode(m.handle, g.handle, _ptr(out)))
    return out


def dgi_export_activations(m: DGI, layer: int):
    """Test hook: the last step's (Y_l, Z_l), stacked [pos; neg], as fp32 arrays."""
    nt = m.saved_rows()
    if nt == 0:
        raise MarsError(MARS_ESTATE, "no step has run since the last encode")
    R = 2 * nt
    cin = m.F if layer == 1 else m.H
    Y = np.zeros((R, cin), np.float32)
    Z = np.zeros((R, m.H), np.float32)
    _check(lib().mars_dgi_export_activations(m.handle, layer, _ptr(Y), _ptr(Z)))
    return Y, Z


GEMM_IMPLS = {"auto": 0, "simt": 1}   # MARS_GEMM_* (include/mars.h)


# ------------------------------------------------------------------ placer (NEXT-2)
class Placer:
    """The segment-level seq2seq placer (mars_placer*)."""

    def __init__(self, handle, cfg: PlacerConfig):
        self.handle = handle
        self.cfg = cfg
        self.P = int(lib().mars_placer_num_params(ctypes.byref(cfg)))

    def get_params(self) -> np.ndarray:
        p = np.zeros(self.P, np.float32)
        _check(lib().mars_placer_get_params(self.handle, _ptr(p)))
        return p

    def set_params(self, params):
        p = np.ascontiguousarray(params, np.float32)
        _check(lib().mars_placer_set_params(self.handle, _ptr(p)))

    def sample(self, embeddings, num_samples: int, sample_seed: int = 0, forced=None):
        """mars_placer_sample: (placements [S x N] int32, logp [S x N], entropy [S x N])."""
        E = np.ascontiguousarray(embeddings, np.float32)
        N = E.shape[0]
        S = int(num_samples)
        f = None if forced is None else np.ascontiguousarray(forced, np.int32).reshape(S, N)
        place = np.zeros((S, N), np.int32)
        logp = np.zeros((S, N), np.float32)
        ent = np.zeros((S, N), np.float32)
        _check(lib().mars_placer_sample(self.handle, _ptr(E), N, S, sample_seed & (2 ** 64 - 1),
                                        None if f is None else _ptr(f), _ptr(place), _ptr(logp),
                                        _ptr(ent)))
        return place, logp, ent

    def ppo_grad(self, embeddings, placements, logp_old, adv, clip_eps=0.2, ent_coef=0.001):
        """mars_placer_ppo_grad: (loss, grads [P], dL/dE [N x H])."""
        E = np.ascontiguousarray(embeddings, np.float32)
        N = E.shape[0]
        pl = np.ascontiguousarray(placements, np.int32)
        S = pl.shape[0]
        lo = np.ascontiguousarray(logp_old, np.float32).reshape(S, N)
        ad = np.ascontiguousarray(adv, np.float32).reshape(S)
        loss = np.zeros(1, np.float32)
        g = np.zeros(self.P, np.float32)
        dE = np.zeros_like(E)
        _check(lib().mars_placer_ppo_grad(self.handle, _ptr(E), N, S, _ptr(pl), _ptr(lo), _ptr(ad),
                                          float(clip_eps), float(ent_coef), _ptr(loss), _ptr(g),
                                          _ptr(dE)))
        return float(loss[0]), g, dE

    def free(self):
        if self.handle:
            lib().mars_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def placer_create(in_dim=256, enc_hidden=256, attn_dim=512, dev_embed=64, num_devices=4,
                  segment=128, seed=0, init_params=None, device=0) -> Placer:
    c = PlacerConfig()
    lib().mars_placer_config_default(ctypes.byref(c))
    c.in_dim, c.enc_hidden, c.attn_dim, c.dev_embed = in_dim, enc_hidden, attn_dim, dev_embed
    c.num_devices, c.segment, c.seed, c.device = num_devices, segment, seed & (2 ** 64 - 1), device
    keep = None
    if init_params is not None:
        keep = np.ascontiguousarray(init_params, np.float32)
        c.init_params = keep.ctypes.data
    h = ctypes.c_void_p()
    _check(lib().mars_placer_create(ctypes.byref(c), ctypes.byref(h)))
    c.init_params = None
    del keep
    return Placer(h, c)


def debug_gemm(op: str, A, B, impl: str = "auto", iters: int = 0, device: int = 0):
    """mars_debug_gemm: op 'rows' -> A[M×K]·Bᵀ (B [N×K]); op 'dw' -> Aᵀ·B (A [M×K],
    B [M×N]).  Returns (C, mean ms per launch)."""
    A = np.ascontiguousarray(A, np.float32)
    B = np.ascontiguousarray(B, np.float32)
    M, K = A.shape
    if op == "rows":
        N = B.shape[0]
        C = np.zeros((M, N), np.float32)
    else:
        N = B.shape[1]
        C = np.zeros((K, N), np.float32)
    ms = ctypes.c_float()
    _check(lib().mars_debug_gemm(device, 0 if op == "rows" else 1, GEMM_IMPLS[impl],
                                 _ptr(A), _ptr(B), _ptr(C), M, N, K, iters, ctypes.byref(ms)))
    return C, ms.value


def free(handle_obj):
    handle_obj.free()


# ------------------------------------------------------------------ PPO (NEXT-3)
class Ppo:
    """PPO training of a placer (mars_ppo*)."""

    def __init__(self, handle, cfg: PpoConfig, placer: "Placer"):
        self.handle, self.cfg, self.placer = handle, cfg, placer

    @property
    def num_samples(self):
        return self.cfg.samples_per_policy * self.cfg.policies

    def iteration(self, embeddings, graph):
        """mars_ppo_iteration on one op graph (an object with num_nodes, indptr,
        indices and dims [N x 8]).  Returns dict(placements, step_times,
        advantages, loss)."""
        E = np.ascontiguousarray(embeddings, np.float32)
        N = E.shape[0]
        dims = np.ascontiguousarray(graph.dims, np.int64).reshape(N, 8)
        ip = np.ascontiguousarray(graph.indptr, np.int64)
        ix = np.ascontiguousarray(graph.indices, np.int32)
        S = self.num_samples
        pl = np.zeros((S, N), np.int32)
        t = np.zeros(S, np.float32)
        a = np.zeros(S, np.float32)
        loss = np.zeros(1, np.float32)
        _check(lib().mars_ppo_iteration(self.handle, _ptr(E), N, _ptr(dims), _ptr(ip),
                                        _ptr(ix) if ix.size else None, _ptr(pl), _ptr(t), _ptr(a),
                                        _ptr(loss)))
        return dict(placements=pl, step_times=t, advantages=a, loss=float(loss[0]))

    def iteration_joint(self, g: Graph, graph):
        """mars_ppo_iteration_joint: the encoder's embeddings of the loaded op graph
        g (one graph), the step-time model from `graph` (dims, indptr, indices)."""
        N = g.total_nodes
        dims = np.ascontiguousarray(graph.dims, np.int64).reshape(N, 8)
        ip = np.ascontiguousarray(graph.indptr, np.int64)
        ix = np.ascontiguousarray(graph.indices, np.int32)
        S = self.num_samples
        pl = np.zeros((S, N), np.int32)
        t = np.zeros(S, np.float32)
        a = np.zeros(S, np.float32)
        loss = np.zeros(1, np.float32)
        _check(lib().mars_ppo_iteration_joint(self.handle, g.handle, _ptr(dims), _ptr(ip),
                                              _ptr(ix) if ix.size else None, _ptr(pl), _ptr(t),
                                              _ptr(a), _ptr(loss)))
        return dict(placements=pl, step_times=t, advantages=a, loss=float(loss[0]))

    def free(self):
        if self.handle:
            lib().mars_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def ppo_create(placer: Placer, encoder: "DGI | None" = None, **kw) -> Ppo:
    c = PpoConfig()
    lib().mars_ppo_config_default(ctypes.byref(c))
    for k, v in kw.items():
        setattr(c, k, v)
    h = ctypes.c_void_p()
    _check(lib().mars_ppo_create(placer.handle, None if encoder is None else encoder.handle,
                                 ctypes.byref(c), ctypes.byref(h)))
    return Ppo(h, c, placer)

