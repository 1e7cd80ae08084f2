"""Row-sharded single graph (include/mars.h "Row-sharded
single graph") on one GPU: P shards of one op graph, each its own model,
connected in one process (mars_shard_connect_local) -- the same kernels, peer
gathers and device barriers as P GPUs, with every shard's buffers on device 0.

Checks:
  * forward activations of the owned rows are BITWISE those of the unsharded
    step (same neighbour order and arithmetic; halo rows only change where a
    row is read from);
  * loss and gradients are bitwise identical on every shard, within 1e-5 of
    the unsharded step (only the readout / dv / dW reduction grouping differs)
    and the loss within 1e-5 of the fp64 oracle;
  * the corruption permutation of the whole graph is the oracle's (bit-exact);
  * several captured steps keep the shards' parameters bitwise identical and
    within 1e-5 of the unsharded trajectory; bf16 within 2e-2.
"""
import numpy as np
import pytest

import oracle
import paper_conf_icpp_lancl21_b200 as mars
from synth import graphs as SG
from tests.util import scaled_err, split_params

pytestmark = pytest.mark.gpu
TOL = 1e-5


def _sharded(graph, P, F, H, seed, precision=mars.MARS_FP32):
    gs = [mars.graph_load_shard(graph, P, p) for p in range(P)]
    ms = [mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed, precision=precision)
          for _ in range(P)]
    for m, g in zip(ms, gs):
        mars.shard_attach(m, g)
    mars.shard_connect_local(ms)
    return gs, ms


def _step_all(gs, ms, step):
    for m, g in zip(ms, gs):            # enqueue every shard before reading any
        m.step(g, step, 0, global_batch=1)
    return [m.read_step() for m in ms]


def test_shard_geometry():
    graph = SG.cached("gnmt", 0)
    P = 4
    infos = []
    for p in range(P):
        g = mars.graph_load_shard(graph, P, p)
        infos.append(mars.graph_shard_info(g))
        g.free()
    ref = oracle.csr(graph.num_nodes, graph.indptr, graph.indices)
    assert infos[0]["row_begin"] == 0 and infos[-1]["row_end"] == graph.num_nodes
    for a, b in zip(infos, infos[1:]):
        assert a["row_end"] == b["row_begin"] and a["row_end"] > a["row_begin"]
    assert sum(i["local_nnz"] for i in infos) == len(ref.colind)
    for i in infos:
        r0, r1 = i["row_begin"], i["row_end"]
        cols = ref.colind[ref.rowptr[r0]:ref.rowptr[r1]]
        assert i["local_nnz"] == len(cols)
        assert i["halo_rows"] == len(np.unique(cols[(cols < r0) | (cols >= r1)]))
        # balanced by nnz: no shard above 1/P + one row's worth
        assert i["local_nnz"] <= len(ref.colind) / P + np.max(np.diff(ref.rowptr)) + 1


@pytest.mark.parametrize("name,P,H", [("inception", 2, 128), ("inception", 3, 128),
                                      ("gnmt", 4, 256)])
def test_shard_step_matches_unsharded(name, P, H):
    _shard_case(SG.cached(name, 0), P, H)


def test_shard_long_rows():
    """A hub row of ~2600 entries (the long-row path of spmm.cu: segments
    aggregated by several warps, combined in order) owned by one shard, its
    halo gathered from the other shard."""
    from tests.test_gpu_spmm_edge import star_graph
    _shard_case(star_graph(), 2, 256)


def _shard_case(graph, P, H):
    F, seed = 64, 5
    N = graph.num_nodes
    g1 = mars.graph_load([graph])
    m1 = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed)
    p0 = m1.get_state()[0]
    ref = m1.step(g1, 0, 0, global_batch=1, want_loss=True, want_grads=True, want_perms=True)
    ref_acts = {l: m1.export_activations(l) for l in (1, 2, 3)}

    gs, ms = _sharded(graph, P, F, H, seed)
    outs = _step_all(gs, ms, 0)
    # identical on every shard
    for loss, grads in outs[1:]:
        assert loss == outs[0][0] and np.array_equal(grads, outs[0][1])
    loss, grads = outs[0]
    assert abs(loss - ref["loss"]) / abs(ref["loss"]) <= TOL
    for k, blk in split_params(grads, F, H).items():
        e = scaled_err(blk, split_params(ref["grads"], F, H)[k])
        assert e <= TOL, (k, e)
    # forward of the owned rows is bitwise the unsharded one
    for g, m in zip(gs, ms):
        info = mars.graph_shard_info(g)
        r0, r1 = info["row_begin"], info["row_end"]
        rows = np.r_[r0:r1, N + r0:N + r1]
        for l in (1, 2, 3):
            Y, Z = m.export_activations(l)
            assert np.array_equal(Y, ref_acts[l][0][rows]), (l, "Y")
            assert np.array_equal(Z, ref_acts[l][1][rows]), (l, "Z")
    # loss against the fp64 oracle at the same permutation
    b = oracle.Batch([graph])
    perms = b.perms(seed, 0, 0)
    assert np.array_equal(ref["perms"], perms)
    lo, _, _, _ = oracle.step_grads(b, H, p0.astype(np.float64), perms)
    assert abs(loss - lo) / abs(lo) <= TOL


def test_shard_training_trajectory():
    graph = SG.cached("inception", 1)
    F, H, seed, P, n = 64, 128, 8, 3, 5
    g1 = mars.graph_load([graph])
    m1 = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed)
    ref_losses = [m1.step(g1, t, 0, global_batch=1, want_loss=True)["loss"] for t in range(n)]
    gs, ms = _sharded(graph, P, F, H, seed)
    outs = [_step_all(gs, ms, t)[0] for t in range(n)]        # steps >= 2 replay captured graphs
    losses = [o[0] for o in outs]
    states = [m.get_state() for m in ms]
    for st in states[1:]:
        assert np.array_equal(st[0], states[0][0]) and st[3] == n
    # the gradients of the first step agree at the fp32 bar (measured 3e-7);
    # after n Adam steps the parameters are compared at 1e-4: Adam's per-element
    # normalisation m/sqrt(v) turns rounding differences of ~1e-7 on near-zero
    # gradient components (sharded and unsharded dW reduce over different row
    # chunks) into parameter differences of up to O(lr)
    g1.free()
    g1 = mars.graph_load([graph])
    m0 = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed)
    g0 = m0.step(g1, 0, 0, global_batch=1, want_grads=True)["grads"]
    assert scaled_err(outs[0][1], g0) <= TOL
    assert scaled_err(states[0][0], m1.get_state()[0]) <= 1e-4
    assert scaled_err(losses, ref_losses) <= TOL


def test_shard_bf16():
    graph = SG.cached("gnmt", 1)
    F, H, seed, P = 64, 256, 3, 2
    g1 = mars.graph_load([graph])
    m1 = mars.dgi_create(in_dim=F, hidden_dim=H, seed=seed, precision=mars.MARS_BF16)
    ref = m1.step(g1, 0, 0, global_batch=1, want_loss=True, want_grads=True)
    gs, ms = _sharded(graph, P, F, H, seed, precision=mars.MARS_BF16)
    outs = _step_all(gs, ms, 0)
    assert outs[0][0] == outs[1][0] and np.array_equal(outs[0][1], outs[1][1])
    assert abs(outs[0][0] - ref["loss"]) / abs(ref["loss"]) <= 2e-2
    for k, blk in split_params(outs[0][1], F, H).items():
        assert scaled_err(blk, split_params(ref["grads"], F, H)[k]) <= 2e-2, k


def test_shard_misuse_rejected():
    graph = SG.cached("inception", 0)
    with pytest.raises(mars.MarsError):
        mars.graph_load_shard(graph, 9, 0)                  # more than 8 shards
    with pytest.raises(mars.MarsError):
        mars.graph_load_shard(graph, 2, 2)                  # shard index out of range
    g = mars.graph_load_shard(graph, 2, 0)
    m = mars.dgi_create(in_dim=64, hidden_dim=32, seed=0)   # H=32: no tcgen05 path
    with pytest.raises(mars.MarsError):
        mars.shard_attach(m, g)
    plain = mars.graph_load([graph])
    m2 = mars.dgi_create(in_dim=64, hidden_dim=128, seed=0)
    with pytest.raises(mars.MarsError):
        mars.shard_attach(m2, plain)                        # not a shard graph


def test_shard_contrastive_variants_rejected():
    """A row-sharded model runs the default DGI step only: re-setting the
    default is a no-op (the attached workspace is kept and the step still
    runs), any NEXT-4 variant or the SAGE encoder is refused."""
    graph = SG.cached("inception", 0)
    gs, ms = _sharded(graph, 2, 64, 128, 3)
    ms[0].set_contrastive()
    for bad in (dict(num_neg=2), dict(readout="mean"), dict(loss="infonce"),
                dict(aggregator="sage_gcn")):
        with pytest.raises(mars.MarsError):
            ms[0].set_contrastive(**bad)
    out = _step_all(gs, ms, 0)
    assert all(np.isfinite(o[0]) for o in out)
    ms_sage = mars.dgi_create(in_dim=64, hidden_dim=128, seed=3, encoder="sage")
    with pytest.raises(mars.MarsError):
        mars.shard_attach(ms_sage, mars.graph_load_shard(graph, 2, 0))
    for m in ms + [ms_sage]:
        m.free()
    for g in gs:
        g.free()
