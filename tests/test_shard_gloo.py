"""Row-sharded single graph -- the host logic and the
decomposition of one DGI step over shards, on CPU with world_size 2 (gloo).

Each rank owns the row block libmars's host-only mars_shard_partition gives
it, computes its rows of Â_n act(T) with the fp64 oracle, receives ONLY its
halo rows from the peer (every other remote row is NaN, so reading anything
outside the halo poisons the result), and exchanges exactly what the GPU
shards exchange: the readout column sums (Eq. 4), dv and the loss partials
(Eqs. 5-6), and the W partial gradients.  The reassembled loss, dM and dW3
must equal the whole-graph oracle step, and both ranks must agree bitwise.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

F, H, SEED, STEP, N = 16, 32, 11, 3, 300


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _graph():
    from synth import graphs as SG
    return SG.tiny(5, N=N, F=F)


def _prelu(z, a):
    return np.where(z > 0, z, a * z)


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import paper_conf_icpp_lancl21_b200 as mars
    b = oracle.Batch([_graph()])
    starts = mars.shard_partition(b.rowptr, world)
    allst = [None] * world
    dist.all_gather_object(allst, starts.tolist())
    assert all(s == allst[0] for s in allst)
    r0, r1 = int(starts[rank]), int(starts[rank + 1])
    rows = np.r_[r0:r1, N + r0:N + r1]
    cols = b.colind[b.rowptr[r0]:b.rowptr[r1]]
    halo = np.unique(cols[(cols < r0) | (cols >= r1)])

    p = oracle.xavier(SEED, F, H).astype(np.float64)
    o = 0
    W = []
    for cin in (F, H, H):
        W.append(p[o:o + cin * H].reshape(cin, H)); o += cin * H
    M = p[o:o + H * H].reshape(H, H); o += H * H
    alpha = p[o:o + 3]
    perms = b.perms(SEED, STEP, 0)                     # every shard permutes the whole graph

    def gather_halo(Zloc):
        """The peer's rows, reduced to this rank's halo; all else NaN."""
        blocks = [None] * world
        dist.all_gather_object(blocks, (r0, r1, Zloc))
        T = np.full((2 * N, Zloc.shape[1]), np.nan)
        for (a, c, Zb) in blocks:
            n = c - a
            keep = np.arange(a, c) if a == r0 else halo[(halo >= a) & (halo < c)]
            T[keep] = Zb[keep - a]
            T[N + keep] = Zb[n + keep - a]
        return T

    Y, Z = [], []
    T = oracle.layer1_input(b, perms)                  # X and X~ are replicated inputs
    for l in range(3):
        y = oracle.spmm_rows(b, T, rows, None if l == 0 else alpha[l - 1])
        z = y @ W[l]
        assert np.all(np.isfinite(y)), f"layer {l + 1} read a non-halo remote row"
        Y.append(y); Z.append(z)
        if l < 2:
            T = gather_halo(z)
    n = r1 - r0
    H3 = _prelu(Z[2], alpha[2])
    cs = torch.tensor(H3[:n].sum(0)); dist.all_reduce(cs)          # readout exchange
    s = 1.0 / (1.0 + np.exp(-cs.numpy() / N))
    v = M @ s
    lg = H3 @ v
    lp, ln_ = lg[:n], lg[n:]
    sp = lambda x: np.logaddexp(0.0, x)
    dl = np.concatenate([(1 / (1 + np.exp(-lp)) - 1), 1 / (1 + np.exp(-ln_))]) / (2 * N)
    ex = torch.tensor(np.concatenate([dl @ H3, [np.sum(sp(-lp)) + np.sum(sp(ln_))]]))
    dist.all_reduce(ex)                                                # dv + loss exchange
    dv, loss = ex.numpy()[:H], ex.numpy()[H] / (2 * N)
    dM = np.outer(dv, s)
    dm = (M.T @ dv) * s * (1 - s) / N
    dH3 = np.outer(dl, v)
    dH3[:n] += dm
    dZ3 = np.where(Z[2] > 0, dH3, alpha[2] * dH3)
    dW3 = torch.tensor(Y[2].T @ dZ3); dist.all_reduce(dW3)             # gradient exchange
    q.put((rank, loss, dM, dW3.numpy(), starts, len(halo)))
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_two_shard_step_equals_whole_graph():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r[0], r[1:]) for r in [q.get(timeout=240) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import oracle
    b = oracle.Batch([_graph()])
    p = oracle.xavier(SEED, F, H).astype(np.float64)
    loss, grads, _, _ = oracle.step_grads(b, H, p, b.perms(SEED, STEP, 0))
    o = F * H + 2 * H * H
    dM_ref = grads[o:o + H * H].reshape(H, H)
    dW3_ref = grads[F * H + H * H:o].reshape(H, H)
    for r in range(world):
        l, dM, dW3, starts, nh = res[r]
        assert abs(l - loss) <= 1e-13 * abs(loss)
        assert np.max(np.abs(dM - dM_ref)) <= 1e-12 * np.max(np.abs(dM_ref))
        assert np.max(np.abs(dW3 - dW3_ref)) <= 1e-12 * np.max(np.abs(dW3_ref))
        assert nh > 0                                  # the split really has a halo
    assert res[0][0] == res[1][0] and np.array_equal(res[0][2], res[1][2])


def test_partition_rule():
    """mars_shard_partition: contiguous, >= 1 row each, balanced by nnz."""
    import oracle
    import paper_conf_icpp_lancl21_b200 as mars
    b = oracle.Batch([_graph()])
    for P in (1, 2, 3, 5, 8):
        st = mars.shard_partition(b.rowptr, P)
        assert st[0] == 0 and st[-1] == N and np.all(np.diff(st) >= 1)
        nnz = b.rowptr[st[1:]] - b.rowptr[st[:-1]]
        assert nnz.sum() == b.rowptr[-1]
        assert nnz.max() <= b.rowptr[-1] / P + np.max(np.diff(b.rowptr)) + 1
    # degenerate: as many shards as rows -> one row each
    rp = np.arange(0, 9, dtype=np.int32)
    assert list(mars.shard_partition(rp, 8)) == list(range(9))
    with pytest.raises(mars.MarsError):
        mars.shard_partition(rp, 9)
