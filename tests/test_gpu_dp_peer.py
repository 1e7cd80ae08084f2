"""Data parallelism across PROCESSES with libmars's own peer-memory gradient
exchange (a13, mars_dp_*), on the one GPU of the test box:
two processes (the one-process-per-GPU deployment, here both on device 0 --
two contexts time-slice one GPU, so this checks correctness, not speed) each
own two of the four (graph, sample) pairs, assigned by LPT with every graph
keeping its global pair index.  They exchange CUDA IPC blobs through
torch.distributed (gloo); inside the captured step each rank signals a device
barrier, sums both ranks' partial gradients + loss in rank order (fp64) from
the other process's memory, and passes a second barrier before Adam.

Checked: both ranks hold bitwise identical gradients, losses and parameters
after every step; the gradients and loss equal the single-process four-graph
step (same pair indices) within the fp32 bar; the loss equals the oracle's
four-graph loss; the step-0 gradients match the oracle's fp64 backward at the
single-process GPU's own activations (P3)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from tests.util import scaled_err

pytestmark = pytest.mark.gpu
F, H, SEED, WORLD, PER, STEPS = 64, 128, 12, 2, 2, 3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _graphs():
    from synth import graphs as SG
    return [SG.cached("inception", i) for i in range(WORLD * PER)]


def _worker(rank, port, q, variant=None):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(WORLD), LOCAL_RANK="0")
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        import paper_conf_icpp_lancl21_b200 as mars
        from paper_conf_icpp_lancl21_b200 import dp
        gs = _graphs()
        mine = dp.lpt_assign([dp.graph_cost(x) for x in gs], WORLD, PER)[rank]
        g = mars.graph_load([gs[i] for i in mine], device=0)
        g.set_pair_offsets(mine)                   # global pair index = global graph index
        m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=SEED, device=0, world_size=WORLD,
                            rank=rank)
        if variant:
            m.set_contrastive(**variant)
        dp.connect_peers(m)
        dist.barrier()
        out = []
        for t in range(STEPS):
            m.step(g, t, 0, global_batch=WORLD * PER)   # asynchronous: peers wait on device
            out.append(m.read_step())
        dist.barrier()                      # the peer may still read this rank's gradients
        q.put((rank, mine, out, m.get_state()[0], None))
        dist.barrier()
        m.free(); g.free()
    except Exception as e:                  # report instead of hanging the parent
        q.put((rank, None, None, None, repr(e)))
    dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_two_process_peer_dp_matches_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(WORLD):
        r, mine, out, params, err = q.get(timeout=500)
        res[r] = (mine, out, params, err)
    for p in procs:
        p.join(timeout=60)
    for r in range(WORLD):
        assert res[r][3] is None, res[r][3]
    assert sorted(res[0][0] + res[1][0]) == list(range(WORLD * PER))
    for t in range(STEPS):                            # ranks bitwise identical
        assert res[0][1][t][0] == res[1][1][t][0]
        assert np.array_equal(res[0][1][t][1], res[1][1][t][1])
    assert np.array_equal(res[0][2], res[1][2])

    import oracle
    import paper_conf_icpp_lancl21_b200 as mars
    gs = _graphs()
    g = mars.graph_load(gs)
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=SEED)
    p0 = m.get_state()[0].astype(np.float64)
    b = oracle.Batch(gs)
    for t in range(STEPS):
        o = m.step(g, t, 0, want_loss=True, want_grads=True)
        loss_dp, grads_dp = res[0][1][t]
        assert abs(loss_dp - o["loss"]) <= 1e-5 * abs(o["loss"]), t
        e = scaled_err(grads_dp, o["grads"])
        print("step", t, "dp vs single-process grads", e)
        assert e <= 1e-5, t
        if t == 0:
            acts = {}
            for l in (1, 2, 3):
                acts[f"Y{l}"], acts[f"Z{l}"] = m.export_activations(l)
            loss_o, grads_o, _ = oracle.backward(b, H, p0, acts)
            assert abs(loss_dp - loss_o) <= 1e-5 * abs(loss_o)
            assert scaled_err(grads_dp, grads_o) <= 1e-5
    assert scaled_err(res[0][2], m.get_state()[0]) <= 1e-5


@pytest.mark.timeout(600)
def test_two_process_peer_dp_contrastive_variant():
    """NEXT-4 under the peer exchange: K = 3 corruption samples per graph
    sharing the positive branch (sample k of graph g = pair g K + k with the
    global g) and the InfoNCE loss; both ranks bitwise identical and equal to
    the single-process step on all four graphs."""
    variant = dict(num_neg=3, loss="infonce", corruption="mask", mask_rate=0.2)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q, variant)) for r in range(WORLD)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(WORLD):
        r, mine, out, params, err = q.get(timeout=500)
        res[r] = (mine, out, params, err)
    for p in procs:
        p.join(timeout=60)
    for r in range(WORLD):
        assert res[r][3] is None, res[r][3]
    for t in range(STEPS):
        assert res[0][1][t][0] == res[1][1][t][0]
        assert np.array_equal(res[0][1][t][1], res[1][1][t][1])
    import paper_conf_icpp_lancl21_b200 as mars
    g = mars.graph_load(_graphs())
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=SEED)
    m.set_contrastive(**variant)
    for t in range(STEPS):
        o = m.step(g, t, 0, want_loss=True, want_grads=True)
        loss_dp, grads_dp = res[0][1][t]
        assert abs(loss_dp - o["loss"]) <= 1e-5 * abs(o["loss"]), t
        e = scaled_err(grads_dp, o["grads"])
        print("variant step", t, "dp vs single-process grads", e)
        assert e <= 1e-5, t
    m.free(); g.free()
