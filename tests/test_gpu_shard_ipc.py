"""Row-sharded graph across PROCESSES (the one-process-per-GPU deployment of
SURVEY §8(e)(ii)), on the one GPU of the test box: two processes, each owning
one shard, exchange their CUDA IPC blobs through torch.distributed (gloo) and
step together; peers' buffers are opened with cudaIpcOpenMemHandle, the SpMM
kernels gather halo rows from the other process's memory, and the device
barriers synchronise the two contexts.  (Two contexts on one GPU are
time-sliced, so this checks correctness, not speed.)  Loss, gradients and the
parameters after two steps must equal the in-process sharded run bitwise."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
F, H, SEED, P, STEPS = 64, 128, 6, 2, 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(P), LOCAL_RANK="0")
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=P)
    try:
        import paper_conf_icpp_lancl21_b200 as mars
        from synth import graphs as SG
        graph = SG.cached("inception", 0)
        g = mars.graph_load_shard(graph, P, rank, device=0)
        m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=SEED, device=0)
        mars.shard_attach(m, g)
        blobs = [None] * P
        dist.all_gather_object(blobs, mars.shard_export(m))
        mars.shard_connect(m, blobs)
        dist.barrier()
        out = []
        for t in range(STEPS):
            m.step(g, t, 0, global_batch=1)
            out.append(m.read_step())
        dist.barrier()                      # peers may still read this shard's buffers
        q.put((rank, out, m.get_state()[0], None))
        dist.barrier()
        m.free(); g.free()
    except Exception as e:                  # report instead of hanging the parent
        q.put((rank, None, None, repr(e)))
    dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_two_process_shards_match_in_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(P)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(P):
        r, out, params, err = q.get(timeout=500)
        res[r] = (out, params, err)
    for p in procs:
        p.join(timeout=60)
    for r in range(P):
        assert res[r][2] is None, res[r][2]
    import paper_conf_icpp_lancl21_b200 as mars
    from synth import graphs as SG
    graph = SG.cached("inception", 0)
    gs = [mars.graph_load_shard(graph, P, p) for p in range(P)]
    ms = [mars.dgi_create(in_dim=F, hidden_dim=H, seed=SEED) for _ in range(P)]
    for m, g in zip(ms, gs):
        mars.shard_attach(m, g)
    mars.shard_connect_local(ms)
    for t in range(STEPS):
        for m, g in zip(ms, gs):
            m.step(g, t, 0, global_batch=1)
        ref = ms[0].read_step()
        for r in range(P):
            loss, grads = res[r][0][t]
            assert loss == ref[0] and np.array_equal(grads, ref[1]), (r, t)
    for r in range(P):
        assert np.array_equal(res[r][1], ms[0].get_state()[0])
