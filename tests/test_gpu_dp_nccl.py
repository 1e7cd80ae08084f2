"""Data parallelism across PROCESSES with libmars's NCCL allreduce (a13,
DESIGN.md §8.1), on the one GPU of the test box: two processes (the
one-process-per-GPU deployment, here both on device 0), each owning two of the
four (graph, sample) pairs, exchange libmars's ncclUniqueId through
torch.distributed (gloo) and step together; the gradient + loss allreduce runs
inside the captured step.  With several GPUs each rank takes its own device.  Every rank must end with the global-batch gradient
and loss of the single-process four-graph step (up to the summation order of
the allreduce), and identical parameters on both ranks.  NCCL may refuse two
ranks on one device; the test then skips with NCCL's message."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from tests.util import scaled_err

pytestmark = pytest.mark.gpu
F, H, SEED, WORLD, PER, STEPS = 16, 32, 12, 2, 2, 3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, q):
    import torch
    dev = rank % max(1, torch.cuda.device_count())    # one GPU per rank where there are several
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(WORLD), LOCAL_RANK=str(dev))
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        import paper_conf_icpp_lancl21_b200 as mars
        from paper_conf_icpp_lancl21_b200 import dp
        from synth import graphs as SG
        uid = dp.broadcast_unique_id(mars.nccl_get_unique_id)
        base, B = dp.pair_range(rank, WORLD, PER)
        g = mars.graph_load([SG.tiny(i) for i in dp.graph_indices(rank, WORLD, PER)], device=dev)
        m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=SEED, device=dev, world_size=WORLD,
                            rank=rank, nccl_unique_id=uid)
        out = []
        for t in range(STEPS):
            m.step(g, t, base, global_batch=B)
            out.append(m.read_step())
        q.put((rank, out, m.get_state()[0], None))
        dist.barrier()
        m.free()
        g.free()
    except Exception as e:                  # report instead of hanging the parent
        q.put((rank, None, None, repr(e)))
    dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_two_process_nccl_dp_matches_full_batch():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(WORLD):
        r, out, params, err = q.get(timeout=500)
        res[r] = (out, params, err)
    for p in procs:
        p.join(timeout=60)
    errs = [res[r][2] for r in range(WORLD) if res[r][2]]
    if errs:
        if any("NCCL" in e or "ENCCL" in e or "nccl" in e for e in errs):
            pytest.skip(f"NCCL refused two ranks on one device: {errs[0][:200]}")
        raise AssertionError(errs)
    import paper_conf_icpp_lancl21_b200 as mars
    from synth import graphs as SG
    g = mars.graph_load([SG.tiny(i) for i in range(WORLD * PER)])
    m = mars.dgi_create(in_dim=F, hidden_dim=H, seed=SEED)
    for t in range(STEPS):
        m.step(g, t, 0, global_batch=WORLD * PER)
        loss, grads = m.read_step()
        for r in range(WORLD):
            lr, gr = res[r][0][t]
            assert abs(lr - loss) <= 1e-6 * abs(loss), (r, t, lr, loss)
            assert scaled_err(gr, grads) <= 1e-6, (r, t)
    # replicated Adam on identical allreduced gradients: bitwise equal parameters
    assert np.array_equal(res[0][1], res[1][1])
    assert scaled_err(res[0][1], m.get_state()[0]) <= 1e-5
