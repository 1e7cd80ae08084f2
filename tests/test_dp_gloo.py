"""Multi-process (world_size 2, gloo, CPU) checks of the data-parallel host
logic (a13, reading c15): contiguous pair assignment, gradients pre-scaled by
1/B_global on each rank, allreduce(sum), the ncclUniqueId broadcast path.
Each rank computes its share with the fp64 oracle; the sum must equal the
single-process full-batch result, and one replicated Adam step must leave the
ranks bit-identical."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_lancl21_b200 import dp

F, H, SEED, STEP, PER_RANK = 16, 32, 13, 4, 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from synth import graphs as SG
    r, w, _ = dp.env()
    base, B = dp.pair_range(r, w, PER_RANK)
    gs = [SG.tiny(i) for i in dp.graph_indices(r, w, PER_RANK)]
    b = oracle.Batch(gs)
    p = oracle.xavier(SEED, F, H).astype(np.float64)
    loss, grads, _, _ = oracle.step_grads(b, H, p, b.perms(SEED, STEP, base), B=B)
    t = torch.tensor(np.concatenate([grads, [loss]]))
    dist.all_reduce(t)
    uid = dp.broadcast_unique_id(lambda: bytes(range(128)))
    g_all = t.numpy()
    p1, _, _ = oracle.adam(p, np.zeros_like(p), np.zeros_like(p), g_all[:-1], 1)
    q.put((rank, g_all, p1, uid))
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_two_rank_allreduce_equals_full_batch():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r, (g, p1, u)) for r, g, p1, u in [q.get(timeout=240) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import oracle
    from synth import graphs as SG
    gs = [SG.tiny(i) for i in range(world * PER_RANK)]
    b = oracle.Batch(gs)
    p = oracle.xavier(SEED, F, H).astype(np.float64)
    loss, grads, _, _ = oracle.step_grads(b, H, p, b.perms(SEED, STEP, 0))
    g0 = res[0][0]
    assert abs(g0[-1] - loss) < 1e-14
    assert np.max(np.abs(g0[:-1] - grads)) <= 1e-13 * np.max(np.abs(grads))
    assert np.array_equal(res[0][0], res[1][0])          # identical reduced gradients
    assert np.array_equal(res[0][1], res[1][1])          # replicated Adam: identical params
    assert res[0][2] == res[1][2] == bytes(range(128))   # unique-id broadcast


def test_pair_range():
    assert dp.pair_range(0, 1, 16) == (0, 16)
    assert dp.pair_range(3, 8, 16) == (48, 128)
    assert dp.graph_indices(1, 2, 3) == [3, 4, 5]
    with pytest.raises(ValueError):
        dp.pair_range(2, 2, 1)


def test_lpt_assign_deterministic_and_balanced():
    from synth import graphs as SG
    costs = [dp.graph_cost(SG.cached("gnmt", i)) for i in range(32)]
    for world in (1, 2, 4, 8):
        per = 32 // world
        a = dp.lpt_assign(costs, world, per)
        assert a == dp.lpt_assign(list(costs), world, per)          # deterministic
        assert sorted(sum(a, [])) == list(range(32))                  # a partition
        assert all(len(x) == per for x in a)                          # b graphs per rank
        loads = [sum(costs[i] for i in x) for x in a]
        # LPT's bound: no rank exceeds the mean by more than one graph
        assert max(loads) <= sum(costs) / world + max(costs)
        blocks = [sum(costs[i] for i in dp.graph_indices(r, world, per)) for r in range(world)]
        assert max(loads) <= max(blocks)                              # never worse than blocks
    with pytest.raises(ValueError):
        dp.lpt_assign(costs, 3, 10)


def _lpt_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from synth import graphs as SG
    gl = [SG.tiny(i) for i in range(world * PER_RANK)]
    mine = dp.lpt_assign([dp.graph_cost(g) for g in gl], world, PER_RANK)[rank]
    gs = [gl[i] for i in mine]
    b = oracle.Batch(gs)
    p = oracle.xavier(SEED, F, H).astype(np.float64)
    # pair index of each graph = its global index (mars_graph_set_pair_offsets)
    perms = np.concatenate([oracle.perm(SEED, STEP, i, gl[i].num_nodes) for i in mine])
    loss, grads, _, _ = oracle.step_grads(b, H, p, perms.astype(np.int32), B=world * PER_RANK)
    t = torch.tensor(np.concatenate([grads, [loss]]))
    dist.all_reduce(t)
    q.put((rank, mine, t.numpy()))
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_two_rank_lpt_with_global_pair_ids_equals_full_batch():
    """LPT-assigned graphs keeping their global pair index: the reduced
    gradient is the single-process full batch's (pair index = graph index),
    i.e. independent of which rank ran which graph (c15)."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_lpt_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r, (mine, g)) for r, mine, g in [q.get(timeout=240) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert sorted(res[0][0] + res[1][0]) == list(range(world * PER_RANK))
    import oracle
    from synth import graphs as SG
    gs = [SG.tiny(i) for i in range(world * PER_RANK)]
    b = oracle.Batch(gs)
    p = oracle.xavier(SEED, F, H).astype(np.float64)
    loss, grads, _, _ = oracle.step_grads(b, H, p, b.perms(SEED, STEP, 0))
    g0 = res[0][1]
    assert abs(g0[-1] - loss) < 1e-14
    assert np.max(np.abs(g0[:-1] - grads)) <= 1e-13 * np.max(np.abs(grads))
