"""Host-side data-parallel plumbing (a13).

Data parallelism over independent (graph, sample) pairs (reading c15).  Each
graph keeps its GLOBAL index as its pair index, whatever rank runs it, so a
graph's corruption permutation does not depend on the rank count.  Graphs are
assigned to ranks by deterministic LPT (longest processing time first) on
their cost, b graphs per rank (weak scaling); every rank scales its partial
gradients by 1/B_global inside the kernels, so one sum over the ranks gives
the global-batch mean and the replicated Adam keeps parameters identical.

The exchange itself runs in libmars, captured in the step's CUDA Graph:
either its own peer-memory kernel (mars_dp_*: rank-ordered fp64 sum reading
the peers' gradients over NVLink, between two device barriers) or an NCCL
allreduce.  torch.distributed is only the rendezvous that all-gathers the
peer-memory blobs or broadcasts the ncclUniqueId.
"""
from __future__ import annotations

import os


def env():
    """(rank, world_size, local_rank) from the torchrun environment."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def pair_range(rank: int, world: int, per_rank: int):
    """(pair_base, global_batch) of `rank` under contiguous block assignment."""
    if not (0 <= rank < world) or per_rank < 1:
        raise ValueError("bad rank / world / per_rank")
    return rank * per_rank, world * per_rank


def graph_indices(rank: int, world: int, per_rank: int):
    base, _ = pair_range(rank, world, per_rank)
    return list(range(base, base + per_rank))


def lpt_assign(costs, world: int, per_rank: int):
    """Deterministic LPT: graphs in decreasing cost (ties: lower index first),
    each to the rank with the smallest load so far among ranks holding fewer
    than per_rank graphs (ties: lower rank).  len(costs) must equal
    world * per_rank.  Returns world sorted lists of global graph indices."""
    n = len(costs)
    if world < 1 or per_rank < 1 or n != world * per_rank:
        raise ValueError("need exactly world * per_rank costs")
    order = sorted(range(n), key=lambda i: (-costs[i], i))
    load = [0] * world
    out = [[] for _ in range(world)]
    for i in order:
        r = min((q for q in range(world) if len(out[q]) < per_rank), key=lambda q: (load[q], q))
        out[r].append(i)
        load[r] += costs[i]
    return [sorted(x) for x in out]


def graph_cost(g) -> int:
    """Work proxy of one op graph: N + 2E (the stored entries of Â before
    deduplication bound the SpMM's gathers; the dense parts scale with N)."""
    return int(g.num_nodes) + 2 * int(g.indptr[g.num_nodes])


def broadcast_unique_id(get_id, group=None) -> bytes | None:
    """Rank 0 calls get_id() (libmars's mars_nccl_get_unique_id) and every rank
    receives the same 128 bytes through torch.distributed."""
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return None
    obj = [get_id() if dist.get_rank() == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def connect_peers(m, group=None):
    """Peer-memory gradient exchange: all-gather every rank's mars_dp_export
    blob in rank order through torch.distributed and mars_dp_connect."""
    import torch.distributed as dist
    from . import mars as _m
    blobs = [None] * dist.get_world_size(group)
    dist.all_gather_object(blobs, _m.dp_export(m), group=group)
    _m.dp_connect(m, blobs)
