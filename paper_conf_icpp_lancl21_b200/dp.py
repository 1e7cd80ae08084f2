"""Host-side data-parallel plumbing (a13).

Data parallelism over independent (graph, sample) pairs (reading c15): rank r
owns the contiguous global pair indices [r*b, (r+1)*b); every rank scales its
partial gradients by 1/B_global inside the kernels, so one NCCL allreduce(sum)
of the flat gradient (+ loss) inside libmars gives the global-batch mean on
every rank and the replicated Adam keeps parameters identical.

torch.distributed is only the rendezvous: it broadcasts libmars's 128-byte
ncclUniqueId from rank 0 (the gradient collective itself is issued by libmars
on its own stream, captured in the step's CUDA Graph).
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


def broadcast_unique_id(get_id, group=None) -> bytes | None:
    """Rank 0 calls get_id() (libmars's mars_nccl_get_unique_id) and every rank
    receives the same 128 bytes through torch.distributed."""
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return None
    obj = [get_id() if dist.get_rank() == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]
