"""Multi-GPU plumbing: one process per GPU, torch.distributed
for the process group, and the library context's own NCCL communicator for
the data path.  This module holds no method arithmetic: every exchange and
every combine of per-rank results (the (score desc, index asc) pick, the
vector gather, the frontier all-reduces, the per-scenario aggregate sum) runs
inside libproteus.so (csrc/comm.cu) on the context's stream.

    dist.init_process_group("nccl", ...)
    px = Proteus(local_rank)
    init_comm(px)                 # NCCL unique id from rank 0 over the group
    px.solve_batch(...)           # distributed: every rank gets the optima
    px.replay(...)                # distributed: scenarios split by owner

Work split (the library's; shard_range mirrors it for the callers that size
buffers):
  * flat / multiset search: contiguous index-range slices, one ncclAllGather
    of the materialised per-rank winners, a device pick per vector;
  * factored batched re-solve (c4, the f4 re-solves): demand-vector slices,
    one ncclAllGather of the solutions;
  * Fig. 1b frontier: index slices, ncclAllReduce(MAX) of the best accuracy
    per capacity + ncclAllReduce(MIN) of the lowest index per point;
  * replay / closed loop (c5, f2, f4): scenario s on rank owner[s]
    (proteus_scenario_owner: a cost-balanced greedy), one
    ncclAllReduce(SUM) of the per-scenario aggregates.

Without NCCL (e.g. a gloo group) the per-rank results can be moved by any
transport and combined by the library: combine_batch_over_group.
"""

from __future__ import annotations

import numpy as np


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous slice r of [0, n) -- the split the library uses."""
    return n * rank // world, n * (rank + 1) // world


def broadcast_unique_id(uid: bytes | None, group=None) -> bytes:
    """The 128-byte NCCL unique id of rank 0, on every rank of `group` (any
    torch.distributed backend)."""
    import torch.distributed as dist
    obj = [uid if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def init_comm(px, group=None):
    """Give the Proteus context `px` an NCCL communicator over the ranks of
    `group` (rank 0 draws the id, torch.distributed broadcasts it); later
    library calls are distributed (include/proteus.h, multi-GPU)."""
    import torch.distributed as dist
    from . import Proteus
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    uid = broadcast_unique_id(Proteus.comm_unique_id() if rank == 0 else None, group)
    px.comm_init(uid, world, rank)
    return world, rank


def combine_batch_over_group(px, local: dict, ncand: int, D: int, group=None):
    """Transport-agnostic combine of a sliced batched flat search (modes 0/1,
    proteus_solve_batch with shard_rank / shard_world): the per-rank outputs
    are all-gathered over `group` (gloo or anything torch.distributed
    offers) and combined on this rank's GPU by proteus_combine_solutions.
    Returns (dict of arrays, candidates of the whole space per vector)."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    parts = [None] * world
    dist.all_gather_object(parts, ({k: np.asarray(v) for k, v in local.items()}, int(ncand)), group=group)
    return px.combine_solutions([p[0] for p in parts], [p[1] for p in parts], D)
