"""Multi-GPU sharding of the allocation search.

Flat / multiset search (modes 0/1): rank r scans the r-th contiguous slice of
the candidate index space on its own GPU, then ONE all-reduce over the process
group combines the per-rank winners: every rank writes its (score, index) into
its own two slots of an int64[2 * world] vector (zeros elsewhere), the SUM
all-reduce assembles all slots, and every rank picks the lexicographic maximum
(score desc, index asc) -- the same order as the in-GPU warp/block/grid
argmax, so the result is identical for every world size.  128 bytes at 8
ranks; NCCL over NVLink on GPUs, gloo in the CPU tests.

Batched flat search (the bench step): every rank scans its slice for every
demand vector of the batch in one library call, and ONE all-gather of the
per-rank winners -- each already materialised -- gives every rank the batch's
optima (solve_sharded_batch; no re-materialisation).

Factored batched re-solve (mode 2, config c4): demand vectors are
independent; rank r solves vectors [r*n/world, (r+1)*n/world) -- no collective
on the data path (weak scaling).

Replay / closed loop (c5, f2, f4): scenarios are independent; rank r replays
its slice and one SUM all-reduce of a zero-padded [3][S] vector gathers the
per-scenario aggregates (replay_sharded).  Fig. 1b: index-range slices and a
host-side frontier merge (pareto_merge).
"""

from __future__ import annotations

import numpy as np

U64 = (1 << 64) - 1


def _to_i64(u: int) -> int:
    u &= U64
    return u - (1 << 64) if u >= (1 << 63) else u


def _to_u64(i: int) -> int:
    return int(i) & U64


def slot_vector(rank: int, world: int, score: int, index: int) -> np.ndarray:
    v = np.zeros(2 * world, np.int64)
    v[2 * rank] = _to_i64(score)
    v[2 * rank + 1] = _to_i64(index)
    return v


def pick_best(slots) -> tuple[int, int, int]:
    """(score, index, rank) of the lexicographic maximum (score desc, index asc)."""
    slots = np.asarray(slots, dtype=np.int64)
    best = None
    for r in range(len(slots) // 2):
        s, i = _to_u64(slots[2 * r]), _to_u64(slots[2 * r + 1])
        if best is None or s > best[0] or (s == best[0] and i < best[1]):
            best = (s, i, r)
    return best


def allreduce_best(score: int, index: int, group=None, device=None) -> tuple[int, int, int]:
    """The slot all-reduce.  `device`: torch device of the collective's tensor
    (cuda for NCCL, cpu for gloo)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    t = torch.from_numpy(slot_vector(rank, world, score, index))
    if device is not None:
        t = t.to(device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return pick_best(t.cpu().numpy())


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous slice r of [0, n) -- the same split the library uses."""
    return n * rank // world, n * (rank + 1) // world


def solve_sharded(px, device_type, slo_us, demand, mode=0, group=None, comm_device=None):
    """Modes 0/1 on every rank of `group`: local slice on this GPU, one slot
    all-reduce, then the winner's full solution (placement + z) materialised
    locally from its canonical index.  Returns (Solution, local Solution)."""
    import torch.distributed as dist
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    local = px.solve(device_type, slo_us, demand, mode=mode, shard_rank=rank, shard_world=world)[0]
    s, i, _ = allreduce_best(local.score, local.index, group, comm_device)
    sol = px.materialize(device_type, slo_us, demand, i, mode=mode)
    assert sol.score == s
    return sol, local


def solve_vectors_sharded(px, device_type, slo_us, demand_vectors, group=None):
    """Mode 2 over a batch of demand vectors, split by vector across ranks."""
    import torch.distributed as dist
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    lo, hi = shard_range(len(demand_vectors), rank, world)
    if hi <= lo:
        return lo, []
    return lo, px.solve(device_type, slo_us, demand_vectors[lo:hi], mode=2)


def pareto_merge(parts):
    """Frontier of the union of shard frontiers (Fig. 1b, proteus_pareto with
    shard_rank/shard_world): a point dominated inside a shard is dominated in
    the whole space, so the union holds every frontier point; keep the points
    strictly more accurate than everything of higher capacity (exact integer
    cross-multiplication), the lowest index among equal points.  Host-side
    combination of <= a few hundred points per shard, like pick_best."""
    pts = {}
    for p in parts:
        for c, a, i in zip(p["cap"].tolist(), p["accsum"].tolist(), p["index"].tolist()):
            key = (int(c), int(a))
            if key not in pts or int(i) < pts[key]:
                pts[key] = int(i)
    by_cap = {}
    for (c, a), i in pts.items():  # at one capacity only the largest accuracy sum can survive
        if c not in by_cap or a > by_cap[c][0] or (a == by_cap[c][0] and i < by_cap[c][1]):
            by_cap[c] = (a, i)
    out, ra, rc = [], 0, 0
    for c in sorted(by_cap, reverse=True):
        a, i = by_cap[c]
        above = a * rc > ra * c if (c > 0 and rc > 0) else (a > 0 if c > 0 else (rc == 0 and ra == 0))
        if above:
            out.append((c, a, i))
            ra, rc = a, c
    out.reverse()
    return dict(cap=np.array([o[0] for o in out], np.int64), accsum=np.array([o[1] for o in out], np.int64),
                index=np.array([o[2] for o in out], np.uint64),
                n_configs=sum(int(p["n_configs"]) for p in parts), n_front=len(out))


def gather_aggregates(lo: int, hi: int, S: int, parts: dict, group=None, device=None) -> dict:
    """Per-scenario aggregates of scenarios [lo, hi) from every rank into full
    [S] arrays on every rank: each rank writes its slice into a zero
    int64[3][S] tensor, one SUM all-reduce assembles it (scenario slices are
    disjoint, so the sum is a gather).  768 bytes per 32 scenarios."""
    import torch
    import torch.distributed as dist
    v = np.zeros((3, S), np.int64)
    for k, name in enumerate(("violations", "on_time", "acc_sum")):
        v[k, lo:hi] = np.asarray(parts[name], dtype=np.uint64).astype(np.int64)
    t = torch.from_numpy(v)
    if device is not None:
        t = t.to(device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    out = t.cpu().numpy().astype(np.uint64)
    return dict(violations=out[0], on_time=out[1], acc_sum=out[2])


def replay_sharded(replay, scenarios, group=None, comm_device=None, **kw):
    """Replay (c5) / closed loop (f4) with the scenarios split by rank
    (scenarios are independent): this rank runs slice
    shard_range(S) through `replay(scenarios=..., **kw)` (Proteus.replay or
    Proteus.replay_epochs, keyword arguments) and the per-scenario aggregates
    are gathered to every rank; per-query latencies stay on their rank.
    Returns (aggregates over all S, this rank's result, (lo, hi))."""
    import torch.distributed as dist
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    sc = np.asarray(scenarios, dtype=np.int32)
    S = len(sc)
    lo, hi = shard_range(S, rank, world)
    if hi > lo:
        local = replay(scenarios=sc[lo:hi], **kw)
    else:
        local = dict(latency=None, violations=np.zeros(0, np.uint64), on_time=np.zeros(0, np.uint64),
                     acc_sum=np.zeros(0, np.uint64))
    return gather_aggregates(lo, hi, S, local, group, comm_device), local, (lo, hi)


# ------------------------------------------------ batched flat search --
BATCH_HEAD = ("score", "index", "served", "unmet", "accsum", "eff_acc_micro")


def pack_batch(out: dict, D: int, ncand: int) -> np.ndarray:
    """proteus_solve_batch arrays of this rank -> int64 rows [n][7 + 2D]:
    the BATCH_HEAD fields (uint64 score / index as their bit patterns), the
    rank's slice size, option[D], z[D]."""
    n = len(out["score"])
    cols = [np.asarray(out[k]).astype(np.uint64).view(np.int64).reshape(n, 1) if k in ("score", "index")
            else np.asarray(out[k], np.int64).reshape(n, 1) for k in BATCH_HEAD]
    cols.append(np.full((n, 1), ncand, np.int64))
    cols += [np.asarray(out["option"], np.int64).reshape(n, D), np.asarray(out["z_qps"], np.int64).reshape(n, D)]
    return np.ascontiguousarray(np.concatenate(cols, axis=1))


def pick_batch(gathered: np.ndarray, D: int):
    """gathered [world][n][7 + 2D]: per vector the rank with the
    lexicographic maximum (score desc, index asc) -- its local winner is the
    global one, already materialised (placement, z, value).  Returns (dict of
    arrays, candidates of the whole space per vector)."""
    s = gathered[:, :, 0].view(np.uint64)
    i = gathered[:, :, 1].view(np.uint64)
    best = s.max(axis=0)
    r = np.where(s == best[None, :], i, np.uint64(U64)).argmin(axis=0)
    rows = gathered[r, np.arange(gathered.shape[1])]
    out = {k: rows[:, c] for c, k in enumerate(BATCH_HEAD)}
    out["score"] = rows[:, 0].view(np.uint64)
    out["index"] = rows[:, 1].view(np.uint64)
    out["option"] = rows[:, 7:7 + D].astype(np.int32)
    out["z_qps"] = rows[:, 7 + D:].astype(np.int32)
    return out, int(gathered[:, 0, 6].sum()) if gathered.shape[1] else 0


def solve_sharded_batch(px, device_type, slo_us, demand, mode=0, group=None, comm_device=None):
    """Modes 0/1 for a batch of demand vectors on every rank of `group`: one
    proteus_solve_batch call scans this rank's index slice for every vector
    (one host synchronisation), then ONE all-gather of the per-rank winners,
    each already materialised, and the per-vector (score desc, index asc)
    pick, all in numpy -- no re-materialisation, no per-vector host objects.
    Returns (dict of arrays over the batch, this rank's dict, candidates of
    the whole space per vector, candidates of this rank's slice per vector)."""
    import torch
    import torch.distributed as dist
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    D = len(device_type)
    local, ncand = px.solve_batch(device_type, slo_us, demand, mode=mode, shard_rank=rank, shard_world=world)
    t = torch.from_numpy(pack_batch(local, D, ncand))
    if comm_device is not None:
        t = t.to(comm_device)
    if t.is_cuda:  # NCCL: one flat buffer, one device-to-host copy
        flat = torch.empty((world,) + tuple(t.shape), dtype=t.dtype, device=t.device)
        dist.all_gather_into_tensor(flat, t, group=group)
        gathered = flat.cpu().numpy()
    else:
        parts = [torch.empty_like(t) for _ in range(world)]
        dist.all_gather(parts, t, group=group)
        gathered = np.stack([p.numpy() for p in parts])
    best, n_all = pick_batch(gathered, D)
    return best, local, n_all, ncand
