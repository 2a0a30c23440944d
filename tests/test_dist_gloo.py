"""Multi-process (world_size 2, gloo, CPU) coverage of the N > 1 host logic
(SURVEY §8(e)): the NCCL unique-id broadcast that joins the library contexts,
the work splits the library uses (index slices, demand-vector slices, the
scenario owners of proteus_scenario_owner -- host code of libproteus.so that
runs without a GPU), and that each split is exact: per-rank results combined
in the library's order reproduce the single-process answer.  The per-rank
GPU work is stood in for by the oracle; the library's device-side combine
(NCCL all-gather / all-reduce + pick kernels) is covered by -m gpu
(tests/test_gpu_solve.py: combine_solutions, the world-1 NCCL communicator)."""

import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _run(worker, world=2, timeout=600):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = [q.get(timeout=timeout) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out, key=lambda o: o[0])


def _init(rank, world, port):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    return dist


def _rank_best(prof, dev, slo, dem, lo, hi):
    """Best (score, index) over flat indices [lo, hi) by the oracle: device 0
    is the most significant digit (reading C9); ascending order + strict >
    keeps the lowest index among ties."""
    import oracle
    K, D = 1 + prof.M, len(dev)
    best = None
    for idx in range(lo, hi):
        opt = [(idx // K ** (D - 1 - d)) % K for d in range(D)]
        r = oracle.score_placement(prof, dev, slo, dem, np.array(opt))
        sc = (r["served"] << 42) | r["accsum"]
        if best is None or sc > best[0]:
            best = (sc, idx)
    return best if best else (0, (1 << 64) - 1)


def _id_worker(rank, world, port, q):
    dist = _init(rank, world, port)
    try:
        from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, scenario_owner, workloads as W
        from paper_conf_asplos_ahmadgfwsw24_b200.dist import broadcast_unique_id, shard_range
        uid = broadcast_unique_id(Proteus.comm_unique_id() if rank == 0 else None)
        sc = np.concatenate([W.scenarios_64(0, 0), W.scenarios_fig6(0), W.scenarios_64(0, 1)])
        owner = scenario_owner(sc, world)
        lo, hi = shard_range(3600, rank, world)
        q.put((rank, uid, owner.tolist(), lo, hi))
    finally:
        dist.destroy_process_group()


def test_world2_comm_id_broadcast_and_splits():
    """Rank 0's 128-byte NCCL id reaches every rank unchanged (the bytes
    proteus_comm_init needs); every rank computes the same scenario owners
    (each scenario owned once, loads balanced) and disjoint vector slices."""
    out = _run(_id_worker)
    assert len(out[0][1]) == 128 and out[0][1] == out[1][1]
    assert out[0][2] == out[1][2]
    owner = np.array(out[0][2])
    assert set(owner.tolist()) <= {0, 1} and abs(int(np.sum(owner == 0)) - int(np.sum(owner == 1))) <= 24
    assert (out[0][3], out[0][4], out[1][3], out[1][4]) == (0, 1800, 1800, 3600)


def _flat_worker(rank, world, port, q):
    dist = _init(rank, world, port)
    try:
        from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
        from paper_conf_asplos_ahmadgfwsw24_b200.dist import shard_range
        cfg = W.config("c1")
        prof, cl = cfg["prof"], cfg["cluster"]
        dems = np.array([[0, 0], [300, 100], [600, 0], [800, 700]], np.int32)
        n = (1 + prof.M) ** len(cl.device_type)
        lo, hi = shard_range(n, rank, world)
        mine = [_rank_best(prof, cl.device_type, cl.slo_us, d, lo, hi) for d in dems]
        parts = [None] * world
        dist.all_gather_object(parts, mine)
        q.put((rank, parts))
    finally:
        dist.destroy_process_group()


def test_world2_flat_slices_combine_to_the_optimum(oracle_mod):
    """Index-range slices (the library's split) of c1: the (score desc,
    index asc) maximum of the per-rank slice winners -- the order of
    k_pick_solrec -- is the single-process optimum for every demand vector,
    on every rank."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c1")
    prof, cl = cfg["prof"], cfg["cluster"]
    dems = np.array([[0, 0], [300, 100], [600, 0], [800, 700]], np.int32)
    refs = [oracle_mod.solve(prof, cl.device_type, cl.slo_us, d, 0) for d in dems]
    for _, parts in _run(_flat_worker):
        for v, r in enumerate(refs):
            cands = [p[v] for p in parts]
            best = max(cands, key=lambda si: (si[0], -si[1]))
            assert best == ((r["served"] << 42) | r["accsum"], r["index"])


def _replay_worker(rank, world, port, q):
    dist = _init(rank, world, port)
    try:
        import torch
        import oracle
        from paper_conf_asplos_ahmadgfwsw24_b200 import scenario_owner, workloads as W
        cfg = W.config("c3", totals=(12000,))
        prof, cl = cfg["prof"], cfg["cluster"]
        r = oracle.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
        a, f = W.query_trace(8000, 12000.0, cfg["weights"], 17, "gamma")
        sc = oracle.scenario_rows(np.concatenate([W.scenarios_64(0, 0)[::9], W.scenarios_fig6(0)[::13]]))
        mine = np.flatnonzero(scenario_owner(sc, world) == rank)
        agg = np.zeros((3, len(sc)), np.int64)
        if len(mine):
            o = oracle.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f,
                              sc[mine], want_latency=False)
            for k, name in enumerate(("violations", "on_time", "acc_sum")):
                agg[k, mine] = o[name].astype(np.int64)
        t = torch.from_numpy(agg)
        dist.all_reduce(t)  # zero-padded per-scenario aggregates: the sum is a gather
        q.put((rank, mine.tolist(), t.numpy().tolist()))
    finally:
        dist.destroy_process_group()


def test_world2_scenario_owner_replay(oracle_mod):
    """§8(e) replay split: scenario s on rank owner[s]; the zero-padded
    per-scenario aggregates summed over ranks (the library's all-reduce)
    equal the single-process aggregates; each scenario ran exactly once."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3", totals=(12000,))
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    a, f = W.query_trace(8000, 12000.0, cfg["weights"], 17, "gamma")
    sc = np.concatenate([W.scenarios_64(0, 0)[::9], W.scenarios_fig6(0)[::13]])
    ref = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f, sc,
                            want_latency=False)
    out = _run(_replay_worker)
    assert sorted(out[0][1] + out[1][1]) == list(range(len(sc)))
    for _, _, agg in out:
        for k, name in enumerate(("violations", "on_time", "acc_sum")):
            assert agg[k] == ref[name].astype(np.int64).tolist(), name


@pytest.mark.parametrize("world", [3, 8])
def test_scenario_owner_balance(world):
    """proteus_scenario_owner (host code of the library): deterministic, every
    scenario owned once, and the measured-cost model balances
    the expensive scenarios: §5 scenarios with batch cap > 1 differ by at most
    one per rank, and the Nexus scenarios (the slowest lanes) spread evenly --
    unlike contiguous slices, which would put all of them on the last ranks."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import scenario_owner, workloads as W
    sc = W.scenarios_64(0)
    o = scenario_owner(sc, world)
    assert o.tolist() == scenario_owner(sc, world).tolist()
    assert set(o.tolist()) == set(range(world))
    heavy = np.bincount(o[sc[:, 1] != 1], minlength=world)
    assert heavy.max() - heavy.min() <= 1
    mixed = np.concatenate([W.scenarios_64(0, 0), W.scenarios_64(0, 1)[:16]])
    om = scenario_owner(mixed, world)
    nex = np.bincount(om[mixed[:, 3] == 1], minlength=world)
    assert nex.max() - nex.min() <= 1
