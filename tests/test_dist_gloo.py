"""Multi-process (world_size 2, gloo, CPU) coverage of the N > 1 host logic:
the slot all-reduce that combines per-rank search winners, the index-range
and demand-vector splits.  The per-rank search itself is stood in for by the
oracle over the rank's index range (the GPU kernels are covered by -m gpu)."""

import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _rank_best(prof, dev, slo, dem, lo, hi):
    """Best (score, index) over flat indices [lo, hi): device 0 is the most
    significant digit (reading C9); ascending order + strict > keeps the
    lowest index among ties."""
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


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    from paper_conf_asplos_ahmadgfwsw24_b200.dist import allreduce_best, shard_range
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        cfg = W.config("c1")
        prof, cl, dem = cfg["prof"], cfg["cluster"], cfg["demand"][0]
        n = (1 + prof.M) ** len(cl.device_type)
        lo, hi = shard_range(n, rank, world)
        s, i = _rank_best(prof, cl.device_type, cl.slo_us, dem, lo, hi)
        gs, gi, grank = allreduce_best(s, i)
        # demand-vector split of the batched re-solve covers every vector once
        vlo, vhi = shard_range(3600, rank, world)
        cover = np.zeros(3600, np.int64)
        cover[vlo:vhi] = 1
        import torch
        t = torch.from_numpy(cover)
        dist.all_reduce(t)
        q.put((rank, gs, gi, grank, int(t.min()), int(t.max())))
    finally:
        dist.destroy_process_group()


def test_world2_slot_allreduce_matches_single_process(oracle_mod):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c1")
    prof, cl, dem = cfg["prof"], cfg["cluster"], cfg["demand"][0]
    ref = oracle_mod.solve(prof, cl.device_type, cl.slo_us, dem, 0)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, gs, gi, grank, cmin, cmax in out:
        assert gi == ref["index"]
        assert gs == (ref["served"] << 42) | ref["accsum"]
        assert (cmin, cmax) == (1, 1)
    assert len({o[3] for o in out}) == 1


def test_pick_best_order_and_sign():
    """Slots carry uint64 bit patterns in int64; the combine order is (score
    desc, index asc) -- the same as the in-GPU reduction."""
    from paper_conf_asplos_ahmadgfwsw24_b200.dist import pick_best, slot_vector
    big = (1 << 63) + 5
    v = slot_vector(0, 3, big, 7) + slot_vector(1, 3, big, 3) + slot_vector(2, 3, 10, 0)
    assert pick_best(v) == (big, 3, 1)
    v = slot_vector(0, 2, 4, 9) + slot_vector(1, 2, 4, 9)
    assert pick_best(v)[:2] == (4, 9)


def _replay_worker(rank, world, port, q):
    """Scenario-split replay: the per-rank replay is stood in for by the
    oracle over this rank's scenario slice."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    import oracle
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    from paper_conf_asplos_ahmadgfwsw24_b200.dist import replay_sharded
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        cfg = W.config("c3", totals=(12000,))
        prof, cl = cfg["prof"], cfg["cluster"]
        r = oracle.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
        a, f = W.query_trace(8000, 12000.0, cfg["weights"], 17, "gamma")
        sc = np.concatenate([W.scenarios_64(0, 0)[::9], W.scenarios_fig6(0)[::13]])

        def rep(scenarios):
            return oracle.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f,
                                 scenarios, want_latency=False)

        agg, _, (lo, hi) = replay_sharded(rep, sc)
        q.put((rank, lo, hi, {k: v.tolist() for k, v in agg.items()}))
    finally:
        dist.destroy_process_group()


def test_world2_scenario_split_replay(oracle_mod):
    """§8(e) replay: scenarios split by rank, aggregates gathered by one SUM
    all-reduce -- every rank ends with the single-process aggregates."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3", totals=(12000,))
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    a, f = W.query_trace(8000, 12000.0, cfg["weights"], 17, "gamma")
    sc = np.concatenate([W.scenarios_64(0, 0)[::9], W.scenarios_fig6(0)[::13]])
    ref = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f, sc,
                            want_latency=False)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_replay_worker, args=(rk, 2, port, q)) for rk in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    spans = sorted((lo, hi) for _, lo, hi, _ in out)
    assert spans[0][0] == 0 and spans[0][1] == spans[1][0] and spans[1][1] == len(sc)
    for _, _, _, agg in out:
        for k in ("violations", "on_time", "acc_sum"):
            assert agg[k] == ref[k].tolist(), k


def _batch_worker(rank, world, port, q):
    """Batched flat search split by index range: the per-rank library call is
    stood in for by a fake `px` whose solve() returns, per demand vector, the
    oracle's best over the rank's index slice, materialised by the oracle."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    import oracle
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    from paper_conf_asplos_ahmadgfwsw24_b200.dist import shard_range, solve_sharded_batch
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        cfg = W.config("c1")
        prof, cl = cfg["prof"], cfg["cluster"]
        dems = np.array([[0, 0], [300, 100], [600, 0], [800, 700]], np.int32)
        K, D = 1 + prof.M, len(cl.device_type)

        class FakePx:
            def solve_batch(self, device_type, slo_us, demand, mode, shard_rank, shard_world):
                n = K ** D
                lo, hi = shard_range(n, shard_rank, shard_world)
                out = {k: [] for k in ("score", "index", "served", "unmet", "accsum", "eff_acc_micro", "option",
                                       "z_qps")}
                for dem in demand:
                    s, i = _rank_best(prof, device_type, slo_us, dem, lo, hi)
                    opt = np.array([(i // K ** (D - 1 - d)) % K for d in range(D)], np.int32)
                    r = oracle.score_placement(prof, device_type, slo_us, dem, opt)
                    for k, v in (("score", s), ("index", i), ("served", r["served"]), ("unmet", r["unmet"]),
                                 ("accsum", r["accsum"]), ("eff_acc_micro", r["eff"]), ("option", opt),
                                 ("z_qps", r["z"])):
                        out[k].append(v)
                out = {k: np.array(v, np.uint64 if k in ("score", "index") else np.int64) for k, v in out.items()}
                return out, hi - lo

        best, _, ncand, _ = solve_sharded_batch(FakePx(), cl.device_type, cl.slo_us, dems, mode=0)
        q.put((rank, [(int(best["score"][v]), int(best["index"][v]), int(best["served"][v]),
                       int(best["accsum"][v]), ncand, best["option"][v].tolist(), best["z_qps"][v].tolist())
                      for v in range(len(dems))]))
    finally:
        dist.destroy_process_group()


def test_world2_batched_flat_search(oracle_mod):
    """One all-gather of the per-rank winners (already materialised) per
    batch of demand vectors: every rank ends with the single-process optimum,
    placement and z of every vector."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c1")
    prof, cl = cfg["prof"], cfg["cluster"]
    dems = np.array([[0, 0], [300, 100], [600, 0], [800, 700]], np.int32)
    refs = [oracle_mod.solve(prof, cl.device_type, cl.slo_us, d, 0) for d in dems]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_batch_worker, args=(rk, 2, port, q)) for rk in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=600) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for _, sols in out:
        for (sc, idx, served, accsum, ncand, opt, z), r in zip(sols, refs):
            assert idx == r["index"] and sc == (r["served"] << 42) | r["accsum"]
            assert (served, accsum) == (r["served"], r["accsum"])
            assert ncand == r["n_candidates"]
            assert opt == r["option"].tolist() and z == r["z"].tolist()
