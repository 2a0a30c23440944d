"""GPU parity of proteus_replay against the oracle's event-driven simulator:
every per-query latency bit-exact, and the per-scenario aggregates."""

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def px():
    from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus
    return Proteus(0)


def _alloc(oracle_mod, cfg, v=0):
    prof, cl = cfg["prof"], cfg["cluster"]
    return oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][v], 2)


def _compare(px, oracle_mod, prof, cl, option, z, demand, arr, fam, sc):
    px.load_profiles(prof)
    g = px.replay(arr, fam, option, z, cl.device_type, demand, cl.slo_us, sc)
    o = oracle_mod.replay(prof, cl.device_type, option, z, demand, cl.slo_us, arr, fam, sc)
    for s in range(len(sc)):
        if not np.array_equal(g["latency"][s], o["latency"][s]):
            bad = np.nonzero(g["latency"][s] != o["latency"][s])[0]
            raise AssertionError(f"scenario {sc[s]}: {len(bad)} latencies differ, first at {bad[0]}: "
                                 f"gpu {g['latency'][s][bad[0]]} oracle {o['latency'][s][bad[0]]}")
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    return g


PATHS = {"chunked": {}, "small_chunks": {"PROTEUS_REPLAY_CHUNK": "16"}, "odd_chunks": {"PROTEUS_REPLAY_CHUNK": "37"},
         "stitch_only": {"PROTEUS_REPLAY_ROUNDS": "0", "PROTEUS_REPLAY_CHUNK": "37"},
         "one_round_then_stitch": {"PROTEUS_REPLAY_ROUNDS": "1", "PROTEUS_REPLAY_CHUNK": "100"},
         "rounds_to_convergence": {"PROTEUS_REPLAY_ROUNDS": "1000000", "PROTEUS_REPLAY_CHUNK": "64"},
         "no_scans": {"PROTEUS_REPLAY_SCAN1": "0", "PROTEUS_REPLAY_BSCAN": "0", "PROTEUS_REPLAY_CHUNK": "512"},
         "scans_small_chunks_rounds": {"PROTEUS_REPLAY_ROUNDS": "3", "PROTEUS_REPLAY_CHUNK": "200",
                                       "PROTEUS_REPLAY_BSCAN": "1"},
         "backlog_scan": {"PROTEUS_REPLAY_BSCAN": "1"},
         "chunk_300": {"PROTEUS_REPLAY_CHUNK": "300"},
         "simple": {"PROTEUS_REPLAY_SIMPLE": "1"},
         "warmup": {"PROTEUS_REPLAY_WARMUP": "4096"},
         "warmup_small_chunks": {"PROTEUS_REPLAY_CHUNK": "37", "PROTEUS_REPLAY_WARMUP": "50"},
         "warmup_long_small_chunks": {"PROTEUS_REPLAY_CHUNK": "16", "PROTEUS_REPLAY_WARMUP": "1000"},
         "warmup_rounds": {"PROTEUS_REPLAY_ROUNDS": "3", "PROTEUS_REPLAY_CHUNK": "64", "PROTEUS_REPLAY_WARMUP": "100"},
         "warmup_bscan": {"PROTEUS_REPLAY_BSCAN": "1", "PROTEUS_REPLAY_CHUNK": "200", "PROTEUS_REPLAY_WARMUP": "300"}}
# the chunk-run / stitch path (the default; PROTEUS_REPLAY_CHAIN=0) under every
# knob, with duplicate lanes (same policy, Bmax and SLO on a device) replayed
# once and copied (default) or each replayed; the window path with windows of
# 1, 3, 16 (default) and 32 tiles of 512 queries; the opt-in chain path: chunk
# tables for every lane (chunks of 256 / 300 / 2048 / 8192 heads, K = 0..8
# greedy batches per chain), full-batch walks for every lane, mixed with the
# chunk runs + stitch (serial or pipelined, or running beside them)
PATHS = {k: dict(v, PROTEUS_REPLAY_WINDOW="0", PROTEUS_REPLAY_CHAIN="0") for k, v in PATHS.items()}
PATHS["no_dedup"] = {"PROTEUS_REPLAY_DEDUP": "0"}
PATHS["finish_fused"] = {"PROTEUS_REPLAY_FINISH": "1"}
_T = {"PROTEUS_REPLAY_CHAIN": "1", "PROTEUS_REPLAY_CHAIN_MINBATCH": "0", "PROTEUS_REPLAY_CHAIN_RHO_PCT": "100000"}
PATHS["chain"] = {"PROTEUS_REPLAY_CHAIN": "1"}
PATHS["chain_tables_c256"] = dict(_T, PROTEUS_REPLAY_CHAIN_C="256")
PATHS["chain_tables_c300_k0"] = dict(_T, PROTEUS_REPLAY_CHAIN_C="300", PROTEUS_REPLAY_CHAIN_K="0")
PATHS["chain_tables_c8192"] = dict(_T, PROTEUS_REPLAY_CHAIN_C="8192")
PATHS["chain_tables_no_dedup"] = dict(_T, PROTEUS_REPLAY_DEDUP="0", PROTEUS_REPLAY_CHAIN_K="3")
PATHS["chain_backlog_all"] = {"PROTEUS_REPLAY_CHAIN": "1", "PROTEUS_REPLAY_CHAIN_RHO_PCT": "0",
                              "PROTEUS_REPLAY_CHAIN_C": "256"}
PATHS["chain_mixed_minb9"] = dict(_T, PROTEUS_REPLAY_CHAIN_MINB="9", PROTEUS_REPLAY_CHUNK="37")
PATHS["chain_mixed_serial"] = {"PROTEUS_REPLAY_CHAIN": "1", "PROTEUS_REPLAY_CHAIN_MINBATCH": "0",
                               "PROTEUS_REPLAY_CHAIN_RHO_PCT": "150", "PROTEUS_REPLAY_CHAIN_MINB": "17",
                               "PROTEUS_REPLAY_OVERLAP": "0"}
PATHS["chain_beside"] = {"PROTEUS_REPLAY_CHAIN": "1", "PROTEUS_REPLAY_CHAIN_MINBATCH": "4",
                         "PROTEUS_REPLAY_CHAIN_BESIDE": "1"}
PATHS["chain_no_scan1"] = dict(_T, PROTEUS_REPLAY_SCAN1="0", PROTEUS_REPLAY_CHAIN_C="256")
# the stitch with chunk tables for every lane with Bmax >= 2 / >= 4, and with none
PATHS["tables_all"] = {"PROTEUS_REPLAY_CHAIN": "0", "PROTEUS_REPLAY_TABLES": "1", "PROTEUS_REPLAY_TABLES_MINB": "2", "PROTEUS_REPLAY_CHUNK": "300"}
PATHS["tables_min4_chunk64"] = {"PROTEUS_REPLAY_CHAIN": "0", "PROTEUS_REPLAY_TABLES": "1", "PROTEUS_REPLAY_TABLES_MINB": "4",
                                "PROTEUS_REPLAY_CHUNK": "64"}
PATHS["tables_default"] = {"PROTEUS_REPLAY_CHAIN": "0", "PROTEUS_REPLAY_TABLES": "1"}
PATHS["serial_spec_stitch"] = {"PROTEUS_REPLAY_CHAIN": "0", "PROTEUS_REPLAY_OVERLAP": "0"}
PATHS["pipelined_small_chunks"] = {"PROTEUS_REPLAY_CHAIN": "0", "PROTEUS_REPLAY_CHUNK": "37"}
PATHS.update({"window": {"PROTEUS_REPLAY_WINDOW": "1"},  # the window path takes its scenarios before the chain
              "window_wt1": {"PROTEUS_REPLAY_WINDOW": "1", "PROTEUS_REPLAY_WIN_TILES": "1"},
              "window_wt3": {"PROTEUS_REPLAY_WINDOW": "1", "PROTEUS_REPLAY_WIN_TILES": "3"},
              "window_wt32": {"PROTEUS_REPLAY_WINDOW": "1", "PROTEUS_REPLAY_WIN_TILES": "32"}})


@pytest.mark.parametrize("path", sorted(PATHS))
@pytest.mark.parametrize("kind", ["poisson", "gamma", "uniform"])
def test_replay_small_all_scenarios(px, oracle_mod, kind, path, monkeypatch):
    """60k queries x 64 scenarios x both routings; `small_chunks` /
    `odd_chunks` cut the device arrays every 16 / 37 queries so the fix-up
    rounds and the stitch (backlogged jumps, re-walks, meeting tests) run at
    every chunk; `stitch_only` / `one_round_then_stitch` /
    `rounds_to_convergence` take each finishing path alone; `simple` is one
    thread per (device, scenario) lane."""
    for k, v in PATHS[path].items():
        monkeypatch.setenv(k, v)
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    r = _alloc(oracle_mod, cfg, 0)
    rate = float(cfg["demand"][0].sum())
    arr, fam = W.query_trace(60_000, rate, cfg["weights"], 9, kind)
    for routing in (0, 1):
        _compare(px, oracle_mod, cfg["prof"], cfg["cluster"], r["option"], r["z"], cfg["demand"][0], arr, fam,
                 W.scenarios_64(routing))


@pytest.mark.parametrize("path", sorted(PATHS))
def test_replay_overload_with_sink(px, oracle_mod, path, monkeypatch):
    for k, v in PATHS[path].items():
        monkeypatch.setenv(k, v)
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    r = _alloc(oracle_mod, cfg, 1)
    assert r["unmet"] > 0
    arr, fam = W.query_trace(80_000, float(cfg["demand"][1].sum()), cfg["weights"], 10, "gamma")
    g = _compare(px, oracle_mod, cfg["prof"], cfg["cluster"], r["option"], r["z"], cfg["demand"][1], arr, fam,
                 W.scenarios_64(0))
    assert np.all(g["violations"] + g["on_time"] == len(arr))


@pytest.mark.parametrize("epochs", [False, True], ids=["replay", "closed_loop"])
def test_replay_nonmonotone_latency_mixed_paths(px, oracle_mod, epochs):
    """A profile whose T(b) decreases at some batch sizes for half of the
    variants: those lanes leave the chain path (the chain's idle decision is a
    binary search that needs T non-decreasing) for the chunk runs + stitch
    (the closed loop: every lane, its domain check fails), the others stay --
    both paths in one call, against the oracle (whose rule does not assume
    monotone T)."""
    import dataclasses
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    prof = cfg["prof"]
    lat = prof.lat_us.copy()
    for m in range(0, prof.M, 2):  # every other variant: T(4) and T(9) below their predecessors
        for t in range(prof.T):
            for b in (3, 8):
                if lat[t, m, b] > 0 and lat[t, m, b - 1] > 2:
                    lat[t, m, b] = lat[t, m, b - 1] - 1
    prof2 = dataclasses.replace(prof, lat_us=lat)
    cl = cfg["cluster"]
    r = oracle_mod.solve(prof2, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    px.set_timing(True)
    if not epochs:
        arr, fam = W.query_trace(60_000, float(cfg["demand"][0].sum()), cfg["weights"], 21, "gamma")
        _compare(px, oracle_mod, prof2, cl, r["option"], r["z"], cfg["demand"][0], arr, fam, W.scenarios_64(0))
        names = {n for n, _ in px.kernel_times()}
        px.set_timing(False)
        assert {"replay_chain", "replay_stitch"} <= names, names  # both paths ran
        return
    f4 = W.config("f4", n_seconds=6, lam_mid=3000.0)
    E, D = len(f4["demand"]), len(cl.device_type)
    opts = np.stack([r["option"]] * E).astype(np.int32)
    zs = np.stack([r["z"]] * E).astype(np.int32)
    dem = np.stack([cfg["demand"][0]] * E).astype(np.int32)
    sc = np.array([(m, c, 0, 0) for m in (1000, 3000) for c in (4, 32, 0)], np.int32)
    px.load_profiles(prof2)
    g = px.replay_epochs(f4["arrival_us"], f4["family"], f4["epoch_us"], opts, zs, cl.device_type, dem, cl.slo_us, sc)
    names = {n for n, _ in px.kernel_times()}
    px.set_timing(False)
    assert "loop_stitch" in names and "loop_chain" in names, names  # domain check ran, the stitch replayed
    o = oracle_mod.replay_epochs(prof2, cl.device_type, opts, zs, dem, cl.slo_us, f4["arrival_us"], f4["family"],
                                 f4["epoch_us"], sc)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    assert np.array_equal(g["latency"], o["latency"])


def test_replay_edge_cases(px, oracle_mod):
    from paper_conf_asplos_ahmadgfwsw24_b200 import ProteusError, workloads as W
    cfg = W.config("c3")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = _alloc(oracle_mod, cfg, 0)
    sc = np.array([[1000, 0, 0], [2000, 1, 0], [1500, 4, 1]], np.int32)
    # empty trace
    px.load_profiles(prof)
    g = px.replay(np.zeros(0, np.uint32), np.zeros(0, np.uint8), r["option"], r["z"], cl.device_type,
                  cfg["demand"][0], cl.slo_us, sc)
    assert g["latency"].shape == (3, 0) and g["violations"].sum() == 0
    # one query; all simultaneous; ragged sizes around the 1024-query tiles
    for n in (1, 31, 1023, 1025, 4097):
        arr = np.sort(np.random.default_rng(n).integers(0, 2_000, size=n)).astype(np.uint32)
        fam = np.random.default_rng(n + 1).integers(0, prof.Q, size=n).astype(np.uint8)
        _compare(px, oracle_mod, prof, cl, r["option"], r["z"], cfg["demand"][0], arr, fam, sc)
    arr = np.zeros(500, np.uint32)
    fam = np.zeros(500, np.uint8)
    _compare(px, oracle_mod, prof, cl, r["option"], r["z"], cfg["demand"][0], arr, fam, sc)
    # all demand zero -> everything of a routed family goes to the sink
    _compare(px, oracle_mod, prof, cl, r["option"], np.zeros_like(r["z"]), np.zeros(prof.Q, np.int32),
             np.arange(100, dtype=np.uint32), np.zeros(100, np.uint8), sc)
    # unsorted timestamps -> ERANGE
    with pytest.raises(ProteusError) as e:
        px.replay(np.array([5, 3], np.uint32), np.zeros(2, np.uint8), r["option"], r["z"], cl.device_type,
                  cfg["demand"][0], cl.slo_us, sc)
    assert e.value.code == -5


def test_replay_c5_full_size(px, oracle_mod):
    """Config 5 at full size: 10M Poisson queries x 64 scenarios on the c3
    allocation, latencies written to HBM in the bench's launch configuration;
    compared with the oracle on every query of every scenario."""
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c5")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    arr, fam, sc = cfg["arrival_us"], cfg["family"], cfg["scenarios"]
    px.load_profiles(prof)
    lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
    g = px.replay(torch.from_numpy(arr).cuda(), torch.from_numpy(fam).cuda(), r["option"], r["z"], cl.device_type,
                  cfg["demand"][0], cl.slo_us, sc, latency=lat)
    o = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, arr, fam, sc)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    glat = lat.cpu().numpy()
    assert np.array_equal(glat, o["latency"])
    # the chunk runs + stitch on the same lanes (PROTEUS_REPLAY_CHAIN=0)
    import os
    os.environ["PROTEUS_REPLAY_CHAIN"] = "0"
    try:
        lat.fill_(0)
        g = px.replay(torch.from_numpy(arr).cuda(), torch.from_numpy(fam).cuda(), r["option"], r["z"],
                      cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
    finally:
        del os.environ["PROTEUS_REPLAY_CHAIN"]
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    assert np.array_equal(lat.cpu().numpy(), o["latency"])


def test_replay_c5_full_size_routing1(px, oracle_mod):
    """Config 5 at full size with routing 1 ("w/o QA": uniform
    weights over the hosting devices that fit, no sink): the 64 §5 scenarios
    on the default chain path, every latency against the oracle."""
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c5")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    arr, fam = cfg["arrival_us"], cfg["family"]
    sc = W.scenarios_64(1)
    px.load_profiles(prof)
    lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
    g = px.replay(torch.from_numpy(arr).cuda(), torch.from_numpy(fam).cuda(), r["option"], r["z"], cl.device_type,
                  cfg["demand"][0], cl.slo_us, sc, latency=lat)
    o = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, arr, fam, sc)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    assert np.array_equal(lat.cpu().numpy(), o["latency"])


@pytest.mark.parametrize("policy", [1, 2])
def test_replay_baselines_c5_full_size(px, oracle_mod, policy):
    """§8(f2) at the bench's size and launch configuration: the c5 trace (10M
    queries) x 64 scenarios of one baseline policy, every latency compared."""
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c5")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    arr, fam = cfg["arrival_us"], cfg["family"]
    sc = W.scenarios_64(0, policy)
    px.load_profiles(prof)
    lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
    g = px.replay(torch.from_numpy(arr).cuda(), torch.from_numpy(fam).cuda(), r["option"], r["z"], cl.device_type,
                  cfg["demand"][0], cl.slo_us, sc, latency=lat)
    o = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, arr, fam, sc)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    assert np.array_equal(lat.cpu().numpy(), o["latency"])


def test_replay_aggregates_without_latencies(px, oracle_mod):
    """latency=None (aggregates only: the separate count pass) equals the
    oracle's aggregates, as the fused count in the un-permute pass does."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = _alloc(oracle_mod, cfg, 1)
    arr, fam = W.query_trace(50_000, float(cfg["demand"][1].sum()), cfg["weights"], 12, "gamma")
    sc = np.concatenate([W.scenarios_64(0)[::3], W.scenarios_64(1)[::5]])
    px.load_profiles(prof)
    g = px.replay(arr, fam, r["option"], r["z"], cl.device_type, cfg["demand"][1], cl.slo_us, sc, latency=None)
    o = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][1], cl.slo_us, arr, fam, sc)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k


@pytest.mark.parametrize("kind", ["poisson", "gamma", "uniform"])
@pytest.mark.parametrize("policy", [1, 2])
def test_replay_baseline_policies(px, oracle_mod, kind, policy):
    """§8(f2): Nexus early drop (1) and Clipper AIMD (2) lanes (k_wc_lanes)
    bit-exact against the oracle's event-driven simulators, 64 scenarios x
    both routings, light load and overload (sink)."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    for v, n in ((0, 60_000), (1, 40_000)):
        r = _alloc(oracle_mod, cfg, v)
        arr, fam = W.query_trace(n, float(cfg["demand"][v].sum()), cfg["weights"], 11 + v, kind)
        for routing in (0, 1):
            g = _compare(px, oracle_mod, cfg["prof"], cfg["cluster"], r["option"], r["z"], cfg["demand"][v], arr,
                         fam, W.scenarios_64(routing, policy))
            assert np.all(g["violations"] + g["on_time"] == len(arr))


@pytest.mark.parametrize("kind", ["poisson", "gamma"])
@pytest.mark.parametrize("rho", ["0", "95"])
def test_replay_nexus_overload_scan(px, oracle_mod, kind, rho, monkeypatch):
    """§8(f2) Nexus lanes through the opt-in overload scan (k_nx_*): the first
    walk stops at a lane's first overload stretch, the scan takes the stretch
    as far as it is valid, the second walk the rest (every Nexus lane selected
    at rho 0); bit-exact against the oracle, light load and overload."""
    monkeypatch.setenv("PROTEUS_REPLAY_NXSCAN", "1")
    monkeypatch.setenv("PROTEUS_REPLAY_NXSCAN_RHO_PCT", rho)
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    for v, n in ((0, 60_000), (1, 80_000)):
        r = _alloc(oracle_mod, cfg, v)
        arr, fam = W.query_trace(n, float(cfg["demand"][v].sum()), cfg["weights"], 17 + v, kind)
        for routing in (0, 1):
            _compare(px, oracle_mod, cfg["prof"], cfg["cluster"], r["option"], r["z"], cfg["demand"][v], arr, fam,
                     W.scenarios_64(routing, 1))


def test_replay_mixed_policies_one_call(px, oracle_mod):
    """All three policies in one call (Fig. 6 grid, both routings): the §5
    scenarios take the chunk/stitch path, the baselines k_wc_lanes, and the
    counts / sink / un-permute see every scenario."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    r = _alloc(oracle_mod, cfg, 1)
    arr, fam = W.query_trace(50_000, float(cfg["demand"][1].sum()), cfg["weights"], 13, "gamma")
    sc = np.concatenate([W.scenarios_fig6(0), W.scenarios_fig6(1)])
    rng = np.random.default_rng(5)
    sc = sc[rng.permutation(len(sc))]
    _compare(px, oracle_mod, cfg["prof"], cfg["cluster"], r["option"], r["z"], cfg["demand"][1], arr, fam, sc)


def test_replay_baseline_edge_cases(px, oracle_mod):
    """Tiny traces: one query, all simultaneous, and a tight SLO that drops
    nearly everything under Nexus."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    r = _alloc(oracle_mod, cfg, 0)
    for arr in (np.array([5], np.uint32), np.zeros(300, np.uint32), np.arange(0, 3000, 10, dtype=np.uint32)):
        fam = np.zeros(len(arr), np.uint8)
        sc = np.array([(m, c, 0, p) for m in (100, 1000) for c in (1, 4, 0) for p in (0, 1, 2)], np.int32)
        _compare(px, oracle_mod, cfg["prof"], cfg["cluster"], r["option"], r["z"], cfg["demand"][0], arr, fam, sc)


def test_replay_scenario_errors(px, oracle_mod):
    """Invalid scenario rows are rejected before any output is written:
    policy outside 0..2, routing outside 0..1, negative multiplier or cap."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import ProteusError, workloads as W
    cfg = W.config("c3")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    a, f = W.query_trace(1000, 3000.0, cfg["weights"], 3, "poisson")
    px.load_profiles(prof)
    for bad in ([1000, 0, 0, 3], [1000, 0, 2, 0], [-1, 0, 0, 0], [1000, -2, 0, 1]):
        lat = np.full((1, len(a)), 7, np.uint32)
        with pytest.raises(ProteusError):
            px.replay(a, f, r["option"], r["z"], cl.device_type, cfg["demand"][0], cl.slo_us,
                      np.array([bad], np.int32), latency=lat)
        assert np.all(lat == 7)


@pytest.mark.parametrize("env", [{"PROTEUS_REPLAY_CHUNK": "16"}, {"PROTEUS_REPLAY_CHUNK": "37"},
                                 {"PROTEUS_REPLAY_CHUNK": "1000"}, {"PROTEUS_REPLAY_WCSPEC": "0"}])
def test_replay_baseline_chunk_runs(px, oracle_mod, env, monkeypatch):
    """AIMD lanes meeting k_wc_spec's chunk runs at free heads in the same
    limit (tiny chunks: batches straddling chunk ends, exits several chunks
    ahead), and the walk without chunk runs; light load and overload."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    for v, kind in ((0, "poisson"), (1, "gamma")):
        r = _alloc(oracle_mod, cfg, v)
        arr, fam = W.query_trace(40_000, float(cfg["demand"][v].sum()), cfg["weights"], 21 + v, kind)
        sc = np.concatenate([W.scenarios_64(0, 2), W.scenarios_64(0, 1)[::5]])
        _compare(px, oracle_mod, cfg["prof"], cfg["cluster"], r["option"], r["z"], cfg["demand"][v], arr, fam, sc)
