"""GPU parity of the §8(f4) closed loop (proteus_replay_epochs /
Proteus.closed_loop) against the oracle's epoch-aware replay: allocations per
epoch from the oracle's factored solve of the controller's demand (previous
epoch's counts), every per-query latency and the aggregates bit-exact."""

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def px():
    from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus
    return Proteus(0)


def _oracle_allocs(oracle_mod, cfg):
    prof, cl = cfg["prof"], cfg["cluster"]
    opts, zs = [], []
    for e in range(len(cfg["demand"])):
        r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][e], 2)
        opts.append(r["option"])
        zs.append(r["z"])
    return np.array(opts, np.int32), np.array(zs, np.int32)


def _compare(px, oracle_mod, cfg, opts, zs, sc):
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    a, f = cfg["arrival_us"], cfg["family"]
    g = px.replay_epochs(a, f, cfg["epoch_us"], opts, zs, cl.device_type, cfg["demand"], cl.slo_us, sc)
    o = oracle_mod.replay_epochs(prof, cl.device_type, opts, zs, cfg["demand"], cl.slo_us, a, f, cfg["epoch_us"], sc)
    for s in range(len(sc)):
        if not np.array_equal(g["latency"][s], o["latency"][s]):
            bad = np.nonzero(g["latency"][s] != o["latency"][s])[0]
            raise AssertionError(f"scenario {sc[s]}: {len(bad)} latencies differ, first at {bad[0]}: "
                                 f"gpu {g['latency'][s][bad[0]]} oracle {o['latency'][s][bad[0]]}")
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    return g


SC = np.array([(m, c, 0, 0) for m in (1000, 2000, 5000) for c in (1, 4, 32, 0)], np.int32)


@pytest.mark.parametrize("lam", [1500.0, 4000.0])
def test_closed_loop_parity(px, oracle_mod, lam):
    """20 one-second epochs of the c4-shaped demand (light and overloaded:
    sink drops and backlogs carried across epoch boundaries)."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("f4", n_seconds=20, lam_mid=lam)
    opts, zs = _oracle_allocs(oracle_mod, cfg)
    g = _compare(px, oracle_mod, cfg, opts, zs, SC)
    assert np.all(g["violations"] + g["on_time"] == len(cfg["arrival_us"]))


@pytest.mark.parametrize("env", [{"PROTEUS_LOOP_CHAIN": "0"},
                                 {"PROTEUS_REPLAY_CHAIN_C": "256", "PROTEUS_REPLAY_CHAIN_SEG": "16"},
                                 {"PROTEUS_REPLAY_CHAIN_C": "300", "PROTEUS_REPLAY_CHAIN_K": "0"},
                                 {"PROTEUS_REPLAY_CHAIN_C": "8192", "PROTEUS_REPLAY_CHAIN_K": "64"}],
                         ids=["stitch", "chain_c256_seg16", "chain_c300_k0", "chain_c8192_k64"])
def test_closed_loop_paths(px, oracle_mod, env, monkeypatch):
    """The closed loop's two replay paths: the chain path (default; small
    chunks and segments put many epoch boundaries inside chunks, segments
    and runs) and the chunk runs + stitch (PROTEUS_LOOP_CHAIN=0), light load
    and overload, against the oracle's closed-loop simulator."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    for lam in (1500.0, 4000.0):
        cfg = W.config("f4", n_seconds=12, lam_mid=lam)
        opts, zs = _oracle_allocs(oracle_mod, cfg)
        g = _compare(px, oracle_mod, cfg, opts, zs, SC)
        assert np.all(g["violations"] + g["on_time"] == len(cfg["arrival_us"]))


def test_closed_loop_short_epochs(px, oracle_mod):
    """100 ms epochs (allocations switching while queues are non-empty) and
    the epoch-boundary carry exercised on every device."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("f4", n_seconds=4, lam_mid=3000.0)
    # re-cut the same demand into 40 epochs of 100 ms: counts scaled down 10x
    counts = np.repeat(cfg["counts"], 10, axis=0) // 10
    arr, fam = W.epoch_trace(counts, 100_000, 707)
    cfg = dict(cfg, counts=counts, demand=W.controller_demand(counts * 10), arrival_us=arr, family=fam,
               epoch_us=100_000)
    opts, zs = _oracle_allocs(oracle_mod, cfg)
    _compare(px, oracle_mod, cfg, opts, zs, SC)


def test_single_epoch_equals_replay(px, oracle_mod):
    """E = 1: proteus_replay_epochs = proteus_replay (and the oracle)."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][1], 2)
    a, f = W.query_trace(30_000, float(cfg["demand"][1].sum()), cfg["weights"], 12, "gamma")
    px.load_profiles(prof)
    sc = SC
    g1 = px.replay_epochs(a, f, int(a[-1]) + 1, r["option"][None], r["z"][None], cl.device_type,
                          cfg["demand"][1][None], cl.slo_us, sc)
    g0 = px.replay(a, f, r["option"], r["z"], cl.device_type, cfg["demand"][1], cl.slo_us, sc)
    for k in ("latency", "violations", "on_time", "acc_sum"):
        assert np.array_equal(g1[k], g0[k]), k


def test_closed_loop_api_device_resident(px, oracle_mod):
    """Proteus.closed_loop: batched factored re-solve with device outputs
    feeding the replay; allocations and the replay equal the oracle chain."""
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("f4", n_seconds=16, lam_mid=2500.0)
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    dev = torch.device("cuda:0")
    arr = torch.from_numpy(cfg["arrival_us"]).to(dev)
    fam = torch.from_numpy(cfg["family"]).to(dev)
    dem = torch.from_numpy(cfg["demand"]).to(dev)
    res, alloc = px.closed_loop(arr, fam, cfg["epoch_us"], dem, cl.device_type, cl.slo_us, SC, device=dev)
    opts, zs = _oracle_allocs(oracle_mod, cfg)
    assert np.array_equal(alloc["option"].cpu().numpy(), opts)
    assert np.array_equal(alloc["z_qps"].cpu().numpy(), zs)
    o = oracle_mod.replay_epochs(prof, cl.device_type, opts, zs, cfg["demand"], cl.slo_us, cfg["arrival_us"],
                                 cfg["family"], cfg["epoch_us"], SC)
    assert np.array_equal(res["latency"], o["latency"])
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(res[k], o[k]), k


def test_closed_loop_errors(px):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W, ProteusError
    cfg = W.config("f4", n_seconds=3)
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    D = len(cl.device_type)
    opts = np.zeros((2, D), np.int32)
    zs = np.zeros((2, D), np.int32)
    with pytest.raises(ProteusError):   # arrivals in epoch 2 of a 2-epoch loop
        px.replay_epochs(cfg["arrival_us"], cfg["family"], cfg["epoch_us"], opts, zs, cl.device_type,
                         cfg["demand"][:2], cl.slo_us, SC)
    with pytest.raises(ProteusError):   # routing 1 is not a closed-loop scenario
        px.replay_epochs(cfg["arrival_us"], cfg["family"], cfg["epoch_us"], np.zeros((3, D), np.int32),
                         np.zeros((3, D), np.int32), cl.device_type, cfg["demand"], cl.slo_us,
                         np.array([[1000, 0, 1, 0]], np.int32))


def test_closed_loop_full_hour(px, oracle_mod):
    """§8(f4) at the bench's size and launch configuration: the whole c4 hour
    (3600 one-second epochs, ~10.6M queries) in one proteus_replay_epochs
    call.  Allocations (inputs of the replay) come from the oracle: 48
    demand levels of the hour solved exactly, epoch e running level e mod 48
    with that level's demand as its routing demand (any valid allocation is a
    valid input); every latency and aggregate compared with the oracle."""
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("f4")
    prof, cl = cfg["prof"], cfg["cluster"]
    E = len(cfg["demand"])
    lv = np.linspace(0, E - 1, 48).astype(int)
    sols = [oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][e], 2) for e in lv]
    pick = np.arange(E) % 48
    opts = np.array([sols[k]["option"] for k in pick], np.int32)
    zs = np.array([sols[k]["z"] for k in pick], np.int32)
    dem = np.ascontiguousarray(cfg["demand"][lv][pick])
    sc = np.array([(1000, 8, 0, 0), (3000, 0, 0, 0)], np.int32)
    px.load_profiles(prof)
    a, f = cfg["arrival_us"], cfg["family"]
    lat = torch.empty((len(sc), len(a)), dtype=torch.uint32, device="cuda")
    g = px.replay_epochs(torch.from_numpy(a).cuda(), torch.from_numpy(f).cuda(), cfg["epoch_us"], opts, zs,
                         cl.device_type, dem, cl.slo_us, sc, latency=lat)
    o = oracle_mod.replay_epochs(prof, cl.device_type, opts, zs, dem, cl.slo_us, a, f, cfg["epoch_us"], sc)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    assert np.array_equal(lat.cpu().numpy(), o["latency"])
