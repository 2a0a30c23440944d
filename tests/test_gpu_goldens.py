"""GPU parity at BASELINE.json's full sizes, in the bench's launch
configurations, against every vector / every latency the oracle computes:

* c2: all 64 demand vectors of the bench step (13^8 candidates each), against
  tests/golden/c2bench_oracle.npz (oracle A's exhaustive optimum, written by
  scripts/gen_goldens.py): canonical index, value, placement and z;
* c4: all 3600 per-second vectors of the factored re-solve, against
  tests/golden/c4_oracle.npz;
* f4: the bench's closed loop -- allocations from proteus_solve_batch on the
  previous epoch's counts, left on the device, fed to proteus_replay_epochs
  with the bench's 12 scenarios -- allocations against the fixture, every
  latency against the oracle's closed-loop simulator;
* c5 trace G: 10M Gamma(0.05) queries x 64
  scenarios, every latency against the oracle's event-driven simulator."""

import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


@pytest.fixture(scope="module")
def px():
    from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus
    return Proteus(0)


def _eq(g, ref, keys, what):
    for k in keys:
        a, b = np.asarray(g[k]).astype(np.int64), np.asarray(ref[k]).astype(np.int64)
        if not np.array_equal(a, b):
            bad = np.nonzero((a != b).reshape(len(a), -1).any(axis=1))[0]
            raise AssertionError(f"{what}: {k} differs at {len(bad)} vectors, first {bad[0]}: {a[bad[0]]} vs {b[bad[0]]}")


def test_c2_bench_batch_all_64_vectors(px):
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    ref = np.load(os.path.join(GOLDEN, "c2bench_oracle.npz"))
    cfg = W.config("c2", totals=W.C2_BENCH_TOTALS)
    cl = cfg["cluster"]
    px.load_profiles(cfg["prof"])
    t = lambda x: torch.as_tensor(x, dtype=torch.int32, device="cuda")  # noqa: E731
    g, n = px.solve_batch(t(cl.device_type), t(cl.slo_us), t(cfg["demand"]), mode=0)
    assert n == 13**8
    _eq(g, {"index": ref["index"], "served": ref["served"], "accsum": ref["accsum"], "unmet": ref["unmet"],
            "option": ref["option"], "z_qps": ref["z"]},
        ("index", "served", "accsum", "unmet", "option", "z_qps"), "c2 bench batch")
    assert np.array_equal(np.asarray(g["score"]), (ref["served"].astype(np.uint64) << np.uint64(42)) +
                          ref["accsum"].astype(np.uint64))


def test_c4_all_3600_vectors(px):
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    ref = np.load(os.path.join(GOLDEN, "c4_oracle.npz"))
    cfg = W.config("c4")
    cl = cfg["cluster"]
    px.load_profiles(cfg["prof"])
    t = lambda x: torch.as_tensor(x, dtype=torch.int32, device="cuda")  # noqa: E731
    g, _ = px.solve_batch(t(cl.device_type), t(cl.slo_us), t(cfg["demand"]), mode=2)
    _eq(g, {"served": ref["served"], "accsum": ref["accsum"], "unmet": ref["unmet"], "option": ref["option"],
            "z_qps": ref["z"]}, ("served", "accsum", "unmet", "option", "z_qps"), "c4")


@pytest.mark.parametrize("env", [{}, {"PROTEUS_LOOP_CHAIN": "0"}], ids=["chain", "stitch"])
def test_f4_bench_configuration_full_hour(px, oracle_mod, env, monkeypatch):
    """bench.py's f4 step exactly: solve_batch(mode 2) of the controller's
    demand into device tensors, then replay_epochs of the 10.6M-query hour
    with the 12 scenarios (SLO {1, 2, 3, 5}x x cap {8, 32, depth}); the
    default chain path and the chunk runs + stitch."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    ref = np.load(os.path.join(GOLDEN, "c4_oracle.npz"))
    cfg = W.config("f4")
    prof, cl = cfg["prof"], cfg["cluster"]
    E, D = len(cfg["demand"]), len(cl.device_type)
    px.load_profiles(prof)
    dev = torch.device("cuda")
    arr = torch.from_numpy(cfg["arrival_us"]).to(dev)
    fam = torch.from_numpy(cfg["family"]).to(dev)
    dem = torch.from_numpy(cfg["demand"]).to(dev)
    t_dev = torch.as_tensor(cl.device_type, dtype=torch.int32, device=dev)
    t_slo = torch.as_tensor(cl.slo_us, dtype=torch.int32, device=dev)
    sc = cfg["scenarios"]
    assert len(sc) == 12
    alloc = {"option": torch.empty((E, D), dtype=torch.int32, device=dev),
             "z_qps": torch.empty((E, D), dtype=torch.int32, device=dev)}
    px.solve_batch(t_dev, t_slo, dem, mode=2, out=alloc)
    lat = torch.empty((len(sc), len(cfg["arrival_us"])), dtype=torch.uint32, device=dev)
    g = px.replay_epochs(arr, fam, cfg["epoch_us"], alloc["option"], alloc["z_qps"], t_dev, dem, t_slo, sc,
                         latency=lat)
    # the controller solves epoch e on epoch e-1's counts: fixture rows shifted by one
    rows = np.concatenate([[0], np.arange(E - 1)])
    oopt, oz = ref["option"][rows], ref["z"][rows]
    assert np.array_equal(alloc["option"].cpu().numpy(), oopt)
    assert np.array_equal(alloc["z_qps"].cpu().numpy(), oz)
    o = oracle_mod.replay_epochs(prof, cl.device_type, oopt, oz, cfg["demand"], cl.slo_us, cfg["arrival_us"],
                                 cfg["family"], cfg["epoch_us"], sc)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(g[k], o[k]), k
    glat = lat.cpu().numpy()
    for s in range(len(sc)):
        if not np.array_equal(glat[s], o["latency"][s]):
            bad = np.nonzero(glat[s] != o["latency"][s])[0]
            raise AssertionError(f"f4 scenario {sc[s]}: {len(bad)} latencies differ, first at {bad[0]}")


@pytest.mark.parametrize("policies,env", [((0,), {}), ((1, 2), {}), ((0,), {"PROTEUS_REPLAY_CHAIN": "0"})],
                         ids=["s5", "baselines", "s5_stitch"])
def test_c5_gamma_trace_full_size(px, oracle_mod, policies, env, monkeypatch):
    """Trace G of config 5: 10M queries with Gamma(shape 0.05) inter-arrivals
    (CV 4.47, the paper's bursty trace) at 3000 QPS on the c3
    allocation; the 64 (SLO x cap) scenarios of §5 batching (and, for f2, of
    the two baseline batchers); every latency compared.  `s5` runs the
    default chain path, `s5_stitch` the chunk runs + stitch."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c5", kind="gamma")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    arr, fam = cfg["arrival_us"], cfg["family"]
    assert len(arr) == 10_000_000
    gaps = np.diff(arr.astype(np.int64))
    assert gaps.std() / gaps.mean() > 3.0  # bursty: CV ~ 4.47
    px.load_profiles(prof)
    ta, tf = torch.from_numpy(arr).cuda(), torch.from_numpy(fam).cuda()
    for pol in policies:
        sc = W.scenarios_64(0, pol)
        lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
        g = px.replay(ta, tf, r["option"], r["z"], cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        o = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, arr, fam, sc)
        for k in ("violations", "on_time", "acc_sum"):
            assert np.array_equal(g[k], o[k]), (pol, k)
        glat = lat.cpu().numpy()
        for s in range(len(sc)):
            if not np.array_equal(glat[s], o["latency"][s]):
                bad = np.nonzero(glat[s] != o["latency"][s])[0]
                raise AssertionError(f"gamma policy {pol} scenario {sc[s]}: {len(bad)} latencies differ")
