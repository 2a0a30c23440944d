"""GPU parity of proteus_solve against the oracle (bit-exact: every quantity is
an integer).  Compared per demand vector: packed score, served, unmet, accsum,
effective accuracy, the canonical index (modes 0/1), the placement and z.
Where several placements are optimal the canonical tie-break (reading C9)
makes the answer unique; independently, the GPU's placement is re-scored by
the oracle (catches decode bugs regardless of tie-breaking)."""

import numpy as np
import pytest

from tests._util import golden, packed_score, profiles_from_capacity, random_instance

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def px():
    from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus
    return Proteus(0)


def check(px, oracle_mod, prof, dev, slo, demand, mode, generic=False, threads=0):
    px.load_profiles(prof)
    dem = np.atleast_2d(np.asarray(demand, np.int32))
    sols = px.solve(dev, slo, dem, mode=mode, generic=generic)
    for v, sol in enumerate(sols):
        r = oracle_mod.solve(prof, dev, slo, dem[v], mode, threads=threads)
        got = (sol.served, sol.unmet, sol.accsum, sol.eff_acc_micro)
        assert got == (r["served"], r["unmet"], r["accsum"], r["eff"]), (mode, v, got, r)
        assert sol.score == packed_score(r["served"], r["accsum"])
        if mode in (0, 1):
            assert sol.index == r["index"], (mode, sol.index, r["index"])
            assert sol.n_candidates == r["n_candidates"]
        assert sol.option.tolist() == r["option"].tolist(), (mode, sol.option, r["option"])
        assert sol.z.tolist() == r["z"].tolist()
        chk = oracle_mod.score_placement(prof, dev, slo, dem[v], sol.option)
        assert (chk["served"], chk["accsum"]) == (sol.served, sol.accsum)
        assert chk["z"].tolist() == sol.z.tolist()
    return sols


def test_golden_h1_g1(px, oracle_mod):
    from paper_conf_asplos_ahmadgfwsw24_b200.workloads import Profiles
    g = golden()
    h = g["H1"]
    prof = Profiles(T=1, Q=1, V=np.array(h["V"], np.int32), acc_micro=np.array(h["acc_micro"], np.int32), bmax=1,
                    lat_us=np.array(h["lat_us"], np.int32))
    px.load_profiles(prof)
    for c in h["cases"]:
        for generic in (False, True):
            s = px.solve(h["device_type"], h["slo_us"], c["s"], mode=0, generic=generic)[0]
            assert (s.index, s.served, s.accsum, s.eff_acc_micro) == (c["index"], c["served"], c["accsum"], c["eff"])
            assert s.option.tolist() == c["option"] and s.z.tolist() == c["z"]
    G = g["G1"]
    prof = profiles_from_capacity(G["P"], G["acc_micro"], G["V"])
    px.load_profiles(prof)
    for c in G["cases"]:
        for generic in (False, True):
            s = px.solve(G["device_type"], G["slo_us"], c["s"], mode=0, generic=generic)[0]
            assert (s.index, s.served, s.accsum, s.eff_acc_micro) == (c["index"], c["served"], c["accsum"], c["eff"])
            assert s.option.tolist() == c["option"] and s.z.tolist() == c["z"]
            if "score_hex" in c:
                assert s.score == int(c["score_hex"], 16)
        if "multiset_index" in c:
            assert px.solve(G["device_type"], G["slo_us"], c["s"], mode=1)[0].index == c["multiset_index"]


@pytest.mark.parametrize("total", [600, 1200, 0, 17])
def test_c1_all_modes(px, oracle_mod, total):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c1", total=total)
    prof, cl = cfg["prof"], cfg["cluster"]
    for mode, generic in ((0, False), (0, True), (1, False), (2, False)):
        check(px, oracle_mod, prof, cl.device_type, cl.slo_us, cfg["demand"], mode, generic)


def test_random_small_instances(px, oracle_mod):
    """Random toys incl. tied accuracies, unsorted variant order, P = 0 holes,
    zero demand, D from 1 to 6, 1-4 families."""
    rng = np.random.default_rng(1234)
    for trial in range(60):
        T = int(rng.integers(1, 4))
        Q = int(rng.integers(1, 5))
        D = int(rng.integers(1, 7))
        prof, dev, slo, P = random_instance(rng, T=T, Q=Q, Vmax=3, D=D, Pmax=40, tie_acc=trial % 3 == 0)
        if trial % 4 == 1:  # unsorted accuracy order inside families
            prof.acc_micro = prof.acc_micro[::-1].copy()
            prof.V = prof.V[::-1].copy()
        s = rng.integers(0, 80, size=(2, prof.Q)).astype(np.int32)
        for mode, generic in ((0, False), (0, True), (1, False), (2, False)):
            check(px, oracle_mod, prof, dev, slo, s, mode, generic, threads=2)


def test_c2_flat_full(px, oracle_mod):
    """Config 2 at full size (13^8 = 815 730 721 candidates), both demand
    vectors, specialised kernel; oracle = exhaustive enumeration."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2")
    sols = check(px, oracle_mod, cfg["prof"], cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"], 0)
    assert sols[0].n_candidates == 13**8
    assert sols[1].unmet > 0


def test_c2_flat_full_ties(px, oracle_mod):
    """Config 2 at full size with tiny demands: millions of candidates tie at
    the maximum, spread over every thread of the launch, so the flat kernel's
    grid-wide score bound (threshold G - 1) must still return the lowest index
    among the maxima (reading C9); the all-zero vector ties everywhere at 0
    (answer: index 0).  Oracle = exhaustive enumeration."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2")
    dem = np.array([[5, 5, 5, 5], [0, 0, 0, 0], [1, 0, 0, 0]], dtype=np.int32)
    sols = check(px, oracle_mod, cfg["prof"], cfg["cluster"].device_type, cfg["cluster"].slo_us, dem, 0)
    assert sols[1].index == 0 and sols[1].score == 0


def test_c2_generic_kernel_and_multiset(px, oracle_mod):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2")
    args = (cfg["prof"], cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"])
    a = check(px, oracle_mod, *args, 0, generic=True)
    b = check(px, oracle_mod, *args, 1)
    c = check(px, oracle_mod, *args, 2)
    for x, y, z in zip(a, b, c):
        assert x.score == y.score == z.score  # invariant (iii)


def test_c2_sharded_identical(px, oracle_mod):
    """Index-range shards (as on 1/2/4/8 GPUs) combined on the device by
    proteus_combine_solutions -- the (score desc, index asc) pick the NCCL
    path runs after its all-gather -- give the single-GPU result."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2")
    px.load_profiles(cfg["prof"])
    dev, slo, dem = cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"][:1]
    full, n = px.solve_batch(dev, slo, dem, mode=0)
    for world in (2, 3, 8):
        parts = [px.solve_batch(dev, slo, dem, mode=0, shard_rank=r, shard_world=world) for r in range(world)]
        best, n_all = px.combine_solutions([p[0] for p in parts], [p[1] for p in parts], len(dev))
        assert n_all == n == 13**8
        for k in ("score", "index", "served", "unmet", "accsum", "eff_acc_micro", "option", "z_qps"):
            assert np.array_equal(np.asarray(best[k]), np.asarray(full[k])), (world, k)


def test_c3_factored(px, oracle_mod):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    sols = check(px, oracle_mod, cfg["prof"], cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"], 2)
    assert sols[0].unmet == 0 and sols[1].unmet > 0


def test_c3mini_multiset_vs_factored(px, oracle_mod):
    """c3-mini: flat multiset over a 12-device cluster of the three types
    (5005 * 220^2 = 2.42e8 candidates) = factored optimum (invariant iii);
    both modes bit-exact vs the oracle."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3mini")
    args = (cfg["prof"], cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"])
    f = check(px, oracle_mod, *args, 2)
    m = check(px, oracle_mod, *args, 1)
    assert m[0].n_candidates == 5005 * 220 * 220
    for x, y in zip(f, m):
        assert x.score == y.score


def test_c3mini_20_devices_multiset_full_size(px, oracle_mod):
    """The same families on the full 20-device cluster: 92378 * 2002^2 =
    3.7e11 multisets on the GPU (too many for the oracle); property at full
    size: the multiset optimum equals the factored optimum, which the oracle
    computes exactly, and the returned placement re-scores to that value."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3mini", counts=(10, 5, 5), totals=(12000,))
    prof, cl, dem = cfg["prof"], cfg["cluster"], cfg["demand"]
    px.load_profiles(prof)
    m = px.solve(cl.device_type, cl.slo_us, dem, mode=1)[0]
    assert m.n_candidates == 92378 * 2002 * 2002
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, dem[0], 2)
    assert (m.served, m.accsum) == (r["served"], r["accsum"])
    chk = oracle_mod.score_placement(prof, cl.device_type, cl.slo_us, dem[0], m.option)
    assert (chk["served"], chk["accsum"]) == (m.served, m.accsum)


def test_c4_batched_resolve_sample(px, oracle_mod):
    """All 3600 per-second vectors in one call; a seeded sample of 12 checked
    against the oracle one by one, plus every vector's reported value checked
    by re-scoring its placement."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c4")
    prof, cl, dem = cfg["prof"], cfg["cluster"], cfg["demand"]
    px.load_profiles(prof)
    sols = px.solve(cl.device_type, cl.slo_us, dem, mode=2)
    assert len(sols) == 3600
    rng = np.random.default_rng(404)
    for v in sorted(rng.choice(3600, size=12, replace=False)):
        r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, dem[v], 2)
        s = sols[v]
        assert (s.served, s.accsum, s.unmet) == (r["served"], r["accsum"], r["unmet"])
        assert s.option.tolist() == r["option"].tolist() and s.z.tolist() == r["z"].tolist()
    for v in range(0, 3600, 7):
        chk = oracle_mod.score_placement(prof, cl.device_type, cl.slo_us, dem[v], sols[v].option)
        assert (chk["served"], chk["accsum"]) == (sols[v].served, sols[v].accsum)
    assert any(s.unmet > 0 for s in sols) and any(s.unmet == 0 for s in sols)


def test_errors(px):
    from paper_conf_asplos_ahmadgfwsw24_b200 import ProteusError, workloads as W
    from paper_conf_asplos_ahmadgfwsw24_b200._native import PROTEUS_EINVAL, PROTEUS_ERANGE
    cfg = W.config("c2")
    px.load_profiles(cfg["prof"])
    dev, slo = cfg["cluster"].device_type, cfg["cluster"].slo_us
    with pytest.raises(ProteusError) as e:
        px.solve(dev, slo, cfg["demand"][0], mode=0, max_candidates=10**6)
    assert e.value.code == PROTEUS_ERANGE
    with pytest.raises(ProteusError) as e:
        px.solve(dev, slo, np.full(4, 2**21, np.int32), mode=2)
    assert e.value.code == PROTEUS_ERANGE
    with pytest.raises(ProteusError) as e:
        px.solve(np.full(8, 7, np.int32), slo, cfg["demand"][0], mode=2)
    assert e.value.code == PROTEUS_EINVAL
    assert px.candidate_count(dev, 0) == 13**8
    assert px.candidate_count(dev, 1) == 91 * 455 * 455


def test_device_pointer_inputs(px, oracle_mod):
    """torch CUDA tensors as inputs (the in-HBM path the bench times)."""
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c1")
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    host = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=0)[0]
    t = lambda a: torch.as_tensor(np.asarray(a, np.int32)).cuda()
    dev = px.solve(t(cl.device_type), t(cl.slo_us), t(cfg["demand"]), mode=0)[0]
    assert (dev.score, dev.index, dev.option.tolist()) == (host.score, host.index, host.option.tolist())


def test_c4_solve_batch_outputs(px, oracle_mod):
    """proteus_solve_batch: array outputs on the host and on the device equal
    the per-vector proteus_solve results; a seeded sample is checked against
    the oracle directly."""
    import torch
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c4")
    prof, cl, dem = cfg["prof"], cfg["cluster"], cfg["demand"][:700]
    px.load_profiles(prof)
    sols = px.solve(cl.device_type, cl.slo_us, dem, mode=2)
    host, ncand = px.solve_batch(cl.device_type, cl.slo_us, dem, mode=2)
    assert ncand == sols[0].n_candidates
    D, n = len(cl.device_type), len(dem)
    dev_out = {"score": torch.empty(n, dtype=torch.uint64, device="cuda"),
               "served": torch.empty(n, dtype=torch.int64, device="cuda"),
               "accsum": torch.empty(n, dtype=torch.int64, device="cuda"),
               "option": torch.empty((n, D), dtype=torch.int32, device="cuda"),
               "z_qps": torch.empty((n, D), dtype=torch.int32, device="cuda")}
    t_dem = torch.as_tensor(dem, dtype=torch.int32, device="cuda")
    px.solve_batch(cl.device_type, cl.slo_us, t_dem, mode=2, out=dev_out)
    d = {k: v.cpu().numpy() for k, v in dev_out.items()}
    for v, s in enumerate(sols):
        assert (host["score"][v], host["served"][v], host["unmet"][v], host["accsum"][v], host["eff_acc_micro"][v]) \
            == (s.score, s.served, s.unmet, s.accsum, s.eff_acc_micro)
        assert host["option"][v].tolist() == s.option.tolist() and host["z_qps"][v].tolist() == s.z.tolist()
        assert (int(d["score"][v]), d["served"][v], d["accsum"][v]) == (s.score, s.served, s.accsum)
        assert d["option"][v].tolist() == s.option.tolist() and d["z_qps"][v].tolist() == s.z.tolist()
    rng = np.random.default_rng(405)
    for v in sorted(rng.choice(n, size=6, replace=False)):
        r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, dem[v], 2)
        assert (host["served"][v], host["accsum"][v]) == (r["served"], r["accsum"])
        assert host["option"][v].tolist() == r["option"].tolist()


def test_random_flat_kernel(px, oracle_mod):
    """The specialised flat kernel (sorted accuracies, D >= 3) on random toys
    (row filters by the largest other-family delta, flagged rows re-scanned),
    incl. tied accuracies and P = 0 holes."""
    rng = np.random.default_rng(4321)
    for trial in range(80):
        T = int(rng.integers(1, 4))
        Q = int(rng.integers(1, 5))
        D = int(rng.integers(3, 7))
        prof, dev, slo, P = random_instance(rng, T=T, Q=Q, Vmax=3, D=D, Pmax=40, tie_acc=trial % 3 == 0)
        s = rng.integers(0, 60, size=(3, prof.Q)).astype(np.int32)
        check(px, oracle_mod, prof, dev, slo, s, 0, False, threads=2)


def test_c2_bench_batch_sampled(px, oracle_mod):
    """The bench's launch configuration: the 64-vector c2 batch in one call
    (one flat launch, grid.y = vector) with device-resident inputs.  Sampled
    vectors against the exhaustive oracle; every vector's placement re-scored
    by the oracle, and the batch equal to one-vector calls."""
    import torch
    import bench
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2", totals=bench.C2_TOTALS)
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    dev = torch.device("cuda:0")
    sols = px.solve(torch.as_tensor(cl.device_type, device=dev), torch.as_tensor(cl.slo_us, device=dev),
                    torch.as_tensor(cfg["demand"], device=dev), mode=0)
    assert len(sols) == bench.NVEC
    for v in (0, 13, bench.NVEC - 1):
        r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][v], 0)
        assert (sols[v].index, sols[v].served, sols[v].accsum) == (r["index"], r["served"], r["accsum"])
        assert sols[v].z.tolist() == r["z"].tolist()
    for v, sol in enumerate(sols):
        chk = oracle_mod.score_placement(prof, cl.device_type, cl.slo_us, cfg["demand"][v], sol.option)
        assert (chk["served"], chk["accsum"]) == (sol.served, sol.accsum)
        one = px.solve(cl.device_type, cl.slo_us, cfg["demand"][v:v + 1], mode=0)[0]
        assert (one.score, one.index) == (sol.score, sol.index)


@pytest.mark.parametrize("world", [2, 3, 8])
def test_c2_batch_shards_combine(px, world):
    """The bench's N-GPU combine without NCCL: every rank's
    proteus_solve_batch over its index slice for the 64-vector batch,
    combined by proteus_combine_solutions (the pick kernel of the NCCL path),
    equals the one-GPU batch -- score, index, value, placement and z of every
    vector."""
    import bench
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2", totals=bench.C2_TOTALS)
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    D = len(cl.device_type)
    ref, n = px.solve_batch(cl.device_type, cl.slo_us, cfg["demand"], mode=0)
    parts = [px.solve_batch(cl.device_type, cl.slo_us, cfg["demand"], mode=0, shard_rank=r, shard_world=world)
             for r in range(world)]
    best, n_all = px.combine_solutions([p[0] for p in parts], [p[1] for p in parts], D)
    assert n_all == n == 13**8
    for k in ("score", "index", "served", "unmet", "accsum", "eff_acc_micro", "option", "z_qps"):
        assert np.array_equal(np.asarray(best[k]).astype(np.int64), np.asarray(ref[k]).astype(np.int64)), k


def test_nccl_collective_paths_world1():
    """The library's own NCCL communicator (proteus_comm_init, world 1 on
    cuda:0, in a subprocess with a torch NCCL process group for the id
    broadcast): distributed solve (modes 0, 1, 2), frontier, replay and
    closed loop equal the non-distributed calls (scripts/nccl_world1.py)."""
    import os
    import socket
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    with socket.socket() as s_:
        s_.bind(("127.0.0.1", 0))
        port = s_.getsockname()[1]
    r = subprocess.run([sys.executable, os.path.join(root, "scripts", "nccl_world1.py"), str(port)],
                       capture_output=True, text=True, timeout=600, cwd=root)
    assert r.returncode == 0 and "nccl world-1 ok" in r.stdout, (r.stdout + r.stderr)[-3000:]
