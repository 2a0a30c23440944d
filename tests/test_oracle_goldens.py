"""The oracle-computed fixtures of tests/golden/ (written by
scripts/gen_goldens.py, which calls only oracle/): their inputs are still
the ones workloads.py draws, they are reproducible, and Oracle A agrees with
Oracle B -- the literal Eqs. 2-6 LP in exact rationals -- on
10^4 seeded c2 placements and 10^4 seeded c3 placements with the real
bmax-64 capacity tables ("10^5 seeded-random candidates of
c2/c3")."""

import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")
sys.path.insert(0, os.path.join(ROOT, "scripts"))


def _load(name):
    return np.load(os.path.join(GOLDEN, name))


def _gen():
    import gen_goldens
    return gen_goldens


@pytest.fixture(scope="module")
def lp():
    return _load("lp_literal.npz")


def _lp_cfg(name):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    if name == "c2":
        return W.config("c2", totals=W.C2_TOTALS + W.C2_BENCH_TOTALS[::8])
    c4 = W.config("c4")
    cfg = W.config("c3")
    cfg["demand"] = np.concatenate([cfg["demand"], c4["demand"][::400]])
    return cfg


@pytest.mark.parametrize("name", ["c2", "c3"])
def test_oracle_a_equals_literal_lp_on_1e4_placements(lp, oracle_mod, name):
    """Every stored placement: Oracle A's per-family vertex-enumeration LP
    (oracle.c) gives the literal LP's exact (served, accsum)."""
    cfg = _lp_cfg(name)
    assert str(lp[f"{name}_inputs_sha"]) == _gen().cfg_sha(cfg)
    prof, cl = cfg["prof"], cfg["cluster"]
    opt, vec = lp[f"{name}_option"], lp[f"{name}_vec"]
    served, accsum = lp[f"{name}_served"], lp[f"{name}_accsum"]
    assert len(opt) == 10_000
    bad = 0
    for i in range(len(opt)):
        r = oracle_mod.score_placement(prof, cl.device_type, cl.slo_us, cfg["demand"][vec[i]], opt[i])
        bad += (r["served"], r["accsum"]) != (int(served[i]), int(accsum[i]))
    assert bad == 0
    # the sample is not degenerate: every kind of placement, feasible and not
    assert len(set(served.tolist())) > 50 and np.sum(served == 0) < len(served) // 2


@pytest.mark.parametrize("name,k", [("c2", 40), ("c3", 8)])
def test_literal_lp_fixture_reproducible(lp, name, k):
    """A seeded sample of the stored values re-solved now by the literal LP."""
    from oracle import capacity
    from oracle.lp_exact import literal_assignment_lp
    cfg = _lp_cfg(name)
    prof, cl = cfg["prof"], cfg["cluster"]
    P = capacity(prof, cl.slo_us)[0]
    rng = np.random.default_rng(11)
    for i in rng.choice(len(lp[f"{name}_option"]), size=k, replace=False):
        s = cfg["demand"][lp[f"{name}_vec"][i]]
        sv, ac, _ = literal_assignment_lp(P, prof.acc_micro, prof.V, cl.device_type,
                                          lp[f"{name}_option"][i].tolist(), s.tolist(), presolve=True)
        assert (sv, ac) == (lp[f"{name}_served"][i], lp[f"{name}_accsum"][i])


def test_presolve_does_not_change_the_literal_lp():
    """lp_max's zero-fixing presolve only removes variables the constraints
    force to 0: on c2 placements the full dense LP (every y, z of Table 1)
    and the presolved one give the same optimum."""
    from oracle import capacity
    from oracle.lp_exact import literal_assignment_lp
    cfg = _lp_cfg("c2")
    prof, cl = cfg["prof"], cfg["cluster"]
    P = capacity(prof, cl.slo_us)[0]
    rng = np.random.default_rng(5)
    for _ in range(3):
        o = rng.integers(0, 13, size=8).tolist()
        s = cfg["demand"][rng.integers(0, len(cfg["demand"]))].tolist()
        a = literal_assignment_lp(P, prof.acc_micro, prof.V, cl.device_type, o, s, presolve=False)
        b = literal_assignment_lp(P, prof.acc_micro, prof.V, cl.device_type, o, s, presolve=True)
        assert a[:2] == b[:2]


def _check_solutions(g, prof, cl, demand, P):
    """invariants of stored optima (SURVEY §8(c) pins (i)): 0 <= z <= P of
    the hosted option, sum z = served <= demand per family, unmet = rest"""
    fam = np.repeat(np.arange(prof.Q), prof.V)
    for v in range(len(demand)):
        o, z = g["option"][v], g["z"][v]
        cap = np.array([P[cl.device_type[d], o[d] - 1] if o[d] else 0 for d in range(len(o))])
        assert np.all((z >= 0) & (z <= cap))
        served_q = np.bincount(fam[o[o > 0] - 1], weights=z[o > 0], minlength=prof.Q)
        assert np.all(served_q <= demand[v])
        assert int(served_q.sum()) == int(g["served"][v])
        assert int(g["served"][v]) + int(g["unmet"][v]) == int(demand[v].sum())
        accsum = sum(int(prof.acc_micro[o[d] - 1]) * int(z[d]) for d in range(len(o)) if o[d])
        assert accsum == int(g["accsum"][v])


def test_c2_bench_fixture(oracle_mod):
    """The bench step's 64 c2 vectors: inputs unchanged, invariants hold,
    vectors 0 and 63 re-solved now by the oracle match."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    g = _load("c2bench_oracle.npz")
    cfg = W.config("c2", totals=W.C2_BENCH_TOTALS)
    prof, cl = cfg["prof"], cfg["cluster"]
    assert str(g["inputs_sha"]) == _gen().cfg_sha(cfg)
    assert len(g["index"]) == W.C2_BENCH_NVEC == 64
    P = oracle_mod.capacity(prof, cl.slo_us)[0]
    _check_solutions(g, prof, cl, cfg["demand"], P)
    assert np.sum(g["unmet"] > 0) > 0 and np.sum(g["unmet"] == 0) > 0  # both regimes
    for v in (0, 63):
        r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][v], 0)
        assert (r["index"], r["served"], r["accsum"]) == (g["index"][v], g["served"][v], g["accsum"][v])
        assert r["option"].tolist() == g["option"][v].tolist() and r["z"].tolist() == g["z"][v].tolist()


def test_c4_fixture(oracle_mod):
    """All 3600 c4 vectors: inputs unchanged, invariants hold, a seeded
    sample re-solved now by the oracle's factored search matches; the f4
    controller's demand is the c4 counts shifted by one epoch (so f4's
    allocations are rows of this fixture)."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    g = _load("c4_oracle.npz")
    cfg = W.config("c4")
    prof, cl = cfg["prof"], cfg["cluster"]
    assert str(g["inputs_sha"]) == _gen().cfg_sha(cfg)
    assert len(g["served"]) == 3600
    P = oracle_mod.capacity(prof, cl.slo_us)[0]
    _check_solutions(g, prof, cl, cfg["demand"], P)
    for v in np.random.default_rng(3).choice(3600, size=6, replace=False):
        r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][v], 2)
        assert (r["served"], r["accsum"]) == (g["served"][v], g["accsum"][v])
        assert r["option"].tolist() == g["option"][v].tolist() and r["z"].tolist() == g["z"][v].tolist()
    f4 = W.config("f4")
    assert np.array_equal(f4["demand"][1:], cfg["demand"][:-1]) and np.array_equal(f4["demand"][0], cfg["demand"][0])
