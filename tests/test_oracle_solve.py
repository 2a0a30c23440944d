"""Pins for the solve oracle (oracle/oracle.c, oracle/lp_exact.py).

Nothing here compares the oracle with itself: every check is against a value
derived by hand from the paper, an independent formulation (the literal LP of
Eqs. 2-6 in exact rationals, a float LP solver, fractional brute force), or an
invariant that the mathematics fixes.
"""

import itertools

import numpy as np
import pytest

from tests._util import golden, packed_score, profiles_from_capacity, random_instance

# ---------------------------------------------------------------- a1 -----


def test_capacity_closed_form(oracle_mod):
    """b* = min(SLO bound, memory bound); P = b* / latency.
    Hand table: type 0 latencies 10,12,14,16 us (b = 1..4); SLO 28 ->
    2*lat <= 28 holds for b <= 3 (2*14 = 28, non-strict C5) -> b* = 3,
    P = floor(3e6 / 14) = 214285.  Type 1: batch 3 does not fit (memory) ->
    depth 2, b* = 2, P = floor(2e6 / 12) = 166666.  Type 2: 2*lat(1) = 30 > 28
    -> P = 0."""
    from paper_conf_asplos_ahmadgfwsw24_b200.workloads import Profiles
    lat = np.array([[[10, 12, 14, 16]], [[10, 12, 0, 16]], [[15, 16, 17, 18]]], np.int32)
    prof = Profiles(T=3, Q=1, V=np.array([1], np.int32), acc_micro=np.array([1_000_000], np.int32),
                    bmax=4, lat_us=lat)
    P, bs, dep = oracle_mod.capacity(prof, [28])
    assert P.tolist() == [[214285], [166666], [0]]
    assert bs.tolist() == [[3], [2], [0]]
    assert dep.tolist() == [[4], [2], [4]]


# ------------------------------------------------------- hand-worked -----


def _h1():
    g = golden()["H1"]
    from paper_conf_asplos_ahmadgfwsw24_b200.workloads import Profiles
    prof = Profiles(T=1, Q=1, V=np.array(g["V"], np.int32), acc_micro=np.array(g["acc_micro"], np.int32),
                    bmax=1, lat_us=np.array(g["lat_us"], np.int32))
    return g, prof


def test_h1_hand_worked(oracle_mod):
    """H1: one family, v0 (A = 1.0, P = 10), v1 (A = 0.9, P = 25), two devices,
    options {0 idle, 1 = v0, 2 = v1}, idx = 3*o_0 + o_1.
      s = 30: (1,2) caps 10 + 25; fill v0 first (C10): z = (10, 20);
              accsum = 10*1e6 + 20*9e5 = 28e6; (2,1) ties at idx 7 > 5; (2,2)
              gives 30*9e5 = 27e6; (1,1) serves only 20.
      s = 20: (1,1) serves 20 at accuracy 1.0 = 20e6, idx 4 (beats (1,2) idx 5
              which also gives 20e6 -> lowest index, C9).
      s = 55: nothing serves more than 50 = (2,2); unmet 5 (C1).
      s = 0 : every placement scores 0; idx 0 (all idle)."""
    g, prof = _h1()
    P, _, _ = oracle_mod.capacity(prof, g["slo_us"])
    assert P.tolist() == g["P"]
    for c in g["cases"]:
        r = oracle_mod.solve(prof, g["device_type"], g["slo_us"], c["s"], 0)
        assert r["index"] == c["index"]
        assert r["option"].tolist() == c["option"]
        assert (r["served"], r["accsum"], r["eff"]) == (c["served"], c["accsum"], c["eff"])
        assert r["z"].tolist() == c["z"]
        assert r["unmet"] == sum(c["s"]) - c["served"]


def _g1():
    g = golden()["G1"]
    prof = profiles_from_capacity(g["P"], g["acc_micro"], g["V"])
    return g, prof


def test_g1_hand_worked(oracle_mod):
    """G1 (45, 12): family 1 needs 12 QPS; a GPU at v1 (cap 14, A 0.88) beats
    v2 (A 0.82) and v0 (cap 8 < 12), so one GPU hosts option 5.  Family 0 then
    has two CPUs (caps 4 at v1, 9 at v2) and one GPU; 45 = 4 + 9 + 32 exactly
    with the GPU at v1 (32, A 0.9): accsum = 4*0.9 + 9*0.8 + 32*0.9 ... in 1e-6
    units 4*900000 + 9*800000 + 32*900000 + 12*880000 = 50 160 000; served 57.
    The lowest index among equal placements is (2, 3, 2, 5) = 2*343 + 3*49 +
    2*7 + 5 = 852."""
    g, prof = _g1()
    P, _, _ = oracle_mod.capacity(prof, g["slo_us"])
    assert P.tolist() == g["P"]
    for c in g["cases"]:
        r = oracle_mod.solve(prof, g["device_type"], g["slo_us"], c["s"], 0)
        assert r["index"] == c["index"], c
        assert r["option"].tolist() == c["option"]
        assert (r["served"], r["accsum"], r["eff"]) == (c["served"], c["accsum"], c["eff"])
        assert r["z"].tolist() == c["z"]
        if "score_hex" in c:
            assert packed_score(r["served"], r["accsum"]) == int(c["score_hex"], 16)
        if "multiset_index" in c:
            r1 = oracle_mod.solve(prof, g["device_type"], g["slo_us"], c["s"], 1)
            assert r1["index"] == c["multiset_index"]
            assert (r1["served"], r1["accsum"]) == (c["served"], c["accsum"])
        r2 = oracle_mod.solve(prof, g["device_type"], g["slo_us"], c["s"], 2)
        assert (r2["served"], r2["accsum"]) == (c["served"], c["accsum"])


def test_g1_index_arithmetic():
    """C9: idx = sum_d o_d K^(D-1-d) with K = 7 (1 + 2*3 options, C8)."""
    assert 2 * 7**3 + 3 * 7**2 + 2 * 7 + 5 == 852
    assert 3 * 7**3 + 3 * 7**2 + 3 * 7 + 6 == 1203


# ------------------------------------------- LP against the literal LP ---


def test_family_lp_vs_literal_rational_lp(oracle_mod):
    """Per-candidate value = the literal Eqs. 2-6 LP (exact rationals) on a
    seeded sample of G1 placements and random toy instances."""
    from oracle.lp_exact import literal_assignment_lp
    g, prof = _g1()
    P = np.array(g["P"])
    rng = np.random.default_rng(7)
    cands = [np.array(c["option"]) for c in g["cases"]] + [rng.integers(0, 7, size=4) for _ in range(30)]
    for opt in cands:
        for s in ([45, 12], [80, 30], [7, 3]):
            r = oracle_mod.score_placement(prof, g["device_type"], g["slo_us"], s, opt)
            served, acc, z = literal_assignment_lp(P, g["acc_micro"], g["V"], g["device_type"], opt.tolist(), s)
            assert (r["served"], r["accsum"]) == (served, acc)
    for _ in range(40):
        prof2, dev, slo, P2 = random_instance(rng, T=2, Q=2, Vmax=3, D=4, Pmax=20)
        opt = rng.integers(0, 1 + prof2.M, size=len(dev))
        s = rng.integers(0, 40, size=prof2.Q)
        r = oracle_mod.score_placement(prof2, dev, slo, s, opt)
        served, acc, _ = literal_assignment_lp(P2, prof2.acc_micro, prof2.V, dev, opt.tolist(), s)
        assert (r["served"], r["accsum"]) == (served, acc)


def test_all_c1_candidates_vs_highs_lp(oracle_mod):
    """Every c1 candidate (7^4 = 2401): oracle value = a two-stage float LP
    (scipy HiGHS) over the literal Eqs. 2-6, rounded (values are integral)."""
    scipy_opt = pytest.importorskip("scipy.optimize")
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c1")
    prof, cl, s = cfg["prof"], cfg["cluster"], cfg["demand"][0]
    P, _, _ = oracle_mod.capacity(prof, cl.slo_us)
    fam = np.repeat(np.arange(prof.Q), prof.V)
    D, Q = len(cl.device_type), prof.Q
    for opt in itertools.product(range(1 + prof.M), repeat=D):
        # variables z[d][q] only (y eliminated: y = z/s satisfies Eqs. 2-4)
        ub = np.zeros(D * Q)
        for d in range(D):
            if opt[d]:
                ub[d * Q + fam[opt[d] - 1]] = P[cl.device_type[d], opt[d] - 1]
        A = np.zeros((Q, D * Q))
        for q in range(Q):
            A[q, q::Q] = 1
        r1 = scipy_opt.linprog(-np.ones(D * Q), A_ub=A, b_ub=s, bounds=list(zip([0] * (D * Q), ub)),
                               method="highs")
        served = round(-r1.fun)
        accw = np.zeros(D * Q)
        for d in range(D):
            if opt[d]:
                accw[d * Q + fam[opt[d] - 1]] = prof.acc_micro[opt[d] - 1]
        r2 = scipy_opt.linprog(-accw, A_ub=A, b_ub=s, A_eq=np.ones((1, D * Q)), b_eq=[served],
                               bounds=list(zip([0] * (D * Q), ub)), method="highs")
        acc = round(-r2.fun)
        r = oracle_mod.score_placement(prof, cl.device_type, cl.slo_us, s, np.array(opt))
        assert (r["served"], r["accsum"]) == (served, acc), opt


def test_fractional_brute_force(oracle_mod):
    """Toy inputs: brute force over z on a 1/2 grid (Eqs. 2-6) = the oracle's
    LP value (the LP optimum is integral here: reading C1/TU argument)."""
    from oracle.lp_exact import brute_force_fractional
    rng = np.random.default_rng(11)
    n = 0
    while n < 25:
        prof, dev, slo, P = random_instance(rng, T=2, Q=2, Vmax=2, D=3, Pmax=4)
        opt = rng.integers(0, 1 + prof.M, size=len(dev))
        s = rng.integers(0, 8, size=prof.Q)
        best = brute_force_fractional(P, prof.acc_micro, prof.V, dev, opt.tolist(), s, grid=2)
        r = oracle_mod.score_placement(prof, dev, slo, s, opt)
        assert (r["served"], r["accsum"]) == best
        n += 1


# ----------------------------------------------------- search pins -------


def test_argmax_is_brute_force_over_all_candidates(oracle_mod):
    """Mode 0 argmax = max over score_placement of every candidate, first
    (lowest index, device 0 most significant) among ties."""
    rng = np.random.default_rng(3)
    for trial in range(12):
        prof, dev, slo, P = random_instance(rng, T=2, Q=2, Vmax=2, D=4, Pmax=15, tie_acc=trial % 2 == 0)
        s = rng.integers(0, 40, size=prof.Q)
        K = 1 + prof.M
        best, best_idx = None, None
        for idx, opt in enumerate(itertools.product(range(K), repeat=len(dev))):
            r = oracle_mod.score_placement(prof, dev, slo, s, np.array(opt))
            key = (r["served"], r["accsum"])
            if best is None or key > best:
                best, best_idx = key, idx
        r = oracle_mod.solve(prof, dev, slo, s, 0)
        assert (r["served"], r["accsum"]) == best
        assert r["index"] == best_idx


def test_multiset_index_is_rank_of_sorted_representatives(oracle_mod):
    """Mode 1 canonical index = rank of the candidate among flat candidates
    whose options are non-decreasing within each type (devices sorted by
    type), in flat index order (reading C9)."""
    rng = np.random.default_rng(5)
    for _ in range(8):
        prof, dev, slo, P = random_instance(rng, T=2, Q=2, Vmax=2, D=4, Pmax=15, tie_acc=True)
        s = rng.integers(0, 40, size=prof.Q)
        K = 1 + prof.M
        best, best_rank, rank = None, None, 0
        for opt in itertools.product(range(K), repeat=len(dev)):
            if any(dev[d] == dev[d + 1] and opt[d] > opt[d + 1] for d in range(len(dev) - 1)):
                continue
            r = oracle_mod.score_placement(prof, dev, slo, s, np.array(opt))
            key = (r["served"], r["accsum"])
            if best is None or key > best:
                best, best_rank = key, rank
            rank += 1
        r1 = oracle_mod.solve(prof, dev, slo, s, 1)
        assert r1["n_candidates"] == rank == oracle_mod.enum_count(prof, dev, 1)
        assert (r1["served"], r1["accsum"]) == best
        assert r1["index"] == best_rank


def test_three_modes_agree_and_factored_is_lexmin(oracle_mod):
    """Invariant (iii): flat = multiset = factored optimum value.  The factored
    canonical is the lexicographically smallest count tensor among optima:
    checked by brute force over all flat candidates' count tensors."""
    rng = np.random.default_rng(9)
    for trial in range(15):
        prof, dev, slo, P = random_instance(rng, T=2, Q=2, Vmax=3, D=4, Pmax=15, tie_acc=trial % 3 == 0)
        s = rng.integers(0, 50, size=prof.Q)
        r0 = oracle_mod.solve(prof, dev, slo, s, 0)
        r1 = oracle_mod.solve(prof, dev, slo, s, 1)
        r2 = oracle_mod.solve(prof, dev, slo, s, 2)
        r2u = oracle_mod.solve(prof, dev, slo, s, 2, prune=0)
        vals = {(r["served"], r["accsum"]) for r in (r0, r1, r2, r2u)}
        assert len(vals) == 1
        assert np.array_equal(r2["counts"], r2u["counts"])  # reading C16
        # brute-force lexmin tensor
        K = 1 + prof.M
        fam = np.repeat(np.arange(prof.Q), prof.V)
        off = np.concatenate([[0], np.cumsum(prof.V)[:-1]])
        best_t = None
        for opt in itertools.product(range(K), repeat=len(dev)):
            r = oracle_mod.score_placement(prof, dev, slo, s, np.array(opt))
            if (r["served"], r["accsum"]) != (r0["served"], r0["accsum"]):
                continue
            n = np.zeros((prof.Q, prof.T, 16), np.int32)
            for d, o in enumerate(opt):
                if o:
                    n[fam[o - 1], dev[d], o - 1 - off[fam[o - 1]]] += 1
            key = tuple(n.ravel())
            if best_t is None or key < best_t:
                best_t = key
        assert tuple(r2["counts"].ravel()) == best_t
        # materialised placement realises that tensor and its value
        chk = oracle_mod.score_placement(prof, dev, slo, s, r2["option"])
        assert (chk["served"], chk["accsum"]) == (r0["served"], r0["accsum"])


def test_invariants_z_and_capacity(oracle_mod):
    """(i) 0 <= z_d <= P_d; sum_d z_{d,q} = served_q <= s_q; unmet = sum s - served."""
    rng = np.random.default_rng(13)
    for _ in range(30):
        prof, dev, slo, P = random_instance(rng, T=3, Q=3, Vmax=3, D=5, Pmax=25)
        s = rng.integers(0, 60, size=prof.Q)
        r = oracle_mod.solve(prof, dev, slo, s, 1)
        fam = np.repeat(np.arange(prof.Q), prof.V)
        served_q = np.zeros(prof.Q, np.int64)
        acc = 0
        for d, o in enumerate(r["option"]):
            if o == 0:
                assert r["z"][d] == 0
                continue
            assert 0 <= r["z"][d] <= P[dev[d], o - 1]
            served_q[fam[o - 1]] += r["z"][d]
            acc += int(r["z"][d]) * int(prof.acc_micro[o - 1])
        assert np.all(served_q <= s)
        assert served_q.sum() == r["served"] and acc == r["accsum"]
        assert r["unmet"] == s.sum() - r["served"]
        assert r["eff"] == (acc // r["served"] if r["served"] else 0)


def test_monotone_in_added_device(oracle_mod):
    """(ii) Adding a device never lowers the optimum (it may idle, Eq. 1 '<=')."""
    rng = np.random.default_rng(17)
    for _ in range(20):
        prof, dev, slo, P = random_instance(rng, T=2, Q=2, Vmax=3, D=3, Pmax=20)
        s = rng.integers(0, 60, size=prof.Q)
        r = oracle_mod.solve(prof, dev, slo, s, 0)
        dev2 = np.sort(np.concatenate([dev, [rng.integers(0, 2)]])).astype(np.int32)
        r2 = oracle_mod.solve(prof, dev2, slo, s, 0)
        assert (r2["served"], r2["accsum"]) >= (r["served"], r["accsum"])


def test_permutation_and_scaling(oracle_mod):
    """(vii) permuting same-type devices keeps the score; (ix) scaling every P
    and s by k scales served and accsum by k; (viii) s = 0 -> idx 0."""
    rng = np.random.default_rng(19)
    for _ in range(20):
        prof, dev, slo, P = random_instance(rng, T=2, Q=2, Vmax=3, D=4, Pmax=20)
        s = rng.integers(0, 50, size=prof.Q)
        opt = rng.integers(0, 1 + prof.M, size=4)
        r = oracle_mod.score_placement(prof, dev, slo, s, opt)
        same = [d for d in range(4) if dev[d] == dev[0]]
        opt2 = opt.copy()
        opt2[same] = opt[same][::-1]
        r2 = oracle_mod.score_placement(prof, dev, slo, s, opt2)
        assert (r["served"], r["accsum"]) == (r2["served"], r2["accsum"])
        k = 3
        r3 = oracle_mod.solve(prof, dev, slo, s * k, 0, P=P * k)
        r4 = oracle_mod.solve(prof, dev, slo, s, 0, P=P)
        assert (r3["served"], r3["accsum"]) == (k * r4["served"], k * r4["accsum"])
        r5 = oracle_mod.solve(prof, dev, slo, np.zeros(prof.Q, np.int32), 0)
        assert r5["index"] == 0 and r5["served"] == 0


def test_single_family_textbook_knapsack(oracle_mod):
    """Q = 1 with identical devices: choose counts; the LP is the textbook
    continuous knapsack (greedy by value density = accuracy here)."""
    A = [1_000_000, 900_000, 800_000]
    cap = [5, 9, 20]
    for s in range(0, 60, 3):
        # textbook: fill in decreasing accuracy
        rem, acc = s, 0
        for a, c in zip(A, cap):
            t = min(rem, c)
            acc += a * t
            rem -= t
        assert oracle_mod.family_lp(A, cap, [1, 1, 1], s) == (s - rem, acc)


def test_c1_c2_regimes(oracle_mod):
    """Workload recipe checks: c1/c2 demand at the scaling
    regime mixes variants with unmet = 0; the overload vector has unmet > 0."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    assert r["unmet"] == 0 and r["eff"] < 1_000_000
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][1], 2)
    assert r["unmet"] > 0
    cfg = W.config("c1")
    r = oracle_mod.solve(cfg["prof"], cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"][0], 0)
    assert r["unmet"] == 0 and r["eff"] < 1_000_000 and r["n_candidates"] == 7**4



def test_optimum_dominates_clipper_ht_ha(oracle_mod):
    """(vi) The joint optimum is at least the value of the static Clipper
    placements: Clipper-HT allocates with only each family's
    least accurate variant, Clipper-HA with only its most accurate one -- the
    same search over a subset of the options (the other variants made
    infeasible: latency 0 = does not fit, reading C7).  Also: with a single
    variant per family the restricted and full searches coincide."""
    from paper_conf_asplos_ahmadgfwsw24_b200.workloads import Profiles
    rng = np.random.default_rng(31)
    for _ in range(25):
        prof, dev, slo, P = random_instance(rng, T=2, Q=2, Vmax=3, D=3, Pmax=25)
        s = rng.integers(0, 70, size=prof.Q)
        full = oracle_mod.solve(prof, dev, slo, s, 0)
        off = np.concatenate([[0], np.cumsum(prof.V)[:-1]])
        for pick in ("HT", "HA"):
            lat = prof.lat_us.copy()
            for q in range(prof.Q):
                accs = prof.acc_micro[off[q]:off[q] + prof.V[q]]
                keep = off[q] + (int(np.argmin(accs)) if pick == "HT" else int(np.argmax(accs)))
                for m in range(off[q], off[q] + prof.V[q]):
                    if m != keep:
                        lat[:, m, :] = 0
            sub = Profiles(T=prof.T, Q=prof.Q, V=prof.V, acc_micro=prof.acc_micro, bmax=prof.bmax, lat_us=lat)
            r = oracle_mod.solve(sub, dev, slo, s, 0)
            assert (full["served"], full["accsum"]) >= (r["served"], r["accsum"]), pick
            if all(v == 1 for v in prof.V):
                assert (full["served"], full["accsum"]) == (r["served"], r["accsum"])
