"""Pins for the replay oracle (event-driven §5 simulator + SWRR router).

Closed forms are derived by hand from P:970-1005 (Fig. 3, Case 1 / Case 2) in
tests/golden/h1_g1.json; the invariants below are properties of the rule
that hold on any trace.
"""

import numpy as np
import pytest

from tests._util import golden

T5 = [0, 100, 130, 160, 190, 220]


def test_closed_forms(oracle_mod):
    g = golden()["REPLAY_CLOSED_FORMS"]
    for c in g["cases"]:
        lat = oracle_mod.replay_device(c["arrival"], g["Tproc"], c["Bmax"], g["L"])
        assert lat.tolist() == c["latency"], c["what"]


def _batches(a, lat):
    """Reconstruct batches: consecutive queries sharing a finish time F = a + lat
    (F strictly increases from batch to batch since T(b) > 0)."""
    F = a.astype(np.int64) + lat.astype(np.int64)
    out, h = [], 0
    for j in range(1, len(a) + 1):
        if j == len(a) or F[j] != F[h]:
            out.append((h, j - h, int(F[h])))
            h = j
    return out


def _check_invariants(a, lat, Tp, Bmax, L):
    batches = _batches(a, lat)
    assert sum(b for _, b, _ in batches) == len(a)      # conservation
    prevF = 0
    for h, b, F in batches:
        assert 1 <= b <= Bmax
        t = F - Tp[b]                                    # dispatch time
        assert t >= prevF                                # device serves one batch at a time
        assert t >= a[h + b - 1]                         # every member had arrived
        assert np.all(lat[h:h + b] >= Tp[b])
        # queries arriving by t that were not taken must exceed Bmax (FIFO + R4)
        waiting = np.searchsorted(a, t, side="right") - h
        assert waiting == b or b == Bmax
        if b < Bmax:
            # Case 1 / Case 2: a batch of b < Bmax leaves only once Tmax_wait(b+1) has passed,
            # either by the timer (t = W) or at the event that completed the queue
            W = int(a[h]) + L - Tp[b + 1]
            assert t >= W
            assert t == W or t == max(prevF, int(a[h + b - 1]))
        # proactive guarantee: dispatched by Tmax_wait(b) -> no violation in the batch
        if t <= int(a[h]) + L - Tp[b]:
            assert np.all(lat[h:h + b] <= L)
        prevF = F


@pytest.mark.parametrize("kind", ["poisson", "gamma", "uniform"])
def test_event_sim_invariants(oracle_mod, kind):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    rng = np.random.default_rng(23)
    for trial in range(6):
        a, _ = W.query_trace(3000, float(rng.uniform(200, 3000)), np.array([1.0]), 100 + trial, kind)
        Bmax = int(rng.integers(1, 6))
        L = int(rng.integers(300, 3000))
        lat = oracle_mod.replay_device(a, T5[:Bmax + 1], Bmax, L)
        _check_invariants(a, lat, T5 + [10**9], Bmax, L)


def test_light_load_latency_is_closed_form(oracle_mod):
    """Arrivals far apart: each query is alone, waits until Tmax_wait(2) and
    finishes at a + L - T(2) + T(1) (Case 1)."""
    a = np.arange(0, 50_000 * 40, 50_000, dtype=np.uint32)
    lat = oracle_mod.replay_device(a, T5, 5, 1000)
    assert np.all(lat == 1000 - 130 + 100)


def test_saturated_stream_full_batches(oracle_mod):
    """All queries at t = 0 with Bmax = 4: batches of 4 back to back; batch k
    finishes at (k+1) * T(4) (R4), the last partial batch follows Case 1."""
    a = np.zeros(40, np.uint32)
    lat = oracle_mod.replay_device(a, T5[:5], 4, 10**6)
    assert lat.tolist() == [190 * (k // 4 + 1) for k in range(40)]


def test_swrr_exact_counts_per_period(oracle_mod):
    """R8: within every window of W = sum(weights) consecutive queries of a
    family, member d receives exactly w_d queries (SWRR property)."""
    rng = np.random.default_rng(29)
    for _ in range(10):
        D, Q = 6, 3
        dev_family = rng.integers(-1, Q, size=D).astype(np.int32)
        w = rng.integers(0, 9, size=D).astype(np.int32)
        w_sink = rng.integers(0, 5, size=Q).astype(np.int32)
        fam = rng.integers(0, Q, size=4000).astype(np.uint8)
        tgt = oracle_mod.route_swrr(fam, Q, dev_family, w, w_sink)
        for q in range(Q):
            members = [d for d in range(D) if dev_family[d] == q]
            Wq = int(sum(w[d] for d in members) + w_sink[q])
            tq = tgt[fam == q]
            if Wq == 0:
                assert np.all(tq == D)
                continue
            for k in range(0, len(tq) - Wq + 1, Wq):
                win = tq[k:k + Wq]
                for d in members:
                    assert np.sum(win == d) == w[d]
                assert np.sum(win == D) == w_sink[q]
            assert set(np.unique(tq)) <= set(members) | {D}


def test_swrr_smooth_small_example(oracle_mod):
    """Weights (5, 1, 1) -> the classic smooth sequence a a b a c a a."""
    tgt = oracle_mod.route_swrr(np.zeros(7, np.uint8), 1, np.array([0, 0, 0], np.int32),
                                np.array([5, 1, 1], np.int32), np.array([0], np.int32))
    assert tgt.tolist() == [0, 0, 1, 0, 2, 0, 0]


def test_full_replay_conservation(oracle_mod):
    """(i) conservation: on_time + violations = N per scenario; dropped
    queries (sink) have latency UINT32_MAX and count as violations (R6, R7);
    routing counts match SWRR weights; results identical across thread counts."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3", totals=(12000,))
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    assert r["unmet"] > 0
    a, f = W.query_trace(20000, 12000.0, cfg["weights"], 77, "poisson")
    sc = np.array([(m, c, rt) for m in (1000, 2000) for c in (1, 8, 0) for rt in (0, 1)], np.int32)
    out = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f, sc)
    out1 = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f, sc,
                             threads=1)
    for k in ("violations", "on_time", "acc_sum"):
        assert np.array_equal(out[k], out1[k])
    assert np.array_equal(out["latency"], out1["latency"])
    N = len(a)
    for s in range(len(sc)):
        assert out["on_time"][s] + out["violations"][s] == N
        dropped = np.sum(out["latency"][s] == 0xFFFFFFFF)
        if sc[s, 2] == 0:
            assert dropped > 0
        L = (sc[s, 0] * cl.slo_us[f]) // 1000
        assert out["on_time"][s] == np.sum(out["latency"][s].astype(np.int64) <= L)


def test_uniform_routing_has_no_sink(oracle_mod):
    """Routing mode 1 (w/o QA): weight 1 per hosting device that
    fits batch 1; a family with no such device is dropped entirely."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3", totals=(3000,))
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    a, f = W.query_trace(5000, 3000.0, cfg["weights"], 78, "poisson")
    out = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f,
                            np.array([[2000, 0, 1]], np.int32))
    fam_m = np.repeat(np.arange(prof.Q), prof.V)
    hosted = {int(fam_m[o - 1]) for o in r["option"] if o > 0}
    dropped = out["latency"][0] == 0xFFFFFFFF
    assert set(np.unique(f[dropped]).tolist()) <= set(range(prof.Q)) - hosted


def test_acc_sum_hand_worked(oracle_mod):
    """R9 pin ("accuracy for all the queries successfully
    served"): acc_sum = sum of the serving variant's accuracy over ON-TIME
    queries only; late and dropped queries add nothing.  Worked by hand:

    one family, two variants v0 (A = 1 000 000, option 1) and v1 (A = 900 000,
    option 2); one device type, table depth 1 (so Bmax = 1, R4: every query is
    dispatched alone at max(F, a)), T_v0(1) = 100 us, T_v1(1) = 50 us.  Device
    0 hosts v0 with z = 1, device 1 hosts v1 with z = 1, demand s = 3, so the
    sink weight is unmet = 1 (R7, R8).  SWRR over weights (1, 1, sink 1):
    currents (1,1,1) -> device 0; (-1,2,2) -> device 1; (0,0,3) -> sink; the
    pattern repeats every 3 queries.  Arrivals 0, 0, 0, 10, 10, 20 us:
      q0 -> dev 0 at 0: F = 100, latency 100
      q1 -> dev 1 at 0: F = 50,  latency 50
      q2 -> sink: dropped (UINT32_MAX)
      q3 -> dev 0 at 10, busy until 100: F = 200, latency 190
      q4 -> dev 1 at 10, busy until 50:  F = 100, latency 90
      q5 -> sink: dropped
    SLO base 150 us, multiplier 1x: q3 is late (190 > 150, R6) -> on_time 3,
    violations 3 (one late + two dropped), acc_sum = A0 + A1 + A1 = 2 800 000.
    Multiplier 2x (SLO 300): q3 on time -> on_time 4, violations 2,
    acc_sum = 1e6 + 9e5 + 1e6 + 9e5 = 3 800 000."""
    from paper_conf_asplos_ahmadgfwsw24_b200.workloads import Profiles
    prof = Profiles(T=1, Q=1, V=np.array([2], np.int32), acc_micro=np.array([1_000_000, 900_000], np.int32),
                    bmax=1, lat_us=np.array([[[100], [50]]], np.int32))
    arr = np.array([0, 0, 0, 10, 10, 20], np.uint32)
    fam = np.zeros(6, np.uint8)
    sc = np.array([[1000, 0, 0], [2000, 0, 0]], np.int32)
    out = oracle_mod.replay(prof, np.array([0, 0], np.int32), np.array([1, 2], np.int32),
                            np.array([1, 1], np.int32), np.array([3], np.int32), np.array([150], np.int32),
                            arr, fam, sc)
    U = 0xFFFFFFFF
    assert out["latency"][0].tolist() == [100, 50, U, 190, 90, U]
    assert out["latency"][1].tolist() == [100, 50, U, 190, 90, U]
    assert out["on_time"].tolist() == [3, 4]
    assert out["violations"].tolist() == [3, 2]
    assert out["acc_sum"].tolist() == [2_800_000, 3_800_000]


def test_max_allowed_batch_size_R4prime(oracle_mod):
    """Reading R4': a device batches at most the "maximum allowed
    batch size" -- the largest b <= min(cap, depth) with 2 T(b) <= SLO (the
    half-SLO rule of P:920-926), at least 1.  Worked by hand: one variant,
    T = (100, 130, 160, 190, 220) us for b = 1..5 (depth 5), 7 queries at t = 0,
    one device with z = 7 = demand (no sink).
      SLO 400, cap depth: b* = 4 (2 x 190 <= 400 < 2 x 220): four leave at 0
        (F = 190); three wait until W = 0 + 400 - T(4) = 210, F = 210 + 160 = 370
        -> latencies 190 x 4, 370 x 3, all on time.
      SLO 400, cap 3: three at 0 (F = 160); at 160 four are queued >= 3: three
        more (F = 320); at 320 one is left, W = 400 - T(2) = 270 <= 320: it
        leaves at once, F = 420 -> 160 x 3, 320 x 3, 420 (late).
      SLO 800: b* = 5 = depth: five at 0 (F = 220); two wait until
        W = 800 - T(3) = 640, F = 770 -> 220 x 5, 770 x 2."""
    from paper_conf_asplos_ahmadgfwsw24_b200.workloads import Profiles
    prof = Profiles(T=1, Q=1, V=np.array([1], np.int32), acc_micro=np.array([1_000_000], np.int32), bmax=5,
                    lat_us=np.array([[[100, 130, 160, 190, 220]]], np.int32))
    arr = np.zeros(7, np.uint32)
    fam = np.zeros(7, np.uint8)
    sc = np.array([[1000, 0, 0], [1000, 3, 0], [2000, 0, 0]], np.int32)
    out = oracle_mod.replay(prof, np.array([0], np.int32), np.array([1], np.int32), np.array([7], np.int32),
                            np.array([7], np.int32), np.array([400], np.int32), arr, fam, sc)
    assert out["latency"][0].tolist() == [190] * 4 + [370] * 3
    assert out["latency"][1].tolist() == [160] * 3 + [320] * 3 + [420]
    assert out["latency"][2].tolist() == [220] * 5 + [770] * 2
    assert out["on_time"].tolist() == [7, 6, 7] and out["violations"].tolist() == [0, 1, 0]
