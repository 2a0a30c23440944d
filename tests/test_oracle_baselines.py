"""Pins for the §8(f2) baseline batchers in the oracle (§6.4).

Nexus early drop (reading R14) and Clipper AIMD (reading R15) are given by the
paper in prose only ("Nexus dispatches an inference batch to each device as
soon as the previous batch is finished"; "It keeps incrementally
increasing batch size until it experiences latency timeouts, at which point it
backs off multiplicatively"); their constants (the 10 % back-off,
the +1 step, Nexus's batch size) are readings, parity-unpinned against the
paper's numbers.  What is pinned: hand-worked closed forms of the rules as read
(tests/golden/baseline_batchers.json) and properties that hold on any trace.
"""

import numpy as np
import pytest

from tests._util import golden

DROP = 0xFFFFFFFF
T5 = [0, 100, 130, 160, 190, 220]


def _lat(x):
    return [DROP if v is None else v for v in x]


def test_nexus_closed_forms(oracle_mod):
    g = golden("baseline_batchers.json")
    for c in g["NEXUS"]:
        lat = oracle_mod.replay_device_nexus(c["arrival"], g["Tproc"], c["B"], c["L"])
        assert lat.tolist() == _lat(c["latency"]), c["what"]


def test_aimd_closed_forms(oracle_mod):
    g = golden("baseline_batchers.json")
    for c in g["AIMD"]:
        lat = oracle_mod.replay_device_aimd(c["arrival"], g["Tproc"], c["Bmax"], c["L"])
        assert lat.tolist() == _lat(c["latency"]), c["what"]


def _batches(a, lat):
    """Served queries grouped by finish time (F strictly increases between
    batches); dropped queries are skipped."""
    out, cur, curF = [], [], None
    for j in range(len(a)):
        if lat[j] == DROP:
            continue
        F = int(a[j]) + int(lat[j])
        if cur and F != curF:
            out.append((cur, curF))
            cur = []
        cur.append(j)
        curF = F
    if cur:
        out.append((cur, curF))
    return out


def _traces(kind, n_trials=5):
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    rng = np.random.default_rng(41)
    for trial in range(n_trials):
        a, _ = W.query_trace(3000, float(rng.uniform(500, 6000)), np.array([1.0]), 300 + trial, kind)
        yield rng, a


@pytest.mark.parametrize("kind", ["poisson", "gamma", "uniform"])
def test_nexus_invariants(oracle_mod, kind):
    """(i) every served query meets its SLO (the window's head meets its
    deadline and the rest arrived later: the early-drop guarantee);
    (ii) batches are FIFO, consecutive, of 1..B queries, and never overlap;
    (iii) work-conserving: a batch leaves at max(previous finish, the arrival
    of the first query left after the previous batch) -- the drops happen at
    that same instant or at earlier decisions that emptied the queue;
    (iv) the queries between two batches are exactly the dropped ones, and
    the window rule held for the batch: t + T(b) <= a_first + L with
    b = min(B, queued from first)."""
    for rng, a in _traces(kind):
        B = int(rng.integers(1, 6))
        L = int(rng.integers(250, 2000))
        lat = oracle_mod.replay_device_nexus(a, T5[:B + 1], B, L)
        served = lat != DROP
        assert np.all(lat[served].astype(np.int64) <= L)
        prevF, prev_end = 0, 0
        for idx, F in _batches(a, lat):
            first, b = idx[0], len(idx)
            assert idx == list(range(first, first + b)) and 1 <= b <= B
            t = F - T5[b]
            assert t >= prevF and t >= int(a[first + b - 1])
            assert np.all(lat[prev_end:first] == DROP)
            queued = int(np.searchsorted(a, t, side="right")) - first
            assert b == min(B, queued)
            assert t + T5[b] <= int(a[first]) + L
            # work-conserving: t is the previous finish or an arrival time no later than the batch's
            assert t == prevF or t in set(int(x) for x in a[prev_end:first + 1])
            prevF, prev_end = F, first + b
        assert np.all(lat[prev_end:] == DROP)


@pytest.mark.parametrize("kind", ["poisson", "gamma", "uniform"])
def test_aimd_invariants(oracle_mod, kind):
    """(i) conservation, no drops; (ii) work-conserving: every batch leaves at
    max(previous finish, its head's arrival); (iii) the first batch holds one
    query; (iv) the batch-size limit implied by each batch moves by the AIMD
    steps only: a batch smaller than its queue length sets the limit, which
    never exceeds the previous limit + 1 and after a timeout is at most
    floor(9 * previous / 10) (or 1)."""
    for rng, a in _traces(kind):
        Bmax = int(rng.integers(1, 6))
        L = int(rng.integers(250, 2000))
        lat = oracle_mod.replay_device_aimd(a, T5[:Bmax + 1], Bmax, L)
        assert np.all(lat != DROP)
        bs = _batches(a, lat)
        assert sum(len(i) for i, _ in bs) == len(a)
        assert len(bs[0][0]) == 1
        prevF, bound = 0, 1   # bound: the largest limit the rule allows now
        for k, (idx, F) in enumerate(bs):
            h, b = idx[0], len(idx)
            t = F - T5[b]
            assert t == max(prevF, int(a[h]))
            queued = int(np.searchsorted(a, t, side="right")) - h
            assert 1 <= b <= min(queued, Bmax)
            assert b <= bound
            timed_out = np.any(lat[h:h + b].astype(np.int64) > L)
            if b < queued:          # the limit itself: exact bound propagation
                bound = b
            bound = max(1, bound * 9 // 10) if timed_out else min(Bmax, bound + 1)
            prevF = F


def test_full_replay_policies(oracle_mod):
    """orc_replay with policy 1/2 rows: per lane equal to the device-level
    simulators (Nexus batch size = the capacity rule's b*, reading R14);
    conservation per scenario; every Nexus on-time count equals its served
    count (drops are the only violations besides the sink)."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3", totals=(3000,))
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    a, f = W.query_trace(20000, 3000.0, cfg["weights"], 79, "gamma")
    sc = np.array([(m, c, 0, p) for m in (1000, 2500) for c in (4, 0) for p in (0, 1, 2)], np.int32)
    out = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f, sc)
    N = len(a)
    fam_m = np.repeat(np.arange(prof.Q), prof.V)
    for s in range(len(sc)):
        assert out["on_time"][s] + out["violations"][s] == N
        lat = out["latency"][s]
        if sc[s, 3] != 1:
            continue
        L = (sc[s, 0] * cl.slo_us[f]) // 1000
        served = lat != DROP
        assert np.all(lat[served].astype(np.int64) <= L[served])
        assert out["on_time"][s] == np.sum(served)
    # one lane cross-checked against the device-level simulator: route with the
    # literal SWRR, take the busiest device
    dev_family = np.array([fam_m[o - 1] if o > 0 else -1 for o in r["option"]], np.int32)
    wdev = np.array([r["z"][d] if dev_family[d] >= 0 else 0 for d in range(len(dev_family))], np.int32)
    wsink = np.array(cfg["demand"][0], np.int32).copy()
    for d in range(len(dev_family)):
        if dev_family[d] >= 0:
            wsink[dev_family[d]] -= wdev[d]
    tgt = oracle_mod.route_swrr(f, prof.Q, dev_family, wdev, wsink)
    d = int(np.argmax(np.bincount(tgt, minlength=len(dev_family) + 1)[:len(dev_family)]))
    m = r["option"][d] - 1
    row = prof.lat_us[cl.device_type[d], m]
    depth = int(np.argmin(np.append(row > 0, False)))
    for s in range(len(sc)):
        cap = int(sc[s, 1])
        Bmax = min(cap, depth) if cap > 0 else depth
        L = int(sc[s, 0]) * int(cl.slo_us[fam_m[m]]) // 1000
        Tp = [0] + [int(x) for x in row[:Bmax]]
        sel = np.nonzero(tgt == d)[0]
        # the maximum allowed batch size: Nexus's batch (R14) and the
        # §5 policy's cap (R4'); AIMD grows its limit to min(cap, depth) (R15)
        B = max([1] + [b for b in range(1, Bmax + 1) if 2 * Tp[b] <= L])
        if sc[s, 3] == 1:
            ref = oracle_mod.replay_device_nexus(a[sel], Tp, B, L)
        elif sc[s, 3] == 2:
            ref = oracle_mod.replay_device_aimd(a[sel], Tp, Bmax, L)
        else:
            ref = oracle_mod.replay_device(a[sel], Tp[:B + 1], B, L)
        assert np.array_equal(out["latency"][s][sel], ref)
