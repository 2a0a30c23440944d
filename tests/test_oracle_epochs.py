"""Pins for the §8(f4) closed-loop replay in the oracle (readings F1-F4,
DESIGN.md): one allocation per epoch (the per-second re-solve, P:707-723,
P:1369-1370), routing restarted each epoch, a device finishing one epoch's
queue with that epoch's variant before the next epoch's queries.

Pinned against the single-allocation simulator (already pinned by the §5
closed forms), hand-worked two-epoch cases and invariants."""

import numpy as np

T0 = [0, 100, 130, 160, 190, 220]
T1 = [0, 50, 60, 70]


def test_two_epoch_closed_forms(oracle_mod):
    """epoch_us = 500.  Query 0 (epoch 0, L 1000) waits alone until
    Tmax_wait(2) = 870 -- query 1 (epoch 1) arriving at 600 does not join
    (F3) -- and finishes at 970.  Query 1 is then the head: Tmax_wait(2) =
    600 + 400 - 60 = 940 <= 970, so it leaves at once: 970 + 50 = 1020,
    latency 420.  With query 2 (epoch 1) at 650 the queue holds two:
    Tmax_wait(3) = 600 + 400 - 70 = 930 <= 970, batch of 2 finishing at 1030."""
    lat = oracle_mod.replay_device_epochs([0, 600], [0, 1], [T0, T1], [5, 3], [1000, 400])
    assert lat.tolist() == [970, 420]
    lat = oracle_mod.replay_device_epochs([0, 600, 650], [0, 1, 1], [T0, T1], [5, 3], [1000, 400])
    assert lat.tolist() == [970, 430, 380]
    # one epoch: the plain §5 result -- query 1 joins at 600 (<= 870), the queue
    # of 2 then waits until Tmax_wait(3) = 1000 - 160 = 840: F = 840 + 130 = 970
    lat = oracle_mod.replay_device_epochs([0, 600], [0, 0], [T0], [5], [1000])
    assert lat.tolist() == oracle_mod.replay_device([0, 600], T0, 5, 1000).tolist() == [970, 370]


def test_single_epoch_equals_replay(oracle_mod):
    """E = 1: the closed-loop replay is the single-allocation replay."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3", totals=(12000,))
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
    a, f = W.query_trace(20000, 12000.0, cfg["weights"], 81, "gamma")
    sc = np.array([(m, c, 0, 0) for m in (1000, 3000) for c in (1, 8, 0)], np.int32)
    ref = oracle_mod.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, a, f, sc)
    out = oracle_mod.replay_epochs(prof, cl.device_type, r["option"][None], r["z"][None], cfg["demand"][:1],
                                   cl.slo_us, a, f, int(a[-1]) + 1, sc)
    for k in ("latency", "violations", "on_time", "acc_sum"):
        assert np.array_equal(out[k], ref[k]), k


def test_idle_gaps_split_into_independent_replays(oracle_mod):
    """Epoch arrivals confined to the first half of each epoch, with gaps
    longer than any finish: the device is idle at every epoch start, so each
    epoch replays independently from an idle device (R13) with its own
    variant."""
    rng = np.random.default_rng(3)
    rows = [T0, T1, [0, 80, 90, 100, 110]]
    Bm, Ls = [5, 3, 4], [1000, 400, 700]
    E, tau = 6, 100_000
    a, ep = [], []
    for e in range(E):
        k = int(rng.integers(1, 40))
        a += sorted((e * tau + rng.integers(0, tau // 2, size=k)).tolist())
        ep += [e] * k
    pe = [rng.integers(0, 3) for _ in range(E)]
    lat = oracle_mod.replay_device_epochs(a, ep, [rows[p] for p in pe], [Bm[p] for p in pe], [Ls[p] for p in pe])
    a, ep = np.array(a), np.array(ep)
    for e in range(E):
        sel = ep == e
        ref = oracle_mod.replay_device(a[sel], rows[pe[e]], Bm[pe[e]], Ls[pe[e]])
        assert np.array_equal(lat[sel], ref)


def test_closed_loop_invariants(oracle_mod):
    """Conservation per scenario; batches never mix epochs (queries sharing a
    finish time on a device belong to one epoch); routing restarts per epoch:
    per epoch and family, each device receives its SWRR share exactly when
    the epoch holds whole periods."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("f4", n_seconds=12, lam_mid=1500.0)
    prof, cl = cfg["prof"], cfg["cluster"]
    E = len(cfg["demand"])
    opts, zs = [], []
    for e in range(E):
        r = oracle_mod.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][e], 2)
        opts.append(r["option"])
        zs.append(r["z"])
    opts, zs = np.array(opts, np.int32), np.array(zs, np.int32)
    a, f = cfg["arrival_us"], cfg["family"]
    out = oracle_mod.replay_epochs(prof, cl.device_type, opts, zs, cfg["demand"], cl.slo_us, a, f,
                                   cfg["epoch_us"], cfg["scenarios"])
    N = len(a)
    assert np.all(out["violations"] + out["on_time"] == N)
    ep = a // cfg["epoch_us"]
    for s in range(len(cfg["scenarios"])):
        lat = out["latency"][s]
        served = lat != 0xFFFFFFFF
        fin = a.astype(np.int64) + lat
        # same finish time on the same device -> same epoch: check via (finish, epoch) uniqueness per finish
        for Fv in np.unique(fin[served])[:2000]:
            assert len(np.unique(ep[served & (fin == Fv)])) == 1
