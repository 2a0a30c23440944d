"""Pins for the Fig. 1b oracle (oracle.pareto; readings P1-P4 in
DESIGN.md): a hand-worked two-device instance, the 3125-configuration shape of
the paper's example, and properties the definition of a Pareto frontier fixes
(extreme configurations on it, mutual non-dominance, scaling)."""

import itertools
from fractions import Fraction

import numpy as np
import pytest

from tests._util import profiles_from_capacity


def _hand():
    """One family, two variants, one device type: v0 A = 1.0 at P = 10 QPS,
    v1 A = 0.9 at P = 25 QPS."""
    P = np.array([[10, 25]], np.int32)
    prof = profiles_from_capacity(P, [1_000_000, 900_000], [2])
    return prof, np.zeros(2, np.int32), P


def test_hand_worked_no_idle():
    """Configurations (index = 2 o_0 + o_1): (v0, v0) cap 20, accuracy 1.0;
    (v0, v1) and (v1, v0) cap 35, accsum 10e6 + 22.5e6 = 32.5e6 (0.9286);
    (v1, v1) cap 50, accuracy 0.9.  Capacity rises as accuracy falls, so all
    three distinct points are on the frontier; the (v0, v1) point is reported
    with the lower index 1."""
    import oracle
    prof, dev, P = _hand()
    r = oracle.pareto(prof, dev, [4_000_000], 0, P=P)
    assert r["n_configs"] == 4
    assert r["cap"].tolist() == [20, 35, 50]
    assert r["accsum"].tolist() == [20_000_000, 32_500_000, 45_000_000]
    assert r["index"].tolist() == [0, 1, 3]


def test_hand_worked_with_idle():
    """With idle (digit 0): the single-device points (10, 1.0) and (25, 0.9)
    are dominated by (20, 1.0) and (35, 0.9286), the all-idle (0, 0) by
    everything; the frontier is the same three points at radix-3 indices
    (1,1) = 4, (1,2) = 5, (2,2) = 8."""
    import oracle
    prof, dev, P = _hand()
    r = oracle.pareto(prof, dev, [4_000_000], 0, allow_idle=True, P=P)
    assert r["n_configs"] == 9
    assert r["cap"].tolist() == [20, 35, 50]
    assert r["index"].tolist() == [4, 5, 8]


def test_equal_accuracy_keeps_larger_capacity():
    """Two variants of equal accuracy: (cap 10, 1.0) is dominated by
    (cap 20, 1.0) (capacity strictly larger, accuracy equal)."""
    import oracle
    P = np.array([[10, 20]], np.int32)
    prof = profiles_from_capacity(P, [1_000_000, 1_000_000], [2])
    r = oracle.pareto(prof, np.zeros(1, np.int32), [4_000_000], 0, P=P)
    assert r["cap"].tolist() == [20] and r["index"].tolist() == [1]


def test_fig1b_shape_and_properties():
    """5 variants of one family on 5 devices of 3 types: 5^5 = 3125
    configurations.  The frontier is sorted by capacity with
    strictly decreasing accuracy; it contains the maximum-capacity
    configuration and the maximum-accuracy one; no configuration lies strictly
    above it."""
    import oracle
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    prof, cl = cfg["prof"], cfg["cluster"]
    q = 3  # EfficientNet (Table 3 order), 5 variants
    assert prof.V[q] == 5
    dev = np.array([0, 1, 1, 2, 2], np.int32)
    r = oracle.pareto(prof, dev, cl.slo_us, q)
    assert r["n_configs"] == 3125 and r["n_front"] >= 2
    cap, acs = r["cap"].tolist(), r["accsum"].tolist()
    assert all(a < b for a, b in zip(cap, cap[1:]))
    accs = [Fraction(a, c) if c else Fraction(0) for a, c in zip(acs, cap)]
    assert all(a > b for a, b in zip(accs, accs[1:]))
    # every configuration from the capacity table (itertools, exact fractions)
    P, _, _ = oracle.capacity(prof, cl.slo_us)
    off = int(np.sum(prof.V[:q]))
    pts = []
    for i, cfg_ in enumerate(itertools.product(range(5), repeat=5)):
        c = sum(int(P[dev[d], off + o]) for d, o in enumerate(cfg_))
        a = sum(int(P[dev[d], off + o]) * int(prof.acc_micro[off + o]) for d, o in enumerate(cfg_))
        pts.append((c, Fraction(a, c) if c else Fraction(0), i))
    cmax = max(p[0] for p in pts)
    best_at_cmax = max(p[1] for p in pts if p[0] == cmax)
    assert (cap[-1], accs[-1]) == (cmax, best_at_cmax)
    amax = max(p[1] for p in pts)
    cap_at_amax = max(p[0] for p in pts if p[1] == amax)
    assert (cap[0], accs[0]) == (cap_at_amax, amax)
    for c, a, _ in pts:  # nothing dominates a frontier point
        for fc, fa in zip(cap, accs):
            assert not (c >= fc and a >= fa and (c > fc or a > fa))
    # the reported index is the first configuration at that point
    for fc, fa, fi in zip(cap, accs, r["index"].tolist()):
        assert fi == min(i for c, a, i in pts if c == fc and a == fa)


@pytest.mark.parametrize("allow_idle", [False, True])
def test_scaling_capacity_keeps_frontier(allow_idle):
    """Multiplying every capacity by 3 multiplies capacities and accuracy sums
    by 3 and leaves accuracies, hence the frontier's configurations, unchanged."""
    import oracle
    rng = np.random.default_rng(7)
    P = rng.integers(1, 40, size=(2, 4)).astype(np.int32)
    acc = [1_000_000, 950_000, 870_000, 820_000]
    prof = profiles_from_capacity(P, acc, [4])
    dev = np.array([0, 0, 1, 1, 1], np.int32)
    a = oracle.pareto(prof, dev, [4_000_000], 0, allow_idle=allow_idle, P=P)
    b = oracle.pareto(prof, dev, [4_000_000], 0, allow_idle=allow_idle, P=3 * P)
    assert (3 * a["cap"]).tolist() == b["cap"].tolist()
    assert (3 * a["accsum"]).tolist() == b["accsum"].tolist()
    assert a["index"].tolist() == b["index"].tolist()


def test_pareto_shard_decomposition():
    """The multi-GPU split of Fig. 1b (index slices) is exact: a
    point dominated inside a slice is dominated in the whole space, so the
    frontier (definition P3, exact fractions) of the union of the slices'
    frontiers, lowest index per point, equals the oracle's frontier of the
    whole space.  (The product's merge, proteus_pareto_merge, runs on the GPU:
    tests/test_gpu_pareto.py.)"""
    import oracle
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    prof, cl = cfg["prof"], cfg["cluster"]
    dev = np.array([0, 1, 1, 2], np.int32)
    q = 3
    whole = oracle.pareto(prof, dev, cl.slo_us, q)
    P, _, _ = oracle.capacity(prof, cl.slo_us)
    off = int(np.sum(prof.V[:q]))
    pts = []
    for i, c_ in enumerate(itertools.product(range(5), repeat=4)):
        c = sum(int(P[dev[d], off + o]) for d, o in enumerate(c_))
        a = sum(int(P[dev[d], off + o]) * int(prof.acc_micro[off + o]) for d, o in enumerate(c_))
        pts.append((c, a, i))

    def front(sub):  # definition of the frontier (exact fractions), lowest index per point
        keep = {}
        for c, a, i in sub:
            fa = Fraction(a, c) if c else Fraction(0)
            dom = any(c2 >= c and (Fraction(a2, c2) if c2 else Fraction(0)) >= fa and
                      (c2 > c or (Fraction(a2, c2) if c2 else Fraction(0)) > fa) for c2, a2, _ in sub)
            if not dom and ((c, a) not in keep or i < keep[(c, a)]):
                keep[(c, a)] = i
        return sorted((c, a, i) for (c, a), i in keep.items())
    parts = [front(pts[k * 625 // 3:(k + 1) * 625 // 3]) for k in range(3)]
    merged = front([p for part in parts for p in part])
    assert [m[0] for m in merged] == whole["cap"].tolist()
    assert [m[1] for m in merged] == whole["accsum"].tolist()
    assert [m[2] for m in merged] == whole["index"].tolist()
