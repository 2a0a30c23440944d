"""GPU parity of proteus_pareto (Fig. 1b, §8(f3)) against the oracle's brute
force: the frontier points (capacity, accuracy sum) and their canonical
(lowest) configuration index, bit-exact."""

import numpy as np
import pytest

from tests._util import profiles_from_capacity, random_instance

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def px():
    from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus
    return Proteus(0)


def check(px, oracle_mod, prof, dev, slo, q, idle, P=None):
    px.load_profiles(prof)
    g = px.pareto(dev, slo, q, allow_idle=idle)
    o = oracle_mod.pareto(prof, dev, slo, q, allow_idle=idle, P=P)
    assert g["n_configs"] == o["n_configs"]
    assert g["cap"].tolist() == o["cap"].tolist()
    assert g["accsum"].tolist() == o["accsum"].tolist()
    assert g["index"].tolist() == o["index"].tolist()
    return g


@pytest.mark.parametrize("idle", [False, True])
def test_hand_worked(px, oracle_mod, idle):
    P = np.array([[10, 25]], np.int32)
    prof = profiles_from_capacity(P, [1_000_000, 900_000], [2])
    g = check(px, oracle_mod, prof, np.zeros(2, np.int32), np.full(1, 4_000_000, np.int32), 0, idle, P)
    assert g["cap"].tolist() == [20, 35, 50]


@pytest.mark.parametrize("idle", [False, True])
def test_fig1b_efficientnet_5x5(px, oracle_mod, idle):
    """5 EfficientNet variants on 5 devices: 3125 configurations."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    g = check(px, oracle_mod, cfg["prof"], np.array([0, 1, 1, 2, 2], np.int32), cfg["cluster"].slo_us, 3, idle)
    assert g["n_configs"] == (6 if idle else 5) ** 5


def test_random_instances(px, oracle_mod):
    rng = np.random.default_rng(31)
    for _ in range(25):
        prof, dev, slo, P = random_instance(rng, T=int(rng.integers(1, 4)), Q=2, Vmax=4,
                                            D=int(rng.integers(1, 7)), Pmax=60, zero_frac=0.25,
                                            tie_acc=bool(rng.integers(0, 2)))
        for q in range(prof.Q):
            check(px, oracle_mod, prof, dev, slo, q, bool(rng.integers(0, 2)), P)


def test_large_10_devices_and_shards(px, oracle_mod):
    """EfficientNet on 10 devices of the c3 cluster types: 5^10 = 9 765 625
    configurations (several blocks per thread range, carries through every
    digit); three shards merged equal the whole space."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    dev = np.array([0, 0, 0, 0, 1, 1, 1, 2, 2, 2], np.int32)
    g = check(px, oracle_mod, cfg["prof"], dev, cfg["cluster"].slo_us, 3, False)
    parts = [px.pareto(dev, cfg["cluster"].slo_us, 3, shard_rank=r, shard_world=3) for r in range(3)]
    m = px.pareto_merge(parts)  # proteus_pareto_merge (device kernel)
    assert m["n_configs"] == g["n_configs"]
    for k in ("cap", "accsum", "index"):
        assert m[k].tolist() == g[k].tolist(), k


def test_bench_size_5_pow_12(px, oracle_mod):
    """The bench's f3 workload: EfficientNet's 5 variants on 12 devices (4 of
    each c3 type), 5^12 = 244 140 625 configurations, against the oracle's
    brute force (every configuration, pairwise dominance)."""
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c3")
    dev = np.repeat(np.arange(3, dtype=np.int32), 4)
    g = check(px, oracle_mod, cfg["prof"], dev, cfg["cluster"].slo_us, 3, False)
    assert g["n_configs"] == 5 ** 12


def test_pareto_merge_kernel_equal_points_and_ties(px):
    """proteus_pareto_merge on hand-made parts (reading P3): duplicates of one
    point keep the lowest index; a point dominated by another part's point
    drops; capacity 0 has accuracy 0; output sorted by capacity."""
    parts = [dict(cap=np.array([0, 10, 20], np.int64), accsum=np.array([0, 9_000_000, 16_000_000], np.int64),
                  index=np.array([0, 7, 9], np.uint64), n_configs=5),
             dict(cap=np.array([10, 20, 30], np.int64), accsum=np.array([9_000_000, 17_000_000, 21_000_000], np.int64),
                  index=np.array([3, 11, 12], np.uint64), n_configs=5)]
    m = px.pareto_merge(parts)
    # (10, 0.9) idx 3 (lowest of the two); (20, 0.85) beats (20, 0.8); (30, 0.7); (0, 0) is dominated
    assert m["cap"].tolist() == [10, 20, 30]
    assert m["accsum"].tolist() == [9_000_000, 17_000_000, 21_000_000]
    assert m["index"].tolist() == [3, 11, 12]
    assert m["n_configs"] == 10
