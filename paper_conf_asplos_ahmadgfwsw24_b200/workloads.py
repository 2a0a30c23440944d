"""Seeded synthetic inputs shaped like the paper's workloads.

This module draws integer input arrays and nothing else.  It holds none of
the method's arithmetic: no capacity estimate, no assignment LP
(Eqs. 2-6), no batching rule (§5).  Both the CUDA path and the CPU oracle
consume exactly these arrays; neither is imported here.

Shapes follow the paper's evaluation setting (recipe restated in DESIGN.md §3):

* device types (Fig. 1a ordering P:284-286): a CPU-like type and
  two GPU types (1080 Ti-like, V100-like), each with a speed factor, a batching
  overhead fraction and a memory size;
* model families and variant counts from Table 3, capped at 5;
* accuracy normalised per family to its best variant, range 80-100 %
  (P:1137-1142), stored in 1e-6 units;
* latency SLO per family = 2x the CPU latency of its fastest variant at the
  smallest batch;
* demand split across families by Zipf alpha = 1.001,
  Poisson arrivals within each second, macro bursts as
  flat-low/high interleave, micro bursts as Gamma(0.05)
  inter-arrivals, SLO multipliers 1x-3.5x.
"""

from __future__ import annotations

import dataclasses
import math

import numpy as np

# name: (speed factor, batching overhead alpha, memory GB)
DEVICE_TYPES = {
    "cpu": (1.0, 0.05, 64.0),
    "gpu_a": (6.0, 0.60, 11.0),   # GTX 1080 Ti-like
    "gpu_b": (12.0, 0.70, 32.0),  # V100-like
}

# Table 3: family name, variant count (capped at 5), kind
FAMILIES = [
    ("resnet", 5, "cnn"),
    ("densenet", 4, "cnn"),
    ("resnest", 4, "cnn"),
    ("efficientnet", 5, "cnn"),
    ("mobilenet", 4, "cnn"),
    ("yolov5", 5, "cnn"),
    ("bert", 5, "transformer"),
    ("t5", 5, "transformer"),
    ("gpt2", 4, "gpt"),
]
FAMILY_INDEX = {f[0]: i for i, f in enumerate(FAMILIES)}

ZIPF_ALPHA = 1.001
GAMMA_SHAPE = 0.05
SLO_CPU_MULT = 2
UINT32_MAX = 0xFFFFFFFF


@dataclasses.dataclass
class Profiles:
    """Profile store: latency per (device type, variant, batch)."""
    T: int
    Q: int
    V: np.ndarray          # int32[Q]
    acc_micro: np.ndarray  # int32[sum V], family-major, caller's variant order
    bmax: int
    lat_us: np.ndarray     # int32[T][sum V][bmax]; [t][m][b-1]; 0 => batch b does not fit
    type_names: tuple = ()
    family_names: tuple = ()

    @property
    def M(self) -> int:
        return int(self.V.sum())


@dataclasses.dataclass
class Cluster:
    device_type: np.ndarray  # int32[D], devices sorted by type
    slo_us: np.ndarray       # int32[Q]


def _accuracies(rng, V):
    if V == 1:
        return [1_000_000]
    lo = int(rng.integers(800_000, 850_001))
    mids = sorted(set(int(x) for x in rng.integers(lo + 1, 1_000_000, size=4 * V)), reverse=True)
    pick = sorted(rng.choice(len(mids), size=V - 2, replace=False)) if V > 2 else []
    return [1_000_000] + [mids[i] for i in pick] + [lo]


def make_profiles(seed: int, type_names, family_names, n_variants=None, bmax: int = 64) -> Profiles:
    """Draw a latency table.  Variant v of a family costs base * r**(V-1-v) ms
    at CPU batch 1 (v = 0 is the most accurate and the slowest); batch b on
    type t takes ceil(1000 * cost / speed_t * (alpha_t + (1 - alpha_t) * b)) us
    while weights + b * activations fit in the type's memory."""
    rng = np.random.default_rng(seed)
    T = len(type_names)
    fams = [FAMILIES[FAMILY_INDEX[n]] for n in family_names]
    Vs = [min(f[1], n_variants) if n_variants else f[1] for f in fams]
    M = sum(Vs)
    lat = np.zeros((T, M, bmax), dtype=np.int64)
    acc = []
    m = 0
    for (name, _, kind), V in zip(fams, Vs):
        if kind == "cnn":
            base = math.exp(rng.uniform(math.log(2.0), math.log(40.0)))
            wbase, wgrow = rng.uniform(0.05, 0.4), 1.6
        elif kind == "transformer":
            base = math.exp(rng.uniform(math.log(10.0), math.log(80.0)))
            wbase, wgrow = rng.uniform(0.6, 1.5), 2.2
        else:  # gpt: heavyweight, fits only the largest-memory GPU
            base = math.exp(rng.uniform(math.log(10.0), math.log(80.0)))
            wbase, wgrow = rng.uniform(12.0, 13.0), 1.2
        r = rng.uniform(1.4, 2.0)
        acc += _accuracies(rng, V)
        for v in range(V):
            cost = base * r ** (V - 1 - v)
            w_gb = wbase * wgrow ** (V - 1 - v)
            a_gb = 0.01 * w_gb + 0.002
            for t, tn in enumerate(type_names):
                speed, alpha, mem = DEVICE_TYPES[tn]
                for b in range(1, bmax + 1):
                    if w_gb + b * a_gb > mem:
                        break
                    lat[t, m, b - 1] = math.ceil(1000.0 * cost / speed * (alpha + (1.0 - alpha) * b))
            m += 1
    assert lat.max() < 2**31
    return Profiles(T=T, Q=len(fams), V=np.array(Vs, dtype=np.int32),
                    acc_micro=np.array(acc, dtype=np.int32), bmax=bmax,
                    lat_us=lat.astype(np.int32), type_names=tuple(type_names),
                    family_names=tuple(family_names))


def slo_from_cpu_rule(prof: Profiles, cpu_type: int = 0, mult: int = SLO_CPU_MULT) -> np.ndarray:
    """SLO_q = 2 x latency of the family's fastest CPU-capable
    variant at the smallest batch.  (Workload setup, not the method.)"""
    out = np.zeros(prof.Q, dtype=np.int32)
    m0 = 0
    for q in range(prof.Q):
        lats = [int(prof.lat_us[cpu_type, m, 0]) for m in range(m0, m0 + int(prof.V[q]))]
        lats = [x for x in lats if x > 0]
        out[q] = mult * min(lats)
        m0 += int(prof.V[q])
    return out


def zipf_weights(Q: int, seed: int, alpha: float = ZIPF_ALPHA) -> np.ndarray:
    """Zipf popularity over families; ranks permuted by seed."""
    rng = np.random.default_rng(seed)
    ranks = rng.permutation(Q) + 1
    w = 1.0 / ranks.astype(np.float64) ** alpha
    return w / w.sum()


def split_demand(total_qps: int, weights: np.ndarray) -> np.ndarray:
    """Integer QPS per family, largest-remainder rounding so it sums to total."""
    raw = total_qps * weights
    base = np.floor(raw).astype(np.int64)
    rem = total_qps - int(base.sum())
    order = np.argsort(-(raw - base), kind="stable")
    base[order[:rem]] += 1
    return base.astype(np.int32)


def demand_trace(n_seconds: int, lam_mid: float, weights: np.ndarray, seed: int) -> np.ndarray:
    """Per-second demand vectors (config 4): diurnal sine x flat-low/high
    burst interleave, Poisson counts per family."""
    rng = np.random.default_rng(seed)
    t = np.arange(n_seconds, dtype=np.float64)
    burst = np.zeros(n_seconds)
    for a, b in ((600, 720), (1500, 1560), (2400, 2580), (3200, 3260)):
        burst[(t >= a * n_seconds / 3600) & (t < b * n_seconds / 3600)] = 1.0
    lam = lam_mid * (1.0 + 0.6 * np.sin(2 * np.pi * (t - 900.0) / 3600.0)) * (1.0 + 1.5 * burst)
    lam_q = lam[:, None] * weights[None, :]
    return rng.poisson(lam_q).astype(np.int32)


def query_trace(n: int, rate_qps: float, weights: np.ndarray, seed: int, kind: str = "poisson"):
    """Arrival timestamps (uint32 us, sorted) and family ids (uint8).

    kind: "poisson" (exponential inter-arrivals), "gamma" (shape 0.05, same
    mean), "uniform" (constant inter-arrival)."""
    rng = np.random.default_rng(seed)
    mean_us = 1e6 / rate_qps
    if kind == "poisson":
        gaps = rng.exponential(mean_us, size=n)
    elif kind == "gamma":
        gaps = rng.gamma(GAMMA_SHAPE, mean_us / GAMMA_SHAPE, size=n)
    elif kind == "uniform":
        gaps = np.full(n, mean_us)
    else:
        raise ValueError(kind)
    arr = np.floor(np.cumsum(gaps) - gaps[0]).astype(np.int64)
    if n and arr[-1] >= UINT32_MAX:
        raise ValueError("trace longer than 2^32 us")
    fam = rng.choice(len(weights), size=n, p=weights).astype(np.uint8)
    return arr.astype(np.uint32), fam


def epoch_trace(counts: np.ndarray, epoch_us: int, seed: int):
    """Arrivals for per-epoch family counts [E][Q] (§8(f4)): counts[e][q]
    queries of family q uniformly at random in epoch e (a Poisson process
    conditioned on its count: "Poisson inter-arrivals within each second",
    P:1155-1157), merged and sorted.  Returns (uint32 us, uint8 family)."""
    rng = np.random.default_rng(seed)
    E, Q = counts.shape
    if E * epoch_us >= UINT32_MAX:
        raise ValueError("trace longer than 2^32 us")
    tot = counts.sum(axis=1)
    ep = np.repeat(np.arange(E, dtype=np.int64), tot)
    fam = np.concatenate([np.repeat(np.arange(Q, dtype=np.uint8), counts[e]) for e in range(E)]) if E else \
        np.zeros(0, np.uint8)
    t = ep * epoch_us + rng.integers(0, epoch_us, size=len(ep))
    order = np.lexsort((rng.random(len(ep)), t))
    return t[order].astype(np.uint32), fam[order].astype(np.uint8)


def controller_demand(counts: np.ndarray) -> np.ndarray:
    """The controller's estimate for epoch e: the counts observed in epoch
    e - 1 (epoch 0: its own), per-second re-solve on the last second's
    statistics."""
    return np.concatenate([counts[:1], counts[:-1]]).astype(np.int32)


# -------------------------------------------------------------- scenarios --
SLO_MULTS_MILLI = (1000, 1500, 2000, 2500, 3000, 3500, 4000, 5000)   # covers P:1817-1818
BATCH_CAPS = (1, 2, 4, 8, 16, 32, 64, 0)                               # 1 = "w/o AB"; 0 = table depth


def scenarios_64(routing: int = 0, policy: int | None = None) -> np.ndarray:
    """64 (SLO multiplier, batch cap) scenarios as an int32[S][3] array of
    (slo_mult_milli, batch_cap, routing), or int32[S][4] with a policy column
    (0 §5 batching, 1 Nexus early drop, 2 Clipper AIMD; §6.4)."""
    if policy is None:
        rows = [(m, c, routing) for m in SLO_MULTS_MILLI for c in BATCH_CAPS]
    else:
        rows = [(m, c, routing, policy) for m in SLO_MULTS_MILLI for c in BATCH_CAPS]
    return np.array(rows, dtype=np.int32)


def scenarios_fig6(routing: int = 0) -> np.ndarray:
    """Fig. 6 / §6.4 comparison grid: the three batching
    policies x SLO multipliers x batch caps {8, 32, depth}: int32[72][4]."""
    rows = [(m, c, routing, p) for p in (0, 1, 2) for m in SLO_MULTS_MILLI for c in (8, 32, 0)]
    return np.array(rows, dtype=np.int32)


# ---------------------------------------------------------------- configs --
C1_FAMILIES = ("resnet", "bert")
C2_FAMILIES = ("resnet", "efficientnet", "yolov5", "bert")
C3_FAMILIES = tuple(f[0] for f in FAMILIES)
C3MINI_FAMILIES = ("resnet", "yolov5", "bert")


def cluster_types(counts) -> np.ndarray:
    return np.concatenate([np.full(n, t, dtype=np.int32) for t, n in enumerate(counts)])


def config(name: str, **kw) -> dict:
    """Concrete inputs for BASELINE.json's configs.

    Demand totals are absolute constants (calibrated once against the oracle's
    capacity table and recorded in DESIGN.md), so this module never computes
    the method's capacity estimate."""
    if name == "c1":
        prof = make_profiles(101, ("cpu", "gpu_b"), C1_FAMILIES, n_variants=3, bmax=16)
        cl = Cluster(cluster_types((2, 2)), slo_from_cpu_rule(prof))
        w = zipf_weights(prof.Q, 101)
        dem = np.stack([split_demand(kw.get("total", C1_TOTAL), w)])
    elif name == "c2":
        prof = make_profiles(202, ("cpu", "gpu_a", "gpu_b"), C2_FAMILIES, n_variants=3, bmax=64)
        cl = Cluster(cluster_types((2, 3, 3)), slo_from_cpu_rule(prof))
        w = zipf_weights(prof.Q, 202)
        dem = np.stack([split_demand(t, w) for t in kw.get("totals", C2_TOTALS)])
    elif name in ("c3", "c3mini"):
        fams = C3_FAMILIES if name == "c3" else C3MINI_FAMILIES
        prof = make_profiles(303, ("cpu", "gpu_a", "gpu_b"), fams,
                             n_variants=None if name == "c3" else 3, bmax=64)
        cl = Cluster(cluster_types(kw.get("counts", (10, 5, 5) if name == "c3" else C3MINI_COUNTS)),
                     slo_from_cpu_rule(prof))
        w = zipf_weights(prof.Q, 303)
        totals = kw.get("totals", C3_TOTALS if name == "c3" else C3MINI_TOTALS)
        dem = np.stack([split_demand(t, w) for t in totals])
    elif name == "c4":
        prof = make_profiles(303, ("cpu", "gpu_a", "gpu_b"), C3_FAMILIES, bmax=64)
        cl = Cluster(cluster_types((10, 5, 5)), slo_from_cpu_rule(prof))
        w = zipf_weights(prof.Q, 303)
        dem = demand_trace(kw.get("n_seconds", 3600), kw.get("lam_mid", C4_LAM_MID), w, 404)
    elif name == "c5":
        prof = make_profiles(303, ("cpu", "gpu_a", "gpu_b"), C3_FAMILIES, bmax=64)
        cl = Cluster(cluster_types((10, 5, 5)), slo_from_cpu_rule(prof))
        w = zipf_weights(prof.Q, 303)
        rate = kw.get("rate", C5_RATE)
        dem = np.stack([split_demand(rate, w)])
        n = kw.get("n", 10_000_000)
        arr, fam = query_trace(n, rate, w, 505, kw.get("kind", "poisson"))
        return dict(name=name, prof=prof, cluster=cl, demand=dem, arrival_us=arr, family=fam,
                    scenarios=scenarios_64(kw.get("routing", 0)), weights=w)
    elif name == "f4":
        # §8(f4) closed loop on the c4 demand: every epoch's true counts make
        # the trace; the controller solves epoch e on epoch e - 1's counts
        prof = make_profiles(303, ("cpu", "gpu_a", "gpu_b"), C3_FAMILIES, bmax=64)
        cl = Cluster(cluster_types((10, 5, 5)), slo_from_cpu_rule(prof))
        w = zipf_weights(prof.Q, 303)
        E = kw.get("n_seconds", 3600)
        counts = demand_trace(E, kw.get("lam_mid", C4_LAM_MID), w, 404)
        epoch_us = kw.get("epoch_us", 1_000_000)
        arr, fam = epoch_trace(counts, epoch_us, 606)
        return dict(name=name, prof=prof, cluster=cl, counts=counts, demand=controller_demand(counts),
                    arrival_us=arr, family=fam, epoch_us=epoch_us, weights=w,
                    scenarios=np.array([(m, c, 0, 0) for m in (1000, 2000, 3000, 5000) for c in (8, 32, 0)],
                                       np.int32))
    else:
        raise ValueError(name)
    return dict(name=name, prof=prof, cluster=cl, demand=dem, weights=w)


# Calibrated absolute demand totals (QPS); see DESIGN.md §3 for how they were chosen.
C1_TOTAL = 600
C2_TOTALS = (3000, 7000)
# the bench step's batch (bench.py): 64 demand vectors, totals 1500..7500 QPS
# (from the all-most-accurate regime to overload)
C2_BENCH_NVEC = 64
C2_BENCH_TOTALS = tuple(int(t) for t in np.linspace(1500, 7500, C2_BENCH_NVEC))
C3_TOTALS = (3000, 12000)
C3MINI_TOTALS = (8000, 30000)
C3MINI_COUNTS = (6, 3, 3)   # 12 devices: multiset space 5005 * 220^2 = 2.42e8
C4_LAM_MID = 2500.0
C5_RATE = 3000
