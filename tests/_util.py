"""Test helpers: fixtures loading and small instance builders (no method arithmetic)."""

import json
import os

import numpy as np

from paper_conf_asplos_ahmadgfwsw24_b200.workloads import Profiles

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def golden(name="h1_g1.json"):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def profiles_from_capacity(P, acc, V, slo=4_000_000):
    """bmax = 1 latency table whose capacity floor(1e6 / lat) is exactly P
    (0 = does not fit).  Requires 2 * lat <= slo for every P > 0."""
    P = np.asarray(P, dtype=np.int64)
    T, M = P.shape
    lat = np.zeros((T, M, 1), np.int32)
    for t in range(T):
        for m in range(M):
            p = int(P[t, m])
            if p > 0:
                lat_v = 1_000_000 // p
                while 1_000_000 // lat_v != p:
                    lat_v -= 1
                assert 2 * lat_v <= slo
                lat[t, m, 0] = lat_v
    return Profiles(T=T, Q=len(V), V=np.asarray(V, np.int32), acc_micro=np.asarray(acc, np.int32),
                    bmax=1, lat_us=lat)


def random_instance(rng, T=2, Q=2, Vmax=3, D=4, Pmax=30, bmax=1, slo=4_000_000, zero_frac=0.2,
                    tie_acc=False):
    """Small random instance given through a capacity table."""
    V = rng.integers(1, Vmax + 1, size=Q)
    M = int(V.sum())
    acc = []
    for q in range(Q):
        if tie_acc:
            a = sorted(rng.choice([800_000, 900_000, 1_000_000], size=V[q]), reverse=True)
        else:
            a = sorted(rng.choice(np.arange(800_000, 1_000_001, 1000), size=V[q], replace=False), reverse=True)
        acc += [int(x) for x in a]
    P = rng.integers(1, Pmax + 1, size=(T, M))
    P[rng.random(size=(T, M)) < zero_frac] = 0
    prof = profiles_from_capacity(P, acc, V, slo)
    dev = np.sort(rng.integers(0, T, size=D)).astype(np.int32)
    return prof, dev, np.full(Q, slo, np.int32), P


def packed_score(served, accsum):
    """The CUDA path's packed score (served << 42 | accsum), for comparing."""
    return (int(served) << 42) | int(accsum)
