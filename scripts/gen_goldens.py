"""Write the oracle-computed expected values under tests/golden/ (test
infrastructure: calls only oracle/ and the seeded input generators of
workloads.py -- never the CUDA path).

    python scripts/gen_goldens.py [c2bench] [c4] [lp]      # default: all

* c2bench_oracle.npz -- the bench step's 64 c2 demand vectors (BASELINE
  configs[1], 13^8 candidates each), oracle A's exhaustive flat optimum per
  vector (Eqs. 1-7 with readings C1-C10; canonical index C9).
* c4_oracle.npz -- all 3600 per-second c4 demand vectors (P:192-203,
  P:1369-1370), oracle A's factored optimum per vector (modes 2, C9).  The
  f4 controller's demand (epoch e solves epoch e-1's counts) is a shifted copy
  of these vectors, so f4's allocations are rows of this file too.
* lp_literal.npz -- 10^4 seeded c2 placements and 10^4 seeded c3 placements
  (real bmax-64 capacity tables; uniform random options, perturbations of
  the optimum, single-family placements), each scored by Oracle B: the
  literal Eqs. 2-6 LP of lp_exact.py in exact rationals (two stages, reading
  C1), with its generic zero-fixing presolve (SURVEY §8(c) asks for 10^5
  candidates over c2/c3 in total; the CPU suite re-solves a sample of these).

Each file stores `inputs_sha` = SHA-256 of the input arrays it was computed
from; the tests recompute it from workloads.py and fail if the inputs drift.
"""

from __future__ import annotations

import hashlib
import multiprocessing as mp
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

GOLDEN = os.path.join(ROOT, "tests", "golden")
LP_N = 10_000


def inputs_sha(*arrays) -> str:
    h = hashlib.sha256()
    for a in arrays:
        a = np.ascontiguousarray(a)
        h.update(str(a.dtype).encode() + str(a.shape).encode())
        h.update(a.tobytes())
    return h.hexdigest()


def cfg_sha(cfg) -> str:
    p, cl = cfg["prof"], cfg["cluster"]
    return inputs_sha(p.V, p.acc_micro, p.lat_us, cl.device_type, cl.slo_us, cfg["demand"])


def c2bench():
    import oracle
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c2", totals=W.C2_BENCH_TOTALS)
    prof, cl = cfg["prof"], cfg["cluster"]
    rows = []
    t0 = time.time()
    for v, s in enumerate(cfg["demand"]):
        r = oracle.solve(prof, cl.device_type, cl.slo_us, s, 0, threads=os.cpu_count())
        rows.append(r)
        print(f"c2bench vector {v}: index {r['index']} served {r['served']} ({time.time() - t0:.0f} s)", flush=True)
    np.savez_compressed(
        os.path.join(GOLDEN, "c2bench_oracle.npz"), inputs_sha=cfg_sha(cfg),
        index=np.array([r["index"] for r in rows], np.uint64),
        served=np.array([r["served"] for r in rows], np.int64),
        accsum=np.array([r["accsum"] for r in rows], np.int64),
        unmet=np.array([r["unmet"] for r in rows], np.int64),
        option=np.stack([r["option"] for r in rows]).astype(np.int32),
        z=np.stack([r["z"] for r in rows]).astype(np.int32))


def _c4_one(v):
    import oracle
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = _c4_one.cfg
    if cfg is None:
        cfg = _c4_one.cfg = W.config("c4")
    prof, cl = cfg["prof"], cfg["cluster"]
    r = oracle.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][v], 2, threads=1)
    return r["served"], r["accsum"], r["unmet"], r["option"], r["z"]


_c4_one.cfg = None


def c4():
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    cfg = W.config("c4")
    E = len(cfg["demand"])
    t0 = time.time()
    with mp.Pool(os.cpu_count()) as pool:
        res = pool.map(_c4_one, range(E), chunksize=16)
    print(f"c4: {E} vectors in {time.time() - t0:.0f} s", flush=True)
    np.savez_compressed(
        os.path.join(GOLDEN, "c4_oracle.npz"), inputs_sha=cfg_sha(cfg),
        served=np.array([r[0] for r in res], np.int64), accsum=np.array([r[1] for r in res], np.int64),
        unmet=np.array([r[2] for r in res], np.int64), option=np.stack([r[3] for r in res]).astype(np.int32),
        z=np.stack([r[4] for r in res]).astype(np.int32))


def lp_candidates(name, n, seed):
    """Seeded placements of config `name` (c2 / c3) with the demand vector
    each is scored under: a third uniform random, a third the oracle's
    optimum for that vector with 1-3 devices re-drawn, a third with every
    non-idle device in one family (joint water-fills)."""
    import oracle
    from paper_conf_asplos_ahmadgfwsw24_b200 import workloads as W
    if name == "c2":
        cfg = W.config("c2", totals=W.C2_TOTALS + W.C2_BENCH_TOTALS[::8])
    else:
        c4 = W.config("c4")
        cfg = W.config("c3")
        cfg["demand"] = np.concatenate([cfg["demand"], c4["demand"][::400]])
    prof, cl = cfg["prof"], cfg["cluster"]
    D, K = len(cl.device_type), 1 + int(np.sum(prof.V))
    fam_of = np.repeat(np.arange(prof.Q), prof.V)
    opts = [oracle.solve(prof, cl.device_type, cl.slo_us, s, 0 if name == "c2" else 2)["option"]
            for s in cfg["demand"]]
    rng = np.random.default_rng(seed)
    vec = rng.integers(0, len(cfg["demand"]), size=n).astype(np.int32)
    out = np.zeros((n, D), np.int32)
    for i in range(n):
        kind = i % 3
        if kind == 0:
            out[i] = rng.integers(0, K, size=D)
        elif kind == 1:
            o = opts[vec[i]].copy()
            for d in rng.choice(D, size=rng.integers(1, 4), replace=False):
                o[d] = rng.integers(0, K)
            out[i] = o
        else:
            q = rng.integers(0, prof.Q)
            codes = 1 + np.flatnonzero(fam_of == q)
            out[i] = np.where(rng.random(D) < 0.2, 0, rng.choice(codes, size=D))
    return cfg, vec, out


def _lp_one(args):
    from oracle import capacity
    from oracle.lp_exact import literal_assignment_lp
    name, opt, s = args
    cfg = _lp_one.cfgs[name]
    prof, cl = cfg["prof"], cfg["cluster"]
    P = _lp_one.P.setdefault(name, capacity(prof, cl.slo_us)[0])
    served, acc, _ = literal_assignment_lp(P, prof.acc_micro, prof.V, cl.device_type, opt.tolist(), s.tolist(),
                                           presolve=True)
    assert served.denominator == 1 and acc.denominator == 1
    return int(served), int(acc)


_lp_one.cfgs = {}
_lp_one.P = {}


def lp():
    res = {}
    for name, seed in (("c2", 2020), ("c3", 3030)):
        cfg, vec, opt = lp_candidates(name, LP_N, seed)
        _lp_one.cfgs[name] = cfg
        t0 = time.time()
        with mp.Pool(os.cpu_count()) as pool:
            vals = pool.map(_lp_one, [(name, opt[i], cfg["demand"][vec[i]]) for i in range(LP_N)], chunksize=64)
        print(f"lp {name}: {LP_N} literal LPs in {time.time() - t0:.0f} s", flush=True)
        res[f"{name}_inputs_sha"] = cfg_sha(cfg)
        res[f"{name}_demand"] = cfg["demand"].astype(np.int32)
        res[f"{name}_vec"] = vec
        res[f"{name}_option"] = opt
        res[f"{name}_served"] = np.array([v[0] for v in vals], np.int64)
        res[f"{name}_accsum"] = np.array([v[1] for v in vals], np.int64)
    np.savez_compressed(os.path.join(GOLDEN, "lp_literal.npz"), **res)


if __name__ == "__main__":
    import oracle
    oracle.build()
    what = sys.argv[1:] or ["c2bench", "c4", "lp"]
    for w in what:
        {"c2bench": c2bench, "c4": c4, "lp": lp}[w]()
