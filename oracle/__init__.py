"""CPU oracle for the Proteus hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(paper_conf_asplos_ahmadgfwsw24_b200) never imports it, and it shares no code
with the CUDA path: the arithmetic lives in ``oracle.c`` (plain C, exhaustive
enumeration, exact vertex-enumeration LP, event-driven simulator) and
``lp_exact.py`` (the literal Eqs. 2-6 LP in exact rationals).

Every function cites the passage of PAPER.md it follows; see oracle.c.
"""

from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_DIR = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_DIR, "oracle.c")
_LIB = os.path.join(_DIR, "liboracle.so")
_lib = None

i32p = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
i64p = np.ctypeslib.ndpointer(dtype=np.int64, flags="C_CONTIGUOUS")
u32p = np.ctypeslib.ndpointer(dtype=np.uint32, flags="C_CONTIGUOUS")
u64p = np.ctypeslib.ndpointer(dtype=np.uint64, flags="C_CONTIGUOUS")
u8p = np.ctypeslib.ndpointer(dtype=np.uint8, flags="C_CONTIGUOUS")


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (building the checker is not using it)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-pthread", "-shared", "-fPIC",
                               "-o", _LIB + ".tmp", _SRC])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


class Problem(C.Structure):
    _fields_ = [("T", C.c_int32), ("Q", C.c_int32), ("M", C.c_int32), ("D", C.c_int32),
                ("V", C.c_void_p), ("acc", C.c_void_p), ("P", C.c_void_p),
                ("dev_type", C.c_void_p), ("s", C.c_void_p)]


class Result(C.Structure):
    _fields_ = [("served", C.c_int64), ("accsum", C.c_int64), ("unmet", C.c_int64),
                ("index", C.c_uint64), ("n_candidates", C.c_uint64),
                ("eff", C.c_int32), ("pad", C.c_int32)]


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        L.orc_capacity.argtypes = [C.c_int, C.c_int, C.c_int, i32p, i32p, i32p, i32p, i32p]
        L.orc_family_lp.argtypes = [C.c_int, i64p, i64p, i32p, C.c_int64,
                                    C.POINTER(C.c_int64), C.POINTER(C.c_int64)]
        L.orc_score_placement.argtypes = [C.POINTER(Problem), i32p, C.POINTER(Result), i32p]
        L.orc_enum_count.argtypes = [C.POINTER(Problem), C.c_int, C.POINTER(C.c_uint64)]
        L.orc_solve_enum.argtypes = [C.POINTER(Problem), C.c_int, C.c_int, C.POINTER(Result), i32p, i32p]
        L.orc_solve_factored.argtypes = [C.POINTER(Problem), C.c_int, C.c_int, C.POINTER(Result),
                                         i32p, i32p, i32p]
        L.orc_route_swrr.argtypes = [C.c_int64, u8p, C.c_int, C.c_int, i32p, i32p, i32p, i32p]
        L.orc_replay_device.argtypes = [C.c_int64, u32p, i32p, C.c_int, C.c_int64, u32p]
        L.orc_replay_device_nexus.argtypes = [C.c_int64, u32p, i32p, C.c_int, C.c_int64, u32p]
        L.orc_replay_device_aimd.argtypes = [C.c_int64, u32p, i32p, C.c_int, C.c_int64, u32p]
        L.orc_replay.argtypes = [C.c_int64, u32p, u8p, C.c_int, C.c_int, i32p, i32p, C.c_int, i32p,
                                 C.c_int, i32p, i32p, i32p, i32p, i32p, C.c_int, i32p, C.c_int,
                                 C.c_void_p, u64p, u64p, u64p]
        L.orc_replay_epochs.argtypes = [C.c_int64, u32p, u8p, C.c_int, C.c_int64, C.c_int, C.c_int, i32p, i32p,
                                        C.c_int, i32p, C.c_int, i32p, i32p, i32p, i32p, i32p, C.c_int, i32p,
                                        C.c_void_p, u64p, u64p, u64p]
        L.orc_pareto.argtypes = [C.c_int, i32p, C.c_int, i32p, i32p, C.c_int, C.c_int, C.c_int, C.c_int64,
                                 i64p, i64p, u64p, C.POINTER(C.c_uint64), C.POINTER(C.c_int64)]
        _lib = L
    return _lib


def _i32(x):
    return np.ascontiguousarray(np.asarray(x, dtype=np.int32))


def family_of_variant(V) -> np.ndarray:
    return np.repeat(np.arange(len(V), dtype=np.int32), np.asarray(V))


def capacity(prof, slo_us):
    """a1: P[t][m], b*[t][m], depth[t][m]."""
    M = int(np.sum(prof.V))
    slo_m = _i32(np.asarray(slo_us)[family_of_variant(prof.V)])
    P = np.zeros((prof.T, M), np.int32)
    bs = np.zeros_like(P)
    dep = np.zeros_like(P)
    lib().orc_capacity(prof.T, M, prof.bmax, _i32(prof.lat_us), slo_m, P, bs, dep)
    return P, bs, dep


class _Prob:
    """Keeps the numpy buffers a Problem points at alive."""

    def __init__(self, prof, device_type, slo_us, demand, P=None):
        self.V = _i32(prof.V)
        self.acc = _i32(prof.acc_micro)
        self.P = _i32(capacity(prof, slo_us)[0] if P is None else P)
        self.dev = _i32(device_type)
        self.s = _i32(demand)
        self.st = Problem(prof.T, len(self.V), int(self.V.sum()), len(self.dev),
                          self.V.ctypes.data, self.acc.ctypes.data, self.P.ctypes.data,
                          self.dev.ctypes.data, self.s.ctypes.data)


def _res(r: Result, option=None, z=None, rc=0) -> dict:
    if rc != 0:
        raise RuntimeError(f"oracle returned {rc}")
    out = dict(served=r.served, accsum=r.accsum, unmet=r.unmet, index=r.index,
               n_candidates=r.n_candidates, eff=r.eff)
    if option is not None:
        out["option"] = option
    if z is not None:
        out["z"] = z
    return out


def family_lp(A, cap, mult, s):
    """Per-family LP value (served, accsum) by vertex enumeration."""
    sv, ac = C.c_int64(), C.c_int64()
    rc = lib().orc_family_lp(len(A), np.ascontiguousarray(A, dtype=np.int64),
                             np.ascontiguousarray(cap, dtype=np.int64), _i32(mult), int(s),
                             C.byref(sv), C.byref(ac))
    assert rc == 0
    return sv.value, ac.value


def score_placement(prof, device_type, slo_us, demand, option, P=None):
    pr = _Prob(prof, device_type, slo_us, demand, P)
    r = Result()
    z = np.zeros(len(pr.dev), np.int32)
    rc = lib().orc_score_placement(C.byref(pr.st), _i32(option), C.byref(r), z)
    return _res(r, _i32(option), z, rc)


def enum_count(prof, device_type, mode):
    pr = _Prob(prof, device_type, np.ones(prof.Q, np.int32), np.zeros(prof.Q, np.int32),
               P=np.zeros((prof.T, int(np.sum(prof.V))), np.int32))
    n = C.c_uint64()
    rc = lib().orc_enum_count(C.byref(pr.st), mode, C.byref(n))
    if rc != 0:
        raise OverflowError("candidate space exceeds 2^64")
    return n.value


def solve(prof, device_type, slo_us, demand, mode, threads=0, prune=1, P=None):
    """Exhaustive optimum for one demand vector.  mode 0 flat mixed radix,
    1 per-type multiset, 2 family-factored (reading C9 canonical forms)."""
    pr = _Prob(prof, device_type, slo_us, demand, P)
    r = Result()
    D = len(pr.dev)
    option = np.zeros(D, np.int32)
    z = np.zeros(D, np.int32)
    if mode in (0, 1):
        rc = lib().orc_solve_enum(C.byref(pr.st), mode, threads, C.byref(r), option, z)
        return _res(r, option, z, rc)
    counts = np.zeros((prof.Q, 8, 16), np.int32)
    rc = lib().orc_solve_factored(C.byref(pr.st), threads, prune, C.byref(r), option, z, counts)
    out = _res(r, option, z, rc)
    out["counts"] = counts[:, :prof.T, :]
    return out


def route_swrr(family, Q, dev_family, w_dev, w_sink):
    """R8: literal SWRR; returns target device per query (D = sink)."""
    family = np.ascontiguousarray(family, dtype=np.uint8)
    tgt = np.zeros(len(family), np.int32)
    D = len(dev_family)
    rc = lib().orc_route_swrr(len(family), family, Q, D, _i32(dev_family), _i32(w_dev), _i32(w_sink), tgt)
    assert rc == 0
    return tgt


def replay_device(arrival_us, Tproc, Bmax, L):
    """§5 on one device.  Tproc[b] for b = 1..Bmax (Tproc[0] unused)."""
    a = np.ascontiguousarray(arrival_us, dtype=np.uint32)
    lat = np.zeros(len(a), np.uint32)
    rc = lib().orc_replay_device(len(a), a, _i32(Tproc), int(Bmax), int(L), lat)
    assert rc == 0
    return lat


def replay_device_nexus(arrival_us, Tproc, B, L):
    """§8(f2) Nexus early-drop batching on one device (reading R14); B = the
    window / batch size.  Dropped queries get UINT32_MAX."""
    a = np.ascontiguousarray(arrival_us, dtype=np.uint32)
    lat = np.zeros(len(a), np.uint32)
    rc = lib().orc_replay_device_nexus(len(a), a, _i32(Tproc), int(B), int(L), lat)
    assert rc == 0
    return lat


def replay_device_aimd(arrival_us, Tproc, Bmax, L):
    """§8(f2) Clipper AIMD batching on one device (reading R15)."""
    a = np.ascontiguousarray(arrival_us, dtype=np.uint32)
    lat = np.zeros(len(a), np.uint32)
    rc = lib().orc_replay_device_aimd(len(a), a, _i32(Tproc), int(Bmax), int(L), lat)
    assert rc == 0
    return lat


def scenario_rows(scenarios):
    """[S][3] (policy 0) or [S][4] scenario rows -> int32[S][4]
    (slo_mult_milli, batch_cap, routing, policy)."""
    sc = np.asarray(scenarios, dtype=np.int32)
    sc = sc.reshape(-1, sc.shape[-1]) if sc.size else sc.reshape(0, 4)
    if sc.shape[1] == 3:
        sc = np.concatenate([sc, np.zeros((sc.shape[0], 1), np.int32)], axis=1)
    return np.ascontiguousarray(sc)


def replay(prof, device_type, option, z, demand, slo_base, arrival_us, family, scenarios,
           want_latency=True, threads=0):
    """a11-a13: route + simulate.  Returns dict(latency [S][N] or None,
    violations, on_time, acc_sum) per scenario."""
    a = np.ascontiguousarray(arrival_us, dtype=np.uint32)
    f = np.ascontiguousarray(family, dtype=np.uint8)
    sc = scenario_rows(scenarios)
    S, N = sc.shape[0], len(a)
    lat = np.zeros((S, N), np.uint32) if want_latency else None
    viol = np.zeros(S, np.uint64)
    ont = np.zeros(S, np.uint64)
    accs = np.zeros(S, np.uint64)
    rc = lib().orc_replay(N, a, f, prof.T, prof.Q, _i32(prof.V), _i32(prof.acc_micro), prof.bmax,
                          _i32(prof.lat_us), len(device_type), _i32(option), _i32(z), _i32(device_type),
                          _i32(demand), _i32(slo_base), S, sc, threads,
                          lat.ctypes.data if lat is not None else None, viol, ont, accs)
    if rc != 0:
        raise RuntimeError(f"orc_replay returned {rc}")
    return dict(latency=lat, violations=viol, on_time=ont, acc_sum=accs)


def replay_device_epochs(arrival_us, epoch, Tprocs, Bmaxs, Ls):
    """§8(f4) one device across allocation epochs (readings F3-F4): epoch[j]
    of query j, Tprocs[e] = T(b) row (index b), Bmaxs[e], Ls[e]."""
    a = np.ascontiguousarray(arrival_us, dtype=np.uint32)
    ep = _i32(epoch)
    E = len(Bmaxs)
    rows = [_i32(t) for t in Tprocs]
    ptrs = (C.POINTER(C.c_int32) * E)(*[r.ctypes.data_as(C.POINTER(C.c_int32)) for r in rows])
    lat = np.zeros(len(a), np.uint32)
    L = np.ascontiguousarray(np.asarray(Ls, dtype=np.int64))
    f = lib().orc_replay_device_epochs
    f.argtypes = [C.c_int64, u32p, i32p, C.POINTER(C.POINTER(C.c_int32)), i32p, i64p, u32p]
    rc = f(len(a), a, ep, ptrs, _i32(Bmaxs), L, lat)
    assert rc == 0
    return lat


def replay_epochs(prof, device_type, option, z, demand, slo_base, arrival_us, family, epoch_us, scenarios,
                  want_latency=True):
    """§8(f4) closed-loop replay: option/z [E][D] and demand [E][Q] per epoch
    (readings F1-F4).  Returns dict(latency, violations, on_time, acc_sum)."""
    a = np.ascontiguousarray(arrival_us, dtype=np.uint32)
    f = np.ascontiguousarray(family, dtype=np.uint8)
    sc = scenario_rows(scenarios)
    opt = _i32(option)
    E, D = opt.shape
    S, N = sc.shape[0], len(a)
    lat = np.zeros((S, N), np.uint32) if want_latency else None
    viol, ont, accs = np.zeros(S, np.uint64), np.zeros(S, np.uint64), np.zeros(S, np.uint64)
    rc = lib().orc_replay_epochs(N, a, f, E, int(epoch_us), prof.T, prof.Q, _i32(prof.V), _i32(prof.acc_micro),
                                 prof.bmax, _i32(prof.lat_us), D, opt, _i32(z), _i32(device_type), _i32(demand),
                                 _i32(slo_base), S, sc, lat.ctypes.data if lat is not None else None,
                                 viol, ont, accs)
    if rc != 0:
        raise RuntimeError(f"orc_replay_epochs returned {rc}")
    return dict(latency=lat, violations=viol, on_time=ont, acc_sum=accs)


def pareto(prof, device_type, slo_us, family, allow_idle=False, P=None, max_out=1 << 16):
    """Fig. 1b: every configuration of family `family`'s variants
    on the devices; returns dict(cap, accsum, index) of the Pareto frontier
    sorted by capacity, and n_configs (readings P1-P4)."""
    Pt = _i32(capacity(prof, slo_us)[0] if P is None else P)
    off = int(np.sum(np.asarray(prof.V)[:family]))
    cap = np.zeros(max_out, np.int64)
    acs = np.zeros(max_out, np.int64)
    idx = np.zeros(max_out, np.uint64)
    ncfg, nout = C.c_uint64(), C.c_int64()
    rc = lib().orc_pareto(len(device_type), _i32(device_type), Pt.shape[1], Pt, _i32(prof.acc_micro), off,
                          int(prof.V[family]), int(bool(allow_idle)), max_out, cap, acs, idx,
                          C.byref(ncfg), C.byref(nout))
    if rc != 0:
        raise OverflowError("configuration space too large for the oracle")
    k = min(nout.value, max_out)
    return dict(cap=cap[:k], accsum=acs[:k], index=idx[:k], n_configs=ncfg.value, n_front=nout.value)
