"""Proteus (ASPLOS '24) allocation search and adaptive-batching replay on B200.

Thin Python binding of libproteus.so (include/proteus.h): argument marshalling
only.  Arrays may be numpy arrays (host memory) or CUDA torch tensors (device
memory, passed by pointer); the library detects which.

    px = Proteus()                       # context on cuda:0, torch's current stream
    px.load_profiles(prof)               # workloads.Profiles or equivalent arrays
    sol = px.solve(device_type, slo_us, demand, mode=0)[0]
    out = px.replay(arrival_us, family, sol.option, sol.z, device_type, demand, slo_us, scenarios)
"""

from __future__ import annotations

import ctypes as C
import dataclasses

import numpy as np

from . import _native as N
from ._native import ProteusError  # noqa: F401

__all__ = ["Proteus", "Solution", "ProteusError", "MODE_FLAT", "MODE_MULTISET", "MODE_FACTORED", "scenario_owner"]

MODE_FLAT, MODE_MULTISET, MODE_FACTORED = 0, 1, 2
UINT64_MAX = (1 << 64) - 1


@dataclasses.dataclass
class Solution:
    score: int
    index: int
    served: int
    unmet: int
    accsum: int
    eff_acc_micro: int
    n_candidates: int
    option: np.ndarray
    z: np.ndarray


def _pinned_u32(shape, keep):
    """Host output in page-locked memory (the D2H copy of the latencies runs at
    full PCIe / C2C bandwidth instead of staging through pageable memory)."""
    import torch
    t = torch.empty(shape, dtype=torch.int32, pin_memory=True)
    keep.append(t)
    return t.numpy().view(np.uint32)


def _scenario_rows(scenarios):
    """int32 rows (slo_mult_milli, batch_cap, routing[, policy]) -> [S][4]
    (a missing policy column means 0, §5 batching)."""
    sc = np.asarray(scenarios, dtype=np.int32)
    sc = sc.reshape(-1, sc.shape[-1])
    if sc.shape[1] == 3:
        sc = np.concatenate([sc, np.zeros((sc.shape[0], 1), np.int32)], axis=1)
    if sc.shape[1] != 4:
        raise ValueError("scenario rows have 3 or 4 columns")
    return sc


def scenario_owner(scenarios, world: int) -> np.ndarray:
    """Rank that replays each scenario in a distributed replay
    (proteus_scenario_owner; host only, no GPU needed)."""
    sc = _scenario_rows(scenarios)
    S = sc.shape[0]
    scs = (N.proteus_scenario * max(S, 1))(*[N.proteus_scenario(*map(int, row)) for row in sc])
    owner = np.zeros(max(S, 1), np.int32)
    rc = N.load().proteus_scenario_owner(scs, S, int(world), owner.ctypes.data)
    if rc != 0:
        raise ProteusError(rc, "proteus_scenario_owner")
    return owner[:S]


def _is_torch(x):
    return type(x).__module__.startswith("torch")


def _arg(x, np_dtype, keep):
    """Pointer to x's data: a torch tensor's data_ptr (host or device) or a
    contiguous numpy copy's buffer.  `keep` holds references for the call."""
    if x is None:
        return None
    if _is_torch(x):
        import torch
        want = {np.int32: torch.int32, np.uint32: torch.uint32, np.uint8: torch.uint8,
                np.uint64: torch.uint64, np.int64: torch.int64}[np_dtype]
        if x.dtype != want or not x.is_contiguous():
            raise TypeError(f"tensor must be contiguous {want}, got {x.dtype}")
        keep.append(x)
        return x.data_ptr()
    a = np.ascontiguousarray(x, dtype=np_dtype)
    keep.append(a)
    return a.ctypes.data


class Proteus:
    """One library context: one GPU, one CUDA stream (proteus.h)."""

    def __init__(self, device: int = 0, stream=None):
        self._lib = N.load()
        if stream is None:
            try:
                import torch
                if torch.cuda.is_available():
                    stream = torch.cuda.current_stream(device).cuda_stream
            except ImportError:
                stream = None
        h = C.c_void_p()
        rc = self._lib.proteus_create(C.byref(h), device, C.c_void_p(stream) if stream else None)
        if rc != 0:
            raise ProteusError(rc, f"proteus_create(device={device}) failed (no CUDA device?)")
        self._h = h
        self.device = device
        self.Q = None

    def close(self):
        if getattr(self, "_h", None):
            self._lib.proteus_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, rc):
        if rc != 0:
            msg = self._lib.proteus_last_error(self._h)
            raise ProteusError(rc, msg.decode() if msg else "")

    def set_stream(self, stream):
        self._check(self._lib.proteus_set_stream(self._h, C.c_void_p(stream) if stream else None))

    # ------------------------------------------------------------ profiles --
    def load_profiles(self, prof=None, *, T=None, Q=None, V=None, acc_micro=None, bmax=None, lat_us=None):
        if prof is not None:
            T, Q, V, acc_micro, bmax, lat_us = prof.T, prof.Q, prof.V, prof.acc_micro, prof.bmax, prof.lat_us
        keep = []
        p = N.proteus_profiles(int(T), int(Q), _arg(V, np.int32, keep), _arg(acc_micro, np.int32, keep), int(bmax),
                               _arg(lat_us, np.int32, keep))
        self._check(self._lib.proteus_load_profiles(self._h, C.byref(p)))
        self.Q = int(Q)

    # --------------------------------------------------------------- solve --
    def _solve_args(self, device_type, slo_us, demand, mode, shard_rank, shard_world, max_candidates, generic, keep):
        dem = demand
        if not _is_torch(dem):
            dem = np.atleast_2d(np.asarray(demand, dtype=np.int32))
            n_vec = dem.shape[0]
        else:
            n_vec = dem.shape[0] if dem.dim() == 2 else 1
        D = len(device_type)
        a = N.proteus_solve_args(D, _arg(device_type, np.int32, keep), int(mode), _arg(slo_us, np.int32, keep),
                                 int(n_vec), _arg(dem, np.int32, keep), int(max_candidates), int(shard_rank),
                                 int(shard_world), N.PROTEUS_SOLVE_GENERIC if generic else 0)
        return a, n_vec, D

    def solve(self, device_type, slo_us, demand, mode=MODE_FLAT, shard_rank=0, shard_world=1,
              max_candidates=0, generic=False):
        """Optimal allocation per demand vector (proteus_solve)."""
        keep = []
        a, n_vec, D = self._solve_args(device_type, slo_us, demand, mode, shard_rank, shard_world, max_candidates,
                                       generic, keep)
        opts = np.zeros((n_vec, D), np.int32)
        zs = np.zeros((n_vec, D), np.int32)
        sols = (N.proteus_solution * n_vec)()
        for i in range(n_vec):
            sols[i].option = opts[i].ctypes.data
            sols[i].z_qps = zs[i].ctypes.data
        self._check(self._lib.proteus_solve(self._h, C.byref(a), sols))
        return [self._sol(sols[i], opts[i], zs[i]) for i in range(n_vec)]

    def solve_batch(self, device_type, slo_us, demand, mode=MODE_FACTORED, out=None, fields=None, shard_rank=0,
                    shard_world=1):
        """Many demand vectors at once (proteus_solve_batch).  out: dict of
        preallocated arrays (numpy or CUDA torch) keyed by field name, written
        in place; else host numpy arrays are returned for `fields` (default
        all).  Modes 0/1 may scan one slice of shard_world (as solve()).
        Returns (dict of arrays, n_candidates per vector)."""
        keep = []
        a, n_vec, D = self._solve_args(device_type, slo_us, demand, mode, shard_rank, shard_world, 0, False, keep)
        shapes = {"score": ((n_vec,), np.uint64), "index": ((n_vec,), np.uint64), "served": ((n_vec,), np.int64),
                  "unmet": ((n_vec,), np.int64), "accsum": ((n_vec,), np.int64),
                  "eff_acc_micro": ((n_vec,), np.int32), "option": ((n_vec, D), np.int32),
                  "z_qps": ((n_vec, D), np.int32)}
        if out is None:
            out = {k: np.empty(*shapes[k]) for k in (fields or shapes)}
        b = N.proteus_batch()
        for k, x in out.items():
            setattr(b, k, _arg(x, shapes[k][1], keep))
        self._check(self._lib.proteus_solve_batch(self._h, C.byref(a), C.byref(b)))
        return out, int(b.n_candidates)

    def materialize(self, device_type, slo_us, demand, index, vec=0, mode=MODE_FLAT):
        keep = []
        a, n_vec, D = self._solve_args(device_type, slo_us, demand, mode, 0, 1, 0, False, keep)
        opt = np.zeros(D, np.int32)
        z = np.zeros(D, np.int32)
        s = N.proteus_solution()
        s.option = opt.ctypes.data
        s.z_qps = z.ctypes.data
        self._check(self._lib.proteus_materialize(self._h, C.byref(a), int(vec), int(index), C.byref(s)))
        return self._sol(s, opt, z)

    def candidate_count(self, device_type, mode=MODE_FLAT):
        keep = []
        a, _, _ = self._solve_args(device_type, np.zeros(self.Q, np.int32), np.zeros(self.Q, np.int32), mode, 0, 1,
                                   0, False, keep)
        n = C.c_uint64()
        self._check(self._lib.proteus_candidate_count(self._h, C.byref(a), C.byref(n)))
        return n.value

    @staticmethod
    def _sol(s, opt, z):
        return Solution(s.score, s.index, s.served, s.unmet, s.accsum, s.eff_acc_micro, s.n_candidates,
                        opt.copy(), z.copy())

    # -------------------------------------------------------------- pareto --
    def pareto(self, device_type, slo_us, family, allow_idle=False, shard_rank=0, shard_world=1, max_points=65536):
        """Fig. 1b Pareto frontier (proteus_pareto): dict of numpy arrays
        cap, accsum, index sorted by capacity, plus n_configs."""
        keep = []
        a = N.proteus_pareto_args(len(device_type), _arg(device_type, np.int32, keep), _arg(slo_us, np.int32, keep),
                                  int(family), int(bool(allow_idle)), int(shard_rank), int(shard_world))
        pts = (N.proteus_pareto_point * max(1, max_points))()
        npts, ncfg = C.c_int32(), C.c_uint64()
        self._check(self._lib.proteus_pareto(self._h, C.byref(a), pts, int(max_points), C.byref(npts), C.byref(ncfg)))
        k = min(npts.value, max_points)
        cap = np.array([pts[i].capacity for i in range(k)], np.int64)
        acs = np.array([pts[i].accsum for i in range(k)], np.int64)
        idx = np.array([pts[i].index for i in range(k)], np.uint64)
        return dict(cap=cap, accsum=acs, index=idx, n_configs=ncfg.value, n_front=npts.value)

    # -------------------------------------------------------------- replay --
    def replay(self, arrival_us, family, option, z, device_type, demand, slo_base_us, scenarios,
               latency=True, aggregates_out=None):
        """Adaptive-batching replay (proteus_replay).  latency: True -> host
        numpy [S][N]; a CUDA uint32 tensor [S][N] -> written in place; None ->
        not produced.  scenarios: int32 rows (slo_mult_milli, batch_cap,
        routing[, policy]); a missing policy column means 0 (§5 batching)."""
        keep = []
        sc = _scenario_rows(scenarios)
        S = sc.shape[0]
        scs = (N.proteus_scenario * S)(*[N.proteus_scenario(*map(int, row)) for row in sc])
        n = int(arrival_us.shape[0]) if hasattr(arrival_us, "shape") else len(arrival_us)
        lat_np = None
        if latency is True:
            lat_np = _pinned_u32((self.latency_rows(sc), n), keep)
            lat_ptr = lat_np.ctypes.data
        elif latency is None or latency is False:
            lat_ptr = None
        else:
            lat_ptr = _arg(latency, np.uint32, keep)
        if aggregates_out is not None:  # torch uint64 [3][S] on device
            viol = _arg(aggregates_out[0], np.uint64, keep)
            ont = _arg(aggregates_out[1], np.uint64, keep)
            accs = _arg(aggregates_out[2], np.uint64, keep)
            out = None
        else:
            out = np.zeros((3, S), np.uint64)
            viol, ont, accs = out[0].ctypes.data, out[1].ctypes.data, out[2].ctypes.data
        D = len(device_type)
        rc = self._lib.proteus_replay(
            self._h, _arg(arrival_us, np.uint32, keep), _arg(family, np.uint8, keep), n,
            _arg(option, np.int32, keep), _arg(z, np.int32, keep), _arg(device_type, np.int32, keep), D,
            _arg(demand, np.int32, keep), _arg(slo_base_us, np.int32, keep), scs, S, lat_ptr, viol, ont, accs)
        self._check(rc)
        res = {"latency": lat_np if latency is True else latency}
        if out is not None:
            res.update(violations=out[0], on_time=out[1], acc_sum=out[2])
        return res

    # --------------------------------------------------------- closed loop --
    def replay_epochs(self, arrival_us, family, epoch_us, option, z, device_type, demand, slo_base_us, scenarios,
                      latency=True, aggregates_out=None):
        """§8(f4) closed-loop replay (proteus_replay_epochs): option / z
        [E][D] and demand [E][Q], one allocation per epoch of epoch_us
        (numpy or CUDA tensors).  latency / aggregates_out as replay()."""
        keep = []
        sc = _scenario_rows(scenarios)
        S = sc.shape[0]
        scs = (N.proteus_scenario * S)(*[N.proteus_scenario(*map(int, row)) for row in sc])
        n = int(arrival_us.shape[0]) if hasattr(arrival_us, "shape") else len(arrival_us)
        E, D = int(option.shape[0]), int(option.shape[1])
        lat_np = None
        if latency is True:
            lat_np = _pinned_u32((self.latency_rows(sc), n), keep)
            lat_ptr = lat_np.ctypes.data
        elif latency is None or latency is False:
            lat_ptr = None
        else:
            lat_ptr = _arg(latency, np.uint32, keep)
        if aggregates_out is not None:
            viol, ont, accs = (_arg(aggregates_out[k], np.uint64, keep) for k in range(3))
            out = None
        else:
            out = np.zeros((3, S), np.uint64)
            viol, ont, accs = out[0].ctypes.data, out[1].ctypes.data, out[2].ctypes.data
        rc = self._lib.proteus_replay_epochs(
            self._h, _arg(arrival_us, np.uint32, keep), _arg(family, np.uint8, keep), n, E, int(epoch_us),
            _arg(option, np.int32, keep), _arg(z, np.int32, keep), _arg(device_type, np.int32, keep), D,
            _arg(demand, np.int32, keep), _arg(slo_base_us, np.int32, keep), scs, S, lat_ptr, viol, ont, accs)
        self._check(rc)
        res = {"latency": lat_np if latency is True else latency}
        if out is not None:
            res.update(violations=out[0], on_time=out[1], acc_sum=out[2])
        return res

    def closed_loop(self, arrival_us, family, epoch_us, demand, device_type, slo_us, scenarios, latency=True,
                    device=None):
        """§8(f4): per-epoch re-solve (factored, batched) of the controller's
        demand estimates [E][Q] feeding the closed-loop replay; with CUDA
        tensors (or `device`) the allocations stay on the GPU between the two
        calls.  Returns (replay result dict, allocation dict)."""
        E = int(demand.shape[0])
        D = len(device_type)
        if device is not None:
            import torch
            alloc = {"option": torch.empty((E, D), dtype=torch.int32, device=device),
                     "z_qps": torch.empty((E, D), dtype=torch.int32, device=device)}
        else:
            alloc = {"option": np.empty((E, D), np.int32), "z_qps": np.empty((E, D), np.int32)}
        self.solve_batch(device_type, slo_us, demand, mode=MODE_FACTORED, out=alloc)
        res = self.replay_epochs(arrival_us, family, epoch_us, alloc["option"], alloc["z_qps"], device_type, demand,
                                 slo_us, scenarios, latency=latency)
        return res, alloc

    # ----------------------------------------------------------- multi-GPU --
    @staticmethod
    def comm_unique_id() -> bytes:
        """128-byte NCCL unique id (rank 0; broadcast it to the other ranks)."""
        buf = C.create_string_buffer(N.COMM_ID_BYTES)
        rc = N.load().proteus_comm_unique_id(buf)
        if rc != 0:
            raise ProteusError(rc, "proteus_comm_unique_id (NCCL unavailable?)")
        return buf.raw

    def comm_init(self, unique_id: bytes, world: int, rank: int):
        """Join the context's NCCL communicator (collective over the ranks);
        later calls are distributed (proteus.h, multi-GPU)."""
        buf = C.create_string_buffer(bytes(unique_id), N.COMM_ID_BYTES)
        self._check(self._lib.proteus_comm_init(self._h, buf, int(world), int(rank)))

    def comm_enable(self, on: bool = True):
        self._check(self._lib.proteus_comm_enable(self._h, 1 if on else 0))

    def comm_info(self):
        """(world, rank, distributed calls enabled)."""
        w, r = C.c_int32(), C.c_int32()
        on = self._lib.proteus_comm_info(self._h, C.byref(w), C.byref(r))
        return w.value, r.value, bool(on == 1)

    def latency_rows(self, scenarios) -> int:
        """Rows of a replay's latency output: S, or in a distributed replay
        the number of scenarios this rank owns (in ascending order)."""
        sc = _scenario_rows(scenarios)
        world, rank, on = self.comm_info()
        if not on or world == 1:
            return sc.shape[0]
        return int(np.sum(scenario_owner(sc, world) == rank))

    def combine_solutions(self, parts, part_candidates, D):
        """proteus_combine_solutions: per-slice solve_batch outputs (dicts of
        arrays with every field) -> the batch's optima, combined on the GPU."""
        keep = []
        world = len(parts)
        n_vec = len(parts[0]["score"])
        types = {"score": np.uint64, "index": np.uint64, "served": np.int64, "unmet": np.int64,
                 "accsum": np.int64, "eff_acc_micro": np.int32, "option": np.int32, "z_qps": np.int32}
        arr = (N.proteus_batch * world)()
        for r, p in enumerate(parts):
            for k, t in types.items():
                setattr(arr[r], k, _arg(p[k], t, keep))
        out = {"score": np.empty(n_vec, np.uint64), "index": np.empty(n_vec, np.uint64),
               "served": np.empty(n_vec, np.int64), "unmet": np.empty(n_vec, np.int64),
               "accsum": np.empty(n_vec, np.int64), "eff_acc_micro": np.empty(n_vec, np.int32),
               "option": np.empty((n_vec, D), np.int32), "z_qps": np.empty((n_vec, D), np.int32)}
        b = N.proteus_batch()
        for k, x in out.items():
            setattr(b, k, _arg(x, types[k], keep))
        pc = _arg(np.asarray(part_candidates, np.uint64), np.uint64, keep)
        self._check(self._lib.proteus_combine_solutions(self._h, world, n_vec, int(D), arr, pc, C.byref(b)))
        return out, int(b.n_candidates)

    def pareto_merge(self, parts, max_points=65536):
        """proteus_pareto_merge: frontier of the union of shard frontiers
        (dicts from pareto(..., shard_rank, shard_world))."""
        cap = np.concatenate([np.asarray(p["cap"], np.int64) for p in parts])
        acs = np.concatenate([np.asarray(p["accsum"], np.int64) for p in parts])
        idx = np.concatenate([np.asarray(p["index"], np.uint64) for p in parts])
        n = len(cap)
        pts = (N.proteus_pareto_point * max(1, n))()
        for i in range(n):
            pts[i] = N.proteus_pareto_point(int(cap[i]), int(acs[i]), int(idx[i]))
        out = (N.proteus_pareto_point * max(1, max_points))()
        npts = C.c_int32()
        self._check(self._lib.proteus_pareto_merge(self._h, pts, n, out, int(max_points), C.byref(npts)))
        k = min(npts.value, max_points)
        return dict(cap=np.array([out[i].capacity for i in range(k)], np.int64),
                    accsum=np.array([out[i].accsum for i in range(k)], np.int64),
                    index=np.array([out[i].index for i in range(k)], np.uint64),
                    n_configs=sum(int(p["n_configs"]) for p in parts), n_front=npts.value)

    # ----------------------------------------------------- instrumentation --
    def set_timing(self, on=True):
        self._check(self._lib.proteus_set_timing(self._h, 1 if on else 0))

    def kernel_times(self):
        n = self._lib.proteus_kernel_times(self._h, None, None, 0)
        names = (C.c_char_p * max(n, 1))()
        ms = (C.c_float * max(n, 1))()
        self._lib.proteus_kernel_times(self._h, names, ms, n)
        return [(names[i].decode(), ms[i]) for i in range(n)]

    def launch_count(self):
        return int(self._lib.proteus_launch_count(self._h))
