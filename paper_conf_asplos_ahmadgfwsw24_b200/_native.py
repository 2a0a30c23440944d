"""ctypes binding of libproteus.so (include/proteus.h).  Argument marshalling
only: every step of the path runs in the library's CUDA kernels.  There is no
CPU fallback -- if the library cannot be loaded, importing fails loudly."""

from __future__ import annotations

import ctypes as C
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PROTEUS_LIB") or os.path.join(_PKG, "libproteus.so")  # override: diagnostics builds

PROTEUS_OK = 0
PROTEUS_EINVAL = -1
PROTEUS_ENOMEM = -2
PROTEUS_ECUDA = -3
PROTEUS_ENCCL = -4
PROTEUS_ERANGE = -5
PROTEUS_EINTERNAL = -6
PROTEUS_SOLVE_GENERIC = 1

EXPORTED = (
    "proteus_abi_version", "proteus_create", "proteus_destroy", "proteus_set_stream", "proteus_last_error",
    "proteus_load_profiles", "proteus_solve", "proteus_solve_batch", "proteus_materialize", "proteus_candidate_count",
    "proteus_pareto", "proteus_replay", "proteus_replay_epochs", "proteus_set_timing", "proteus_kernel_times", "proteus_launch_count",
    "proteus_comm_unique_id", "proteus_comm_init", "proteus_comm_enable", "proteus_comm_info", "proteus_scenario_owner",
    "proteus_combine_solutions", "proteus_pareto_merge",
)
ABI_VERSION = 3
COMM_ID_BYTES = 128


class proteus_profiles(C.Structure):
    _fields_ = [("T", C.c_int32), ("Q", C.c_int32), ("V", C.c_void_p), ("acc_micro", C.c_void_p),
                ("bmax", C.c_int32), ("lat_us", C.c_void_p)]


class proteus_solve_args(C.Structure):
    _fields_ = [("D", C.c_int32), ("device_type", C.c_void_p), ("mode", C.c_int32), ("slo_us", C.c_void_p),
                ("n_vec", C.c_int32), ("demand_qps", C.c_void_p), ("max_candidates", C.c_uint64),
                ("shard_rank", C.c_int32), ("shard_world", C.c_int32), ("flags", C.c_int32)]


class proteus_solution(C.Structure):
    _fields_ = [("score", C.c_uint64), ("index", C.c_uint64), ("served", C.c_int64), ("unmet", C.c_int64),
                ("accsum", C.c_int64), ("eff_acc_micro", C.c_int32), ("reserved", C.c_int32),
                ("n_candidates", C.c_uint64), ("option", C.c_void_p), ("z_qps", C.c_void_p)]


class proteus_batch(C.Structure):
    _fields_ = [("score", C.c_void_p), ("index", C.c_void_p), ("served", C.c_void_p), ("unmet", C.c_void_p),
                ("accsum", C.c_void_p), ("eff_acc_micro", C.c_void_p), ("option", C.c_void_p),
                ("z_qps", C.c_void_p), ("n_candidates", C.c_uint64)]


class proteus_pareto_args(C.Structure):
    _fields_ = [("D", C.c_int32), ("device_type", C.c_void_p), ("slo_us", C.c_void_p), ("family", C.c_int32),
                ("allow_idle", C.c_int32), ("shard_rank", C.c_int32), ("shard_world", C.c_int32)]


class proteus_pareto_point(C.Structure):
    _fields_ = [("capacity", C.c_int64), ("accsum", C.c_int64), ("index", C.c_uint64)]


class proteus_scenario(C.Structure):
    _fields_ = [("slo_mult_milli", C.c_int32), ("batch_cap", C.c_int32), ("routing", C.c_int32),
                ("policy", C.c_int32)]


class ProteusError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"proteus error {code}: {msg}")
        self.code = code


_lib = None


def load(path: str = LIB_PATH):
    """Load libproteus.so and declare its signatures.  Raises if missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} is missing: build it with `python -m paper_conf_asplos_ahmadgfwsw24_b200.build` "
                          "(there is no CPU fallback)")
    L = C.CDLL(path)
    vp, i32, i64, u64 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64
    L.proteus_abi_version.restype = C.c_int
    L.proteus_create.argtypes = [C.POINTER(vp), C.c_int, vp]
    L.proteus_destroy.argtypes = [vp]
    L.proteus_destroy.restype = None
    L.proteus_set_stream.argtypes = [vp, vp]
    L.proteus_last_error.argtypes = [vp]
    L.proteus_last_error.restype = C.c_char_p
    L.proteus_load_profiles.argtypes = [vp, C.POINTER(proteus_profiles)]
    L.proteus_solve.argtypes = [vp, C.POINTER(proteus_solve_args), C.POINTER(proteus_solution)]
    L.proteus_solve_batch.argtypes = [vp, C.POINTER(proteus_solve_args), C.POINTER(proteus_batch)]
    L.proteus_materialize.argtypes = [vp, C.POINTER(proteus_solve_args), i32, u64, C.POINTER(proteus_solution)]
    L.proteus_candidate_count.argtypes = [vp, C.POINTER(proteus_solve_args), C.POINTER(u64)]
    L.proteus_pareto.argtypes = [vp, C.POINTER(proteus_pareto_args), C.POINTER(proteus_pareto_point), i32,
                                 C.POINTER(i32), C.POINTER(u64)]
    L.proteus_replay.argtypes = [vp, vp, vp, i64, vp, vp, vp, i32, vp, vp, C.POINTER(proteus_scenario), i32,
                                 vp, vp, vp, vp]
    L.proteus_replay_epochs.argtypes = [vp, vp, vp, i64, i32, i64, vp, vp, vp, i32, vp, vp,
                                        C.POINTER(proteus_scenario), i32, vp, vp, vp, vp]
    L.proteus_set_timing.argtypes = [vp, C.c_int]
    L.proteus_kernel_times.argtypes = [vp, C.POINTER(C.c_char_p), C.POINTER(C.c_float), C.c_int]
    L.proteus_launch_count.argtypes = [vp]
    L.proteus_launch_count.restype = u64
    L.proteus_comm_unique_id.argtypes = [vp]
    L.proteus_comm_init.argtypes = [vp, vp, C.c_int, C.c_int]
    L.proteus_comm_enable.argtypes = [vp, C.c_int]
    L.proteus_comm_info.argtypes = [vp, C.POINTER(i32), C.POINTER(i32)]
    L.proteus_scenario_owner.argtypes = [C.POINTER(proteus_scenario), i32, i32, vp]
    L.proteus_combine_solutions.argtypes = [vp, i32, i32, i32, C.POINTER(proteus_batch), vp, C.POINTER(proteus_batch)]
    L.proteus_pareto_merge.argtypes = [vp, C.POINTER(proteus_pareto_point), i32, C.POINTER(proteus_pareto_point),
                                       i32, C.POINTER(i32)]
    if L.proteus_abi_version() != ABI_VERSION:
        raise ImportError("libproteus ABI version mismatch")
    _lib = L
    return L
