"""Small invocations of every kernel, for compute-sanitizer (tests/test_gpu_sanitizer.py)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402


def main():
    px = Proteus(0)
    cfg = W.config("c1")
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    for mode in (0, 1, 2):
        px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=mode)
    px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=0, generic=True)
    # k_flat_fam without the symmetric states (last two devices of different types)
    px.solve(np.array([1, 0, 1, 0], np.int32), cl.slo_us, cfg["demand"], mode=0)
    # the device combines of the multi-GPU path (comm.cu) on 3 slices
    parts = [px.solve_batch(cl.device_type, cl.slo_us, cfg["demand"], mode=0, shard_rank=r, shard_world=3)
             for r in range(3)]
    px.combine_solutions([q[0] for q in parts], [q[1] for q in parts], len(cl.device_type))
    px.solve(cl.device_type, cl.slo_us, np.repeat(cfg["demand"], 9, axis=0), mode=2)  # batched kernel
    cfg = W.config("c3", totals=(3000,))
    px.load_profiles(cfg["prof"])
    px.pareto(np.array([0, 1, 1, 2, 2], np.int32), cfg["cluster"].slo_us, 3)
    px.pareto(np.array([0, 1, 2], np.int32), cfg["cluster"].slo_us, 1, allow_idle=True)
    pp = [px.pareto(np.array([0, 1, 1, 2], np.int32), cfg["cluster"].slo_us, 3, shard_rank=r, shard_world=2)
          for r in range(2)]
    px.pareto_merge(pp)
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    sol = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
    arr, fam = W.query_trace(6000, 3000.0, cfg["weights"], 3, "gamma")
    sc = np.array([[1000, 1, 0], [2000, 4, 0], [3500, 0, 0], [1500, 0, 1]], np.int32)
    os.environ["PROTEUS_REPLAY_CHUNK"] = "16"
    px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
    os.environ["PROTEUS_REPLAY_ROUNDS"] = "1"  # one fix-up round, then the stitch
    px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
    os.environ.pop("PROTEUS_REPLAY_ROUNDS")
    os.environ["PROTEUS_REPLAY_WARMUP"] = "40"  # chunk runs entered after a warm-up
    px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
    os.environ.pop("PROTEUS_REPLAY_WARMUP")
    # §8(f2) baseline batchers (k_wc_lanes), mixed with §5 scenarios
    scb = np.array([[1000, 4, 0, 1], [2000, 0, 0, 2], [1500, 8, 1, 1], [3000, 0, 0, 0]], np.int32)
    px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, scb)
    # duplicate lanes (caps past R4's bound give the same Bmax): one replayed, rows copied
    scd = np.array([[2000, 32, 0], [2000, 64, 0], [2000, 0, 0], [1000, 1, 0], [3000, 16, 1], [3000, 0, 1]], np.int32)
    px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, scd)
    # opt-in replay paths: window path, stitch chunk tables, fused finish, binary-search stitch,
    # the chain path (tables mode for every lane; full-batch walks for every lane)
    for env in ({"PROTEUS_REPLAY_WINDOW": "1", "PROTEUS_REPLAY_WIN_TILES": "2"},
                {"PROTEUS_REPLAY_TABLES": "1", "PROTEUS_REPLAY_TABLES_MINB": "2"},
                {"PROTEUS_REPLAY_FINISH": "1"}, {"PROTEUS_STITCH_BSEARCH": "1"},
                {"PROTEUS_REPLAY_CHAIN": "1", "PROTEUS_REPLAY_CHAIN_MINBATCH": "0", "PROTEUS_REPLAY_CHAIN_RHO_PCT": "100000",
                 "PROTEUS_REPLAY_CHAIN_C": "256", "PROTEUS_REPLAY_CHAIN_K": "2"},
                {"PROTEUS_REPLAY_CHAIN": "1", "PROTEUS_REPLAY_CHAIN_RHO_PCT": "0", "PROTEUS_REPLAY_CHAIN_C": "256"}):
        os.environ.update(env)
        px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
        for k in env:
            os.environ.pop(k)
    os.environ["PROTEUS_REPLAY_SIMPLE"] = "1"
    px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
    os.environ.pop("PROTEUS_REPLAY_SIMPLE")
    # §8(f4) closed loop (k_ep_*), 5 short epochs with switching allocations
    lc = W.config("f4", n_seconds=5, lam_mid=3000.0)
    dem = np.ascontiguousarray(lc["demand"])
    px.load_profiles(lc["prof"])
    px.closed_loop(lc["arrival_us"], lc["family"], lc["epoch_us"], dem, lc["cluster"].device_type,
                   lc["cluster"].slo_us, np.array([[1000, 4, 0, 0], [3000, 0, 0, 0]], np.int32))
    print("sanitize target done")


if __name__ == "__main__":
    main()
