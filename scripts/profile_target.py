"""One invocation of a hot-path workload, for ncu captures (never timed).

    python scripts/profile_target.py c2      # flat search over 13^8 candidates
    python scripts/profile_target.py c4      # factored re-solve, 3600 vectors
    python scripts/profile_target.py c5      # replay 10M queries x 64 scenarios
    python scripts/profile_target.py f2      # c5 trace, Nexus + AIMD, 32 scenarios each
    python scripts/profile_target.py f4      # closed loop, 3600 epochs x 12 scenarios
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402


def main(what):
    px = Proteus(0)
    if what == "c2":  # the bench's step: the c2 batch (flat launches of 32 vectors)
        import bench
        cfg = W.config("c2", totals=bench.C2_TOTALS)
        px.load_profiles(cfg["prof"])
        out, n = px.solve_batch(cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"], mode=0)
        print("c2", int(out["index"][0]), n)
    elif what == "c4":
        cfg = W.config("c4")
        px.load_profiles(cfg["prof"])
        sols = px.solve(cfg["cluster"].device_type, cfg["cluster"].slo_us, cfg["demand"], mode=2)
        print("c4", len(sols), sum(s.unmet for s in sols))
    elif what == "c5":
        cfg = W.config("c5")
        prof, cl = cfg["prof"], cfg["cluster"]
        px.load_profiles(prof)
        a = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
        arr = torch.from_numpy(cfg["arrival_us"]).cuda()
        fam = torch.from_numpy(cfg["family"]).cuda()
        sc = cfg["scenarios"]
        lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
        r = px.replay(arr, fam, a.option, a.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        print("c5", r["violations"][:8])
    elif what == "f2":
        cfg = W.config("c5")
        prof, cl = cfg["prof"], cfg["cluster"]
        px.load_profiles(prof)
        a = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
        arr = torch.from_numpy(cfg["arrival_us"]).cuda()
        fam = torch.from_numpy(cfg["family"]).cuda()
        sc = np.concatenate([W.scenarios_64(0, 1)[::2], W.scenarios_64(0, 2)[::2]])
        lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
        r = px.replay(arr, fam, a.option, a.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        print("f2", r["violations"][:8])
    elif what == "f4":
        cfg = W.config("f4")
        px.load_profiles(cfg["prof"])
        cl = cfg["cluster"]
        arr = torch.from_numpy(cfg["arrival_us"]).cuda()
        fam = torch.from_numpy(cfg["family"]).cuda()
        dem = torch.from_numpy(cfg["demand"]).cuda()
        res, _ = px.closed_loop(arr, fam, cfg["epoch_us"], dem, cl.device_type, cl.slo_us, cfg["scenarios"],
                                latency=None, device=torch.device("cuda:0"))
        print("f4", res["violations"][:8])
    torch.cuda.synchronize()


if __name__ == "__main__":
    main(sys.argv[1])
