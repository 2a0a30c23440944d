"""Measured 1-GPU time of every replay scenario alone (S = 1 per call,
latencies written to HBM), for the scenario-to-rank cost model of the
distributed replay (csrc/comm.cu scenario_cost).

    python scripts/scenario_costs.py > gpurun_out/scenario_costs.json
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402


def timed(fn, reps=2):
    fn()
    best = 1e30
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


px = Proteus(0)
out = {}
for kind in ("poisson", "gamma"):
    cfg = W.config("c5", kind=kind)
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    sol = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
    arr = torch.from_numpy(cfg["arrival_us"]).cuda()
    fam = torch.from_numpy(cfg["family"]).cuda()
    lat = torch.empty((1, len(arr)), dtype=torch.uint32, device="cuda")
    rows = []
    for pol in (0, 1, 2):
        for sc in W.scenarios_64(0, pol):
            ms = timed(lambda: px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us,
                                         sc[None, :], latency=lat))
            rows.append([int(x) for x in sc] + [ms])
    out[kind] = rows
    print(kind, "done", file=sys.stderr, flush=True)
cfg = W.config("f4")
px.load_profiles(cfg["prof"])
cl = cfg["cluster"]
E, D = len(cfg["demand"]), len(cl.device_type)
arr = torch.from_numpy(cfg["arrival_us"]).cuda()
fam = torch.from_numpy(cfg["family"]).cuda()
dem = torch.from_numpy(cfg["demand"]).cuda()
alloc = {"option": torch.empty((E, D), dtype=torch.int32, device="cuda"),
         "z_qps": torch.empty((E, D), dtype=torch.int32, device="cuda")}
px.solve_batch(cl.device_type, cl.slo_us, dem, mode=2, out=alloc)
lat = torch.empty((1, len(arr)), dtype=torch.uint32, device="cuda")
rows = []
for sc in cfg["scenarios"]:
    ms = timed(lambda: px.replay_epochs(arr, fam, cfg["epoch_us"], alloc["option"], alloc["z_qps"], cl.device_type,
                                        dem, cl.slo_us, sc[None, :], latency=lat))
    rows.append([int(x) for x in sc] + [ms])
out["f4"] = rows
print(json.dumps(out))
