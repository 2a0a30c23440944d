"""Which f4 scenarios are slow (diagnostic, GPU): the closed-loop hour, one
scenario at a time, stitch time."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
cfg = W.config("f4")
prof, cl = cfg["prof"], cfg["cluster"]
px = Proteus(0)
px.load_profiles(prof)
dev = torch.device("cuda:0")
arr = torch.from_numpy(cfg["arrival_us"]).to(dev); fam = torch.from_numpy(cfg["family"]).to(dev)
dem = torch.from_numpy(cfg["demand"]).to(dev)
E, D = len(cfg["demand"]), len(cl.device_type)
alloc = {"option": torch.empty((E, D), dtype=torch.int32, device=dev), "z_qps": torch.empty((E, D), dtype=torch.int32, device=dev)}
px.solve_batch(cl.device_type, cl.slo_us, dem, mode=2, out=alloc)
for row in cfg["scenarios"]:
    px.set_timing(True)
    r = px.replay_epochs(arr, fam, cfg["epoch_us"], alloc["option"], alloc["z_qps"], cl.device_type, dem, cl.slo_us,
                         np.array([row], np.int32), latency=None)
    ms = sum(v for n, v in px.kernel_times() if n == "loop_stitch")
    print(tuple(int(x) for x in row), round(ms, 1), "viol", float(r["violations"][0]) / len(cfg["arrival_us"]), flush=True)
