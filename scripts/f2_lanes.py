"""Which f2 scenarios are slow (diagnostic, GPU): c5 trace, one SLO multiplier
x batch cap at a time per policy, replay time."""
import os, statistics, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
cfg = W.config("c5")
prof, cl = cfg["prof"], cfg["cluster"]
px = Proteus(0)
px.load_profiles(prof)
a = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
arr = torch.from_numpy(cfg["arrival_us"]).cuda(); fam = torch.from_numpy(cfg["family"]).cuda()
for pol in (1, 2):
    res = []
    for m in W.SLO_MULTS_MILLI:
        for c in W.BATCH_CAPS:
            sc = np.array([[m, c, 0, pol]], np.int32)
            px.set_timing(True)
            px.replay(arr, fam, a.option, a.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=None)
            ms = sum(v for n, v in px.kernel_times() if n == "replay_baseline")
            res.append((ms, m, c))
    res.sort(reverse=True)
    print("policy", pol, [(round(x, 1), m, c) for x, m, c in res[:10]], flush=True)
