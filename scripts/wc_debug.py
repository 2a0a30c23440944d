import os, sys
sys.path.insert(0, ".")
import numpy as np, torch
os.environ["PROTEUS_REPLAY_DEBUG"] = "300000000"
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
cfg = W.config("c5"); prof, cl = cfg["prof"], cfg["cluster"]
px = Proteus(0); px.load_profiles(prof)
a = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
arr = torch.from_numpy(cfg["arrival_us"]).cuda(); fam = torch.from_numpy(cfg["family"]).cuda()
px.replay(arr, fam, a.option, a.z, cl.device_type, cfg["demand"][0], cl.slo_us, np.array([[1000, 2, 0, 1], [5000, 0, 0, 1]], np.int32), latency=None)
torch.cuda.synchronize()
