"""Per-lane stitch statistics of the c5 replay (diagnostic; needs the
PX_STITCH_DEBUG build: PROTEUS_BUILD_DEFS=-DPX_STITCH_DEBUG, PROTEUS_LIB=...)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
cfg = W.config("c5")
prof, cl = cfg["prof"], cfg["cluster"]
px = Proteus(0)
px.load_profiles(prof)
a = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
print("option", a.option.tolist()); print("z", a.z.tolist())
arr = torch.from_numpy(cfg["arrival_us"]).cuda(); fam = torch.from_numpy(cfg["family"]).cuda()
sc = cfg["scenarios"]
print("scenarios", np.asarray(sc).tolist())
lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
os.environ["PROTEUS_REPLAY_DEBUG"] = sys.argv[1] if len(sys.argv) > 1 else "4000000"
px.replay(arr, fam, a.option, a.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
torch.cuda.synchronize()
