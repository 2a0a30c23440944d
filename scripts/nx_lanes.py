"""Per-lane k_wc_lanes cycles of the c5 Nexus scenarios (diagnostic; kernel printf of
lanes slower than PROTEUS_REPLAY_DEBUG cycles)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402

px = Proteus(0)
cfg = W.config("c5")
prof, cl = cfg["prof"], cfg["cluster"]
px.load_profiles(prof)
sol = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
arr = torch.from_numpy(cfg["arrival_us"]).cuda()
fam = torch.from_numpy(cfg["family"]).cuda()
sc = W.scenarios_64(0, 1)
lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
torch.cuda.synchronize()
