"""window-path diagnostics on c5 (PROTEUS_REPLAY_DEBUG=1): per lane idle hops / busy entries / walked decisions"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["PROTEUS_REPLAY_DEBUG"] = "1"
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402

px = Proteus(0)
cfg = W.config("c5", kind=sys.argv[1] if len(sys.argv) > 1 else "poisson")
prof, cl = cfg["prof"], cfg["cluster"]
px.load_profiles(prof)
sol = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
arr = torch.from_numpy(cfg["arrival_us"]).cuda()
fam = torch.from_numpy(cfg["family"]).cuda()
sc = cfg["scenarios"]
px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=None)
torch.cuda.synchronize()
