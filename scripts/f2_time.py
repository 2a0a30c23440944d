"""f2 timing per variant (diagnostic): the c5 trace x 64 scenarios of one
baseline policy, per-kernel split.   python scripts/f2_time.py [NAME=ENV=V[,ENV=V] ...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402

VARIANTS = [("default", [])]
if len(sys.argv) > 1:
    VARIANTS = []
    for arg in sys.argv[1:]:
        name, rest = arg.split("=", 1)
        VARIANTS.append((name, [tuple(kv.split("=", 1)) for kv in rest.split(",")] if rest else []))
px = Proteus(0)
cfg = W.config("c5")
prof, cl = cfg["prof"], cfg["cluster"]
px.load_profiles(prof)
sol = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
arr = torch.from_numpy(cfg["arrival_us"]).cuda()
fam = torch.from_numpy(cfg["family"]).cuda()
out = {}
keys = {k for _, envs in VARIANTS for k, _ in envs}
for pol in (1, 2):
    sc = W.scenarios_64(0, pol)
    lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
    res = {}
    for name, envs in VARIANTS:
        for k in keys:
            os.environ.pop(k, None)
        for k, v in envs:
            os.environ[k] = v
        px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        px.set_timing(True)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        r = px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        b.record()
        torch.cuda.synchronize()
        split = {}
        for n_, v in px.kernel_times():
            split[n_] = round(split.get(n_, 0.0) + v, 3)
        px.set_timing(False)
        res[name] = {"ms": a.elapsed_time(b), "split": split, "checksum": int(lat.sum().item()),
                     "viol": r["violations"][:8].tolist()}
    out["nexus" if pol == 1 else "aimd"] = res
print(json.dumps(out))
