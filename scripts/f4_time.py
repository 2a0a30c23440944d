"""f4 closed-loop timing per variant (diagnostic): the c4 hour, 12 scenarios,
latencies on the device; checksums and the per-kernel split.
    python scripts/f4_time.py [NAME=ENV=V[,ENV=V] ...]"""
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
cfg = W.config("f4")
px.load_profiles(cfg["prof"])
cl = cfg["cluster"]
arr = torch.from_numpy(cfg["arrival_us"]).cuda()
fam = torch.from_numpy(cfg["family"]).cuda()
dem = torch.from_numpy(cfg["demand"]).cuda()
sc = cfg["scenarios"]
lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
keys = {k for _, envs in VARIANTS for k, _ in envs}
out = {}
for name, envs in VARIANTS:
    for k in keys:
        os.environ.pop(k, None)
    for k, v in envs:
        os.environ[k] = v
    run = lambda: px.closed_loop(arr, fam, cfg["epoch_us"], dem, cl.device_type, cl.slo_us, sc,  # noqa: E731
                                 latency=lat, device=torch.device("cuda:0"))
    run()
    px.set_timing(True)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    res, _ = run()
    b.record()
    torch.cuda.synchronize()
    split = {}
    for n_, v in px.kernel_times():
        split[n_] = round(split.get(n_, 0.0) + v, 3)
    px.set_timing(False)
    out[name] = {"ms": a.elapsed_time(b), "split": split, "checksum": int(lat.sum().item()),
                 "viol": [int(x) for x in res["violations"][:12]]}
print(json.dumps(out))
