"""c5 replay timing per path variant (diagnostic; the bench line is bench.py's).

    python scripts/replay_variants.py [NAME=ENV=VALUE[,ENV=VALUE] ...]

Default variants: the chain path vs the chunk-run/stitch path."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402

VARIANTS = [("chain", [("PROTEUS_REPLAY_CHAIN", "1")]), ("stitch", [("PROTEUS_REPLAY_CHAIN", "0")])]
if len(sys.argv) > 1:
    VARIANTS = []
    for arg in sys.argv[1:]:
        name, rest = arg.split("=", 1)
        VARIANTS.append((name, [tuple(kv.split("=", 1)) for kv in rest.split(",")] if rest else []))
px = Proteus(0)
out = {}
for kind in ("poisson", "gamma"):
    cfg = W.config("c5", kind=kind)
    prof, cl = cfg["prof"], cfg["cluster"]
    px.load_profiles(prof)
    sol = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
    arr = torch.from_numpy(cfg["arrival_us"]).cuda()
    fam = torch.from_numpy(cfg["family"]).cuda()
    sc = cfg["scenarios"]
    lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
    res = {}
    keys = {k for _, envs in VARIANTS for k, _ in envs}
    for name, envs in VARIANTS:
        for k in keys:  # every variant starts from the library defaults
            os.environ.pop(k, None)
        for k, v in envs:
            os.environ[k] = v
        r0 = px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        px.set_timing(True)
        ts = []
        for _ in range(3):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            r = px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        split = {}
        for n_, v in px.kernel_times():
            split[n_] = split.get(n_, 0.0) + v
        px.set_timing(False)
        res[name] = {"ms": min(ts), "split": split, "viol": r["violations"][:8].tolist(),
                     "checksum": int(lat.sum().item())}
    ks = list(res)
    res["same"] = all(res[k]["viol"] == res[ks[0]]["viol"] and res[k]["checksum"] == res[ks[0]]["checksum"] for k in ks)
    out[kind] = res
print(json.dumps(out))
