"""Pipelined spec/stitch vs serial on repeated small replays (race check) and c5 timing."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402

px = Proteus(0)
cfg = W.config("c3")
prof, cl = cfg["prof"], cfg["cluster"]
px.load_profiles(prof)
sol = px.solve(cl.device_type, cl.slo_us, cfg["demand"][:1], mode=2)[0]
arr, fam = W.query_trace(60_000, float(cfg["demand"][0].sum()), cfg["weights"], 9, "gamma")
sc = W.scenarios_64(0)
os.environ["PROTEUS_STITCH_BSEARCH"] = "1"
for chunk in ("37", "64", "4096"):
    os.environ["PROTEUS_REPLAY_CHUNK"] = chunk
    os.environ["PROTEUS_REPLAY_OVERLAP"] = "0"
    ref = px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
    os.environ["PROTEUS_REPLAY_OVERLAP"] = "1"
    t0 = time.time()
    for it in range(20):
        g = px.replay(arr, fam, sol.option, sol.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
        assert np.array_equal(g["latency"], ref["latency"]), (chunk, it)
    print("chunk", chunk, "20 pipelined replays identical", round(time.time() - t0, 2), "s", flush=True)
os.environ.pop("PROTEUS_REPLAY_CHUNK")
c5 = W.config("c5")
px.load_profiles(c5["prof"])
sol = px.solve(c5["cluster"].device_type, c5["cluster"].slo_us, c5["demand"], mode=2)[0]
a = torch.from_numpy(c5["arrival_us"]).cuda()
f = torch.from_numpy(c5["family"]).cuda()
lat = torch.empty((64, len(a)), dtype=torch.uint32, device="cuda")
for ov, bs in (("1", "0"), ("1", "1"), ("0", "1")):
    os.environ["PROTEUS_REPLAY_OVERLAP"] = ov
    os.environ["PROTEUS_STITCH_BSEARCH"] = bs
    px.replay(a, f, sol.option, sol.z, c5["cluster"].device_type, c5["demand"][0], c5["cluster"].slo_us,
              c5["scenarios"], latency=lat)
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        r = px.replay(a, f, sol.option, sol.z, c5["cluster"].device_type, c5["demand"][0], c5["cluster"].slo_us,
                      c5["scenarios"], latency=lat)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print("c5 overlap", ov, "bsearch", bs, "ms", [round(x, 2) for x in ts], r["violations"][:4].tolist(),
          int(lat[:, ::997].sum(dtype=torch.int64).item()), flush=True)
