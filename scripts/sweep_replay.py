"""c5 replay timing sweep over chunk size / warm-up (diagnostic, GPU):
    python scripts/sweep_replay.py CH:WU [CH:WU ...]"""
import os, statistics, sys
import torch
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W

px = Proteus(0)
cfg = W.config("c5")
prof, cl = cfg["prof"], cfg["cluster"]
px.load_profiles(prof)
alloc = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
dev = torch.device("cuda:0")
arr = torch.from_numpy(cfg["arrival_us"]).to(dev)
fam = torch.from_numpy(cfg["family"]).to(dev)
sc = cfg["scenarios"]
lat = torch.empty((len(sc), len(cfg["arrival_us"])), dtype=torch.uint32, device=dev)
ref = None
for spec in sys.argv[1:]:
    ch, wu = spec.split(":")
    os.environ["PROTEUS_REPLAY_CHUNK"] = ch
    os.environ["PROTEUS_REPLAY_WARMUP"] = wu
    px.replay(arr, fam, alloc.option, alloc.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
    px.set_timing(True)
    ts, kk = [], []
    for _ in range(3):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        r = px.replay(arr, fam, alloc.option, alloc.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
        kk.append({n: m for n, m in px.kernel_times() if n in ("replay_spec", "replay_stitch")})
    px.set_timing(False)
    h = int(lat.sum(dtype=torch.int64).item()) if False else None
    v = r["violations"].tolist()
    if ref is None:
        ref = v
    print(f"CH={ch} WU={wu}: {statistics.median(ts):.2f} ms  spec {statistics.median(k['replay_spec'] for k in kk):.2f}"
          f"  stitch {statistics.median(k['replay_stitch'] for k in kk):.2f}  same_aggregates={v == ref}", flush=True)
