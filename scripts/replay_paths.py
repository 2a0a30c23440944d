"""Time the c5 replay through each lane path / chunk size (diagnostic).
Every variant's per-query latencies must equal the first variant's."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
cfg = W.config("c5")
prof, cl = cfg["prof"], cfg["cluster"]
px = Proteus(0)
px.load_profiles(prof)
a = px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=2)[0]
arr = torch.from_numpy(cfg["arrival_us"]).cuda(); fam = torch.from_numpy(cfg["family"]).cuda()
sc = cfg["scenarios"]
lat = torch.empty((len(sc), len(arr)), dtype=torch.uint32, device="cuda")
px.set_timing(True)
KEYS = ("PROTEUS_REPLAY_SIMPLE", "PROTEUS_REPLAY_CHUNK", "PROTEUS_REPLAY_CHECKS", "PROTEUS_REPLAY_ROUNDS", "PROTEUS_REPLAY_DEBUG", "PROTEUS_REPLAY_SCAN1", "PROTEUS_REPLAY_SPLIT", "PROTEUS_REPLAY_BSCAN")
variants = [{}, {"PROTEUS_REPLAY_SPLIT": "0"}, {"PROTEUS_REPLAY_CHUNK": "8192"}, {"PROTEUS_REPLAY_CHUNK": "2048"}]
variants += [eval(v) for v in sys.argv[1:]]
ref = None
for env in variants:
    for k in KEYS: os.environ.pop(k, None)
    os.environ.update(env)
    for rep in range(2):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        r = px.replay(arr, fam, a.option, a.z, cl.device_type, cfg["demand"][0], cl.slo_us, sc, latency=lat)
        torch.cuda.synchronize(); t1 = time.perf_counter()
    kt = {}
    for n, ms in px.kernel_times():
        if n.startswith("replay"):
            kt[n] = round(kt.get(n, 0) + ms, 2)
    nfix = sum(1 for n, _ in px.kernel_times() if n == "replay_fix")
    kt["fix_rounds"] = nfix
    h = int(torch.sum(lat.view(torch.int32).to(torch.int64) * 2654435761 % 1000003).item())
    if ref is None: ref = h
    print(env, f"{(t1-t0)*1e3:.1f} ms", kt, int(r["violations"].sum()), "same" if h == ref else "DIFFERENT", flush=True)
