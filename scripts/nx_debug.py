"""Nexus overload scan diagnostic: c5 trace prefix x Nexus scenarios vs the
oracle, first mismatching query per scenario (with the device and its position)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 300000
cfg = W.config("c5")
prof, cl = cfg["prof"], cfg["cluster"]
r = oracle.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
arr, fam = cfg["arrival_us"][:n], cfg["family"][:n]
sc = W.scenarios_64(0, 1)
px = Proteus(0)
px.load_profiles(prof)
lat = torch.empty((len(sc), n), dtype=torch.uint32, device="cuda")
g = px.replay(torch.from_numpy(arr).cuda(), torch.from_numpy(fam).cuda(), r["option"], r["z"], cl.device_type,
              cfg["demand"][0], cl.slo_us, sc, latency=lat)
o = oracle.replay(prof, cl.device_type, r["option"], r["z"], cfg["demand"][0], cl.slo_us, arr, fam, sc)
gl = lat.cpu().numpy()
# routed device per query (oracle SWRR)
V = np.asarray(prof.V); fam_m = np.repeat(np.arange(prof.Q), V)
opt = r["option"]; D = len(opt)
devfam = np.array([fam_m[x - 1] if x > 0 else -1 for x in opt], np.int32)
wdev = np.array([r["z"][d] if devfam[d] >= 0 else 0 for d in range(D)], np.int32)
wsink = cfg["demand"][0].astype(np.int32).copy()
for d in range(D):
    if devfam[d] >= 0: wsink[devfam[d]] -= r["z"][d]
tgt = oracle.route_swrr(fam, prof.Q, devfam, wdev, wsink)
bad = 0
for s in range(len(sc)):
    if np.array_equal(gl[s], o["latency"][s]):
        continue
    bad += 1
    idx = np.nonzero(gl[s] != o["latency"][s])[0]
    d = tgt[idx[0]]
    pos = np.nonzero(tgt == d)[0]
    p0 = np.searchsorted(pos, idx[0])
    nd = np.sum(tgt[idx] == d)
    print(f"scenario {s} {sc[s].tolist()}: {len(idx)} differ; first query {idx[0]} device {d} pos {p0} of {len(pos)}; "
          f"{nd} on that device; gpu {gl[s][pos[p0-2:p0+3]].tolist()} oracle {o['latency'][s][pos[p0-2:p0+3]].tolist()}")
print("scenarios differing:", bad)
