import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
px = Proteus(0)
cfg = W.config("c3")
prof, cl = cfg["prof"], cfg["cluster"]
r = oracle.solve(prof, cl.device_type, cl.slo_us, cfg["demand"][0], 2)
arr, fam = W.query_trace(60_000, float(cfg["demand"][0].sum()), cfg["weights"], 9, "poisson")
px.load_profiles(prof)
fam_m = np.repeat(np.arange(prof.Q), prof.V)
opt, z = r["option"], r["z"]
dev_family = np.array([fam_m[o-1] if o>0 else -1 for o in opt], np.int32)
wsink = cfg["demand"][0].copy()
for d in range(len(opt)):
    if opt[d]>0: wsink[dev_family[d]] -= z[d]
tgt = oracle.route_swrr(fam, prof.Q, dev_family, z, wsink)
for env in ({}, {"PROTEUS_REPLAY_SIMPLE": "1"}, {"PROTEUS_REPLAY_CHUNK": "16"}, {"PROTEUS_REPLAY_CHUNK": "100000"}):
    for k in ("PROTEUS_REPLAY_SIMPLE", "PROTEUS_REPLAY_CHUNK"):
        os.environ.pop(k, None)
    os.environ.update(env)
    sc = W.scenarios_64(0)
    g = px.replay(arr, fam, opt, z, cl.device_type, cfg["demand"][0], cl.slo_us, sc)
    o = oracle.replay(prof, cl.device_type, opt, z, cfg["demand"][0], cl.slo_us, arr, fam, sc)
    nbad = 0
    for s in range(64):
        bad = np.nonzero(g["latency"][s] != o["latency"][s])[0]
        if len(bad):
            nbad += 1
            if nbad <= 4:
                d = tgt[bad[0]]
                idx = np.nonzero(tgt == d)[0]
                pos = np.searchsorted(idx, bad)
                print(env, "scenario", sc[s], "bad", len(bad), "dev", d, "positions", pos[:10], "gpu", g["latency"][s][bad[:5]], "orc", o["latency"][s][bad[:5]])
    aggok = all(np.array_equal(g[k], o[k]) for k in ("violations", "on_time", "acc_sum"))
    print(env, "bad scenarios", nbad, "aggregates equal", aggok)
