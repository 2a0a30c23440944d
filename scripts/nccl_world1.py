"""NCCL path of dist.solve_sharded_batch / replay_sharded on one GPU (world 1
process group over NCCL): the collectives' code path the N-GPU bench takes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import torch.distributed as dist
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
from paper_conf_asplos_ahmadgfwsw24_b200.dist import replay_sharded, solve_sharded_batch

os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
os.environ.setdefault("MASTER_PORT", sys.argv[1] if len(sys.argv) > 1 else "29533")
dev = torch.device("cuda:0")
dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
px = Proteus(0)
cfg = W.config("c2", totals=(1500, 3000, 7500))
cl = cfg["cluster"]
px.load_profiles(cfg["prof"])
t = lambda x: torch.as_tensor(x, dtype=torch.int32, device=dev)  # noqa: E731
best, local, n_all, nc = solve_sharded_batch(px, t(cl.device_type), t(cl.slo_us), t(cfg["demand"]), 0, None, dev)
ref, n = px.solve_batch(cl.device_type, cl.slo_us, cfg["demand"], mode=0)
assert n_all == n == nc
for k in ("score", "index", "served", "accsum", "option", "z_qps"):
    assert np.array_equal(np.asarray(best[k]).astype(np.int64), np.asarray(ref[k]).astype(np.int64)), k
c3 = W.config("c3")
px.load_profiles(c3["prof"])
sol = px.solve(c3["cluster"].device_type, c3["cluster"].slo_us, c3["demand"][:1], mode=2)[0]
a, f = W.query_trace(20000, 3000.0, c3["weights"], 5, "gamma")
sc = W.scenarios_64(0)[::7]
agg, _, _ = replay_sharded(px.replay, sc, None, dev, arrival_us=a, family=f, option=sol.option, z=sol.z,
                           device_type=c3["cluster"].device_type, demand=c3["demand"][0],
                           slo_base_us=c3["cluster"].slo_us, latency=None)
ref = px.replay(a, f, sol.option, sol.z, c3["cluster"].device_type, c3["demand"][0], c3["cluster"].slo_us, sc,
                latency=None)
for k in ("violations", "on_time", "acc_sum"):
    assert np.array_equal(agg[k], ref[k]), k
dist.destroy_process_group()
print("nccl world-1 ok")
