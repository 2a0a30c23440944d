"""The library's own NCCL communicator on one GPU (world 1): proteus_comm_init
after the id broadcast over a torch NCCL process group, then every
distributed call -- flat and multiset solve (ncclAllGather of the per-rank
winners + device pick), factored batched solve (vector split + ncclAllGather),
the Fig. 1b frontier (two ncclAllReduce), the replay and the closed loop
(ncclAllReduce of the aggregates) -- against the same call with the
communicator disabled.  A world-1 communicator runs the same code path as N
ranks (collectives over one rank).  Run by
tests/test_gpu_solve.py::test_nccl_collective_paths_world1."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402
from paper_conf_asplos_ahmadgfwsw24_b200.dist import init_comm  # noqa: E402

os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
os.environ.setdefault("MASTER_PORT", sys.argv[1] if len(sys.argv) > 1 else "29533")
dev = torch.device("cuda:0")
dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
px = Proteus(0)
assert init_comm(px) == (1, 0)
assert px.comm_info() == (1, 0, True)
t = lambda x: torch.as_tensor(x, dtype=torch.int32, device=dev)  # noqa: E731


def both(fn):
    """fn() distributed, then with the communicator disabled"""
    px.comm_enable(True)
    a = fn()
    px.comm_enable(False)
    b = fn()
    px.comm_enable(True)
    return a, b


def same(a, b, what):
    for k in b:
        if k in ("latency",) or b[k] is None:
            continue
        assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), (what, k)


launches0 = px.launch_count()
cfg = W.config("c2", totals=(1500, 3000, 7500))
cl = cfg["cluster"]
px.load_profiles(cfg["prof"])
for mode in (0, 1):
    (a, na), (b, nb) = both(lambda: px.solve_batch(t(cl.device_type), t(cl.slo_us), t(cfg["demand"]), mode=mode))
    assert na == nb
    same(a, b, f"c2 mode {mode}")
    sa, sb = both(lambda: px.solve(cl.device_type, cl.slo_us, cfg["demand"], mode=mode))
    assert [(s.score, s.index, s.option.tolist(), s.z.tolist()) for s in sa] == \
        [(s.score, s.index, s.option.tolist(), s.z.tolist()) for s in sb]
c4 = W.config("c4", n_seconds=37)
px.load_profiles(c4["prof"])
(a, _), (b, _) = both(lambda: px.solve_batch(c4["cluster"].device_type, c4["cluster"].slo_us, c4["demand"], mode=2))
same(a, b, "c4 37 vectors")
c3 = W.config("c3")
px.load_profiles(c3["prof"])
pdev = np.array([0, 0, 1, 1, 2, 2, 2], np.int32)
a, b = both(lambda: px.pareto(pdev, c3["cluster"].slo_us, 3))
same(a, b, "pareto")
sol = px.solve(c3["cluster"].device_type, c3["cluster"].slo_us, c3["demand"][:1], mode=2)[0]
arr, fam = W.query_trace(20000, 3000.0, c3["weights"], 5, "gamma")
sc = np.concatenate([W.scenarios_64(0, 0)[::7], W.scenarios_64(0, 1)[::16], W.scenarios_64(0, 2)[::16]])
a, b = both(lambda: px.replay(arr, fam, sol.option, sol.z, c3["cluster"].device_type, c3["demand"][0],
                              c3["cluster"].slo_us, sc))
same(a, b, "replay")
assert np.array_equal(a["latency"], b["latency"])  # world 1 owns every scenario
f4 = W.config("f4", n_seconds=4, lam_mid=800.0)
px.load_profiles(f4["prof"])
(ra, aa), (rb, ab) = both(lambda: px.closed_loop(f4["arrival_us"], f4["family"], f4["epoch_us"], f4["demand"],
                                                 f4["cluster"].device_type, f4["cluster"].slo_us, f4["scenarios"]))
same(ra, rb, "closed loop")
same(aa, ab, "closed-loop allocations")
assert np.array_equal(ra["latency"], rb["latency"])
dist.destroy_process_group()
print(f"nccl world-1 ok ({px.launch_count() - launches0} launches)")
