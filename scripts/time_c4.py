"""Time the c4 batched re-solve (3600 vectors) per kernel (diagnostic)."""
import os, statistics, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
cfg = W.config("c4")
prof, cl = cfg["prof"], cfg["cluster"]
px = Proteus(0)
px.load_profiles(prof)
dev = torch.device("cuda")
t_dev = torch.as_tensor(cl.device_type, dtype=torch.int32, device=dev)
t_slo = torch.as_tensor(cl.slo_us, dtype=torch.int32, device=dev)
t_dem = torch.as_tensor(cfg["demand"], dtype=torch.int32, device=dev)
n, D = len(cfg["demand"]), len(cl.device_type)
out = {"score": torch.empty(n, dtype=torch.uint64, device=dev), "option": torch.empty((n, D), dtype=torch.int32, device=dev)}
px.set_timing(True)
for rep in range(5):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    px.solve_batch(t_dev, t_slo, t_dem, mode=2, out=out)
    t1 = time.perf_counter()
    print(f"{(t1 - t0) * 1e3:.2f} ms", [(k, round(v, 3)) for k, v in px.kernel_times()], flush=True)
h = int((out["score"].view(torch.int64) % 1000003).sum().item()), int(out["option"].sum().item())
print("checksum", h)
