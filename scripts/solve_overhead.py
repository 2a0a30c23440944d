"""Per-call overhead of the c2 bench step (diagnostic): device-timed step vs
the flat kernel, and the host phase times (PROTEUS_HOST_TIMING)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W  # noqa: E402

px = Proteus(0)
cfg = W.config("c2", totals=W.C2_BENCH_TOTALS)
cl = cfg["cluster"]
px.load_profiles(cfg["prof"])
t = lambda x: torch.as_tensor(x, dtype=torch.int32, device="cuda")  # noqa: E731
d, s, dm = t(cl.device_type), t(cl.slo_us), t(cfg["demand"])
for nv in (64, 1):
    for _ in range(3):
        px.solve_batch(d, s, dm[:nv], mode=0)
    px.set_timing(True)
    ts, ks = [], []
    for _ in range(10):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        h0 = time.perf_counter()
        px.solve_batch(d, s, dm[:nv], mode=0)
        h1 = time.perf_counter()
        b.record()
        torch.cuda.synchronize()
        ts.append((a.elapsed_time(b), (h1 - h0) * 1e3))
        ks.append(px.kernel_times())
    px.set_timing(False)
    print("nvec", nv, "step ms (device, host):", ts[-3:])
    print("kernels:", ks[-1])
os.environ["PROTEUS_HOST_TIMING"] = "1"
