import sys, time, statistics
sys.path.insert(0, ".")
import torch, numpy as np
from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, workloads as W
px = Proteus(0)
cfg = W.config("c2"); prof, cl = cfg["prof"], cfg["cluster"]
px.load_profiles(prof)
dev = torch.device("cuda:0")
td = torch.as_tensor(cl.device_type, dtype=torch.int32, device=dev)
ts = torch.as_tensor(cl.slo_us, dtype=torch.int32, device=dev)
tm = torch.as_tensor(cfg["demand"][:1], dtype=torch.int32, device=dev)
for _ in range(5): px.solve(td, ts, tm, mode=0)
px.set_timing(True)
ev, host, kts = [], [], []
st = torch.cuda.current_stream()
for _ in range(20):
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(st); t0 = time.perf_counter()
    px.solve(td, ts, tm, mode=0)
    t1 = time.perf_counter(); b.record(st); torch.cuda.synchronize()
    ev.append(a.elapsed_time(b)); host.append((t1 - t0) * 1e3); kts.append(px.kernel_times())
print("event ms", statistics.median(ev), "host ms", statistics.median(host))
print(kts[-1])
px.set_timing(False)
ev = []
for _ in range(20):
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(st); px.solve(td, ts, tm, mode=0); b.record(st); torch.cuda.synchronize()
    ev.append(a.elapsed_time(b))
print("event ms (no timing)", statistics.median(ev))
h = [np.asarray(cl.device_type, np.int32), np.asarray(cl.slo_us, np.int32), np.asarray(cfg["demand"][:1], np.int32)]
ev = []
for _ in range(20):
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(st); px.solve(*h, mode=0); b.record(st); torch.cuda.synchronize()
    ev.append(a.elapsed_time(b))
print("event ms (host inputs)", statistics.median(ev))
