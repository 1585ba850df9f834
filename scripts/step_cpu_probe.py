"""Probe: host enqueue time vs device time of the C3 step (is the clean step launch-bound?)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
import paper_conf_isca_jainpmtp18_b200 as gist
import workloads as WL

dev = torch.device("cuda:0")
cfg = WL.CONFIGS["C3"]
wl = bench.Workload(gist, cfg, 64, 0.8, 16, 0, dev, True)
for _ in range(5):
    wl.step()
torch.cuda.synchronize()
K = 30
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
t0 = time.perf_counter()
for _ in range(K):
    wl.step()
t1 = time.perf_counter()
e1.record()
torch.cuda.synchronize()
t2 = time.perf_counter()
print(f"host enqueue {1e3 * (t1 - t0) / K:.3f} ms/step, device {e0.elapsed_time(e1) / K:.3f} ms/step, "
      f"wall {1e3 * (t2 - t0) / K:.3f} ms/step")
