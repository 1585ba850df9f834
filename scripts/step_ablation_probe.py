"""Probe: clean (PDL-chained) C3 step time with one kind of call removed, vs that kind's
per-launch-event time (marginal cost of each row inside the chain)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
import paper_conf_isca_jainpmtp18_b200 as gist
import workloads as WL

dev = torch.device("cuda:0")
wl = bench.Workload(gist, WL.CONFIGS["C3"], 64, 0.8, 16, 0, dev, True)
names = {"a2": "gist_maxpool_fwd_argmax", "a3": "gist_pool_relu_bwd", "a4": "gist_ssdc_encode",
         "a5": "gist_ssdc_decode", "a6": "gist_dpr_encode", "a7": "gist_dpr_decode"}
orig = {k: getattr(gist, v) for k, v in names.items()}


def timed(K=30):
    for _ in range(5):
        wl.step()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(K):
        wl.step()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / K


full = timed()
print(f"full step {full:.4f} ms")
timer = bench.KernelTimer(torch.cuda.current_stream(dev))
for _ in range(10):
    wl.step(timer)
torch.cuda.synchronize()
per = {}
for kind, d, s, e in timer.records:
    per[kind] = per.get(kind, 0.0) + s.elapsed_time(e) / 10
for k, v in names.items():
    setattr(gist, v, lambda *a, **kw: None)
    t = timed()
    setattr(gist, v, orig[k])
    inst = [val for kk, val in per.items() if kk.startswith(k)]
    print(f"without {k}: {t:.4f} ms  marginal {full - t:.4f} ms  per-launch-event {sum(inst):.4f} ms")
