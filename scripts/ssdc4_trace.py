"""Timing experiment: per (CTA, local tile) timeline of ssdc_encode4_kernel
(var/libgist_trace4.so, built with -DGIST_SSDC4_TRACE)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("GIST_LIBRARY", "var/libgist_trace4.so")
import numpy as np
import torch
import paper_conf_isca_jainpmtp18_b200 as gist
import workloads as WL

dev = torch.device("cuda:0")
CH = 512
G = gist.gist_num_sms()
buf = torch.zeros(G * CH * 8, dtype=torch.int64, device=dev)
fn = gist.lib.gist_debug_ssdc4_trace
fn.argtypes = [ctypes.c_void_p]
fn.restype = ctypes.c_int
s = float(sys.argv[1]) if len(sys.argv) > 1 else 0.8
x = WL.relu_map((64, 64, 224, 224), s, 5, dev)
ws = torch.empty(gist.gist_ssdc_workspace_bytes(x.numel()), dtype=torch.uint8, device=dev)
out = gist.gist_ssdc_encode(x, workspace=ws)
torch.cuda.synchronize()
print("set", fn(buf.data_ptr()))
names = ["issued", "landed", "counted", "allocated", "compacted", "resolved", "stored"]
for run in range(2):
    buf.zero_()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    gist.gist_ssdc_encode(x, row_end=out[0], col=out[1], val=out[2], nnz=out[3], workspace=ws)
    e1.record()
    torch.cuda.synchronize()
    print(f"run {run}: {e0.elapsed_time(e1)*1e3:.0f} us")
    t = buf.view(G, CH, 8).cpu().numpy().astype(np.int64)[:, :, :7]
    valid = (t > 0).all(axis=2)
    t0 = t[t > 0].min()
    T = (t - t0) / 1e3
    cnt = valid.sum(1)
    print(f"  tiles per CTA: min {cnt.min()} median {np.median(cnt):.0f} max {cnt.max()}")
    for a in range(6):
        d = (T[:, :, a + 1] - T[:, :, a])[valid]
        print(f"  {names[a]:>9s} -> {names[a+1]:<9s} median {np.median(d):7.2f} p90 {np.percentile(d, 90):7.2f} max {d.max():8.2f} us")
    c = 0
    print("  CTA 0 first tiles:")
    for j in range(0, 24):
        if valid[c, j]:
            print("   ", j, [round(float(v), 2) for v in T[c, j]])
