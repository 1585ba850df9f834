"""Timing experiment: per-tile hand-off timeline of ssdc_encode_kernel (variants/libgist_trace.so)."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("GIST_LIBRARY", "variants/libgist_trace.so")
import torch
import paper_conf_isca_jainpmtp18_b200 as gist
import workloads as WL
dev = torch.device("cuda:0")
buf = torch.zeros(4 * 256 * 8, dtype=torch.int64, device=dev)
fn = gist.lib.gist_debug_ssdc_trace; fn.argtypes = [ctypes.c_void_p]; fn.restype = ctypes.c_int
s = float(sys.argv[1]) if len(sys.argv) > 1 else 0.8
x = WL.relu_map((64, 64, 224, 224), s, 5, dev)
for _ in range(3): gist.gist_ssdc_encode(x)
torch.cuda.synchronize()
print("set", fn(buf.data_ptr()))
gist.gist_ssdc_encode(x); torch.cuda.synchronize()
t = buf.view(4, 256, 8).cpu().numpy().astype('int64')
import numpy as np
names = ["claim", "landed", "counted", "resolved", "compacted", "stored"]
for c in range(2):
    valid = t[c, :, 0] > 0
    T = t[c][valid][:, :6]
    t0 = T[:, 0].min()
    print(f"CTA {c}: {valid.sum()} tiles; span {(T[:,5].max()-t0)/1e3:.1f} us")
    d = np.diff(T, axis=1)
    for k in range(5):
        dd = d[:, k]; dd = dd[dd > -1e8]
        print(f"  {names[k]:>9s} -> {names[k+1]:<9s}: median {np.median(dd)/1e3:6.2f} us  p90 {np.percentile(dd,90)/1e3:6.2f}")
    lbs = t[c][valid][:, 6]; rp = t[c][valid][:, 7]
    print(f"  counted -> LB start: median {np.median(lbs - T[:,2])/1e3:.2f} us; LB start -> resolved: median {np.median(T[:,3]-lbs)/1e3:.2f} us")
    print(f"  look-back rounds: median {np.median(rp // 1000000):.0f} p90 {np.percentile(rp // 1000000, 90):.0f}; polls median {np.median(rp % 1000000):.0f} p90 {np.percentile(rp % 1000000, 90):.0f}")
    inter = np.diff(T[:, 0]); print(f"  claim interval median {np.median(inter)/1e3:.2f} us; stored interval {np.median(np.diff(T[:,5]))/1e3:.2f} us")
    for j in range(8, 14): print("   ", j, [round((v - t0)/1e3, 2) for v in T[j]])
