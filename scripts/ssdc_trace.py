"""Timing experiment: per (CTA, local tile) timeline of ssdc_encode_kernel
(var/libgist_trace.so, built with -DGIST_SSDC_TRACE).  Back-to-back calls like a timing loop;
the trace keeps the last call of each burst."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("GIST_LIBRARY", "var/libgist_trace.so")
import numpy as np
import torch
import paper_conf_isca_jainpmtp18_b200 as gist
import workloads as WL

dev = torch.device("cuda:0")
CH = 256
G = gist.gist_num_sms()
buf = torch.zeros(G * CH * 4, dtype=torch.int64, device=dev)
fn = gist.lib.gist_debug_ssdc_trace
fn.argtypes = [ctypes.c_void_p]
fn.restype = ctypes.c_int
s = float(sys.argv[1]) if len(sys.argv) > 1 else 0.8
shape = tuple(int(v) for v in sys.argv[2].split("x")) if len(sys.argv) > 2 else (64, 64, 224, 224)
x = WL.relu_map(shape, s, 5, dev)
print("shape", shape, "tiles", -(-x.numel() // 8192))
ws = gist.gist_ssdc_workspace(x.numel(), dev)
out = gist.gist_ssdc_encode(x, workspace=ws)
torch.cuda.synchronize()
print("set", fn(buf.data_ptr()))
for run in range(4):
    buf.zero_()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(4)]
    for e0, e1 in evs:
        e0.record()
        gist.gist_ssdc_encode(x, row_end=out[0], col=out[1], val=out[2], nnz=out[3], workspace=ws)
        e1.record()
    torch.cuda.synchronize()
    print("back-to-back us:", [round(a.elapsed_time(b) * 1e3) for a, b in evs])
    t = buf.view(G, CH, 4).cpu().numpy().astype(np.int64)
    smid = t[:, CH - 1, 3].copy()
    t[:, CH - 1, :] = 0
    valid = (t[:, :, 0] > 0) & (t[:, :, 3] > 0)
    t0 = t[:, :, 0][t[:, :, 0] > 0].min()
    T = np.where(t > 0, (t - t0) / 1e3, np.nan)
    cnt = valid.sum(1)
    print(f"  tiles per CTA: min {cnt.min()} median {np.median(cnt):.0f} max {cnt.max()}")
    for name, a, b in [("issue->publish", 0, 1), ("publish->resolved", 1, 2), ("resolved->written", 2, 3)]:
        d = (T[:, :, b] - T[:, :, a])[valid]
        print(f"  {name:18s} median {np.median(d):6.2f} p90 {np.percentile(d, 90):6.2f} max {np.max(d):7.2f} us")
    per = np.diff(T[:, :, 3], axis=1)[valid[:, 1:] & valid[:, :-1]]
    print(f"  per-CTA tile period (writer) median {np.median(per):.2f} us p90 {np.percentile(per, 90):.2f}")
    end = np.nanmax(T[:, :, 3], axis=1)
    print(f"  CTA end time: min {np.nanmin(end):.1f} median {np.nanmedian(end):.1f} max {np.nanmax(end):.1f} us")
    first = T[:, 0, :]
    print("  first tile: issue min %.2f max %.2f | publish med %.2f | resolved med %.2f max %.2f | written med %.2f max %.2f" % (
        np.nanmin(first[:, 0]), np.nanmax(first[:, 0]), np.nanmedian(first[:, 1]), np.nanmedian(first[:, 2]),
        np.nanmax(first[:, 2]), np.nanmedian(first[:, 3]), np.nanmax(first[:, 3])))
    lo = np.argsort(cnt)[:6]
    print("  fewest tiles (cta, smid, tiles):", [(int(c), int(smid[c]), int(cnt[c])) for c in lo])
