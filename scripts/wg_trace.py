"""f4 timing experiment: a -DGIST_WG_TRACE build (GIST_LIBRARY) stamps clock64 at the MMA thread's
b_full wait, its issue, the builders' b_empty wait and arrive, and the decoders' K-tile end for CTA 0."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402

dev = torch.device("cuda:0")
N, Ci, Co, H, W = 64, 256, 256, 56, 56
passes = int(sys.argv[1]) if len(sys.argv) > 1 else 3
x = WL.relu_map((N, Ci, H, W), 0.8, 77, dev)
dy = WL.grad_map((N, Co, H, W), 78, dev)
row_end, col, val, nnz = gist.gist_ssdc_encode(x)
buf = torch.zeros(256 * 8, dtype=torch.int64, device=dev)
fn = gist.lib.gist_debug_wg_trace
fn.argtypes = [C.c_void_p]
for _ in range(2):
    gist.gist_conv3x3_wgrad_ssdc(dy, row_end, col, val, x.shape, passes)
fn(buf.data_ptr())
gist.gist_conv3x3_wgrad_ssdc(dy, row_end, col, val, x.shape, passes)
torch.cuda.synchronize()
t = buf.view(256, 8).cpu().tolist()
t0 = t[0][0]
print("stage  mma_wait  mma_got  mma_issued  bld_empty  bld_arrive  dec_tile_done   (cycles from stage 0)")
for g in range(60):
    r = t[g]
    print(g, *[(v - t0) if v else "-" for v in r[:6]])
d = [t[g + 1][2] - t[g][2] for g in range(100, 200) if t[g][2] and t[g + 1][2]]
print("median issue period (stages 100-200):", sorted(d)[len(d) // 2])
w = [t[g][1] - t[g][0] for g in range(100, 200) if t[g][1]]
print("median MMA wait for b_full:", sorted(w)[len(w) // 2])
b = [t[g][4] - t[g][3] for g in range(100, 200) if t[g][4] and t[g][3]]
print("median builder work (b_empty seen -> arrive):", sorted(b)[len(b) // 2])
e = [t[g][3] - t[g - 2][2] for g in range(100, 200) if t[g][3] and t[g - 2][2]]
print("median MMA(g-2) issued -> builder sees b_empty(g):", sorted(e)[len(e) // 2])
