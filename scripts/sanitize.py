"""Small-shape run of every kernel for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402

dev = torch.device("cuda:0")
for g, shape in [(WL.P2S2, (2, 8, 16, 16)), (WL.P2S2, (1, 3, 14, 14)), (WL.P3S2, (2, 4, 13, 13)),
                 (WL.P3S2C, (1, 4, 12, 12)), (WL.P3S1P1, (1, 4, 9, 9)),
                 # odd W with n % 32 == 0: the last 2x2 block of the 3x3/s2 backward sits on element n - 1
                 (WL.P3S2, (1, 32, 13, 13)), (WL.P3S2C, (1, 32, 13, 13))]:
    y = WL.relu_map(shape, 0.5, 1, dev)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, g, fuse_mask=True)
    gist.gist_pool_relu_bwd(torch.randn_like(out), arg, mask, shape, g)
for n in (1, 1000, 4096 * 3 + 5, 256 * 16 * 40 + 17):
    x = WL.relu_map((n,), 0.7, n, dev)
    gist.gist_binarize_encode(x)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x, trim=True)
    gist.gist_ssdc_decode(row_end, col, val, n)
    for b in (16, 10, 8):
        gist.gist_dpr_decode(gist.gist_dpr_encode(x, b), n, b)
# 3x3/s1 plane-tile pools with a ragged last tile and odd planes (pool3.cu)
for shape in [(3, 5, 7, 7), (2, 9, 14, 14)]:
    y = WL.relu_map(shape, 0.5, 3, dev)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, WL.P3S1P1, fuse_mask=True)
    gist.gist_pool_relu_bwd(torch.randn_like(out), arg, mask, shape, WL.P3S1P1)
# 3x3/s2 plane-tile pools (pool3.cu when enabled): ragged tiles, words across planes, ceil, padding 1
for g, shape in [(WL.P3S2, (3, 7, 27, 27)), (WL.P3S2C, (2, 5, 14, 14)), ((3, 3, 2, 2, 1, 1, 0), (2, 3, 15, 15))]:
    y = WL.relu_map(shape, 0.5, 4, dev)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, g, fuse_mask=True)
    gist.gist_pool_relu_bwd(torch.randn_like(out), arg, mask, shape, g)
# f4: decode-in-GEMM weight gradient, both precisions, a vector (W % 4 == 0) and a scalar shape
for N, Ci, Co, H, W in [(1, 16, 128, 8, 8), (1, 16, 128, 6, 10)]:
    x = WL.relu_map((N, Ci, H, W), 0.8, 5, dev)
    dy = WL.grad_map((N, Co, H, W), 6, dev)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x)
    for passes in (3, 1):
        gist.gist_conv3x3_wgrad_ssdc(dy, row_end, col, val, (N, Ci, H, W), passes=passes)
torch.cuda.synchronize()
print("sanitize workload done")
