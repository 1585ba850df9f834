#!/usr/bin/env python
"""SSDC encode timing on one VGG16 relu1_1 b64 map at the given sparsities (developer tool for
timing-only variants: GIST_LIBRARY=var/exp_*.so).  python scripts/a4_one.py 0.8 0.9"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402

dev = torch.device("cuda:0")
shape = (64, 64, 224, 224)
n = 64 * 64 * 224 * 224
ws = gist.gist_ssdc_workspace(n, dev)
row_end = torch.empty((n + 255) // 256, dtype=torch.int32, device=dev)
col = torch.empty(n, dtype=torch.uint8, device=dev)
val = torch.empty(n, dtype=torch.float32, device=dev)
nnz = torch.empty(1, dtype=torch.int64, device=dev)
for s in [float(a) for a in sys.argv[1:]] or [0.8]:
    x = WL.relu_map(shape, s, 5, dev)
    fn = lambda: gist.gist_ssdc_encode(x, row_end=row_end, col=col, val=val, nnz=nnz, workspace=ws)
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(20):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    k = int(nnz.item())
    print(f"s={s} ms {sorted(ts)[10]:.4f} nnz {k}")
