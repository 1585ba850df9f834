"""Run one f4 wgrad shape (debug helper): python scripts/wgrad_one.py N Ci Co H W passes"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle as ref  # noqa: E402
import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402

N, Ci, Co, H, W, passes = (int(v) for v in sys.argv[1:7])
dev = torch.device("cuda:0")
x = WL.relu_map((N, Ci, H, W), 0.8, 1, dev)
dy = WL.grad_map((N, Co, H, W), 2, dev)
row_end, col, val, nnz = gist.gist_ssdc_encode(x)
dw = gist.gist_conv3x3_wgrad_ssdc(dy, row_end, col, val, tuple(x.shape), passes=passes)
torch.cuda.synchronize()
want, mag = ref.conv3x3_wgrad(dy.cpu().numpy(), x.cpu().numpy())
err = np.abs(dw.cpu().numpy().astype(np.float64) - want) / np.maximum(mag, 1e-30)
print(sys.argv[1:7], "normwise", float(err.max()))
