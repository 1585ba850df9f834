#!/usr/bin/env python
"""f4 accuracy evidence: normwise error |dW - dW_ref| / sum|dY X| (max and median over entries) of
the decode-in-GEMM weight gradient (3xTF32 and 1xTF32) and, for scale, of cuDNN's own fp32 and
TF32 weight gradients on the same dense inputs, against the binary64 oracle (O8).

  python scripts/wgrad_accuracy.py [--json out.json]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle as ref  # noqa: E402
import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402

SHAPES = [(2, 48, 128, 56, 56), (8, 16, 128, 28, 28), (4, 32, 128, 14, 14), (1, 16, 128, 112, 112)]


def err(got, want, mag):
    e = np.abs(got.astype(np.float64) - want) / np.maximum(mag, 1e-30)
    return {"max": float(e.max()), "median": float(np.median(e))}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--json", default=None)
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    out = []
    for shape in SHAPES:
        N, Ci, Co, H, W = shape
        x = WL.relu_map((N, Ci, H, W), 0.8, sum(shape), dev)
        dy = WL.grad_map((N, Co, H, W), sum(shape) + 1, dev)
        want, mag = ref.conv3x3_wgrad(dy.cpu().numpy(), x.cpu().numpy())
        row_end, col, val, nnz = gist.gist_ssdc_encode(x)
        r = {"shape": list(shape), "K": N * H * W}
        for passes in (3, 1):
            dw = gist.gist_conv3x3_wgrad_ssdc(dy, row_end, col, val, tuple(x.shape), passes=passes)
            r[f"gist_{passes}xtf32"] = err(dw.cpu().numpy(), want, mag)
        for tf32 in (False, True):
            torch.backends.cudnn.allow_tf32 = tf32
            dw = torch.nn.grad.conv2d_weight(x, (Co, Ci, 3, 3), dy, stride=1, padding=1)
            r["cudnn_" + ("tf32" if tf32 else "fp32")] = err(dw.cpu().numpy(), want, mag)
        torch.backends.cudnn.allow_tf32 = True
        print(json.dumps(r), flush=True)
        out.append(r)
    if args.json:
        with open(args.json, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
