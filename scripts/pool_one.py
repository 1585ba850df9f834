#!/usr/bin/env python
"""One 3x3 pool case (forward, forward + mask, backward) run R times: the target of ncu captures
and A/B timing of pool variants (GIST_LIBRARY=var/libgist_*.so).  Developer tool.

  python scripts/pool_one.py --case alexnet1 [--reps 5] [--time]
"""
from __future__ import annotations

import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402

CASES = {
    "alexnet1": ((128, 96, 55, 55), WL.P3S2),
    "alexnet2": ((128, 256, 27, 27), WL.P3S2),
    "alexnet5": ((128, 256, 13, 13), WL.P3S2),
    "nin2": ((256, 96, 54, 54), WL.P3S2C),
    "nin4": ((256, 256, 27, 27), WL.P3S2C),
    "googlenet1": ((64, 64, 112, 112), WL.P3S2C),
    "inc3a": ((64, 192, 28, 28), WL.P3S1P1),
    "vgg1": ((64, 64, 224, 224), WL.P2S2),
    "vgg3": ((64, 256, 56, 56), WL.P2S2),
    "vgg4": ((64, 512, 28, 28), WL.P2S2),
    "vgg5": ((64, 512, 14, 14), WL.P2S2),
    "inc4a": ((64, 480, 14, 14), WL.P3S1P1),
    "inc4b": ((64, 512, 14, 14), WL.P3S1P1),
    "inc3b": ((64, 256, 28, 28), WL.P3S1P1),
    "inc5a": ((64, 832, 7, 7), WL.P3S1P1),
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--case", default="alexnet1")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--time", action="store_true")
    ap.add_argument("--what", default="fwd,fwdm,bwd")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    cases = list(CASES) if args.case == "all" else args.case.split(",")
    for c in cases:
        shp, g = CASES[c]
        y = WL.relu_map(shp, 0.5, 3, dev)
        m = gist.gist_binarize_encode(y)
        o, a, _ = gist.gist_maxpool_fwd_argmax(y, g)
        d = WL.grad_map(tuple(o.shape), 4, dev)
        dx = torch.empty_like(y)
        n, no = y.numel(), o.numel()
        fns = {
            "fwd": (lambda: gist.gist_maxpool_fwd_argmax(y, g, out=o, argmax=a), 4 * n + 4 * no + no // 2),
            "fwdm": (lambda: gist.gist_maxpool_fwd_argmax(y, g, out=o, argmax=a, mask=m, fuse_mask=True),
                     4 * n + 4 * no + no // 2 + n // 8),
            "bwd": (lambda: gist.gist_pool_relu_bwd(d, a, m, shp, g, dx=dx), 4 * no + no // 2 + n // 8 + 4 * n),
        }
        for w in args.what.split(","):
            fn, b = fns[w]
            for _ in range(2):
                fn()
            torch.cuda.synchronize()
            if not args.time:
                for _ in range(args.reps):
                    fn()
                torch.cuda.synchronize()
                continue
            # R launches captured in one CUDA graph: the device time per launch without the
            # Python call overhead (which exceeds small kernels' run time)
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr):
                for _ in range(args.reps):
                    fn()
            gr.replay()
            torch.cuda.synchronize()
            ts = []
            for _ in range(5):
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                gr.replay()
                e.record()
                torch.cuda.synchronize()
                ts.append(s.elapsed_time(e) / args.reps)
            t = sorted(ts)[2]
            print(f"{c:10s} {w:5s} {t * 1e3:8.2f} us  {b / t / 1e6:7.0f} GB/s  {b / t / 1e6 / 6531.3:.3f}")


if __name__ == "__main__":
    main()
