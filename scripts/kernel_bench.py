#!/usr/bin/env python
"""Isolated per-kernel throughput on full-size maps (evidence for each §8(a) row).

Each kernel runs alone, R times back to back on one large map (inputs > L2), timed with CUDA
events on the launching stream; reported as algorithmic GB/s (SURVEY.md §8(d) bytes) and the
fraction of the measured HBM copy bandwidth (MEASURED_PEAKS.json).

  python scripts/kernel_bench.py [--only a4] [--reps 20] [--json out.json]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402


def words(n, k):
    return -(-n // k)


def timeit(fn, reps, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        a.record(s)
        fn()
        b.record(s)
    torch.cuda.synchronize()
    ts = [a.elapsed_time(b) for a, b in evs]
    if os.environ.get("KB_DIST"):
        print("times_ms", [round(t, 3) for t in ts], flush=True)
    ts = sorted(ts)
    return ts[len(ts) // 2], sum(ts) / len(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default=None, help="comma list of row ids: a1,a2,a3,a4,a5,a6,a7,f3")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--json", default=None)
    ap.add_argument("--small", action="store_true", help="secondary geometries too (3x3 pools)")
    args = ap.parse_args()
    only = set(args.only.split(",")) if args.only else None
    dev = torch.device("cuda:0")
    peak, src = bench.hbm_peak()
    res = []
    clocks = bench.ClockSampler(dev)
    clocks.__enter__()

    def rep(row, name, nbytes, fn, extra=None):
        if only and row not in only:
            return
        med, mean = timeit(fn, args.reps)
        gbs = nbytes / (med * 1e-3) / 1e9
        r = {"row": row, "case": name, "ms_median": round(med, 4), "ms_mean": round(mean, 4),
             "algo_bytes": int(nbytes), "algo_GBps": round(gbs, 1), "frac_hbm": round(gbs / peak, 4)}
        if extra:
            r.update(extra)
        res.append(r)
        print(json.dumps(r), flush=True)

    # VGG16 relu1_2 at batch 64: the largest stashed map (822 MB), 2x2/s2 pool
    shape = (64, 64, 224, 224)
    n = 64 * 64 * 224 * 224
    g = WL.P2S2
    y = WL.relu_map(shape, 0.5, 1, dev)
    mask = torch.empty(words(n, 32), dtype=torch.int32, device=dev)
    rep("a1", "vgg16 relu1_2 b64", 4 * n + 4 * words(n, 32), lambda: gist.gist_binarize_encode(y, mask=mask))
    out, arg, _ = gist.gist_maxpool_fwd_argmax(y, g)
    n_o = out.numel()
    rep("a2", "vgg16 relu1_2 b64 2x2/s2", 4 * n + 4 * n_o + 4 * words(n_o, 8),
        lambda: gist.gist_maxpool_fwd_argmax(y, g, out=out, argmax=arg))
    rep("a2", "vgg16 relu1_2 b64 2x2/s2 +fused mask", 4 * n + 4 * n_o + 4 * words(n_o, 8) + 4 * words(n, 32),
        lambda: gist.gist_maxpool_fwd_argmax(y, g, out=out, argmax=arg, mask=mask))
    xpre = WL.grad_map(shape, 4, dev)  # pre-activation map (the producing conv's output)
    rep("f3", "vgg16 relu1_2 b64 2x2/s2 relu on load + mask (in-place ReLU)",
        4 * n + 4 * n_o + 4 * words(n_o, 8) + 4 * words(n, 32),
        lambda: gist.gist_relu_maxpool_fwd_argmax(xpre, g, out=out, argmax=arg, mask=mask))
    del xpre
    gist.gist_maxpool_fwd_argmax(y, g, out=out, argmax=arg)
    gist.gist_binarize_encode(y, mask=mask)
    dY = WL.grad_map(tuple(out.shape), 2, dev)
    dx = torch.empty_like(y)
    rep("a3", "vgg16 relu1_2 b64 2x2/s2", 4 * n_o + 4 * words(n_o, 8) + 4 * words(n, 32) + 4 * n,
        lambda: gist.gist_pool_relu_bwd(dY, arg, mask, shape, g, dx=dx))
    del out, arg, dY
    if args.small:
        for name, shp, gg in [("alexnet relu1 b128 3x3/s2", (128, 96, 55, 55), WL.P3S2),
                              ("nin relu_cccp2 b256 3x3/s2/ceil", (256, 96, 54, 54), WL.P3S2C),
                              ("googlenet inc3a pool b64 3x3/s1/p1", (64, 192, 28, 28), WL.P3S1P1)]:
            yy = WL.relu_map(shp, 0.5, 3, dev)
            m2 = gist.gist_binarize_encode(yy)
            oo, aa, _ = gist.gist_maxpool_fwd_argmax(yy, gg)
            nn, no = yy.numel(), oo.numel()
            rep("a2", name, 4 * nn + 4 * no + 4 * words(no, 8), lambda: gist.gist_maxpool_fwd_argmax(yy, gg, out=oo, argmax=aa))
            rep("a2", name + " +mask", 4 * nn + 4 * no + 4 * words(no, 8) + 4 * words(nn, 32),
                lambda: gist.gist_maxpool_fwd_argmax(yy, gg, out=oo, argmax=aa, mask=m2))
            dd = WL.grad_map(tuple(oo.shape), 4, dev)
            dxx = torch.empty_like(yy)
            rep("a3", name, 4 * no + 4 * words(no, 8) + 4 * words(nn, 32) + 4 * nn,
                lambda: gist.gist_pool_relu_bwd(dd, aa, m2, shp, gg, dx=dxx))
            del yy, m2, oo, aa, dd, dxx

    # SSDC on VGG16 relu1_1 b64 (822 MB) across the paper's sparsity range
    ws = gist.gist_ssdc_workspace(n, dev)
    row_end = torch.empty(words(n, 256), dtype=torch.int32, device=dev)
    col = torch.empty(n, dtype=torch.uint8, device=dev)
    val = torch.empty(n, dtype=torch.float32, device=dev)
    nnz = torch.empty(1, dtype=torch.int64, device=dev)
    xd = torch.empty(n, dtype=torch.float32, device=dev)
    for s in (0.5, 0.8, 0.9):
        if only and not ({"a4", "a5"} & only):
            break
        x = WL.relu_map(shape, s, 5, dev)
        gist.gist_ssdc_encode(x, row_end=row_end, col=col, val=val, nnz=nnz, workspace=ws)
        k = int(nnz.item())
        b = 4 * n + 5 * k + 4 * words(n, 256)
        rep("a4", f"vgg16 relu1_1 b64 s={s}", b,
            lambda: gist.gist_ssdc_encode(x, row_end=row_end, col=col, val=val, nnz=nnz, workspace=ws),
            {"nnz": k, "ratio": round(4 * n / (5 * k + 4 * words(n, 256)), 4)})
        rep("a5", f"vgg16 relu1_1 b64 s={s}", b, lambda: gist.gist_ssdc_decode(row_end, col, val, n, x=xd))
        del x
    del col, val, ws
    # DPR on the same map size, all three widths
    x = WL.dpr_map(shape, 6, dev)
    for bits in (16, 10, 8):
        if only and not ({"a6", "a7"} & only):
            break
        packed = torch.empty(gist.gist_dpr_words(n, bits), dtype=torch.int32, device=dev)
        b = 4 * n + 4 * gist.gist_dpr_words(n, bits)
        rep("a6", f"fp{bits} 205.5M elems", b, lambda: gist.gist_dpr_encode(x, bits, packed=packed))
        rep("a7", f"fp{bits} 205.5M elems", b, lambda: gist.gist_dpr_decode(packed, n, bits, x=xd))
        del packed
    clocks.__exit__(None, None, None)
    clk = clocks.summary()
    print(json.dumps({"clocks": clk}), flush=True)
    if args.json:
        with open(args.json, "w") as f:
            json.dump({"peak_GBps": peak, "peak_source": src, "gpu": torch.cuda.get_device_name(dev),
                       "clocks": clk, "results": res}, f, indent=1)


if __name__ == "__main__":
    main()
