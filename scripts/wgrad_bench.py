#!/usr/bin/env python
"""f4 measurement: the decode-in-GEMM weight gradient (gist_conv3x3_wgrad_ssdc) on VGG16 convs at
batch 64, against the unfused path (SSDC decode to a dense fp32 buffer + cuDNN's weight gradient).

TFLOP/s counts the GEMM's useful work 2*Co*Ci*9*N*H*W; the tensor roofline is TF32:
MEASURED_PEAKS.json bf16_tflops x (1.13/2.25), the guide's nominal TF32:BF16 ratio.  3xTF32 issues
three TF32 MMAs per useful product, so its attainable ceiling is 1/3 of that peak.

  python scripts/wgrad_bench.py [--reps 20] [--json out.json] [--layers conv3_2,...]
"""
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

LAYERS = {  # name: (N, Ci, Co, H, W); X = the ReLU output feeding the conv (SSDC site)
    "conv2_2": (64, 128, 128, 112, 112),
    "conv3_2": (64, 256, 256, 56, 56),
    "conv4_2": (64, 512, 512, 28, 28),
    "conv5_2": (64, 512, 512, 14, 14),
}


def timeit(fn, reps, stream):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(reps):
        a.record(stream)
        fn()
        b.record(stream)
        b.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--json", default=None)
    ap.add_argument("--layers", default=",".join(LAYERS))
    ap.add_argument("--sparsity", type=float, default=0.8)
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream(dev)
    with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
        peaks = json.load(f)
    tf32_peak = peaks["bf16_tflops"] * 1.13 / 2.25
    out = {"tf32_peak_tflops": round(tf32_peak, 1), "peak_source": "MEASURED_PEAKS.json bf16_tflops x 1.13/2.25",
           "sparsity": args.sparsity, "layers": {}}
    with bench.ClockSampler(dev) as clocks:
        for name in args.layers.split(","):
            N, Ci, Co, H, W = LAYERS[name]
            x = WL.relu_map((N, Ci, H, W), args.sparsity, 77, dev)
            dy = WL.grad_map((N, Co, H, W), 78, dev)
            row_end, col, val, nnz = gist.gist_ssdc_encode(x, trim=True)
            flops = 2.0 * Co * Ci * 9 * N * H * W
            dw = torch.empty((Co, Ci, 3, 3), device=dev)
            ws = torch.empty(gist.gist_conv3x3_wgrad_workspace_bytes(N, Ci, Co, H, W), dtype=torch.uint8, device=dev)
            r = {"shape": [N, Ci, Co, H, W], "gflop": round(flops / 1e9, 2), "nnz": int(nnz.item()),
                 "csr_bytes": 5 * int(nnz.item()) + 4 * row_end.numel(), "dense_x_bytes_avoided": 4 * x.numel()}
            for passes in (3, 1):
                ms = timeit(lambda: gist.gist_conv3x3_wgrad_ssdc(dy, row_end, col, val, x.shape, passes, dw=dw,
                                                                 workspace=ws), args.reps, stream)
                tf = flops / ms / 1e9
                ceil = tf32_peak / passes
                r[f"gist_{passes}xtf32"] = {"ms": round(ms, 4), "tflops": round(tf, 1),
                                            "frac_tf32_peak": round(tf / tf32_peak, 4),
                                            "frac_of_attainable": round(tf / ceil, 4)}
            # unfused baseline: decode to dense fp32, then cuDNN's weight gradient (fp32 and TF32)
            xd = torch.empty_like(x)

            def unfused():
                gist.gist_ssdc_decode(row_end, col, val, x.numel(), x=xd.view(-1))
                torch.ops.aten.convolution_backward(dy, xd, dw, None, [1, 1], [1, 1], [1, 1], False, [0, 0], 1,
                                                    [False, True, False])
            for tf32 in (False, True):
                torch.backends.cudnn.allow_tf32 = tf32
                ms = timeit(unfused, max(5, args.reps // 2), stream)
                r[f"decode+cudnn_{'tf32' if tf32 else 'fp32'}"] = {"ms": round(ms, 4), "tflops": round(flops / ms / 1e9, 1)}
            torch.backends.cudnn.allow_tf32 = True
            out["layers"][name] = r
            print(name, json.dumps(r), flush=True)
            del x, dy, xd, ws, row_end, col, val
            torch.cuda.empty_cache()
    out["clocks"] = clocks.summary()
    print(json.dumps(out["clocks"]))
    if args.json:
        with open(args.json, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
