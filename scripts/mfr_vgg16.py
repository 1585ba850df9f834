#!/usr/bin/env python
"""Memory footprint ratio (MFR) and step overhead of Gist's stash-time encodings on
one random-init VGG16 training step (batch 64, 224x224 synthetic images).

Baseline: a plain VGG16 (conv / relu / max_pool2d / linear) whose stash is fp32 feature maps.
Gist: the same weights, with relu->maxpool as Binarize (mask + argmax), relu->conv and pool->conv
as SSDC, and every other stashed activation as DPR (FP16 for VGG16).  Reported: peak
CUDA memory of forward+backward (torch.cuda.max_memory_allocated, parameters and their grads
included, as in a real step), time per step, and the max relative gradient error vs baseline.

  python scripts/mfr_vgg16.py [--batch 64] [--bits 16] [--lossless]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import torch.nn as nn  # noqa: E402
import torch.nn.functional as F  # noqa: E402

from paper_conf_isca_jainpmtp18_b200 import stash  # noqa: E402

CFG = [(3, 64, 2), (64, 128, 2), (128, 256, 3), (256, 512, 3), (512, 512, 3)]
# SSDC-stashed maps per image in forward_gist: (channels, side) of every relu->conv and pool->conv input
SSDC_SHAPES = [(cout, 224 >> b) for b, (_, cout, k) in enumerate(CFG) for _ in range(k - 1)] + \
    [(cin, 224 >> b) for b, (cin, _, _) in enumerate(CFG) if b > 0]


class VGG16(nn.Module):
    def __init__(self, num_classes=1000):
        super().__init__()
        self.convs = nn.ModuleList()
        for cin, cout, k in CFG:
            for i in range(k):
                self.convs.append(nn.Conv2d(cin if i == 0 else cout, cout, 3, padding=1))
        self.fc6 = nn.Linear(512 * 7 * 7, 4096)
        self.fc7 = nn.Linear(4096, 4096)
        self.fc8 = nn.Linear(4096, num_classes)

    def forward_baseline(self, x):
        c = 0
        for _, _, k in CFG:
            for _ in range(k):
                x = F.relu(self.convs[c](x))
                c += 1
            x = F.max_pool2d(x, 2, 2)
        x = torch.flatten(x, 1)
        x = F.relu(self.fc6(x))
        x = F.relu(self.fc7(x))
        return self.fc8(x)

    def forward_gist(self, x, bits, lossless=False, plan=None):
        # DPR (lossy) wraps everything; the Binarize/SSDC functions save only their encodings;
        # with an arena plan each block's SSDC stashes are single-pass appends into the block's own
        # arena (no host sync in the forward; freed once the block's backward has decoded them)
        ctx = stash.dpr_saved_tensors(bits, self.parameters()) if not lossless else _null()
        with ctx:
            c = 0
            z = self.convs[0](x)  # the input image: an "other" stashed map (DPR)
            c = 1
            for b, (cin, cout, k) in enumerate(CFG):
                side = 224 >> b
                default = x.shape[0] * side * side * ((k - 1) * cout + (cin if b else 0)) * 6 // 10
                actx = stash.ssdc_arena(plan.arena(b, default)) if plan is not None else _null()
                with actx:
                    for i in range(1 if b == 0 else 0, k):
                        conv = self.convs[c]
                        c += 1
                        if i == 0:  # pool -> conv: SSDC of the pool output
                            z = stash.stashed_conv(z, conv)
                        else:  # relu -> conv: SSDC of the ReLU output
                            z = stash.relu_conv(z, conv)
                z = stash.relu_maxpool(z, 2, 2)  # relu -> maxpool: Binarize
            z = torch.flatten(z, 1)
            z = F.relu(self.fc6(z))
            z = F.relu(self.fc7(z))
            return self.fc8(z)


class _null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


def step(model, x, target, fwd, marks=None):
    model.zero_grad(set_to_none=True)
    plan = ARENA.get("plan")
    try:
        loss = F.cross_entropy(fwd(x), target)
        out = _finish(loss, marks)
    except stash.StashOverflow:  # a block's arena was too small: resize from this step's ends, redo
        if plan is None:
            raise
        loss = None
        ARENA["last"] = plan.update()
        ARENA["grown"] = ARENA.get("grown", 0) + 1
        model.zero_grad(set_to_none=True)
        loss = F.cross_entropy(fwd(x), target)
        out = _finish(loss, marks)
    if plan is not None:
        ARENA["last"] = plan.update()  # one host read per step, after the backward
    return out


ARENA = {}


def _finish(loss, marks):
    if marks is not None:  # the stash: everything alive between the forward and the backward
        torch.cuda.synchronize()
        marks["after_forward_bytes"] = torch.cuda.memory_allocated()
        marks["forward_peak_bytes"] = torch.cuda.max_memory_allocated()
        torch.cuda.reset_peak_memory_stats()
    loss.backward()
    if marks is not None:
        torch.cuda.synchronize()
        marks["backward_peak_bytes"] = torch.cuda.max_memory_allocated()
    return loss.detach()


def measure(model, x, target, fwd, reps=5):
    step(model, x, target, fwd)  # warm-up (cuDNN algorithm selection, allocator)
    torch.cuda.synchronize()
    model.zero_grad(set_to_none=True)
    torch.cuda.empty_cache()
    torch.cuda.reset_peak_memory_stats()
    base = torch.cuda.memory_allocated()
    marks = {}
    loss = step(model, x, target, fwd, marks)
    torch.cuda.synchronize()
    peak = max(marks["forward_peak_bytes"], marks["backward_peak_bytes"])
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        step(model, x, target, fwd)
    b.record()
    torch.cuda.synchronize()
    return {"peak_bytes": peak, "peak_above_inputs_bytes": peak - base,
            "stash_bytes": marks["after_forward_bytes"] - base, "forward_peak_bytes": marks["forward_peak_bytes"],
            "backward_peak_bytes": marks["backward_peak_bytes"], "ms_per_step": a.elapsed_time(b) / reps,
            "loss": float(loss)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=64)
    ap.add_argument("--bits", type=int, default=16)
    ap.add_argument("--lossless", action="store_true", help="Binarize + SSDC only (no DPR)")
    ap.add_argument("--json", default=None)
    ap.add_argument("--no-arena", dest="arena", action="store_false",
                    help="exact-size SSDC stashes (count pass + host read of nnz per conv) instead of the arena")
    ap.add_argument("--cap-gb", type=float, default=None,
                    help="largest-minibatch mode: cap the process at this many GB (P:38: Gist fits larger "
                         "minibatches) and search the largest batch each arm can train")
    ap.add_argument("--bias-shift", type=float, default=0.0,
                    help="subtract this from every conv bias (x the layer's output std) to emulate the >80%% ReLU "
                         "sparsity of trained VGG16 (P:76); 0 = plain random init (~50%%)")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    torch.backends.cudnn.benchmark = False
    torch.manual_seed(0)
    model = VGG16().to(dev)
    # ReLU-like feature maps need real sparsity: a random-init VGG16 gives ~50% ReLU zeros
    x = torch.randn(args.batch, 3, 224, 224, device=dev)
    target = torch.randint(0, 1000, (args.batch,), device=dev)
    if args.bias_shift:
        with torch.no_grad():  # calibrate each conv bias on one forward so P(relu(z) > 0) drops
            h = x[:4]
            c = 0
            for _, _, k in CFG:
                for _ in range(k):
                    z = model.convs[c](h)
                    model.convs[c].bias -= args.bias_shift * z.std(dim=(0, 2, 3))
                    h = F.relu(model.convs[c](h))
                    c += 1
                h = F.max_pool2d(h, 2, 2)
    with torch.no_grad():  # measured ReLU sparsity of the conv outputs
        h, zs, c = x[:4], [], 0
        for _, _, k in CFG:
            for _ in range(k):
                h = F.relu(model.convs[c](h))
                zs.append(float((h == 0).float().mean()))
                c += 1
            h = F.max_pool2d(h, 2, 2)
    args.sparsity_note = {"mean": round(sum(zs) / len(zs), 3), "per_conv": [round(v, 3) for v in zs]}

    if args.cap_gb:
        total = torch.cuda.get_device_properties(dev).total_memory
        torch.cuda.set_per_process_memory_fraction(args.cap_gb * 1e9 / total, dev)
        res = {}
        for name, fwd in (("baseline", model.forward_baseline),
                          ("gist", lambda t: model.forward_gist(t, args.bits, args.lossless))):
            best = 0
            for bsz in (16, 24, 32, 48, 64, 80, 96, 112, 128, 160, 192, 224, 256):
                torch.cuda.empty_cache()
                try:
                    xb = torch.randn(bsz, 3, 224, 224, device=dev)
                    tb = torch.randint(0, 1000, (bsz,), device=dev)
                    step(model, xb, tb, fwd)
                    torch.cuda.synchronize()
                    best = bsz
                except torch.OutOfMemoryError:
                    break
                finally:
                    xb = tb = None
                    model.zero_grad(set_to_none=True)
            res[name] = best
        out = {"model": "VGG16 random init", "cap_gb": args.cap_gb, "largest_batch": res,
               "encodings": "Binarize + SSDC" + ("" if args.lossless else f" + DPR-fp{args.bits}"),
               "relu_sparsity_mean": args.sparsity_note["mean"],
               "batch_ratio": round(res["gist"] / max(1, res["baseline"]), 3)}
        print(json.dumps(out, indent=1))
        if args.json:
            with open(args.json, "w") as f:
                json.dump(out, f, indent=1)
        return

    base = measure(model, x, target, model.forward_baseline)
    g_base = [p.grad.clone() for p in model.parameters()]
    if args.arena:  # per-block arenas sized from the previous step (60% of the elements at first)
        ARENA["plan"] = stash.ArenaPlan(dev)
    gist = measure(model, x, target, lambda t: model.forward_gist(t, args.bits, args.lossless, ARENA.get("plan")))
    g_gist = [p.grad for p in model.parameters()]
    rel = max(float((a - b).abs().max() / (a.abs().max() + 1e-30)) for a, b in zip(g_base, g_gist))
    out = {
        "model": "VGG16 random init", "batch": args.batch, "image": 224,
        "encodings": "Binarize + SSDC" + ("" if args.lossless else f" + DPR-fp{args.bits}"),
        "baseline": base, "gist": gist,
        "ssdc_stash": ({"mode": "per-block arenas (one encode pass per stash, no host sync in the forward; "
                                "capacities from the previous step, one host read per step after the backward)",
                        "blocks_used_capacity": {str(k): v for k, v in ARENA.get("last", {}).items()},
                        "regrown_steps": ARENA.get("grown", 0)} if args.arena else
                       {"mode": "exact-size (count pass + host read of nnz + encode pass per stash)"}),
        "mfr_peak": round(base["peak_bytes"] / gist["peak_bytes"], 3),
        "mfr_above_inputs": round(base["peak_above_inputs_bytes"] / gist["peak_above_inputs_bytes"], 3),
        "stash_ratio": round(base["stash_bytes"] / gist["stash_bytes"], 3),
        "relu_sparsity": args.sparsity_note,
        "cudnn_workspace_cap_mib": os.environ.get("CUDNN_CONV_WSCAP_DBG"),
        "step_overhead": round(gist["ms_per_step"] / base["ms_per_step"] - 1.0, 4),
        "max_rel_grad_diff_vs_baseline": rel,
    }
    print(json.dumps(out, indent=1))
    if args.json:
        with open(args.json, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
