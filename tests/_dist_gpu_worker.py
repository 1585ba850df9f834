"""Worker for tests/test_gpu_dist.py, launched under torchrun with 2 ranks on ONE GPU (gloo for the
tally; the hot path has no collective).  Each rank runs bench.py's Workload step
(the libgist kernels through the C ABI) on its shard of a strong-scaled GoogLeNet-shaped minibatch
(C4's split, shard_bounds) and checks every encoding and decoded map against the oracle on that
rank's shard; the cross-rank tally must equal the single-process count of the whole minibatch."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import bench  # noqa: E402
import oracle as ref  # noqa: E402
import paper_conf_isca_jainpmtp18_b200 as gist  # noqa: E402
import workloads as WL  # noqa: E402
from paper_conf_isca_jainpmtp18_b200.shard import shard_bounds, tally  # noqa: E402

BATCH = 5  # global minibatch (odd: the ranks get 3 and 2 images)
SITES = 9  # the stem, and the first inception module's sites (every encoding kind and pool geometry)


def same(a, b, what):
    a = np.ascontiguousarray(a).view(np.uint8)
    b = np.ascontiguousarray(b).view(np.uint8)
    if a.shape != b.shape or not np.array_equal(a, b):
        raise SystemExit(f"rank {dist.get_rank()}: {what} differs from the oracle")


def main():
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    cfg = WL.CONFIGS["C4"]
    lo, hi = shard_bounds(BATCH, world, rank)
    full_sites = WL.sites_for(cfg)
    wl = bench.Workload(gist, cfg, range(lo, hi), cfg.sparsity, cfg.dpr_bits, dev, True)
    wl.sites = wl.sites[:SITES]
    # inputs are seeded per GLOBAL image: this shard equals its slice of the whole minibatch
    whole = bench.Workload(gist, cfg, range(BATCH), cfg.sparsity, cfg.dpr_bits, dev, True)
    for d, w in zip(wl.sites, whole.sites[:SITES]):
        assert torch.equal(d["y"], w["y"][lo:hi]), d["site"].name
    del whole
    # one step, keeping each decoded map (the bench reuses one scratch buffer)
    g, nnz_mine = gist, 0
    for d in wl.sites:
        s = d["site"]
        yh = d["y"].cpu().numpy()
        if s.kind in ("relu_pool", "pool_only"):
            g.gist_maxpool_fwd_argmax(d["y"], s.pool, out=d["out"], argmax=d["arg"], mask=d["mask"])
            dx = g.gist_pool_relu_bwd(d["dY"], d["arg"], d["mask"], d["shape"], s.pool)
            r_out, r_arg = ref.maxpool_fwd_argmax(yh, s.pool)
            r_mask = ref.binarize_encode(yh) if d["mask"] is not None else None
            same(d["out"].cpu().numpy(), r_out, f"{s.name} out")
            same(d["arg"].cpu().numpy(), r_arg, f"{s.name} argmax")
            if r_mask is not None:
                same(d["mask"].cpu().numpy(), r_mask, f"{s.name} mask")
            same(dx.cpu().numpy(), ref.pool_relu_bwd(d["dY"].cpu().numpy(), r_arg, r_mask, d["shape"], s.pool),
                 f"{s.name} dx")
        elif s.kind == "ssdc":
            g.gist_ssdc_encode(d["y"], capacity=d["n"], row_end=d["row_end"], col=d["col"], val=d["val"],
                               nnz=d["nnz"], workspace=d["ws"])
            back = g.gist_ssdc_decode(d["row_end"], d["col"], d["val"], d["n"])
            r_row_end, r_col, r_val = ref.ssdc_encode(yh)
            k = int(d["nnz"].item())
            assert k == r_col.size, s.name
            nnz_mine += k
            same(d["row_end"].cpu().numpy(), r_row_end, f"{s.name} row_end")
            same(d["col"][:k].cpu().numpy(), r_col, f"{s.name} col")
            same(d["val"][:k].cpu().numpy(), r_val, f"{s.name} val")
            same(back.cpu().numpy(), yh.reshape(-1), f"{s.name} round trip")
        else:
            g.gist_dpr_encode(d["y"], wl.bits, packed=d["packed"])
            back = g.gist_dpr_decode(d["packed"], d["n"], wl.bits)
            r_p = ref.dpr_encode(yh, wl.bits)
            same(d["packed"].cpu().numpy(), r_p, f"{s.name} dpr words")
            same(back.cpu().numpy(), ref.dpr_decode(r_p, d["n"], wl.bits), f"{s.name} dpr decode")
    torch.cuda.synchronize()
    fp32 = 4 * sum(d["n"] for d in wl.sites)
    totals, tmax = tally(dist, {"fp32_bytes": fp32, "nnz": nnz_mine}, elapsed_ms=1.0 + rank)
    if rank == 0:
        # single-process count of the whole minibatch (oracle)
        n_all, nnz_all = 0, 0
        for si, s in enumerate(full_sites[:SITES]):
            n_all += s.numel(BATCH)
            if s.kind == "ssdc":
                seed0 = WL.image_seed(bench.CONFIG_INDEX["C4"], si, 0)
                y = WL.per_image(lambda sh, sd, dv: WL.relu_map(sh, cfg.sparsity, sd, dv), s.chw, range(BATCH), seed0,
                                 dev)
                nnz_all += ref.ssdc_encode(y.cpu().numpy())[1].size
        assert totals["fp32_bytes"] == 4 * n_all, (totals, n_all)
        assert totals["nnz"] == nnz_all, (totals, nnz_all)
        assert tmax == float(world), tmax
        print(f"dist OK: {world} ranks, shards {[shard_bounds(BATCH, world, r) for r in range(world)]}, "
              f"nnz {nnz_all}", flush=True)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
