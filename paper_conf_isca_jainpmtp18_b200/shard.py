"""Data-parallel sharding of the stash-time encode/decode path.

Every encoding is a pure function of one rank's own minibatch tensor: pool windows never cross
an image boundary in NCHW, SSDC rows and packing words are cut from the rank's own shard, so the
hot path has no exchange step.  Ranks take contiguous image ranges; the only collective is an
after-the-fact footprint tally (sum of byte counters, max of elapsed time), which runs over
whatever process group the caller initialised (NCCL on the GPU box, gloo in CPU tests).
"""
from __future__ import annotations

import torch


def shard_bounds(batch: int, world: int, rank: int) -> tuple[int, int]:
    """Images [lo, hi) of rank `rank` when `batch` images are split over `world` ranks
    (strong scaling: C4's 64 images over 1/2/4/8 GPUs).  The first batch % world ranks take
    one extra image."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    base, extra = divmod(batch, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


TALLY_FIELDS = ("fp32_bytes", "binarize_bytes", "ssdc_bytes", "dpr_bytes", "nnz")


def tally(dist, counters: dict, elapsed_ms: float, device=None) -> tuple[dict, float]:
    """Cross-rank footprint tally: SUM of the int64 counters, MAX of elapsed time.
    `dist` is torch.distributed (initialised) or None for a single process."""
    vec = torch.tensor([int(counters.get(f, 0)) for f in TALLY_FIELDS], dtype=torch.int64, device=device)
    t = torch.tensor([float(elapsed_ms)], dtype=torch.float64, device=device)
    if dist is not None and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(vec, op=dist.ReduceOp.SUM)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return dict(zip(TALLY_FIELDS, (int(v) for v in vec.tolist()))), float(t.item())
