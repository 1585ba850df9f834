"""Multi-process (world_size 2, gloo, CPU) coverage of the data-parallel host logic
(SURVEY.md §8(e)): minibatch sharding has no exchange step, so the per-rank encodings of a
rank's image range, tallied with one all_reduce (SUM of byte counters, MAX of time), must
equal the single-process encoding of the whole minibatch.  Encodings here come from the
oracle (no GPU in CI); bench.py runs the same sharding + tally over NCCL with the kernels."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_isca_jainpmtp18_b200.shard import shard_bounds, tally

BATCH, C, H, W = 6, 8, 14, 14
G = (3, 3, 2, 2, 0, 0, 1)


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def encode_images(lo, hi):
    """Byte counters of encoding images [lo, hi) (per-image seeds: content independent of the
    sharding)."""
    import oracle as ref
    import workloads as WL
    cnt = {"fp32_bytes": 0, "binarize_bytes": 0, "ssdc_bytes": 0, "dpr_bytes": 0, "nnz": 0}
    for img in range(lo, hi):
        y = WL.relu_map((1, C, H, W), 0.5, 100 + img).numpy()
        x = WL.relu_map((1, C, H, W), 0.8, 200 + img).numpy()
        d = WL.dpr_map((1, C, H, W), 300 + img).numpy()
        _, arg = ref.maxpool_fwd_argmax(y, G)
        mask = ref.binarize_encode(y)
        row_end, col, val = ref.ssdc_encode(x)
        packed = ref.dpr_encode(d, 10)
        cnt["fp32_bytes"] += 4 * (y.size + x.size + d.size)
        cnt["binarize_bytes"] += mask.nbytes + arg.nbytes
        cnt["ssdc_bytes"] += row_end.nbytes + col.nbytes + val.nbytes
        cnt["dpr_bytes"] += packed.nbytes
        cnt["nnz"] += col.size
    return cnt


def worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    lo, hi = shard_bounds(BATCH, world, rank)
    cnt = encode_images(lo, hi)
    totals, tmax = tally(dist, cnt, elapsed_ms=10.0 * (rank + 1))
    if rank == 0:
        out.put((totals, tmax))
    dist.barrier()
    dist.destroy_process_group()


def test_shard_bounds_partition():
    for batch in (1, 7, 64, 256):
        for world in (1, 2, 3, 4, 8):
            spans = [shard_bounds(batch, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == batch
            assert all(a[1] == b[0] for a, b in zip(spans, spans[1:]))
            sizes = [hi - lo for lo, hi in spans]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        shard_bounds(8, 2, 2)


def test_two_rank_gloo_tally_equals_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    totals, tmax = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    single, t1 = tally(None, encode_images(0, BATCH), elapsed_ms=10.0)
    assert totals == single
    assert tmax == 20.0  # MAX over ranks, not a sum
    # per-encoding compression ratios from the tally
    assert single["fp32_bytes"] > 0 and single["nnz"] > 0
