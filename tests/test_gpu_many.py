"""Many maps per launch (gist_*_many, "these conversions can happen in parallel"): every
job's outputs equal the oracle's for that map, bit for bit, including ragged sizes, empty maps,
capacity truncation, more jobs than one launch holds, and the chained stash arena (append mode)."""
import numpy as np
import pytest
import torch

import workloads as WL

pytestmark = pytest.mark.gpu


def host(t):
    return t.detach().cpu().numpy()


def same(got, expect, what):
    got, expect = np.ascontiguousarray(got).view(np.uint8), np.ascontiguousarray(expect).view(np.uint8)
    assert got.shape == expect.shape and np.array_equal(got, expect), what


SIZES = [1, 255, 8193, 256 * 32 * 70 + 5, 0, 200_704, 1_000_003, 256 * 32, 3]


def maps(sizes, seed, cuda):
    return [WL.relu_map((n,), [0.0, 0.5, 0.8, 0.9, 1.0][k % 5], seed + k, cuda, negative_zero=True) if n else
            torch.empty(0, device=cuda) for k, n in enumerate(sizes)]


def test_ssdc_encode_decode_many(gist, ref, cuda):
    xs = maps(SIZES, 10, cuda)
    caps = [None, None, 100, None, None, None, 12345, None, None]
    plan = gist.SsdcEncodeMany([{"x": x, "capacity": c} for x, c in zip(xs, caps)])
    for rep in range(2):  # the workspace is reused by the second call
        outs = plan()
        torch.cuda.synchronize()
        for k, (x, (row_end, col, val, nnz)) in enumerate(zip(xs, outs)):
            r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
            m = r_col.size
            assert int(nnz.item()) == m, (rep, k)
            same(host(row_end), r_row_end, f"row_end {k}")
            cap = m if caps[k] is None else min(caps[k], m)
            same(host(col)[:cap], r_col[:cap], f"col {k}")
            same(host(val)[:cap], r_val[:cap], f"val {k}")
    backs = gist.gist_ssdc_decode_many([{"row_end": o[0], "col": o[1], "val": o[2], "n": x.numel()}
                                        for x, o, c in zip(xs, outs, caps) if c is None])
    for x, b in zip([x for x, c in zip(xs, caps) if c is None], backs):
        assert torch.equal(b.view(torch.int32), x.view(torch.int32))


def test_ssdc_many_more_jobs_than_one_launch(gist, ref, cuda):
    sizes = [256 * (k % 7) + 31 * k + 1 for k in range(130)]  # 130 maps: 3 encode launches, 3 decode
    xs = maps(sizes, 77, cuda)
    plan = gist.SsdcEncodeMany([{"x": x} for x in xs])  # (initialises its workspace: one launch)
    launches0 = gist.gist_launch_count()
    outs = plan()
    assert gist.gist_launch_count() - launches0 == 3  # 48 + 48 + 34 maps
    dec = gist.SsdcDecodeMany([{"row_end": o[0], "col": o[1], "val": o[2], "n": x.numel()} for x, o in zip(xs, outs)])
    launches0 = gist.gist_launch_count()
    backs = dec()
    assert gist.gist_launch_count() - launches0 == 3  # 64 + 64 + 2 maps
    torch.cuda.synchronize()
    for k, (x, (row_end, col, val, nnz), b) in enumerate(zip(xs, outs, backs)):
        r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
        assert int(nnz.item()) == r_col.size
        same(host(row_end), r_row_end, f"row_end {k}")
        same(host(col)[:r_col.size], r_col, f"col {k}")
        assert torch.equal(b.view(torch.int32), x.view(torch.int32)), k


@pytest.mark.parametrize("start", [0, 13])
def test_ssdc_chained_arena(gist, ref, cuda, start):
    """Append mode: map k's entries follow map k-1's in one arena (offset = previous nnz), all in
    one launch; row_end is absolute; decode takes the same offsets.  The arena holds exactly
    sum(nnz) entries after `start`: no host synchronization sizes it."""
    sizes = [256 * 32 * 40 + 7, 5000, 1, 256 * 33, 777_777]
    xs = maps(sizes, 5, cuda)
    cap = start + sum(sizes)
    extra = 9999  # room for the single-job append at the end
    col = torch.zeros(cap + extra, dtype=torch.uint8, device=cuda)
    val = torch.zeros(cap + extra, dtype=torch.float32, device=cuda)
    offs = torch.zeros(len(sizes) + 1, dtype=torch.int64, device=cuda)
    offs[0] = start
    jobs = [{"x": x, "col": col, "val": val, "capacity": cap, "offset": offs[k:k + 1], "nnz": offs[k + 1:k + 2]}
            for k, x in enumerate(xs)]
    outs = gist.gist_ssdc_encode_many(jobs)
    torch.cuda.synchronize()
    o = offs.tolist()
    for k, x in enumerate(xs):
        r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
        assert o[k + 1] - o[k] == r_col.size, k
        same(host(outs[k][0]), (r_row_end.astype(np.int64) + o[k]).astype(np.int32), f"row_end {k}")
        same(host(col[o[k]:o[k + 1]]), r_col, f"col {k}")
        same(host(val[o[k]:o[k + 1]]), r_val, f"val {k}")
    backs = gist.gist_ssdc_decode_many([{"row_end": outs[k][0], "col": col, "val": val, "offset": offs[k:k + 1],
                                         "n": x.numel()} for k, x in enumerate(xs)])
    for x, b in zip(xs, backs):
        assert torch.equal(b.view(torch.int32), x.view(torch.int32))
    # single-job append mode (offset known from an earlier call)
    more = WL.relu_map((extra,), 0.6, 99, cuda)
    tail = torch.zeros(1, dtype=torch.int64, device=cuda)
    rows = gist.gist_ssdc_encode_many([{"x": more, "col": col, "val": val, "capacity": cap + extra,
                                        "offset": offs[-1:], "nnz": tail}])
    t = int(tail.item())
    r_row_end, r_col, r_val = ref.ssdc_encode(host(more))
    assert t - o[-1] == r_col.size
    same(host(rows[0][0]), (r_row_end.astype(np.int64) + o[-1]).astype(np.int32), "append row_end")
    same(host(col[o[-1]:t]), r_col, "append col")
    same(host(val[o[-1]:t]), r_val, "append val")


@pytest.mark.parametrize("bits", [16, 10, 8])
def test_dpr_many(gist, ref, cuda, bits):
    sizes = [1, 7, 383, 384, 385, 1000, 65537, 0, 200_704, 1_000_003, 11]
    xs = [WL.dpr_map((n,), n + bits, cuda) for n in sizes]
    packed = gist.gist_dpr_encode_many(xs, bits)
    backs = gist.gist_dpr_decode_many(packed, sizes, bits)
    for k, (x, p, b) in enumerate(zip(xs, packed, backs)):
        r = ref.dpr_encode(host(x), bits)
        same(host(p), r, f"fp{bits} words {k}")
        same(host(b), ref.dpr_decode(r, x.numel(), bits), f"fp{bits} decode {k}")


def test_dpr_many_more_jobs_than_one_launch(gist, ref, cuda):
    sizes = [37 * k + 5 for k in range(200)]
    xs = [WL.dpr_map((n,), n, cuda) for n in sizes]
    packed = gist.gist_dpr_encode_many(xs, 10)
    backs = gist.gist_dpr_decode_many(packed, sizes, 10)
    for k, (x, p, b) in enumerate(zip(xs, packed, backs)):
        r = ref.dpr_encode(host(x), 10)
        same(host(p), r, f"words {k}")
        same(host(b), ref.dpr_decode(r, x.numel(), 10), f"decode {k}")
