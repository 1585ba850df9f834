"""GPU parity: every CUDA kernel, called through the C ABI (Python binding), against the
CPU oracle on the same seeded inputs — bit-exact (the north star's bar: encodings and
recomputed gradients identical; no float reduction order differs, reading R6).

Sizes span several tiles/warps with ragged tails; the full-size cases use BASELINE.json's
configurations in the launch configuration bench.py times."""
import numpy as np
import pytest
import torch

import workloads as WL
from pool_cases import GEOMS, gid

pytestmark = pytest.mark.gpu


def host(t):
    return t.detach().cpu().numpy()


def u32(a):
    return np.ascontiguousarray(a).view(np.uint32)


def assert_bits_equal(got, expect, what=""):
    got, expect = np.ascontiguousarray(got), np.ascontiguousarray(expect)
    assert got.shape == expect.shape, (what, got.shape, expect.shape)
    g, e = got.view(np.uint8), expect.view(np.uint8)
    if not np.array_equal(g, e):
        bad = np.flatnonzero(got.reshape(-1).view(np.uint32 if got.itemsize == 4 else np.uint8)
                             != expect.reshape(-1).view(np.uint32 if expect.itemsize == 4 else np.uint8))
        raise AssertionError(f"{what}: {bad.size} mismatches, first at {bad[:8]}")


def mixed_values(n, seed, device):
    g = torch.Generator(device=device).manual_seed(seed)
    x = torch.randn(n, generator=g, device=device)
    r = torch.rand(n, generator=g, device=device)
    x = torch.where(r < 0.3, torch.zeros_like(x), x)
    x = torch.where((r >= 0.3) & (r < 0.35), torch.full_like(x, -0.0), x)
    x = torch.where((r >= 0.35) & (r < 0.36), torch.full_like(x, float("nan")), x)
    x = torch.where((r >= 0.36) & (r < 0.37), torch.full_like(x, float("inf")), x)
    x = torch.where((r >= 0.37) & (r < 0.38), torch.full_like(x, -float("inf")), x)
    return x


RAGGED = [1, 7, 31, 32, 33, 255, 256, 257, 1000, 1023, 1024, 1025, 4097, 8191, 8192, 8193, 65537,
          200_704, 1_000_003]


# ------------------------------------------------------------------------ a1 Binarize
@pytest.mark.parametrize("n", RAGGED)
def test_binarize(gist, ref, cuda, n):
    y = mixed_values(n, n, cuda)
    got = gist.gist_binarize_encode(y)
    torch.cuda.synchronize()
    assert_bits_equal(host(got), ref.binarize_encode(host(y)), "mask")


def test_binarize_offset_views_rejected(gist, cuda):
    y = torch.zeros(1000, device=cuda)
    with pytest.raises(gist.GistError):
        gist.gist_binarize_encode(y[1:])  # 4-byte offset -> GIST_ERR_MISALIGNED


# ------------------------------------------------------------------------ a2/a3 pooling
def pool_case(shape, g, seed, cuda, ties=True):
    y = WL.relu_map(shape, 0.5, seed, cuda)
    if ties:  # quantize so windows hold exact ties; plant -inf / NaN / -0.0
        y = torch.round(y * 2) / 2
        r = torch.rand(shape, generator=torch.Generator(device=cuda).manual_seed(seed + 1), device=cuda)
        y = torch.where(r < 0.01, torch.full_like(y, float("nan")), y)
        y = torch.where((r >= 0.01) & (r < 0.03), torch.full_like(y, -float("inf")), y)
        y = torch.where((r >= 0.03) & (r < 0.1), torch.full_like(y, -0.0), y)
    return y


SHAPES = [(1, 1, 5, 7), (2, 3, 13, 13), (1, 64, 56, 56), (2, 5, 27, 27), (1, 7, 14, 14), (3, 2, 55, 55),
          (1, 3, 9, 16), (2, 4, 12, 24), (1, 1, 1, 1), (2, 3, 8, 32), (1, 5, 6, 16), (1, 2, 10, 112),
          # fused 2x2/s2 + mask: several word-aligned units with a partial last one (V = 2 and 4),
          # tiny rows, and a row too wide for one unit (fallback)
          (2, 9, 14, 14), (3, 7, 28, 28), (1, 3, 6, 6), (1, 1, 2, 2050)]


@pytest.mark.parametrize("g", GEOMS, ids=gid)
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: "x".join(map(str, s)))
def test_maxpool_fwd_and_fused_bwd(gist, ref, cuda, g, shape):
    N, Cc, H, W = shape
    if H + 2 * g[4] < g[0] or W + 2 * g[5] < g[1]:
        pytest.skip("window larger than padded input")
    y = pool_case(shape, g, sum(shape) + g[0], cuda)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, g, fuse_mask=True)
    r_out, r_arg = ref.maxpool_fwd_argmax(host(y), g)
    assert_bits_equal(host(out), r_out, "out")
    assert_bits_equal(host(arg), r_arg, "argmax")
    assert_bits_equal(host(mask), ref.binarize_encode(host(y)), "fused mask")
    dout = WL.grad_map(tuple(out.shape), 7, cuda)
    dout = torch.where(torch.rand_like(dout) < 0.05, torch.full_like(dout, -0.0), dout)
    for m, rm in ((mask, ref.binarize_encode(host(y))), (None, None)):
        dx = gist.gist_pool_relu_bwd(dout, arg, m, shape, g)
        r_dx = ref.pool_relu_bwd(host(dout), r_arg, rm, shape, g)
        assert_bits_equal(host(dx), r_dx, "dx" + (" (pool-only)" if m is None else ""))


@pytest.mark.parametrize("shape", [(64, 192, 28, 28), (64, 480, 14, 14), (64, 832, 7, 7), (5, 37, 9, 11)],
                         ids=lambda s: "x".join(map(str, s)))
def test_pool3s1_full_googlenet_sizes(gist, ref, cuda, shape):
    """GoogLeNet's in-module 3x3/s1/p1 pools at batch 64 (C4): the plane-group backward stages
    many planes per group (odd plane sizes give every argmax-word and mask-word phase) and a
    partial last group; pool-only and with a mask."""
    g = (3, 3, 1, 1, 1, 1, 0)
    y = pool_case(shape, g, 11, cuda)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, g, fuse_mask=True)
    r_out, r_arg = ref.maxpool_fwd_argmax(host(y), g)
    assert_bits_equal(host(arg), r_arg, "argmax")
    assert_bits_equal(host(mask), ref.binarize_encode(host(y)), "fused mask")
    dout = WL.grad_map(tuple(out.shape), 5, cuda)
    for m, rm in ((None, None), (mask, ref.binarize_encode(host(y)))):
        dx = gist.gist_pool_relu_bwd(dout, arg, m, shape, g)
        r_dx = ref.pool_relu_bwd(host(dout), r_arg, rm, shape, g)
        assert_bits_equal(host(dx), r_dx, "dx" + (" (pool-only)" if m is None else ""))


@pytest.mark.parametrize("g", GEOMS, ids=gid)
@pytest.mark.parametrize("shape", SHAPES + [(64, 64, 56, 56)], ids=lambda s: "x".join(map(str, s)))
def test_relu_maxpool_fwd_in_place_relu(gist, ref, cuda, g, shape):
    """f3: the pre-activation map goes in; out/argmax/mask equal the oracle's on
    relu(x) (torch's ReLU, R21), and the fused-backward from them matches as well."""
    N, Cc, H, W = shape
    if H + 2 * g[4] < g[0] or W + 2 * g[5] < g[1]:
        pytest.skip("window larger than padded input")
    gen = torch.Generator(device=cuda).manual_seed(sum(shape) + 17)
    x = torch.round(torch.randn(shape, device=cuda, generator=gen) * 2) / 2  # ties, negatives, zeros
    r = torch.rand(shape, device=cuda, generator=gen)
    x = torch.where(r < 0.01, torch.full_like(x, float("nan")), x)
    x = torch.where((r >= 0.01) & (r < 0.02), torch.full_like(x, -float("inf")), x)
    x = torch.where((r >= 0.02) & (r < 0.05), torch.full_like(x, -0.0), x)
    x = torch.where((r >= 0.05) & (r < 0.06), torch.full_like(x, float("inf")), x)
    y = torch.relu(x.cpu()).numpy()  # the definition of ReLU the path follows (R21)
    out, arg, mask = gist.gist_relu_maxpool_fwd_argmax(x, g)
    r_out, r_arg = ref.maxpool_fwd_argmax(y, g)
    assert_bits_equal(host(out), r_out, "out")
    assert_bits_equal(host(arg), r_arg, "argmax")
    assert_bits_equal(host(mask), ref.binarize_encode(y), "mask")


@pytest.mark.parametrize("bands", [2, 3, 5])
@pytest.mark.parametrize("shape,g", [((2, 5, 48, 48), (3, 3, 2, 2, 0, 0, 1)), ((3, 4, 32, 32), (3, 3, 2, 2, 0, 0, 1)),
                                     ((1, 6, 80, 80), (3, 3, 2, 2, 0, 0, 1))],
                         ids=["48x48ceil", "32x32ceil", "80x80ceil"])
def test_pool3_banded_stride2_forward(gist, ref, cuda, monkeypatch, bands, shape, g):
    """The stride-2 forward in bands of output rows (the path of planes larger than a stage, e.g.
    GoogLeNet's 112x112 stem), forced on small planes with GIST_POOL3_BANDS: out, argmax and the
    fused mask (with and without the in-place ReLU) equal the oracle's, including a ragged last band."""
    monkeypatch.setenv("GIST_POOL3_BANDS", str(bands))
    y = pool_case(shape, g, sum(shape) + bands, cuda)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, g, fuse_mask=True)
    r_out, r_arg = ref.maxpool_fwd_argmax(host(y), g)
    assert_bits_equal(host(out), r_out, "out")
    assert_bits_equal(host(arg), r_arg, "argmax")
    assert_bits_equal(host(mask), ref.binarize_encode(host(y)), "mask")
    out2, arg2, _ = gist.gist_maxpool_fwd_argmax(y, g)
    assert_bits_equal(host(out2), r_out, "out (no mask)")
    assert_bits_equal(host(arg2), r_arg, "argmax (no mask)")
    x = WL.grad_map(shape, sum(shape), cuda)
    xr = torch.relu(x.cpu()).numpy()
    out3, arg3, mask3 = gist.gist_relu_maxpool_fwd_argmax(x, g)
    r_out3, r_arg3 = ref.maxpool_fwd_argmax(xr, g)
    assert_bits_equal(host(out3), r_out3, "out (relu on load)")
    assert_bits_equal(host(arg3), r_arg3, "argmax (relu on load)")
    assert_bits_equal(host(mask3), ref.binarize_encode(xr), "mask (relu on load)")


def test_fused_bwd_equals_torch_autograd_on_gpu_inputs(gist, cuda):
    # Same chain as the CPU pin, but on the GPU kernels: relu -> max_pool2d (AlexNet 3x3/s2).
    g = (3, 3, 2, 2, 0, 0, 0)
    z = WL.grad_map((4, 16, 55, 55), 3, cuda)
    y = torch.relu(z)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, g, fuse_mask=True)
    dout = WL.grad_map(tuple(out.shape), 4, cuda)
    dx = gist.gist_pool_relu_bwd(dout, arg, mask, y.shape, g)
    zc = z.cpu().requires_grad_()
    oc = torch.nn.functional.max_pool2d(torch.relu(zc), 3, 2)
    oc.backward(dout.cpu())
    assert_bits_equal(host(out), oc.detach().numpy(), "out vs torch")
    assert_bits_equal(host(dx), zc.grad.numpy(), "dx vs torch autograd")


# ------------------------------------------------------------------------ a4/a5 SSDC
@pytest.mark.parametrize("n", RAGGED + [256 * 32 * 70 + 5])
@pytest.mark.parametrize("s", [0.0, 0.5, 0.9, 1.0])
def test_ssdc_round_trip(gist, ref, cuda, n, s):
    x = WL.relu_map((n,), s, n, cuda, negative_zero=True) if s < 1 else torch.zeros(n, device=cuda)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x, trim=True)
    r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
    assert int(nnz.item()) == r_col.size
    assert_bits_equal(host(row_end), r_row_end, "row_end")
    assert_bits_equal(host(col), r_col, "col")
    assert_bits_equal(host(val), r_val, "val")
    back = gist.gist_ssdc_decode(row_end, col, val, n)
    assert_bits_equal(host(back), host(x), "decode(encode(x))")
    assert_bits_equal(host(back), ref.ssdc_decode(r_row_end, r_col, r_val, n), "decode vs oracle")


# Several encode chunks (one chunk = grid x 8192 elements, ~2.4 M on 148 SMs) with ragged ends.
@pytest.mark.parametrize("n", [148 * 2 * 8192 + 1, 7_777_777, 25_000_001])
@pytest.mark.parametrize("s", [0.0, 0.5, 0.9])
def test_ssdc_multi_chunk(gist, ref, cuda, n, s):
    x = WL.relu_map((n,), s, n + 17, cuda, negative_zero=True)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x, trim=True)
    r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
    assert int(nnz.item()) == r_col.size
    assert_bits_equal(host(row_end), r_row_end, "row_end")
    assert_bits_equal(host(col), r_col, "col")
    assert_bits_equal(host(val), r_val, "val")
    cap = r_col.size // 3 + 5
    row_end2, col2, val2, nnz2 = gist.gist_ssdc_encode(x, capacity=cap)
    assert int(nnz2.item()) == r_col.size
    assert_bits_equal(host(row_end2), r_row_end, "row_end (capacity)")
    assert_bits_equal(host(col2)[:cap], r_col[:cap], "col prefix")
    assert_bits_equal(host(val2)[:cap], r_val[:cap], "val prefix")


def test_ssdc_structured_sparsity(gist, ref, cuda):
    x = WL.relu_map((2, 64, 56, 56), 0.8, 11, cuda, structured=True)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x, trim=True)
    r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
    assert_bits_equal(host(row_end), r_row_end, "row_end")
    assert_bits_equal(host(col), r_col, "col")
    assert_bits_equal(host(val), r_val, "val")


@pytest.mark.parametrize("cap_frac", [0.0, 0.3, 0.999])
def test_ssdc_capacity(gist, ref, cuda, cap_frac):
    n = 256 * 32 * 9 + 77
    x = WL.relu_map((n,), 0.6, 5, cuda)
    r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
    cap = int(cap_frac * r_col.size)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x, capacity=cap)
    assert int(nnz.item()) == r_col.size  # true nnz always published
    assert_bits_equal(host(row_end), r_row_end, "row_end")
    if cap:
        assert_bits_equal(host(col)[:cap], r_col[:cap], "col prefix")
        assert_bits_equal(host(val)[:cap], r_val[:cap], "val prefix")


def test_ssdc_repeated_calls_reuse_workspace(gist, ref, cuda):
    n = 256 * 1000 + 3
    ws = gist.gist_ssdc_workspace(n, cuda)
    for seed in range(3):
        x = WL.relu_map((n,), 0.7, seed, cuda)
        row_end, col, val, nnz = gist.gist_ssdc_encode(x, workspace=ws, trim=True)
        r_row_end, r_col, _ = ref.ssdc_encode(host(x))
        assert_bits_equal(host(row_end), r_row_end, "row_end")
        assert_bits_equal(host(col), r_col, "col")


def test_ssdc_uninitialised_workspace_is_reported(gist, cuda):
    n = 256 * 32 * 20 + 5
    x = WL.relu_map((n,), 0.7, 7, cuda)
    ws = torch.full((gist.gist_ssdc_workspace_bytes(n),), 0xAB, dtype=torch.uint8, device=cuda)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x, workspace=ws)
    assert int(nnz.item()) == -1
    with pytest.raises(gist.GistError):
        gist.gist_ssdc_encode(x, workspace=ws, trim=True)
    gist.gist_ssdc_workspace_init(ws)
    _, _, _, nnz = gist.gist_ssdc_encode(x, workspace=ws)
    assert int(nnz.item()) == int((x.view(torch.int32) != 0).sum().item())


def test_ssdc_concurrent_streams_distinct_workspaces(gist, ref, cuda):
    """Calls on different streams with distinct workspaces may overlap on the device (the
    library is stateless apart from the workspace)."""
    sizes = [256 * 32 * 900 + 13, 256 * 32 * 500 + 7, 256 * 32 * 60 + 1]
    xs = [WL.relu_map((n,), 0.75, 300 + i, cuda) for i, n in enumerate(sizes)]
    streams = [torch.cuda.Stream(cuda) for _ in sizes]
    wss = [gist.gist_ssdc_workspace(n, cuda) for n in sizes]
    torch.cuda.synchronize()
    outs = []
    for _ in range(3):
        for x, st, ws in zip(xs, streams, wss):
            with torch.cuda.stream(st):
                outs.append(gist.gist_ssdc_encode(x, workspace=ws, stream=st))
    torch.cuda.synchronize()
    for i, (row_end, col, val, nnz) in enumerate(outs):
        x = xs[i % len(xs)]
        r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
        k = r_col.size
        assert int(nnz.item()) == k
        assert_bits_equal(host(row_end), r_row_end, f"row_end {i}")
        assert_bits_equal(host(col)[:k], r_col, f"col {i}")
        assert_bits_equal(host(val)[:k], r_val, f"val {i}")


def test_ssdc_back_to_back_chain_round_trips(gist, cuda):
    """Encodes and decodes of many maps enqueued back to back with no host sync in between
    (the programmatic-dependent-launch chain the bench runs): every map round-trips exactly."""
    sizes = [64 * 512 * 14 * 14, 64 * 256 * 28 * 28, 256 * 33 + 5, 64 * 128 * 56 * 56 // 2, 64 * 512 * 7 * 7]
    xs = [WL.relu_map((n,), 0.8, 900 + i, cuda) for i, n in enumerate(sizes)]
    wss = [gist.gist_ssdc_workspace(n, cuda) for n in sizes]
    torch.cuda.synchronize()
    for _ in range(2):
        encs = [gist.gist_ssdc_encode(x, workspace=ws) for x, ws in zip(xs, wss)]
        outs = [gist.gist_ssdc_decode(e[0], e[1], e[2], x.numel()) for e, x in zip(reversed(encs), reversed(xs))]
        torch.cuda.synchronize()
        for x, y in zip(reversed(xs), outs):
            assert torch.equal(x.view(torch.int32), y.view(torch.int32))


def test_ssdc_workspace_reused_across_sizes(gist, ref, cuda):
    """One workspace, initialised once, serves a sequence of calls of different sizes and
    capacities (the epoch tag makes the previous call's tile totals read as unpublished)."""
    big = 256 * 32 * 300 + 77
    ws = gist.gist_ssdc_workspace(big, cuda)
    for i, (n, cap) in enumerate([(big, None), (5000, None), (big, 0), (256 * 32 * 7, None), (big, None)] +
                                 [(3000 + 97 * k, None) for k in range(40)] + [(big, None)]):
        x = WL.relu_map((n,), 0.6 + 0.3 * (i % 2), 100 + i, cuda)
        r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
        row_end, col, val, nnz = gist.gist_ssdc_encode(x, capacity=cap, workspace=ws)
        assert int(nnz.item()) == r_col.size, (i, n)
        assert_bits_equal(host(row_end), r_row_end, f"row_end call {i}")
        if cap is None:
            k = r_col.size
            assert_bits_equal(host(col)[:k], r_col, f"col call {i}")
            assert_bits_equal(host(val)[:k], r_val, f"val call {i}")


# ------------------------------------------------------------------------ a6/a7 DPR
@pytest.mark.parametrize("bits", [16, 10, 8])
@pytest.mark.parametrize("n", RAGGED)
def test_dpr(gist, ref, cuda, bits, n):
    x = WL.dpr_map((n,), n + bits, cuda)
    if n >= 200:
        sp = WL.dpr_specials().to(cuda)
        x[: sp.numel()] = sp[: n]
    packed = gist.gist_dpr_encode(x, bits)
    r_packed = ref.dpr_encode(host(x), bits)
    assert_bits_equal(host(packed), r_packed, f"fp{bits} packed")
    back = gist.gist_dpr_decode(packed, n, bits)
    assert_bits_equal(host(back), ref.dpr_decode(r_packed, n, bits), f"fp{bits} decode")


@pytest.mark.parametrize("bits", [16, 10, 8])
def test_dpr_decode_every_code(gist, ref, cuda, bits):
    # all 2^bits codes in every field position of the word
    k = {16: 2, 10: 3, 8: 4}[bits]
    codes = np.arange(1 << bits, dtype=np.uint32)
    n = codes.size
    words = np.zeros(-(-n // k), np.uint32)
    idx = np.arange(n)
    np.bitwise_or.at(words, idx // k, codes << (bits * (idx % k)))
    back = gist.gist_dpr_decode(torch.from_numpy(words.view(np.int32)).to(cuda), n, bits)
    assert_bits_equal(host(back), ref.dpr_values(codes, bits), f"fp{bits} all codes")


@pytest.mark.slow
@pytest.mark.parametrize("bits", [16, 10, 8])
def test_dpr_exhaustive_all_fp32_patterns(gist, ref, cuda, bits):
    # Every one of the 2^32 fp32 bit patterns, in chunks; oracle on all host cores.
    import concurrent.futures as cf
    import os
    chunk = 1 << 27
    k = {16: 2, 10: 3, 8: 4}[bits]
    chunk -= chunk % (12 * k)
    workers = max(1, os.cpu_count() or 1)
    with cf.ThreadPoolExecutor(workers) as ex:
        start = 0
        while start < (1 << 32):
            m = min(chunk, (1 << 32) - start)
            pat = torch.arange(start, start + m, dtype=torch.int64, device=cuda).to(torch.int32)
            x = pat.view(torch.float32)
            got = host(gist.gist_dpr_encode(x, bits))
            xs = host(x)
            parts = np.array_split(np.arange(m), workers)
            parts = [p for p in parts if p.size]
            # split on word boundaries
            bounds = [0] + [int(p[-1] + 1) // k * k for p in parts[:-1]] + [m]
            futs = [ex.submit(ref.dpr_encode, xs[a:b], bits) for a, b in zip(bounds[:-1], bounds[1:])]
            expect = np.concatenate([f.result() for f in futs])
            assert_bits_equal(got, expect, f"fp{bits} patterns [{start}, {start + m})")
            start += m


# ------------------------------------------------------------------------ full-size configs
def _vgg_site(name):
    return next(s for s in WL.NETS["vgg16"] if s.name == name)


@pytest.mark.parametrize("site", ["relu1_2", "relu5_3"])
def test_full_size_vgg16_relu_pool(gist, ref, cuda, site):
    """C3 (VGG16 b64) ReLU->Pool site at full size: every output compared."""
    s = _vgg_site(site)
    shape = (64,) + s.chw
    y = WL.relu_map(shape, 0.8, 3_000_000 + 1, cuda)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, s.pool, fuse_mask=True)  # fused a1 where possible
    assert torch.equal(mask, gist.gist_binarize_encode(y))
    dout = WL.grad_map(tuple(out.shape), 17, cuda)
    dx = gist.gist_pool_relu_bwd(dout, arg, mask, shape, s.pool)
    yh = host(y)
    r_out, r_arg = ref.maxpool_fwd_argmax(yh, s.pool)
    r_mask = ref.binarize_encode(yh)
    assert_bits_equal(host(mask), r_mask, "mask")
    assert_bits_equal(host(out), r_out, "out")
    assert_bits_equal(host(arg), r_arg, "arg")
    del yh
    assert_bits_equal(host(dx), ref.pool_relu_bwd(host(dout), r_arg, r_mask, shape, s.pool), "dx")


def test_full_size_vgg16_ssdc_and_dpr(gist, ref, cuda):
    s = _vgg_site("relu1_1")
    x = WL.relu_map((64,) + s.chw, 0.8, 3_000_000 + 2, cuda)
    row_end, col, val, nnz = gist.gist_ssdc_encode(x, trim=True)
    xh = host(x)
    r_row_end, r_col, r_val = ref.ssdc_encode(xh)
    assert int(nnz.item()) == r_col.size
    assert_bits_equal(host(row_end), r_row_end, "row_end")
    assert_bits_equal(host(col), r_col, "col")
    assert_bits_equal(host(val), r_val, "val")
    back = gist.gist_ssdc_decode(row_end, col, val, x.numel())
    assert torch.equal(back.view(torch.int32), x.reshape(-1).view(torch.int32))
    for bits in (16, 10, 8):
        packed = gist.gist_dpr_encode(x, bits)
        assert_bits_equal(host(packed), ref.dpr_encode(xh, bits), f"fp{bits}")


# ------------------------------------------------------------------------ f1: DPR over SSDC values
@pytest.mark.parametrize("bits", [16, 10, 8])
@pytest.mark.parametrize("n", [1000, 256 * 16 * 33 + 7])
def test_ssdc_values_dpr(gist, ref, cuda, bits, n):
    # DPR of the CSR value array only; the count comes from the device nnz.
    x = WL.relu_map((n,), 0.7, n + bits, cuda) * torch.exp2(torch.randint(-8, 8, (n,), device=cuda).float())
    row_end, col, val, nnz = gist.gist_ssdc_encode(x)
    k = int(nnz.item())
    packed = gist.gist_ssdc_dpr_encode(val, nnz, bits)
    r_row_end, r_col, r_val = ref.ssdc_encode(host(x))
    r_packed = ref.dpr_encode(r_val, bits)
    assert_bits_equal(host(packed)[:r_packed.size], r_packed, "dpr(val)")
    back = gist.gist_ssdc_dpr_decode(packed, nnz, bits, n)
    assert_bits_equal(host(back)[:k], ref.dpr_decode(r_packed, k, bits), "dpr^-1")
    dense = gist.gist_ssdc_decode(row_end, col, back[:max(k, 1)], n)
    expect = ref.ssdc_decode(r_row_end, r_col, ref.dpr_decode(r_packed, k, bits), n)
    assert_bits_equal(host(dense), expect, "ssdc_decode(dpr^-1(dpr(val)))")


# ------------------------------------------------------------------------ full-size code paths (round 2)
def test_full_size_dpr_decode_all_widths(gist, ref, cuda):
    """a7 at the bench's full size (VGG16 relu1_1 b64, 205.5 M values): the unrolled multi-group
    decode loops (u >= 1) and the FP10 multi-pass chunk loop, element by element vs the oracle."""
    s = _vgg_site("relu1_1")
    x = WL.dpr_map((64,) + s.chw, 3_000_000 + 7, cuda)
    sp = WL.dpr_specials().to(cuda)
    x.view(-1)[: sp.numel()] = sp
    xh = host(x).reshape(-1)
    n = x.numel()
    for bits in (16, 10, 8):
        packed = gist.gist_dpr_encode(x, bits)
        r_packed = ref.dpr_encode(xh, bits)
        assert_bits_equal(host(packed), r_packed, f"fp{bits} packed")
        back = gist.gist_dpr_decode(packed, n, bits)
        assert_bits_equal(host(back), ref.dpr_decode(r_packed, n, bits), f"fp{bits} decode")
        del packed, back, r_packed


FULL_3X3 = [("alexnet", "relu1", 128), ("nin", "relu_cccp2", 256), ("googlenet", "relu_conv1", 64),
            ("alexnet", "relu5", 128), ("googlenet", "inc3b_out", 64)]


@pytest.mark.parametrize("net,site,batch", FULL_3X3, ids=lambda v: str(v))
def test_full_size_3x3_pools(gist, ref, cuda, net, site, batch):
    """3x3/s2 floor (AlexNet) and ceil (NiN, GoogLeNet) at the configs' full batch: the generic
    forward and the 3x3/s2 block backward run their grid-stride loops past one pass of the capped
    grid.  Forward with and without the mask, backward with the mask and pool-only."""
    s = next(t for t in WL.NETS[net] if t.name == site)
    shape = (batch,) + s.chw
    y = WL.relu_map(shape, 0.5, 4_000_000 + batch, cuda)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, s.pool, fuse_mask=True)
    out2, arg2, _ = gist.gist_maxpool_fwd_argmax(y, s.pool)
    assert torch.equal(out, out2) and torch.equal(arg, arg2)
    yh = host(y)
    r_out, r_arg = ref.maxpool_fwd_argmax(yh, s.pool)
    r_mask = ref.binarize_encode(yh)
    del yh
    assert_bits_equal(host(out), r_out, "out")
    assert_bits_equal(host(arg), r_arg, "argmax")
    assert_bits_equal(host(mask), r_mask, "mask")
    dout = WL.grad_map(tuple(out.shape), 19, cuda)
    dh = host(dout)
    for m, rm in ((mask, r_mask), (None, None)):
        dx = gist.gist_pool_relu_bwd(dout, arg, m, shape, s.pool)
        assert_bits_equal(host(dx), ref.pool_relu_bwd(dh, r_arg, rm, shape, s.pool),
                          "dx" + (" (pool-only)" if m is None else ""))
        del dx


def test_full_size_2x2_pair_kernels_without_mask(gist, ref, cuda):
    """The 2x2/s2 pair forward (no mask requested) and the pool-only pair backward at the C3 size."""
    s = _vgg_site("relu1_2")
    shape = (64,) + s.chw
    y = WL.relu_map(shape, 0.8, 3_000_000 + 11, cuda)
    out, arg, mask = gist.gist_maxpool_fwd_argmax(y, s.pool)
    assert mask is None
    r_out, r_arg = ref.maxpool_fwd_argmax(host(y), s.pool)
    assert_bits_equal(host(out), r_out, "out")
    assert_bits_equal(host(arg), r_arg, "argmax")
    dout = WL.grad_map(tuple(out.shape), 23, cuda)
    dx = gist.gist_pool_relu_bwd(dout, arg, None, shape, s.pool)
    assert_bits_equal(host(dx), ref.pool_relu_bwd(host(dout), r_arg, None, shape, s.pool), "dx (pool-only)")


@pytest.mark.parametrize("g", GEOMS, ids=gid)
@pytest.mark.parametrize("shape", [(2, 3, 13, 13), (1, 64, 56, 56), (3, 7, 28, 28), (1, 1, 2, 2050)],
                         ids=lambda s: "x".join(map(str, s)))
def test_relu_maxpool_then_fused_bwd(gist, ref, cuda, g, shape):
    """f3 -> a3: the backward fed by the in-place-ReLU forward's argmax and mask equals the
    oracle's backward of relu(x), and torch CPU autograd of relu -> max_pool2d where torch
    supports the geometry (the f3 docstring's promise)."""
    N, Cc, H, W = shape
    if H + 2 * g[4] < g[0] or W + 2 * g[5] < g[1]:
        pytest.skip("window larger than padded input")
    gen = torch.Generator(device=cuda).manual_seed(sum(shape) + 29)
    x = torch.round(torch.randn(shape, device=cuda, generator=gen) * 2) / 2
    out, arg, mask = gist.gist_relu_maxpool_fwd_argmax(x, g)
    y = torch.relu(x.cpu()).numpy()
    r_out, r_arg = ref.maxpool_fwd_argmax(y, g)
    r_mask = ref.binarize_encode(y)
    dout = WL.grad_map(tuple(out.shape), 31, cuda)
    dx = gist.gist_pool_relu_bwd(dout, arg, mask, shape, g)
    r_dx = ref.pool_relu_bwd(host(dout), r_arg, r_mask, shape, g)
    assert_bits_equal(host(dx), r_dx, "dx from f3 encodings")
    kh, kw, sh, sw, ph, pw, cm = g
    xc = x.cpu().requires_grad_()
    oc = torch.nn.functional.max_pool2d(torch.relu(xc), (kh, kw), (sh, sw), (ph, pw), ceil_mode=bool(cm))
    oc.backward(dout.cpu())
    assert_bits_equal(host(out), oc.detach().numpy(), "out vs torch")
    assert_bits_equal(host(dx), xc.grad.numpy(), "dx vs torch autograd")


def test_binding_checks_dtype_device_and_size(gist, cuda):
    """a bf16 map (autocast) read as fp32 would overrun its buffer; the binding refuses it."""
    y16 = torch.zeros(64, 16, 16, device=cuda, dtype=torch.bfloat16).view(1, 64, 16, 16)
    with pytest.raises(ValueError):
        gist.gist_binarize_encode(y16)
    with pytest.raises(ValueError):
        gist.gist_maxpool_fwd_argmax(y16, (2, 2, 2, 2, 0, 0, 0))
    with pytest.raises(ValueError):
        gist.gist_ssdc_encode(y16)
    with pytest.raises(ValueError):
        gist.gist_dpr_encode(y16, 16)
    y = torch.zeros(1, 64, 16, 16, device=cuda)
    with pytest.raises(ValueError):  # mask too small
        gist.gist_maxpool_fwd_argmax(y, (2, 2, 2, 2, 0, 0, 0), mask=torch.zeros(3, dtype=torch.int32, device=cuda))
    with pytest.raises(ValueError):  # float argmax words
        gist.gist_maxpool_fwd_argmax(y, (2, 2, 2, 2, 0, 0, 0), argmax=torch.zeros(1024, device=cuda))
