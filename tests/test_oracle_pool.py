"""Pins for oracles O2 (MaxPool fwd + Y->X argmax map; §IV-A) and O3 (fused
pool+ReLU backward from the encodings; §III-A, §IV-A).

Library pins: torch CPU max_pool2d(return_indices=True) for values and argmax, torch CPU
autograd of relu -> max_pool2d for the backward, bit for bit."""
import itertools

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from pool_cases import GEOMS, gid


def torch_pool(x, g, **kw):
    kh, kw_, sh, sw, ph, pw, cm = g
    return F.max_pool2d(x, (kh, kw_), (sh, sw), (ph, pw), ceil_mode=bool(cm), **kw)


def planted(shape, seed, specials=True):
    rng = np.random.default_rng(seed)
    # few distinct values -> many ties; plus NaN / -inf / +-0 planted
    y = rng.integers(-3, 4, size=shape).astype(np.float32)
    if specials:
        r = rng.random(shape)
        y[r < 0.05] = -np.inf
        y[(r >= 0.05) & (r < 0.1)] = -0.0
        y[(r >= 0.1) & (r < 0.12)] = np.nan
    return y


def nibbles(arg, n_out):
    k = np.arange(n_out)
    return (arg[k >> 3] >> (4 * (k & 7))) & 0xF


@pytest.mark.parametrize("g", GEOMS, ids=gid)
@pytest.mark.parametrize("H,W", [(1, 1), (5, 7), (9, 9), (27, 27), (14, 13), (56, 56)])
def test_out_dims_match_torch(ref, g, H, W):
    kh, kw, sh, sw, ph, pw, cm = g
    if ph > kh // 2 or pw > kw // 2:
        pytest.skip("torch requires pad <= k/2")
    if H + 2 * ph < kh or W + 2 * pw < kw:
        pytest.skip("window larger than padded input")
    out = torch_pool(torch.zeros(1, 1, H, W), g)
    assert ref.pool_out_dim(H, kh, sh, ph, cm) == out.shape[2]
    assert ref.pool_out_dim(W, kw, sw, pw, cm) == out.shape[3]


def to_local(idx, g, Ho, Wo, W):
    """torch's flat in-plane index -> window-local dy*kw+dx (reading R2)."""
    kh, kw, sh, sw, ph, pw, cm = g
    oh = np.arange(Ho).reshape(Ho, 1)
    ow = np.arange(Wo).reshape(1, Wo)
    ih, iw = idx // W, idx % W
    return (ih - (oh * sh - ph)) * kw + (iw - (ow * sw - pw))


@pytest.mark.parametrize("g", GEOMS, ids=gid)
@pytest.mark.parametrize("seed", range(4))
def test_fwd_matches_torch(ref, g, seed):
    N, Cc, H, W = 2, 3, 11 + seed, 13 - seed
    y = planted((N, Cc, H, W), seed)
    out, arg = ref.maxpool_fwd_argmax(y, g)
    t_out, t_idx = torch_pool(torch.from_numpy(y), g, return_indices=True)
    assert out.shape == tuple(t_out.shape)
    assert np.array_equal(out.view(np.uint32), t_out.numpy().view(np.uint32))
    Ho, Wo = out.shape[2:]
    local = to_local(t_idx.numpy(), g, Ho, Wo, W)
    assert np.array_equal(nibbles(arg, out.size).reshape(out.shape), local)
    assert local.max() < g[0] * g[1] <= 16  # fits in 4 bits
    # padding nibbles of the last word are zero (R2)
    last = out.size % 8
    if last:
        assert arg[-1] >> (4 * last) == 0


def brute_argmax(y, g):
    """Brute force straight from the definition, for tiny tensors."""
    kh, kw, sh, sw, ph, pw, cm = g
    N, Cc, H, W = y.shape
    outs = []
    for n, c in itertools.product(range(N), range(Cc)):
        t = torch_pool(torch.from_numpy(y[n:n + 1, c:c + 1]), g)
        Ho, Wo = t.shape[2:]
        for oh, ow in itertools.product(range(Ho), range(Wo)):
            cand = [(dy * kw + dx, y[n, c, oh * sh - ph + dy, ow * sw - pw + dx])
                    for dy in range(kh) for dx in range(kw)
                    if 0 <= oh * sh - ph + dy < H and 0 <= ow * sw - pw + dx < W]
            nans = [a for a, v in cand if np.isnan(v)]
            if nans:
                outs.append(nans[-1])
            else:
                m = max(v for _, v in cand)
                outs.append(next(a for a, v in cand if v == m))
    return np.array(outs)


@pytest.mark.parametrize("g", GEOMS, ids=gid)
def test_fwd_brute_force_tiny(ref, g):
    for seed, (H, W) in enumerate([(3, 3), (4, 5), (6, 6), (7, 9)]):
        if H + 2 * g[4] < g[0] or W + 2 * g[5] < g[1]:
            continue
        y = planted((1, 2, H, W), 100 + seed)
        out, arg = ref.maxpool_fwd_argmax(y, g)
        assert np.array_equal(nibbles(arg, out.size), brute_argmax(y, g))


def torch_relu_pool_grad(z, dy, g, relu=True):
    zt = torch.from_numpy(z).requires_grad_()
    y = torch.relu(zt) if relu else zt * 1.0
    out = torch_pool(y, g)
    out.backward(torch.from_numpy(dy))
    return y.detach().numpy(), zt.grad.numpy()


@pytest.mark.parametrize("g", GEOMS, ids=gid)
@pytest.mark.parametrize("seed", range(3))
def test_fused_bwd_matches_torch_autograd(ref, g, seed):
    # relu -> max_pool2d; dx must be bit-identical to torch's autograd (R6, R7).
    N, Cc, H, W = 2, 4, 15 + seed, 12 + 2 * seed
    rng = np.random.default_rng(seed)
    z = rng.standard_normal((N, Cc, H, W)).astype(np.float32)
    z[rng.random(z.shape) < 0.2] = 0.0  # ties among zeros after ReLU
    y, grad = None, None
    Ho = ref.pool_out_dim(H, g[0], g[2], g[4], g[6])
    Wo = ref.pool_out_dim(W, g[1], g[3], g[5], g[6])
    dy = rng.standard_normal((N, Cc, Ho, Wo)).astype(np.float32)
    dy[rng.random(dy.shape) < 0.05] = -0.0
    y, grad = torch_relu_pool_grad(z, dy, g)
    mask = ref.binarize_encode(y)
    _, arg = ref.maxpool_fwd_argmax(y, g)
    dx = ref.pool_relu_bwd(dy, arg, mask, y.shape, g)
    assert np.array_equal(dx.view(np.uint32), grad.view(np.uint32))


@pytest.mark.parametrize("g", GEOMS, ids=gid)
def test_pool_only_bwd_matches_torch(ref, g):
    # mask = NULL -> plain max-pool backward (GoogLeNet in-module pools).
    rng = np.random.default_rng(7)
    y = rng.standard_normal((2, 3, 10, 11)).astype(np.float32)
    Ho = ref.pool_out_dim(10, g[0], g[2], g[4], g[6])
    Wo = ref.pool_out_dim(11, g[1], g[3], g[5], g[6])
    dy = rng.standard_normal((2, 3, Ho, Wo)).astype(np.float32)
    _, grad = torch_relu_pool_grad(y, dy, g, relu=False)
    _, arg = ref.maxpool_fwd_argmax(y, g)
    dx = ref.pool_relu_bwd(dy, arg, None, y.shape, g)
    assert np.array_equal(dx.view(np.uint32), grad.view(np.uint32))


def test_non_overlapping_bwd_is_pure_select(ref):
    # Special case: 2x2/s2 windows never overlap, so dx is dY routed to the argmax and
    # masked — every dY value appears exactly once (or is masked to +0).
    g = (2, 2, 2, 2, 0, 0, 0)
    rng = np.random.default_rng(1)
    y = np.maximum(rng.standard_normal((1, 2, 8, 8)), 0).astype(np.float32)
    dy = rng.standard_normal((1, 2, 4, 4)).astype(np.float32)
    _, arg = ref.maxpool_fwd_argmax(y, g)
    dx = ref.pool_relu_bwd(dy, arg, None, y.shape, g)
    assert np.count_nonzero(dx) == dy.size
    assert np.array_equal(np.sort(dx[dx != 0]), np.sort(dy.reshape(-1)))


def test_relu_pool_ratio_close_to_16x(ref):
    # "a compression of close to 16x (32x for ReLU output and 8x for MaxPool
    # output)"; closed form 32/(1 + 4*n_o/n) (reading R20).
    for H in (224, 112, 56, 28, 14):  # VGG16 ReLU-Pool sites, 2x2/s2 -> exactly 16x
        n = 64 * H * H
        Ho = ref.pool_out_dim(H, 2, 2, 0, 0)
        n_o = 64 * Ho * Ho
        enc = 4 * ref.binarize_words(n) + 4 * ref.argmax_words(n_o)
        assert 4 * n / enc == 16.0
    n, n_o = 96 * 55 * 55, 96 * 27 * 27  # AlexNet relu1 3x3/s2
    assert 4 * n / (4 * ref.binarize_words(n) + 4 * ref.argmax_words(n_o)) == pytest.approx(
        32 / (1 + 4 * n_o / n), rel=1e-4)
    assert (4 * n_o) / (4 * ref.argmax_words(n_o)) == pytest.approx(8.0, rel=1e-4)


def test_relu_reading_r21_matches_torch():
    """R21: the in-place ReLU of f3 is relu(v) = (v < 0 ? +0.0 : v) — torch's ReLU bit for bit
    (-0.0 and NaN payloads pass through, -inf -> +0.0)."""
    import numpy as np
    v = np.array([-0.0, 0.0, -1.5, 2.5, np.inf, -np.inf, np.nan, 1e-45, -1e-45,
                  np.frombuffer(np.uint32(0xFFC00001).tobytes(), np.float32)[0]], dtype=np.float32)
    ours = np.where(v < 0, np.float32(0.0), v).astype(np.float32)
    theirs = torch.relu(torch.from_numpy(v)).numpy()
    assert np.array_equal(ours.view(np.uint32), theirs.view(np.uint32))
