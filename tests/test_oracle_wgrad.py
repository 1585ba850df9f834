"""Pins of the f4 reference (oracle O8, the conv weight gradient of P:128 that the decode-in-GEMM
kernel computes): torch's own conv2d weight gradient in float64 (a library routine), the
single-impulse special case (one nonzero in dY and X gives one known dW entry), and the
exact sum-of-products on an all-ones map (dW counts the in-bounds pairs)."""
import numpy as np
import pytest
import torch


@pytest.mark.parametrize("shape", [(1, 3, 2, 5, 4), (2, 4, 3, 7, 8), (3, 2, 5, 1, 1), (1, 1, 1, 3, 3)])
def test_wgrad_matches_torch_float64(ref, shape):
    N, Ci, Co, H, W = shape
    g = torch.Generator().manual_seed(sum(shape))
    x = torch.relu(torch.randn(N, Ci, H, W, generator=g))
    dy = torch.randn(N, Co, H, W, generator=g)
    dw, mag = ref.conv3x3_wgrad(dy.numpy(), x.numpy())
    want = torch.nn.grad.conv2d_weight(x.double(), (Co, Ci, 3, 3), dy.double(), stride=1, padding=1)
    np.testing.assert_allclose(dw, want.numpy(), rtol=1e-12, atol=1e-12)
    wabs = torch.nn.grad.conv2d_weight(x.double().abs(), (Co, Ci, 3, 3), dy.double().abs(), stride=1, padding=1)
    np.testing.assert_allclose(mag, wabs.numpy(), rtol=1e-12, atol=1e-12)


def test_wgrad_single_impulse(ref):
    N, Ci, Co, H, W = 2, 3, 2, 6, 5
    x = np.zeros((N, Ci, H, W), np.float32)
    dy = np.zeros((N, Co, H, W), np.float32)
    x[1, 2, 3, 1] = 1.5  # ih, iw
    dy[1, 0, 2, 2] = -2.0  # oh, ow -> kh = ih - oh + 1 = 2, kw = iw - ow + 1 = 0
    dw, _ = ref.conv3x3_wgrad(dy, x)
    expect = np.zeros((Co, Ci, 3, 3))
    expect[0, 2, 2, 0] = -3.0
    assert np.array_equal(dw, expect)


def test_wgrad_all_ones_counts_pairs(ref):
    N, Ci, Co, H, W = 2, 1, 1, 4, 6
    dw, mag = ref.conv3x3_wgrad(np.ones((N, Co, H, W), np.float32), np.ones((N, Ci, H, W), np.float32))
    for kh in range(3):
        for kw in range(3):
            rows = H - abs(kh - 1)
            cols = W - abs(kw - 1)
            assert dw[0, 0, kh, kw] == N * rows * cols == mag[0, 0, kh, kw]
