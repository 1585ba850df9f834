"""Pins for oracle O1 (Binarize encode; §III-A, §IV-A)."""
import numpy as np
import pytest

from golden_io import binarize_cases


@pytest.mark.parametrize("case", list(binarize_cases()), ids=lambda c: f"n{c[0].size}")
def test_golden(ref, case):
    x, words = case
    assert np.array_equal(ref.binarize_encode(x), words)


@pytest.mark.parametrize("n", [0, 1, 31, 32, 33, 255, 256, 1000, 4097, 200_704])
def test_matches_numpy_packbits(ref, n):
    # Library pin: numpy.packbits(y > 0, bitorder='little') viewed as little-endian u32.
    rng = np.random.default_rng(n)
    y = rng.standard_normal(n).astype(np.float32)
    y[rng.random(n) < 0.1] = -0.0
    y[rng.random(n) < 0.01] = np.nan
    bits = np.packbits(y > 0, bitorder="little")
    bits = np.concatenate([bits, np.zeros((-bits.size) % 4, np.uint8)])
    expect = bits.view("<u4")
    got = ref.binarize_encode(y)
    assert got.size == (n + 31) // 32
    assert np.array_equal(got, expect)


def test_compression_ratio_32x(ref):
    # 32x for the ReLU output (1 bit vs fp32) when n is a multiple of 32.
    n = 64 * 56 * 56
    assert (4 * n) / (4 * ref.binarize_words(n)) == 32.0


def test_mask_is_relu_backward(ref):
    # ReLU backward dX = dY where Y > 0 else 0 — the mask must reproduce torch's
    # threshold_backward selection bit for bit.
    import torch
    rng = np.random.default_rng(3)
    z = torch.from_numpy(rng.standard_normal(1000).astype(np.float32)).requires_grad_()
    y = torch.relu(z)
    dy = torch.from_numpy(rng.standard_normal(1000).astype(np.float32))
    y.backward(dy)
    mask = ref.binarize_encode(y.detach().numpy())
    bit = (mask[np.arange(1000) >> 5] >> (np.arange(1000) & 31)) & 1
    sel = np.where(bit == 1, dy.numpy(), np.float32(0))
    assert np.array_equal(sel.view(np.uint32), z.grad.numpy().view(np.uint32))
