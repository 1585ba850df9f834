"""Pins for oracles O4/O5 (SSDC encode/decode; P:158-P:164 §IV-A)."""
import numpy as np
import pytest
import torch


def relu_like(n, s, seed, negzero=False):
    rng = np.random.default_rng(seed)
    x = rng.standard_normal(n).astype(np.float32)
    x[rng.random(n) < s] = 0.0
    if negzero:
        x[rng.random(n) < 0.05] = -0.0
    return x


@pytest.mark.parametrize("n,s", [(256, 0.5), (256 * 37, 0.8), (256 * 100, 0.0), (256 * 9, 1.0)])
def test_matches_torch_csr(ref, n, s):
    # Library pin: torch to_sparse_csr on x.view(rows, 256) (n % 256 == 0, no -0.0):
    # crow[1:] == row_end, col_indices == col, values == val.
    x = relu_like(n, s, n)
    row_end, col, val = ref.ssdc_encode(x)
    csr = torch.from_numpy(x).view(-1, 256).to_sparse_csr()
    assert np.array_equal(row_end, csr.crow_indices()[1:].numpy())
    assert np.array_equal(col, csr.col_indices().numpy())
    assert np.array_equal(val.view(np.uint32), csr.values().numpy().view(np.uint32))


@pytest.mark.parametrize("n", [0, 1, 255, 256, 257, 1000, 200_704, 256 * 50 + 3])
@pytest.mark.parametrize("negzero", [False, True])
def test_round_trip_is_bit_exact(ref, n, negzero):
    # Lossless: decode(encode(x)) is memcmp-identical, including -0.0 (R8).
    x = relu_like(n, 0.7, n + 1, negzero)
    row_end, col, val = ref.ssdc_encode(x)
    assert row_end.size == (n + 255) // 256
    y = ref.ssdc_decode(row_end, col, val, n)
    assert np.array_equal(x.view(np.uint32), y.view(np.uint32))
    # nnz == number of nonzero bit patterns (R8)
    assert col.size == np.count_nonzero(x.view(np.uint32))
    # columns ascend within each row, and are < 256 (1-byte index)
    starts = np.concatenate([[0], row_end[:-1]]) if n else np.zeros(0, np.int64)
    for r in range(0, row_end.size, max(1, row_end.size // 16)):
        cols = col[starts[r]:row_end[r]]
        assert np.all(np.diff(cols.astype(int)) > 0)


def test_size_closed_form_and_break_even(ref):
    # Closed form: 5*nnz + 4*rows bytes (fp32 value + 1-byte column, R10 row ends).
    n = 256 * 1000
    for s in (0.0, 0.2, 0.5, 0.8, 0.9, 0.99):
        x = relu_like(n, s, 5)
        row_end, col, val = ref.ssdc_encode(x)
        nnz = col.size
        assert col.nbytes + val.nbytes + row_end.nbytes == 5 * nnz + 4 * (n // 256)
    # NVO lowers the minimum useful sparsity from 50% (4-byte index) to 20%.
    # 4n > 5(1-s)n + 4n/256  <=>  s > 1 - (4 - 4/256)/5 = 0.2031...
    s_star = 1 - (4 - 4 / 256) / 5
    assert 0.20 < s_star < 0.21
    s_star_int32 = 1 - (4 - 4 / 256) / 8  # same with 4-byte indices: 50.2%
    assert 0.50 < s_star_int32 < 0.51
    for s, compresses in ((0.19, False), (0.22, True)):
        nnz = round((1 - s) * n)
        assert (4 * n > 5 * nnz + 4 * (n // 256)) == compresses


def test_empty_rows_and_full_rows(ref):
    x = np.zeros(256 * 4, np.float32)
    x[256:512] = 1.0       # a full row
    x[3 * 256 + 255] = -2  # last column only
    row_end, col, val = ref.ssdc_encode(x)
    assert row_end.tolist() == [0, 256, 256, 257]
    assert col[-1] == 255 and val[-1] == -2
