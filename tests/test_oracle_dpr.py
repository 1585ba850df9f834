"""Pins for oracles O6/O7 (DPR encode/decode; P:166-P:171 §IV-A)."""
import numpy as np
import pytest
import torch

from golden_io import dpr_cases

FMT = {16: (5, 10), 10: (5, 4), 8: (4, 3)}


@pytest.mark.parametrize("case", list(dpr_cases()), ids=lambda c: f"fp{c[0]}-{c[1].tolist()}")
def test_golden(ref, case):
    bits, x, code, packed = case
    if packed:
        assert ref.dpr_encode(x, bits).tolist() == [code]
    else:
        assert ref.dpr_codes(x, bits)[0] == code


def _patterns(step=257, extra_ranges=()):
    """A strided sample of all 2^32 fp32 patterns plus dense ranges."""
    parts = [np.arange(0, 2 ** 32, step, dtype=np.uint64)]
    for lo, hi in extra_ranges:
        parts.append(np.arange(lo, hi, dtype=np.uint64))
    u = np.concatenate(parts).astype(np.uint32)
    return u.view(np.float32)


def test_fp16_matches_numpy_on_sampled_patterns(ref):
    # Library pin: numpy.float16 of the value clamped to +-65504 ("clamped"),
    # for ~17M fp32 patterns (every 257th + dense around the half range edges).
    x = _patterns(257, [(0x33000000 - 4096, 0x33000000 + 4096),     # 2^-25 ties
                        (0x38800000 - 65536, 0x38800000 + 65536),   # min normal
                        (0x477FE000 - 8192, 0x477FE000 + 8192)])    # 65504 / 65520
    x = np.concatenate([x, -x])
    got = ref.dpr_codes(x, 16)
    nan = np.isnan(x)
    clamped = np.clip(np.where(nan, 0, x), -65504, 65504).astype(np.float32)
    expect = clamped.astype(np.float16).view(np.uint16).astype(np.uint32)
    sign = (x.view(np.uint32) >> 31).astype(np.uint32)
    expect = np.where(nan, 0x7E00 | (sign << 15), expect)
    assert np.array_equal(got, expect)


def test_fp16_decode_all_codes_matches_numpy(ref):
    codes = np.arange(65536, dtype=np.uint32)
    got = ref.dpr_values(codes, 16)
    expect = codes.astype(np.uint16).view(np.float16).astype(np.float32)
    assert np.array_equal(got.view(np.uint32), expect.view(np.uint32))


def test_fp8_matches_float8_e4m3fn_in_normal_range(ref):
    # Library pin: torch float8_e4m3fn agrees with our FP8 on |x| in [2^-6, 464): it is
    # the same 1-4-3 layout with bias 7 (R13); it differs only by reserving 0x7F for NaN
    # (we use it for 480, R14) and by keeping subnormals (we flush).
    rng = np.random.default_rng(0)
    mag = np.exp2(rng.uniform(-6, np.log2(464), 400_000)).astype(np.float32)
    # every exact midpoint between consecutive normal codes
    vals = ref.dpr_values(np.arange(0x08, 0x7E, dtype=np.uint32), 8).astype(np.float64)
    mids = ((vals[:-1] + vals[1:]) / 2).astype(np.float32)
    x = np.concatenate([mag, mids, vals.astype(np.float32)])
    x = np.concatenate([x, -x])
    x = x[(np.abs(x) >= 2 ** -6) & (np.abs(x) < 464)]
    got = ref.dpr_codes(x, 8)
    expect = torch.from_numpy(x).to(torch.float8_e4m3fn).view(torch.uint8).numpy().astype(np.uint32)
    assert np.array_equal(got, expect)


def _codebook(ref, bits):
    E, M = FMT[bits]
    codes = np.array([c for c in range(1 << (E + M)) if (c >> M) != 0], np.uint32)  # positive normals
    return codes, ref.dpr_values(codes, bits).astype(np.float64)


@pytest.mark.parametrize("bits", [8, 10])
def test_decode_closed_form_table(ref, bits):
    # Every code: exponent field 0 -> +-0 (R14), else +-2^(e-bias)(1 + m/2^M), exact.
    E, M = FMT[bits]
    bias = 2 ** (E - 1) - 1
    codes = np.arange(1 << (1 + E + M), dtype=np.uint32)
    got = ref.dpr_values(codes, bits)
    s = (codes >> (E + M)) & 1
    e = (codes >> M) & ((1 << E) - 1)
    m = codes & ((1 << M) - 1)
    mag = np.where(e == 0, 0.0, np.ldexp(1 + m / 2.0 ** M, e.astype(int) - bias))
    expect = np.where(s == 1, -mag, mag).astype(np.float32)
    assert np.array_equal(got.view(np.uint32), expect.view(np.uint32))
    assert got[(1 << (E + M)) - 1] == {8: 480.0, 10: 126976.0}[bits]


@pytest.mark.parametrize("bits", [8, 10, 16])
def test_idempotent_on_codes(ref, bits):
    # encode(decode(c)) == c for every code with a nonzero exponent field (FP16: every
    # finite code; subnormals included).
    E, M = FMT[bits]
    codes = np.arange(1 << (1 + E + M), dtype=np.uint32)
    e = (codes >> M) & ((1 << E) - 1)
    keep = (e != 0) if bits != 16 else (e != 31)
    codes = codes[keep]
    assert np.array_equal(ref.dpr_codes(ref.dpr_values(codes, bits), bits), codes)


@pytest.mark.parametrize("bits", [8, 10])
def test_nearest_code_brute_force(ref, bits):
    # Brute force over the whole codebook: the code is the nearest representable value,
    # ties to the even mantissa (P:171 round-to-nearest, R15), in [min normal, max].
    codes, vals = _codebook(ref, bits)
    rng = np.random.default_rng(bits)
    lo, hi = vals.min(), vals.max()
    x = np.exp2(rng.uniform(np.log2(lo), np.log2(hi), 20_000))
    mids = (vals[:-1] + vals[1:]) / 2
    x = np.concatenate([x, mids, vals]).astype(np.float32)
    x = x[(x >= lo) & (x <= hi)]
    got = ref.dpr_codes(x, bits)
    d = np.abs(x.astype(np.float64)[:, None] - vals[None, :])
    best = d.min(axis=1, keepdims=True)
    cand = d == best
    even = (codes & 1) == 0
    pick = np.where(cand.sum(1) > 1, np.argmax(cand & even[None, :], axis=1), np.argmax(cand, axis=1))
    assert np.array_equal(got, codes[pick])
    # relative error bound in the normal range: <= 2^-(M+1)
    rel = np.abs(ref.dpr_values(got, bits) - x) / x
    assert rel.max() <= 2.0 ** -(FMT[bits][1] + 1)


@pytest.mark.parametrize("bits", [8, 10])
def test_saturate_and_flush(ref, bits):
    E, M = FMT[bits]
    maxcode = ((1 << E) - 1) << M | ((1 << M) - 1)
    x = np.array([1e30, -1e30, np.inf, -np.inf, 1e-30, -1e-30, 1e-45], np.float32)
    got = ref.dpr_codes(x, bits)
    sb = 1 << (E + M)
    assert got.tolist() == [maxcode, sb | maxcode, maxcode, sb | maxcode, 0, sb, 0]


@pytest.mark.parametrize("bits,k", [(16, 2), (10, 3), (8, 4)])
@pytest.mark.parametrize("n", [0, 1, 2, 3, 4, 5, 11, 12, 1000, 4099])
def test_packing_and_ratio(ref, bits, k, n):
    # 2/3/4 values per 4-byte word; FP10 leaves bits 30-31 unused (zero);
    # tail fields zero (R19).  Ratios exactly 2x/3x/4x for n % k == 0.
    rng = np.random.default_rng(n)
    x = (rng.standard_normal(n) * np.exp2(rng.uniform(-8, 8, n))).astype(np.float32)
    w = ref.dpr_encode(x, bits)
    assert w.size == -(-n // k)
    codes = ref.dpr_codes(x, bits)
    for i in range(n):
        assert (int(w[i // k]) >> (bits * (i % k))) & ((1 << bits) - 1) == codes[i]
    if bits == 10 and w.size:
        assert np.all(w >> 30 == 0)
    if n % k:
        assert int(w[-1]) >> (bits * (n % k)) == 0
    if n and n % k == 0:
        assert (4 * n) / (4 * w.size) == k
    y = ref.dpr_decode(w, n, bits)
    assert np.array_equal(y.view(np.uint32), ref.dpr_values(codes, bits).view(np.uint32))
