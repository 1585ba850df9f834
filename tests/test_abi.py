"""CPU-only checks of the C-ABI boundary: libgist.so loads, exports every symbol that
include/gist.h declares, its host size helpers follow the closed forms, and its
synchronous argument validation returns the documented status codes without touching a
GPU."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared():
    src = open(os.path.join(ROOT, "include", "gist.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gist_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_seven_calls():
    names = declared()
    for call in ["gist_binarize_encode", "gist_maxpool_fwd_argmax", "gist_pool_relu_bwd", "gist_ssdc_encode",
                 "gist_ssdc_decode", "gist_dpr_encode", "gist_dpr_decode"]:
        assert call in names


def test_library_exports_every_declared_symbol(gist):
    raw = C.CDLL(gist.library_path)
    missing = [n for n in declared() if not hasattr(raw, n)]
    assert not missing, missing


def test_binding_names_match_abi(gist):
    for n in declared():
        if n != "gist_status_string":
            assert callable(getattr(gist, n)), n


def test_status_strings(gist):
    for code, name in gist.STATUS.items():
        assert gist.lib.gist_status_string(code).decode() == name


def test_size_helpers(gist):
    assert gist.gist_binarize_words(0) == 0
    assert gist.gist_binarize_words(33) == 2
    assert gist.gist_argmax_words(9) == 2
    assert gist.gist_ssdc_rows(257) == 2
    assert gist.gist_ssdc_bytes(512, 100) == 5 * 100 + 4 * 2
    for bits, k in ((16, 2), (10, 3), (8, 4)):
        assert gist.gist_dpr_words(10, bits) == -(-10 // k)
    assert gist.gist_dpr_words(10, 12) == -1
    assert gist.gist_ssdc_workspace_bytes(1 << 20) == 128 + 8 * ((1 << 20) // 8192)  # counters + one tagged total per tile
    assert gist.gist_pool2d_out_dims(56, 56, (3, 3, 2, 2, 0, 0, 0)) == (27, 27)
    assert gist.gist_pool2d_out_dims(54, 54, (3, 3, 2, 2, 0, 0, 1)) == (27, 27)  # NiN ceil
    assert gist.gist_pool2d_out_dims(112, 112, (3, 3, 2, 2, 0, 0, 1)) == (56, 56)  # GoogLeNet
    assert gist.gist_pool2d_out_dims(28, 28, (3, 3, 1, 1, 1, 1, 0)) == (28, 28)


def test_pool_dims_match_oracle(gist, ref):
    from pool_cases import GEOMS
    for g in GEOMS:
        for H in range(1, 40):
            if H + 2 * g[4] < g[0]:
                continue
            Ho, _ = gist.gist_pool2d_out_dims(H, H + 2 * g[5] if H + 2 * g[5] >= g[1] else g[1], g)
            assert Ho == ref.pool_out_dim(H, g[0], g[2], g[4], g[6])


OK, INVALID, MISALIGNED, UNSUPPORTED, TOO_LARGE = 0, 1, 2, 3, 4
A, B = 0x10000, 0x20000000  # fake, 16-byte aligned, non-overlapping device addresses


def test_validation_without_gpu(gist):
    L = gist.lib
    P = gist.Pool2d
    # n == 0 launches nothing
    assert L.gist_binarize_encode(None, 0, None, None) == OK
    assert L.gist_dpr_encode(None, 0, 16, None, None) == OK
    assert L.gist_dpr_decode(None, 0, 8, None, None) == OK
    assert L.gist_ssdc_decode(None, None, None, 0, None, None) == OK
    # NULL / negative
    assert L.gist_binarize_encode(None, 10, B, None) == INVALID
    assert L.gist_binarize_encode(A, -1, B, None) == INVALID
    # misaligned
    assert L.gist_binarize_encode(A + 4, 10, B, None) == MISALIGNED
    assert L.gist_dpr_encode(A, 10, 16, B + 8, None) == MISALIGNED
    # overlap
    assert L.gist_binarize_encode(A, 1000, A + 16, None) == INVALID
    assert L.gist_dpr_decode(A, 1000, 16, A, None) == INVALID
    # DPR widths (16, 10, 8 only)
    for bits in (0, 4, 9, 12, 32):
        assert L.gist_dpr_encode(A, 10, bits, B, None) == UNSUPPORTED
        assert L.gist_dpr_decode(A, 10, bits, B, None) == UNSUPPORTED
    # pooling geometry
    g = P(5, 5, 1, 1, 0, 0, 0)  # 25 window positions do not fit 4 bits
    assert L.gist_maxpool_fwd_argmax(A, 1, 1, 8, 8, C.byref(g), B, B + 4096, None, None) == UNSUPPORTED
    g = P(3, 3, 2, 2, 2, 2, 0)  # padding > k/2
    assert L.gist_maxpool_fwd_argmax(A, 1, 1, 8, 8, C.byref(g), B, B + 4096, None, None) == INVALID
    g = P(2, 2, 2, 2, 0, 0, 0)
    assert L.gist_relu_maxpool_fwd_argmax(A, 1, 1, 8, 8, C.byref(g), B, B + 4096, None, None) == INVALID  # f3 needs the mask
    assert L.gist_relu_maxpool_fwd_argmax(A + 4, 1, 1, 8, 8, C.byref(g), B, B + 4096, B + 8192, None) == MISALIGNED
    g = P(3, 3, 0, 2, 0, 0, 0)  # zero stride
    assert L.gist_pool_relu_bwd(A, B, None, 1, 1, 8, 8, C.byref(g), B + 4096, None) == INVALID
    g = P(3, 3, 2, 2, 0, 0, 0)
    assert L.gist_maxpool_fwd_argmax(A, 1, 1, 2, 2, C.byref(g), B, B + 4096, None, None) == INVALID  # Ho < 1
    assert L.gist_maxpool_fwd_argmax(A, 1 << 16, 1 << 10, 64, 64, C.byref(g), B, B + 4096, None, None) == TOO_LARGE
    # SSDC
    n = 1 << 31
    assert L.gist_ssdc_encode(A, n, B, None, None, 0, B + 64, B + 128, 1 << 20, None) == TOO_LARGE
    assert L.gist_ssdc_decode(A, None, None, n, B, None) == TOO_LARGE
    assert L.gist_ssdc_encode(A, 1024, B, None, None, 16, B + 4096, B + 8192, 4096, None) == INVALID  # cap w/o col
    assert L.gist_ssdc_encode(A, 1 << 20, B, B + (1 << 24), B + (1 << 26), 1 << 20, B + (1 << 28), B + (1 << 29),
                              8, None) == INVALID  # workspace too small
    assert L.gist_ssdc_encode(A, 1024, B, None, None, 0, B + 4100, B + 8192, 4096, None) == MISALIGNED  # nnz
    assert L.gist_ssdc_workspace_init(None, 0, None) == OK  # nothing to zero: no CUDA call
    assert L.gist_ssdc_workspace_init(None, 256, None) == INVALID
    assert L.gist_ssdc_workspace_init(B + 4, 256, None) == MISALIGNED
    assert L.gist_ssdc_workspace_init(B, 64, None) == INVALID  # smaller than the counter line
    # f1: DPR over SSDC values (device count)
    assert L.gist_ssdc_dpr_encode(A, B, 0, 16, B + 64, None) == OK
    assert L.gist_ssdc_dpr_encode(A, B, 100, 12, B + 64, None) == UNSUPPORTED
    assert L.gist_ssdc_dpr_encode(A, None, 100, 8, B + 64, None) == INVALID
    assert L.gist_ssdc_dpr_decode(A, B + 4, 100, 8, B + 64, None) == MISALIGNED


def test_wgrad_validation_without_gpu(gist):
    """f4 (gist_conv3x3_wgrad_ssdc): host-side validation returns the documented codes, no launch."""
    L = gist.lib
    N, Ci, Co, H, W = 2, 16, 128, 8, 8
    ws = gist.gist_conv3x3_wgrad_workspace_bytes(N, Ci, Co, H, W)
    assert ws > 0
    args = lambda **k: [k.get("dy", A), B, B + 4096, B + 8192, k.get("N", N), k.get("Ci", Ci), k.get("Co", Co),
                        k.get("H", H), k.get("W", W), k.get("passes", 3), k.get("dw", B + (1 << 20)),
                        k.get("ws", B + (1 << 21)), k.get("wsb", ws), None]
    assert L.gist_conv3x3_wgrad_ssdc(*args(passes=2)) == UNSUPPORTED
    assert L.gist_conv3x3_wgrad_ssdc(*args(Co=64)) == UNSUPPORTED      # M tile of 128 output channels
    assert L.gist_conv3x3_wgrad_ssdc(*args(Ci=24)) == UNSUPPORTED      # 16 input channels per N tile
    assert L.gist_conv3x3_wgrad_ssdc(*args(W=300)) == UNSUPPORTED      # decode slab does not fit
    assert L.gist_conv3x3_wgrad_ssdc(*args(H=7, W=7)) == UNSUPPORTED   # H*W % 4: dY rows are TMA rows
    assert L.gist_conv3x3_wgrad_ssdc(*args(N=-1)) == INVALID
    assert L.gist_conv3x3_wgrad_ssdc(*args(dy=None)) == INVALID
    assert L.gist_conv3x3_wgrad_ssdc(*args(dy=A + 4)) == MISALIGNED
    assert L.gist_conv3x3_wgrad_ssdc(*args(wsb=ws - 1)) == INVALID      # workspace too small
    assert L.gist_conv3x3_wgrad_ssdc(*args(Ci=0)) == OK                 # empty dW: nothing to write
    big = (1 << 31) // (Ci * H * W) + 1
    assert L.gist_conv3x3_wgrad_ssdc(*args(N=big, wsb=1 << 40)) == TOO_LARGE
    assert gist.gist_conv3x3_wgrad_workspace_bytes(N, Ci, 64, H, W) == 0


def test_pool_geometry_overflow_rejected(gist):
    """A window whose kh*kw wraps in int32 (kh=3, kw=1431655766 -> 2 mod 2^32) must not pass the
    4-bit argmax check; huge padded spans must not wrap either."""
    L = gist.lib
    P = gist.Pool2d
    g = P(3, 1431655766, 1, 1, 0, 715827883, 0)
    assert L.gist_maxpool_fwd_argmax(A, 1, 1, 4, 1, C.byref(g), B, B + 4096, None, None) == UNSUPPORTED
    assert L.gist_pool_relu_bwd(A, B, None, 1, 1, 4, 1, C.byref(g), B + 4096, None) == UNSUPPORTED
    g = P(17, 1, 1, 1, 0, 0, 0)
    assert L.gist_maxpool_fwd_argmax(A, 1, 1, 32, 32, C.byref(g), B, B + 4096, None, None) == UNSUPPORTED
    Ho, Wo = C.c_int32(), C.c_int32()
    g = P(3, 3, 1, 1, 1, 1, 0)
    assert L.gist_pool2d_out_dims(2**31 - 1, 8, C.byref(g), C.byref(Ho), C.byref(Wo)) == OK
    assert Ho.value == 2**31 - 1 and Wo.value == 8  # (H + 2 - 3)/1 + 1 computed without wrapping


def test_binding_rejects_wrong_dtypes_and_devices(gist):
    """The C ABI sees raw pointers only; the binding checks dtype, device and size before the call
    (a bf16 map read as fp32 would run 2x past its buffer)."""
    import torch
    with pytest.raises(ValueError):
        gist._ptr(torch.zeros(4), gist._F32, name="y")  # CPU tensor: no fallback
    meta = torch.empty(8, dtype=torch.bfloat16, device="meta")
    with pytest.raises(ValueError):
        gist._ptr(meta, gist._F32, name="y")


def test_many_calls_validation_without_gpu(gist):
    L = gist.lib
    J = gist.SsdcJob
    assert L.gist_ssdc_encode_many(None, 0, None, 0, None) == OK
    assert L.gist_ssdc_encode_many(None, 1, None, 0, None) == INVALID
    assert L.gist_ssdc_decode_many(None, 0, None) == OK
    assert L.gist_dpr_encode_many(None, 0, 16, None) == OK
    assert L.gist_dpr_encode_many(None, 0, 12, None) == UNSUPPORTED
    jobs = (J * 2)()
    jobs[0] = J(A, 1024, B, B + 4096, B + 8192, 1024, B + 16384, None)
    jobs[1] = J(A + 4, 1024, B + 32768, B + 36864, B + 40960, 1024, B + 49152, None)  # misaligned x
    ws = gist.lib.gist_ssdc_workspace_bytes_many(jobs, 2)
    assert ws == 128 + 8 * 2
    assert L.gist_ssdc_encode_many(jobs, 2, B + (1 << 20), ws, None) == MISALIGNED
    jobs[1] = J(A + 8192, 1024, B + 32768, B + 36864, B + 40960, 1024, B + 49152, B + 16384)  # chained: ok so far
    assert L.gist_ssdc_encode_many(jobs, 2, B + (1 << 20), 8, None) == INVALID  # workspace too small
    jobs[1] = J(A + 8192, 1024, B + 32768, B + 36864, B + 40960, 1024, B + 49152, B + 49152)  # own nnz
    assert L.gist_ssdc_encode_many(jobs, 2, B + (1 << 20), ws, None) == INVALID
    D = gist.DprJob
    dj = (D * 1)(D(A, 100, A + 16))  # overlapping in/out
    assert L.gist_dpr_encode_many(dj, 1, 16, None) == INVALID
