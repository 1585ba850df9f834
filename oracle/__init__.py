"""CPU oracle for Gist's stash-time encode/decode hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_isca_jainpmtp18_b200``) never imports it and shares no code with it.

This module is argument marshalling over ``oracle/gist_oracle.c`` (numpy arrays in,
numpy arrays out); every line of arithmetic lives in that C file, which cites the
PAPER.md passage each function follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gist_oracle.c")
_LIB = os.path.join(_HERE, "libgist_oracle.so")

CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-std=c11", "-shared", "-fPIC"]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (strict IEEE binary32/binary64, no contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib() -> C.CDLL:
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        i64, i32, u32, p = C.c_int64, C.c_int32, C.c_uint32, C.c_void_p
        sig = {
            "oracle_binarize_words": (i64, [i64]),
            "oracle_binarize_encode": (None, [p, i64, p]),
            "oracle_pool_out_dim": (i32, [i32, i32, i32, i32, i32]),
            "oracle_argmax_words": (i64, [i64]),
            "oracle_maxpool_fwd_argmax": (None, [p, i32, i32, i32, i32] + [i32] * 7 + [p, p]),
            "oracle_pool_relu_bwd": (None, [p, p, p, i32, i32, i32, i32] + [i32] * 7 + [p]),
            "oracle_ssdc_rows": (i64, [i64]),
            "oracle_ssdc_encode": (i64, [p, i64, p, p, p]),
            "oracle_ssdc_decode": (None, [p, p, p, i64, p]),
            "oracle_dpr_code": (u32, [C.c_float, i32]),
            "oracle_dpr_value": (C.c_float, [u32, i32]),
            "oracle_dpr_per_word": (i32, [i32]),
            "oracle_dpr_words": (i64, [i64, i32]),
            "oracle_dpr_encode": (None, [p, i64, i32, p]),
            "oracle_dpr_decode": (None, [p, i64, i32, p]),
            "oracle_dpr_codes": (None, [p, i64, i32, p]),
            "oracle_dpr_values": (None, [p, i64, i32, p]),
            "oracle_conv3x3_wgrad_entries": (None, [p, p, i32, i32, i32, i32, i32, p, i64, p, p]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(_lib, name)
            fn.restype = res
            fn.argtypes = args
    return _lib


def _ptr(a: np.ndarray | None):
    return None if a is None else a.ctypes.data


def _f32(a) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a


# ---------------------------------------------------------------- O1 Binarize
def binarize_words(n: int) -> int:
    return lib().oracle_binarize_words(n)


def binarize_encode(y) -> np.ndarray:
    y = _f32(y).reshape(-1)
    out = np.empty(binarize_words(y.size), np.uint32)
    lib().oracle_binarize_encode(_ptr(y), y.size, _ptr(out))
    return out


# ---------------------------------------------------------------- O2/O3 pooling
def pool_out_dim(size: int, k: int, s: int, p: int, ceil_mode: bool) -> int:
    return lib().oracle_pool_out_dim(size, k, s, p, int(bool(ceil_mode)))


def argmax_words(n_out: int) -> int:
    return lib().oracle_argmax_words(n_out)


def _geom(pool):
    kh, kw, sh, sw, ph, pw, cm = pool
    return [int(kh), int(kw), int(sh), int(sw), int(ph), int(pw), int(bool(cm))]


def maxpool_fwd_argmax(y, pool):
    """y: float32 [N,C,H,W]; pool = (kh, kw, sh, sw, ph, pw, ceil_mode).
    Returns (out float32 [N,C,Ho,Wo], arg uint32 [ceil(n_out/8)])."""
    y = _f32(y)
    N, Cc, H, W = y.shape
    g = _geom(pool)
    Ho = pool_out_dim(H, g[0], g[2], g[4], g[6])
    Wo = pool_out_dim(W, g[1], g[3], g[5], g[6])
    out = np.empty((N, Cc, Ho, Wo), np.float32)
    arg = np.empty(argmax_words(out.size), np.uint32)
    lib().oracle_maxpool_fwd_argmax(_ptr(y), N, Cc, H, W, *g, _ptr(out), _ptr(arg))
    return out, arg


def pool_relu_bwd(dout, arg, mask, shape, pool):
    """dout float32 [N,C,Ho,Wo]; arg/mask uint32 words (mask may be None);
    shape = (N,C,H,W).  Returns dx float32 [N,C,H,W]."""
    dout = _f32(dout)
    arg = np.ascontiguousarray(arg, np.uint32)
    mask = None if mask is None else np.ascontiguousarray(mask, np.uint32)
    N, Cc, H, W = shape
    dx = np.empty((N, Cc, H, W), np.float32)
    lib().oracle_pool_relu_bwd(_ptr(dout), _ptr(arg), _ptr(mask), N, Cc, H, W, *_geom(pool), _ptr(dx))
    return dx


# ---------------------------------------------------------------- O4/O5 SSDC
def ssdc_rows(n: int) -> int:
    return lib().oracle_ssdc_rows(n)


def ssdc_encode(x):
    """Returns (row_end int32[rows], col uint8[nnz], val float32[nnz])."""
    x = _f32(x).reshape(-1)
    row_end = np.empty(ssdc_rows(x.size), np.int32)
    col = np.empty(max(x.size, 1), np.uint8)
    val = np.empty(max(x.size, 1), np.float32)
    nnz = lib().oracle_ssdc_encode(_ptr(x), x.size, _ptr(row_end), _ptr(col), _ptr(val))
    return row_end, col[:nnz].copy(), val[:nnz].copy()


def ssdc_decode(row_end, col, val, n: int) -> np.ndarray:
    row_end = np.ascontiguousarray(row_end, np.int32)
    col = np.ascontiguousarray(col, np.uint8)
    val = _f32(val)
    x = np.empty(n, np.float32)
    lib().oracle_ssdc_decode(_ptr(row_end), _ptr(col), _ptr(val), n, _ptr(x))
    return x


# ---------------------------------------------------------------- O6/O7 DPR
def dpr_words(n: int, bits: int) -> int:
    return lib().oracle_dpr_words(n, bits)


def dpr_encode(x, bits: int) -> np.ndarray:
    x = _f32(x).reshape(-1)
    out = np.empty(dpr_words(x.size, bits), np.uint32)
    lib().oracle_dpr_encode(_ptr(x), x.size, bits, _ptr(out))
    return out


def dpr_decode(packed, n: int, bits: int) -> np.ndarray:
    packed = np.ascontiguousarray(packed, np.uint32)
    x = np.empty(n, np.float32)
    lib().oracle_dpr_decode(_ptr(packed), n, bits, _ptr(x))
    return x


def dpr_codes(x, bits: int) -> np.ndarray:
    """Per-element code (unpacked), for pin tests over large value sets."""
    x = _f32(x).reshape(-1)
    out = np.empty(x.size, np.uint32)
    lib().oracle_dpr_codes(_ptr(x), x.size, bits, _ptr(out))
    return out


def dpr_values(codes, bits: int) -> np.ndarray:
    codes = np.ascontiguousarray(codes, np.uint32).reshape(-1)
    out = np.empty(codes.size, np.float32)
    lib().oracle_dpr_values(_ptr(codes), codes.size, bits, _ptr(out))
    return out


# ---------------------------------------------------------------- O8 f4 reference (conv weight gradient)
def conv3x3_wgrad_entries(dy, x, entries):
    """dW entries (co, ci, tap) of a 3x3/s1/p1 conv, and sum |dY*X| for each (binary64)."""
    dy, x = _f32(dy), _f32(x)
    N, Co, H, W = dy.shape
    Ci = x.shape[1]
    ent = np.ascontiguousarray(entries, np.int32).reshape(-1, 3)
    dw = np.empty(len(ent), np.float64)
    mag = np.empty(len(ent), np.float64)
    lib().oracle_conv3x3_wgrad_entries(_ptr(dy), _ptr(x), N, Ci, Co, H, W, _ptr(ent), len(ent), _ptr(dw), _ptr(mag))
    return dw, mag


def conv3x3_wgrad(dy, x):
    """The full dW [Co, Ci, 3, 3] (binary64) and sum |dY*X| per entry."""
    Co, Ci = dy.shape[1], x.shape[1]
    ent = np.stack(np.meshgrid(np.arange(Co), np.arange(Ci), np.arange(9), indexing="ij"), -1).reshape(-1, 3)
    dw, mag = conv3x3_wgrad_entries(dy, x, ent)
    return dw.reshape(Co, Ci, 3, 3), mag.reshape(Co, Ci, 3, 3)
