"""Python binding of libgist — Gist's stash-time encode/decode hot path on B200 (sm_100a).

Argument marshalling only: every function below checks what the C ABI cannot see (a torch
tensor's device, dtype, contiguity and element count), allocates outputs with torch on the
input's device when the caller passes none, and forwards raw device pointers plus torch's
current CUDA stream to the same-named C-ABI call in ``include/gist.h`` (ctypes).  All arithmetic runs in the CUDA kernels of ``csrc/``.
There is no CPU fallback: importing this package without ``libgist.so`` raises, and a
non-CUDA tensor is rejected.

Paper: Jain et al., "Gist: Efficient Data Encoding for Deep Neural Network Training",
ISCA 2018 (§IV-A, P:151-P:171).
"""
from __future__ import annotations

import ctypes as C
import os

import torch

__all__ = [
    "GistError", "Pool2d", "lib", "library_path",
    "gist_binarize_words", "gist_argmax_words", "gist_pool2d_out_dims", "gist_ssdc_rows",
    "gist_ssdc_bytes", "gist_ssdc_workspace_bytes", "gist_ssdc_workspace", "gist_ssdc_workspace_init", "gist_dpr_words", "gist_num_sms", "gist_launch_count",
    "gist_binarize_encode", "gist_maxpool_fwd_argmax", "gist_relu_maxpool_fwd_argmax", "gist_pool_relu_bwd",
    "gist_ssdc_encode", "gist_ssdc_decode", "gist_dpr_encode", "gist_dpr_decode",
    "gist_ssdc_dpr_encode", "gist_ssdc_dpr_decode",
    "gist_ssdc_workspace_bytes_many", "gist_ssdc_encode_many", "gist_ssdc_decode_many", "gist_dpr_encode_many",
    "gist_dpr_decode_many", "SsdcEncodeMany", "SsdcDecodeMany", "DprMany",
    "gist_conv3x3_wgrad_workspace_bytes", "gist_conv3x3_wgrad_ssdc",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
library_path = os.environ.get("GIST_LIBRARY") or os.path.join(_HERE, "libgist.so")  # override: tuning variants

STATUS = {0: "GIST_OK", 1: "GIST_ERR_INVALID_ARGUMENT", 2: "GIST_ERR_MISALIGNED",
          3: "GIST_ERR_UNSUPPORTED", 4: "GIST_ERR_TOO_LARGE", 5: "GIST_ERR_CUDA"}


class GistError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {STATUS.get(status, status)}")


class Pool2d(C.Structure):
    """gist_pool2d: (kh, kw, sh, sw, ph, pw, ceil_mode), torch max_pool2d semantics."""
    _fields_ = [(f, C.c_int32) for f in ("kh", "kw", "sh", "sw", "ph", "pw", "ceil_mode")]

    @classmethod
    def of(cls, g) -> "Pool2d":
        if isinstance(g, Pool2d):
            return g
        return cls(*[int(v) for v in g])


class SsdcJob(C.Structure):
    """gist_ssdc_job (include/gist.h)."""
    _fields_ = [("x", C.c_void_p), ("n", C.c_int64), ("row_end", C.c_void_p), ("col", C.c_void_p),
                ("val", C.c_void_p), ("capacity", C.c_int64), ("nnz", C.c_void_p), ("offset", C.c_void_p)]


class SsdcDecodeJob(C.Structure):
    """gist_ssdc_decode_job (include/gist.h)."""
    _fields_ = [("row_end", C.c_void_p), ("col", C.c_void_p), ("val", C.c_void_p), ("offset", C.c_void_p),
                ("n", C.c_int64), ("x", C.c_void_p)]


class DprJob(C.Structure):
    """gist_dpr_job (include/gist.h)."""
    _fields_ = [("x", C.c_void_p), ("n", C.c_int64), ("packed", C.c_void_p)]


def _load() -> C.CDLL:
    if not os.path.exists(library_path):
        raise ImportError(
            f"{library_path} is missing: build it with `python build_gist.py` "
            "(there is no CPU fallback for the Gist kernels)")
    L = C.CDLL(library_path)
    i64, i32, p, sz = C.c_int64, C.c_int32, C.c_void_p, C.c_size_t
    P = C.POINTER(Pool2d)
    sigs = {
        "gist_status_string": (C.c_char_p, [C.c_int]),
        "gist_binarize_words": (i64, [i64]),
        "gist_argmax_words": (i64, [i64]),
        "gist_pool2d_out_dims": (C.c_int, [i32, i32, P, C.POINTER(i32), C.POINTER(i32)]),
        "gist_ssdc_rows": (i64, [i64]),
        "gist_ssdc_bytes": (i64, [i64, i64]),
        "gist_ssdc_workspace_bytes": (sz, [i64]),
        "gist_ssdc_workspace_init": (C.c_int, [p, sz, p]),
        "gist_dpr_words": (i64, [i64, i32]),
        "gist_num_sms": (i32, []),
        "gist_launch_count": (C.c_uint64, []),
        "gist_binarize_encode": (C.c_int, [p, i64, p, p]),
        "gist_maxpool_fwd_argmax": (C.c_int, [p, i32, i32, i32, i32, P, p, p, p, p]),
        "gist_pool_relu_bwd": (C.c_int, [p, p, p, i32, i32, i32, i32, P, p, p]),
        "gist_relu_maxpool_fwd_argmax": (C.c_int, [p, i32, i32, i32, i32, P, p, p, p, p]),
        "gist_ssdc_encode": (C.c_int, [p, i64, p, p, p, i64, p, p, sz, p]),
        "gist_ssdc_decode": (C.c_int, [p, p, p, i64, p, p]),
        "gist_dpr_encode": (C.c_int, [p, i64, i32, p, p]),
        "gist_dpr_decode": (C.c_int, [p, i64, i32, p, p]),
        "gist_ssdc_dpr_encode": (C.c_int, [p, p, i64, i32, p, p]),
        "gist_ssdc_dpr_decode": (C.c_int, [p, p, i64, i32, p, p]),
        "gist_ssdc_workspace_bytes_many": (sz, [p, i32]),
        "gist_ssdc_encode_many": (C.c_int, [p, i32, p, sz, p]),
        "gist_ssdc_decode_many": (C.c_int, [p, i32, p]),
        "gist_dpr_encode_many": (C.c_int, [p, i32, i32, p]),
        "gist_dpr_decode_many": (C.c_int, [p, i32, i32, p]),
        "gist_conv3x3_wgrad_workspace_bytes": (sz, [i32, i32, i32, i32, i32]),
        "gist_conv3x3_wgrad_ssdc": (C.c_int, [p, p, p, p, i32, i32, i32, i32, i32, i32, p, p, sz, p]),
    }
    for name, (res, args) in sigs.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    return L


lib = _load()


# ------------------------------------------------------------------ marshalling helpers
_F32 = (torch.float32,)
_W32 = (torch.int32, torch.uint32)  # uint32 words (the binding allocates int32 views)
_U8 = (torch.uint8,)
_I32 = (torch.int32,)
_I64 = (torch.int64,)


def _ptr(t: torch.Tensor | None, dtypes=None, device=None, numel: int | None = None, name: str = "tensor"):
    """Raw device pointer of `t` after the checks the C ABI cannot make: a CUDA tensor,
    contiguous, of one of `dtypes`, on `device` (when given), with at least `numel` elements."""
    if t is None:
        return None
    if not t.is_cuda:
        raise ValueError(f"libgist takes CUDA tensors only (no CPU fallback): {name} is on {t.device}")
    if not t.is_contiguous():
        raise ValueError(f"libgist takes contiguous tensors: {name}")
    if dtypes is not None and t.dtype not in dtypes:
        raise ValueError(f"{name} must be {' or '.join(str(d) for d in dtypes)}, got {t.dtype}")
    if device is not None and t.device != device:
        raise ValueError(f"{name} is on {t.device}, the call's tensors are on {device}")
    if numel is not None and t.numel() < numel:
        raise ValueError(f"{name} holds {t.numel()} elements, the call needs {numel}")
    return t.data_ptr()


def _stream(t: torch.Tensor, stream=None):
    s = stream if stream is not None else torch.cuda.current_stream(t.device)
    return s.cuda_stream if hasattr(s, "cuda_stream") else s


def _check(status: int, where: str):
    if status != 0:
        raise GistError(status, where)


def _words(n: int, dev, out=None):
    return out if out is not None else torch.empty(max(n, 0), dtype=torch.int32, device=dev)


# ------------------------------------------------------------------ size helpers
def gist_binarize_words(n: int) -> int:
    return lib.gist_binarize_words(n)


def gist_argmax_words(n_out: int) -> int:
    return lib.gist_argmax_words(n_out)


def gist_pool2d_out_dims(H: int, W: int, pool) -> tuple[int, int]:
    Ho, Wo = C.c_int32(), C.c_int32()
    _check(lib.gist_pool2d_out_dims(H, W, C.byref(Pool2d.of(pool)), C.byref(Ho), C.byref(Wo)),
           "gist_pool2d_out_dims")
    return Ho.value, Wo.value


def gist_ssdc_rows(n: int) -> int:
    return lib.gist_ssdc_rows(n)


def gist_ssdc_bytes(n: int, nnz: int) -> int:
    return lib.gist_ssdc_bytes(n, nnz)


def gist_ssdc_workspace_bytes(n: int) -> int:
    return lib.gist_ssdc_workspace_bytes(n)


def gist_ssdc_workspace_init(workspace: torch.Tensor, stream=None) -> torch.Tensor:
    """Zero a gist_ssdc_encode workspace (required once before its first use)."""
    _check(lib.gist_ssdc_workspace_init(_ptr(workspace), workspace.numel() * workspace.element_size(),
                                        _stream(workspace, stream)), "gist_ssdc_workspace_init")
    return workspace


def gist_ssdc_workspace(n: int, device, stream=None) -> torch.Tensor:
    """A workspace for gist_ssdc_encode of up to n elements, initialised with
    gist_ssdc_workspace_init (once; every encode leaves it reusable)."""
    ws = torch.empty(max(gist_ssdc_workspace_bytes(n), 1), dtype=torch.uint8, device=device)
    return gist_ssdc_workspace_init(ws, stream)


def gist_dpr_words(n: int, bits: int) -> int:
    return lib.gist_dpr_words(n, bits)


def gist_num_sms() -> int:
    return lib.gist_num_sms()


def gist_launch_count() -> int:
    """Kernels libgist has enqueued so far in this process."""
    return lib.gist_launch_count()


# ------------------------------------------------------------------ a1..a7
# Every call runs under torch.cuda.device(<the call's device>), so the library's per-device
# launch state (SM count, shared-memory opt-ins) is the one of the device the tensors live on.
def gist_binarize_encode(y: torch.Tensor, mask: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a1: 1-bit ReLU mask, int32 tensor of uint32 words (bit i = y[i] > 0)."""
    n = y.numel()
    dev = y.device
    mask = _words(gist_binarize_words(n), dev, mask)
    with torch.cuda.device(dev):
        _check(lib.gist_binarize_encode(_ptr(y, _F32, name="y"), n,
                                        _ptr(mask, _W32, dev, gist_binarize_words(n), "mask"), _stream(y, stream)),
               "gist_binarize_encode")
    return mask


def _pool_outputs(x, g, out, argmax):
    N, Cc, H, W = x.shape
    Ho, Wo = gist_pool2d_out_dims(H, W, g)
    if out is None:
        out = torch.empty((N, Cc, Ho, Wo), dtype=torch.float32, device=x.device)
    argmax = _words(gist_argmax_words(N * Cc * Ho * Wo), x.device, argmax)
    return (N, Cc, H, W), N * Cc * Ho * Wo, out, argmax


def gist_maxpool_fwd_argmax(y: torch.Tensor, pool, out=None, argmax=None, mask=None, fuse_mask=False,
                            stream=None):
    """a2: returns (out [N,C,Ho,Wo] fp32, argmax int32 words, mask or None).
    fuse_mask=True (or a mask tensor) also writes the a1 mask of y."""
    g = Pool2d.of(pool)
    (N, Cc, H, W), n_out, out, argmax = _pool_outputs(y, g, out, argmax)
    dev = y.device
    if mask is None and fuse_mask:
        mask = _words(gist_binarize_words(y.numel()), dev)
    with torch.cuda.device(dev):
        _check(lib.gist_maxpool_fwd_argmax(
            _ptr(y, _F32, name="y"), N, Cc, H, W, C.byref(g), _ptr(out, _F32, dev, n_out, "out"),
            _ptr(argmax, _W32, dev, gist_argmax_words(n_out), "argmax"),
            _ptr(mask, _W32, dev, gist_binarize_words(y.numel()), "mask"), _stream(y, stream)),
            "gist_maxpool_fwd_argmax")
    return out, argmax, mask


def gist_relu_maxpool_fwd_argmax(x: torch.Tensor, pool, out=None, argmax=None, mask=None, stream=None):
    """f3 (P:139, P:152-P:156): ReLU applied on load to the pre-activation map x, then a2 + a1:
    returns (out, argmax words, mask) equal to gist_maxpool_fwd_argmax(relu(x), pool, fuse_mask=True);
    the ReLU output is never materialised."""
    g = Pool2d.of(pool)
    (N, Cc, H, W), n_out, out, argmax = _pool_outputs(x, g, out, argmax)
    dev = x.device
    mask = _words(gist_binarize_words(x.numel()), dev, mask)
    with torch.cuda.device(dev):
        _check(lib.gist_relu_maxpool_fwd_argmax(
            _ptr(x, _F32, name="x"), N, Cc, H, W, C.byref(g), _ptr(out, _F32, dev, n_out, "out"),
            _ptr(argmax, _W32, dev, gist_argmax_words(n_out), "argmax"),
            _ptr(mask, _W32, dev, gist_binarize_words(x.numel()), "mask"), _stream(x, stream)),
            "gist_relu_maxpool_fwd_argmax")
    return out, argmax, mask


def gist_pool_relu_bwd(dout: torch.Tensor, argmax: torch.Tensor, mask: torch.Tensor | None, shape, pool,
                       dx: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a3: dx [N,C,H,W] from dY, the 4-bit argmax map and the 1-bit mask."""
    N, Cc, H, W = shape
    g = Pool2d.of(pool)
    Ho, Wo = gist_pool2d_out_dims(H, W, g)
    n, n_out = N * Cc * H * W, N * Cc * Ho * Wo
    dev = dout.device
    if dx is None:
        dx = torch.empty((N, Cc, H, W), dtype=torch.float32, device=dev)
    with torch.cuda.device(dev):
        _check(lib.gist_pool_relu_bwd(
            _ptr(dout, _F32, dev, n_out, "dout"), _ptr(argmax, _W32, dev, gist_argmax_words(n_out), "argmax"),
            _ptr(mask, _W32, dev, gist_binarize_words(n), "mask"), N, Cc, H, W, C.byref(g),
            _ptr(dx, _F32, dev, n, "dx"), _stream(dout, stream)), "gist_pool_relu_bwd")
    return dx


def gist_ssdc_encode(x: torch.Tensor, capacity: int | None = None, row_end=None, col=None, val=None, nnz=None,
                     workspace=None, trim: bool = False, stream=None):
    """a4 (P:158-P:164): returns (row_end int32[rows], col uint8[capacity], val fp32[capacity],
    nnz int64[1] on device).  capacity defaults to n (always complete).  trim=True reads nnz
    back (one D2H sync) and returns col/val views of exactly nnz entries."""
    n = x.numel()
    dev = x.device
    cap = n if capacity is None else int(capacity)
    if row_end is None:
        row_end = torch.empty(gist_ssdc_rows(n), dtype=torch.int32, device=dev)
    if col is None:
        col = torch.empty(max(cap, 1), dtype=torch.uint8, device=dev)
    if val is None:
        val = torch.empty(max(cap, 1), dtype=torch.float32, device=dev)
    if nnz is None:
        nnz = torch.empty(1, dtype=torch.int64, device=dev)
    if workspace is None:
        workspace = gist_ssdc_workspace(n, dev, stream)
    with torch.cuda.device(dev):
        _check(lib.gist_ssdc_encode(
            _ptr(x, _F32, name="x"), n, _ptr(row_end, _I32, dev, gist_ssdc_rows(n), "row_end"),
            _ptr(col, _U8, dev, cap, "col"), _ptr(val, _F32, dev, cap, "val"), cap, _ptr(nnz, _I64, dev, 1, "nnz"),
            _ptr(workspace, None, dev, name="workspace"), workspace.numel() * workspace.element_size(),
            _stream(x, stream)), "gist_ssdc_encode")
    if trim:
        k = int(nnz.item())
        if k < 0:
            raise GistError(1, "gist_ssdc_encode: the workspace was not initialised (gist_ssdc_workspace_init)")
        if k > cap:
            raise GistError(4, f"gist_ssdc_encode: nnz {k} exceeds capacity {cap}")
        return row_end, col[:k], val[:k], nnz
    return row_end, col, val, nnz


def gist_ssdc_decode(row_end: torch.Tensor, col: torch.Tensor, val: torch.Tensor, n: int,
                     x: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a5: dense fp32 [n] from the CSR encoding."""
    dev = row_end.device
    if x is None:
        x = torch.empty(n, dtype=torch.float32, device=dev)
    with torch.cuda.device(dev):
        _check(lib.gist_ssdc_decode(_ptr(row_end, _I32, dev, gist_ssdc_rows(n), "row_end"),
                                    _ptr(col, _U8, dev, name="col"), _ptr(val, _F32, dev, name="val"), n,
                                    _ptr(x, _F32, dev, n, "x"), _stream(row_end, stream)), "gist_ssdc_decode")
    return x


def gist_dpr_encode(x: torch.Tensor, bits: int, packed: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a6: fp32 -> FP16/FP10/FP8 codes packed 2/3/4 per 32-bit word (int32 tensor)."""
    n = x.numel()
    words = gist_dpr_words(n, bits)
    if words < 0:
        raise GistError(3, "gist_dpr_encode")
    dev = x.device
    packed = _words(words, dev, packed)
    with torch.cuda.device(dev):
        _check(lib.gist_dpr_encode(_ptr(x, _F32, name="x"), n, bits, _ptr(packed, _W32, dev, words, "packed"),
                                   _stream(x, stream)), "gist_dpr_encode")
    return packed


def gist_dpr_decode(packed: torch.Tensor, n: int, bits: int, x: torch.Tensor | None = None,
                    stream=None) -> torch.Tensor:
    """a7: packed codes -> fp32 [n]."""
    dev = packed.device
    words = gist_dpr_words(n, bits)
    if words < 0:
        raise GistError(3, "gist_dpr_decode")
    if x is None:
        x = torch.empty(n, dtype=torch.float32, device=dev)
    with torch.cuda.device(dev):
        _check(lib.gist_dpr_decode(_ptr(packed, _W32, dev, words, "packed"), n, bits, _ptr(x, _F32, dev, n, "x"),
                                   _stream(packed, stream)), "gist_dpr_decode")
    return x


def gist_ssdc_dpr_encode(val: torch.Tensor, nnz: torch.Tensor, bits: int, capacity: int | None = None,
                         packed: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """f1: DPR of the first min(nnz, capacity) CSR values; nnz is the device int64."""
    cap = val.numel() if capacity is None else int(capacity)
    words = gist_dpr_words(cap, bits)
    if words < 0:
        raise GistError(3, "gist_ssdc_dpr_encode")
    dev = val.device
    packed = _words(words, dev, packed)
    with torch.cuda.device(dev):
        _check(lib.gist_ssdc_dpr_encode(_ptr(val, _F32, dev, cap, "val"), _ptr(nnz, _I64, dev, 1, "nnz"), cap, bits,
                                        _ptr(packed, _W32, dev, words, "packed"), _stream(val, stream)),
               "gist_ssdc_dpr_encode")
    return packed


def gist_ssdc_dpr_decode(packed: torch.Tensor, nnz: torch.Tensor, bits: int, capacity: int,
                         val: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """f1: restore the first min(nnz, capacity) CSR values to fp32."""
    dev = packed.device
    words = gist_dpr_words(int(capacity), bits)
    if words < 0:
        raise GistError(3, "gist_ssdc_dpr_decode")
    if val is None:
        val = torch.empty(max(capacity, 1), dtype=torch.float32, device=dev)
    with torch.cuda.device(dev):
        _check(lib.gist_ssdc_dpr_decode(_ptr(packed, _W32, dev, words, "packed"), _ptr(nnz, _I64, dev, 1, "nnz"),
                                        int(capacity), bits, _ptr(val, _F32, dev, int(capacity), "val"),
                                        _stream(packed, stream)), "gist_ssdc_dpr_decode")
    return val


# ------------------------------------------------------------------ many maps per launch
class SsdcEncodeMany:
    """A prepared gist_ssdc_encode_many call: the job table is marshalled once, and every call
    re-runs it (one persistent launch per up to 48 maps).  jobs: dicts with x and optional
    row_end / col / val / nnz / capacity / offset (append mode: a device int64 start offset);
    missing outputs are allocated like gist_ssdc_encode's.  .outputs[k] = (row_end, col, val, nnz)."""

    def __init__(self, jobs, workspace=None, stream=None):
        self.outputs, self._keep = [], []
        arr = (SsdcJob * max(1, len(jobs)))()
        dev = jobs[0]["x"].device if jobs else None
        for k, jb in enumerate(jobs):
            x = jb["x"]
            n = x.numel()
            cap = n if jb.get("capacity") is None else int(jb["capacity"])
            row_end = jb.get("row_end")
            if row_end is None:
                row_end = torch.empty(gist_ssdc_rows(n), dtype=torch.int32, device=dev)
            col = jb.get("col")
            if col is None:
                col = torch.empty(max(cap, 1), dtype=torch.uint8, device=dev)
            val = jb.get("val")
            if val is None:
                val = torch.empty(max(cap, 1), dtype=torch.float32, device=dev)
            nnz = jb.get("nnz")
            if nnz is None:
                nnz = torch.empty(1, dtype=torch.int64, device=dev)
            off = jb.get("offset")
            arr[k] = SsdcJob(_ptr(x, _F32, dev, name="x"), n, _ptr(row_end, _I32, dev, gist_ssdc_rows(n), "row_end"),
                             _ptr(col, _U8, dev, cap, "col"), _ptr(val, _F32, dev, cap, "val"), cap,
                             _ptr(nnz, _I64, dev, 1, "nnz"), _ptr(off, _I64, dev, 1, "offset"))
            self.outputs.append((row_end, col, val, nnz))
            self._keep += [x, off]
        self.jobs, self.count, self.device = arr, len(jobs), dev
        self.ws_bytes = lib.gist_ssdc_workspace_bytes_many(arr, len(jobs))
        if workspace is None and jobs:
            workspace = torch.empty(self.ws_bytes, dtype=torch.uint8, device=dev)
            gist_ssdc_workspace_init(workspace, stream)
        self.workspace = workspace

    def __call__(self, stream=None):
        if not self.count:
            return self.outputs
        with torch.cuda.device(self.device):
            _check(lib.gist_ssdc_encode_many(self.jobs, self.count, _ptr(self.workspace, None, self.device),
                                             self.workspace.numel() * self.workspace.element_size(),
                                             _stream(self.workspace, stream)), "gist_ssdc_encode_many")
        return self.outputs


class SsdcDecodeMany:
    """A prepared gist_ssdc_decode_many call.  jobs: dicts with row_end, col, val, n and optional
    x / offset.  .outputs[k] = x."""

    def __init__(self, jobs):
        arr = (SsdcDecodeJob * max(1, len(jobs)))()
        dev = jobs[0]["row_end"].device if jobs else None
        self.outputs, self._keep = [], []
        for k, jb in enumerate(jobs):
            n = int(jb["n"])
            x = jb.get("x")
            if x is None:
                x = torch.empty(n, dtype=torch.float32, device=dev)
            off = jb.get("offset")
            arr[k] = SsdcDecodeJob(_ptr(jb["row_end"], _I32, dev, gist_ssdc_rows(n), "row_end"),
                                   _ptr(jb["col"], _U8, dev, name="col"), _ptr(jb["val"], _F32, dev, name="val"),
                                   _ptr(off, _I64, dev, 1, "offset"), n, _ptr(x, _F32, dev, n, "x"))
            self.outputs.append(x)
            self._keep += [jb["row_end"], jb["col"], jb["val"], off]
        self.jobs, self.count, self.device = arr, len(jobs), dev

    def __call__(self, stream=None):
        if self.count:
            with torch.cuda.device(self.device):
                _check(lib.gist_ssdc_decode_many(self.jobs, self.count, _stream(self.outputs[0], stream)),
                       "gist_ssdc_decode_many")
        return self.outputs


class DprMany:
    """A prepared gist_dpr_encode_many (encode=True: jobs of x, optional packed) or
    gist_dpr_decode_many (encode=False: jobs of packed, n, optional x) call."""

    def __init__(self, jobs, bits: int, encode: bool):
        arr = (DprJob * max(1, len(jobs)))()
        key = "x" if encode else "packed"
        dev = jobs[0][key].device if jobs else None
        self.outputs, self._keep = [], []
        for k, jb in enumerate(jobs):
            if encode:
                x = jb["x"]
                n = x.numel()
                words = gist_dpr_words(n, bits)
                if words < 0:
                    raise GistError(3, "gist_dpr_encode_many")
                packed = _words(words, dev, jb.get("packed"))
                self.outputs.append(packed)
            else:
                packed, n = jb["packed"], int(jb["n"])
                words = gist_dpr_words(n, bits)
                if words < 0:
                    raise GistError(3, "gist_dpr_decode_many")
                x = jb.get("x")
                if x is None:
                    x = torch.empty(n, dtype=torch.float32, device=dev)
                self.outputs.append(x)
            arr[k] = DprJob(_ptr(x, _F32, dev, n, "x"), n, _ptr(packed, _W32, dev, words, "packed"))
            self._keep += [x, packed]
        self.jobs, self.count, self.bits, self.encode, self.device = arr, len(jobs), bits, encode, dev

    def __call__(self, stream=None):
        if self.count:
            fn = lib.gist_dpr_encode_many if self.encode else lib.gist_dpr_decode_many
            with torch.cuda.device(self.device):
                _check(fn(self.jobs, self.count, self.bits, _stream(self.outputs[0], stream)),
                       "gist_dpr_encode_many" if self.encode else "gist_dpr_decode_many")
        return self.outputs


def gist_ssdc_workspace_bytes_many(ns) -> int:
    """Workspace bytes of gist_ssdc_encode_many over maps of these sizes."""
    arr = (SsdcJob * max(1, len(ns)))()
    for k, n in enumerate(ns):
        arr[k].n = int(n)
    return lib.gist_ssdc_workspace_bytes_many(arr, len(ns))


def gist_ssdc_encode_many(jobs, workspace=None, stream=None):
    """a4 over several maps in one launch; see SsdcEncodeMany.  Returns [(row_end, col, val, nnz)]."""
    return SsdcEncodeMany(jobs, workspace, stream)(stream)


def gist_ssdc_decode_many(jobs, stream=None):
    """a5 over several maps in one launch; see SsdcDecodeMany.  Returns [x]."""
    return SsdcDecodeMany(jobs)(stream)


def gist_dpr_encode_many(xs, bits: int, stream=None):
    """a6 over several maps in one launch.  Returns [packed]."""
    return DprMany([{"x": x} for x in xs], bits, True)(stream)


def gist_dpr_decode_many(packed, ns, bits: int, stream=None):
    """a7 over several maps in one launch.  Returns [x]."""
    return DprMany([{"packed": p, "n": n} for p, n in zip(packed, ns)], bits, False)(stream)


# ------------------------------------------------------------------ f4: decode inside the consumer GEMM
def gist_conv3x3_wgrad_workspace_bytes(N: int, Ci: int, Co: int, H: int, W: int) -> int:
    return lib.gist_conv3x3_wgrad_workspace_bytes(N, Ci, Co, H, W)


def gist_conv3x3_wgrad_ssdc(dy: torch.Tensor, row_end: torch.Tensor, col: torch.Tensor, val: torch.Tensor,
                            x_shape, passes: int = 3, dw: torch.Tensor | None = None,
                            workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """f4: dW [Co,Ci,3,3] of a 3x3/s1/p1 conv from dY [N,Co,H,W] and the SSDC
    encoding of its input X (shape x_shape = (N, Ci, H, W)); X is decoded inside the tcgen05 GEMM."""
    N, Ci, H, W = (int(v) for v in x_shape)
    Co = int(dy.shape[1])
    dev = dy.device
    if tuple(dy.shape) != (N, Co, H, W):
        raise ValueError(f"dy {tuple(dy.shape)} does not match x_shape {tuple(x_shape)}")
    if dw is None:
        dw = torch.empty((Co, Ci, 3, 3), dtype=torch.float32, device=dev)
    wsb = gist_conv3x3_wgrad_workspace_bytes(N, Ci, Co, H, W)
    if workspace is None:
        workspace = torch.empty(max(wsb, 16), dtype=torch.uint8, device=dev)
    with torch.cuda.device(dev):
        _check(lib.gist_conv3x3_wgrad_ssdc(
            _ptr(dy, _F32, dev, name="dy"), _ptr(row_end, _I32, dev, gist_ssdc_rows(N * Ci * H * W), "row_end"),
            _ptr(col, _U8, dev, name="col"), _ptr(val, _F32, dev, name="val"), N, Ci, Co, H, W, int(passes),
            _ptr(dw, _F32, dev, Co * Ci * 9, "dw"), _ptr(workspace, None, dev, name="workspace"),
            workspace.numel() * workspace.element_size(), _stream(dy, stream)), "gist_conv3x3_wgrad_ssdc")
    return dw
