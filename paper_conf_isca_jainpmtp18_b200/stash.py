"""Stash-time integration with PyTorch autograd (§IV-B).

Gist's Schedule Builder inserts an encode after a feature map's last
forward use and a decode before its backward use, so only the encoding lives through the
long forward->backward gap (Fig 2).  Here the same schedule is expressed with autograd:

* `relu_maxpool(x, pool)` — ReLU->MaxPool pair (Binarize): the forward runs the
  a2 kernel with the a1 mask fused; autograd saves ONLY the 1-bit mask and the 4-bit argmax
  map (neither the ReLU output nor the pool output), and the backward is the a3 kernel.
* `relu_conv(x, conv)` / `stashed_conv(y, conv)` — ReLU->Conv and Pool->Conv (SSDC,
  P:158-164): the conv input is stashed as 256-column CSR (a4) and densified just before the
  conv backward (a5); the dense math stays in cuDNN ("dense compute").  Inside
  `ssdc_arena(...)` every stash appends its entries to one chained arena in a single encode
  pass with device-side offsets (no host synchronization in the forward; one capacity check
  per step, before the first decode); outside it, each stash is sized exactly by a count pass
  and a host read of nnz.
* `dpr_saved_tensors(bits, params)` — every other stashed activation (DPR,
  "applicable to any layer combination") is packed to FP16/FP10/FP8 by the a6 kernel when
  autograd saves it and restored by a7 when the backward unpacks it.

Everything on the encode/decode path is a libgist kernel; torch supplies the dense layers.
"""
from __future__ import annotations

import contextlib

import torch
import torch.nn.functional as F

from . import (gist_dpr_decode, gist_dpr_encode, gist_relu_maxpool_fwd_argmax, gist_pool_relu_bwd,
               gist_ssdc_decode, gist_ssdc_decode_many, gist_ssdc_encode, gist_ssdc_rows, gist_ssdc_workspace,
               gist_ssdc_workspace_bytes, gist_ssdc_workspace_init, SsdcEncodeMany)


def _pool_tuple(kernel_size, stride, padding, ceil_mode):
    k = (kernel_size, kernel_size) if isinstance(kernel_size, int) else tuple(kernel_size)
    s = k if stride is None else ((stride, stride) if isinstance(stride, int) else tuple(stride))
    p = (padding, padding) if isinstance(padding, int) else tuple(padding)
    return (k[0], k[1], s[0], s[1], p[0], p[1], int(bool(ceil_mode)))


class _ReLUMaxPool(torch.autograd.Function):
    @staticmethod
    def forward(ctx, x, pool):
        # in-place ReLU: relu is applied on load, the fp32 ReLU output never exists and
        # is not stashed
        out, arg, mask = gist_relu_maxpool_fwd_argmax(x.contiguous(), pool)
        ctx.save_for_backward(arg, mask)
        ctx.shape, ctx.pool = tuple(x.shape), pool
        return out

    @staticmethod
    def backward(ctx, dout):
        arg, mask = ctx.saved_tensors
        return gist_pool_relu_bwd(dout.contiguous(), arg, mask, ctx.shape, ctx.pool), None


def relu_maxpool(x, kernel_size, stride=None, padding=0, ceil_mode=False):
    """max_pool2d(relu(x)) whose stash is the Binarize encoding (mask + argmax map)."""
    return _ReLUMaxPool.apply(x, _pool_tuple(kernel_size, stride, padding, ceil_mode))


class StashOverflow(RuntimeError):
    """The step's SSDC entries did not fit the arena; `needed` is the entry count it would take."""

    def __init__(self, needed: int, capacity: int):
        super().__init__(f"SSDC stash arena overflow: {needed} entries needed, capacity {capacity}")
        self.needed, self.capacity = needed, capacity


class StashArena:
    """One chained SSDC arena for a training step (the Schedule
    Builder's preallocated stash): each stash's col/val entries follow the previous stash's, the
    start offset is a device scalar (the previous encode's nnz output), so an encode is ONE pass
    over the map with no host synchronization.  Entries past `capacity` are dropped by the kernel
    (which still publishes the true end); `check()` reads the end once and raises StashOverflow
    before any stash of an overflowed arena is decoded."""

    def __init__(self, capacity: int, device, plan=None):
        self.capacity, self.device = int(capacity), torch.device(device)
        self.col = torch.empty(max(1, self.capacity), dtype=torch.uint8, device=self.device)
        self.val = torch.empty(max(1, self.capacity), dtype=torch.float32, device=self.device)
        self.ws, self.plan = None, plan
        self.reset()

    def reset(self):
        self.head = torch.zeros(1, dtype=torch.int64, device=self.device)
        self.used = None  # host value once checked

    def head_ref(self):
        """A callable returning the arena's current end (device tensor) without keeping the arena's
        buffers alive (ArenaPlan reads it after the backward has released them)."""
        box = self._box = [self.head]
        return lambda: box[0]

    def _workspace(self, n: int) -> torch.Tensor:
        if self.plan is not None:
            return self.plan.workspace(n)
        need = gist_ssdc_workspace_bytes(n)
        if self.ws is None or self.ws.numel() < need:
            self.ws = torch.empty(need, dtype=torch.uint8, device=self.device)
            gist_ssdc_workspace_init(self.ws)
        return self.ws

    def append(self, y: torch.Tensor):
        """Encode y after the current end; returns (row_end, start, end) (start/end on the device)."""
        n = y.numel()
        start, end = self.head, torch.empty(1, dtype=torch.int64, device=self.device)
        row_end = torch.empty(gist_ssdc_rows(n), dtype=torch.int32, device=self.device)
        SsdcEncodeMany([{"x": y, "row_end": row_end, "col": self.col, "val": self.val, "capacity": self.capacity,
                         "offset": start, "nnz": end}], workspace=self._workspace(n))()
        self.head = end
        if getattr(self, "_box", None) is not None:
            self._box[0] = end
        return row_end, start, end

    def check(self) -> int:
        """Entries used by the step (one host read per reset); raises StashOverflow."""
        if self.used is None:
            self.used = int(self.head.item())
        if self.used > self.capacity:
            raise StashOverflow(self.used, self.capacity)
        return self.used


class ArenaPlan:
    """Per-group arenas for one training step, sized from the previous step (no host sync in the
    forward).  Each group (e.g. a VGG block) gets a fresh StashArena when `arena(g)` is called; the
    arena is freed by the allocator once the group's last stash has been decoded in the backward, so
    the stash memory shrinks as the backward proceeds (as exact-size stashes do).  `update()`, after
    the backward, reads every arena's end in ONE host synchronization and resizes the groups for the
    next step (used x `slack`); a group that overflowed raises StashOverflow at its first decode."""

    def __init__(self, device, initial: dict | None = None, slack: float = 1.05, floor: int = 1 << 16):
        self.device, self.slack, self.floor = torch.device(device), slack, floor
        self.cap = dict(initial or {})
        self.live = {}
        self.ws = None  # one encode workspace shared by the plan's arenas (stream-ordered reuse)

    def workspace(self, n: int) -> torch.Tensor:
        need = gist_ssdc_workspace_bytes(n)
        if self.ws is None or self.ws.numel() < need:
            self.ws = torch.empty(need, dtype=torch.uint8, device=self.device)
            gist_ssdc_workspace_init(self.ws)
        return self.ws

    def arena(self, group, default_capacity: int) -> "StashArena":
        cap = self.cap.get(group, default_capacity)
        a = StashArena(cap, self.device, plan=self)
        self.live[group] = (a.head_ref(), cap)
        return a

    def update(self):
        if not self.live:
            return {}
        groups = list(self.live)
        used = torch.cat([self.live[g][0]() for g in groups]).cpu().tolist()  # one synchronization
        out = {}
        for g, u in zip(groups, used):
            self.cap[g] = max(self.floor, int(u * self.slack))
            out[g] = (int(u), self.live[g][1])
        self.live = {}
        return out


_ARENA: list = []


@contextlib.contextmanager
def ssdc_arena(arena: StashArena):
    """Stashes made inside this context append to `arena` (one encode pass each, no host sync)."""
    _ARENA.append(arena)
    try:
        yield arena
    finally:
        _ARENA.pop()


class CSRStash:
    """SSDC encoding of a dense fp32 map: appended to the active arena (one pass), else exact-size
    (one count pass, a host read of nnz, one encode pass)."""

    def __init__(self, y: torch.Tensor):
        y = y.contiguous()
        self.shape, self.n = tuple(y.shape), y.numel()
        self.arena = _ARENA[-1] if _ARENA else None
        if self.arena is not None:
            self.row_end, self.start, self.end = self.arena.append(y)
            return
        ws = gist_ssdc_workspace(self.n, y.device)
        nnz = torch.empty(1, dtype=torch.int64, device=y.device)
        row_end = torch.empty(gist_ssdc_rows(self.n), dtype=torch.int32, device=y.device)
        gist_ssdc_encode(y, capacity=0, row_end=row_end, nnz=nnz, workspace=ws)  # count only
        k = int(nnz.item())
        col = torch.empty(max(k, 1), dtype=torch.uint8, device=y.device)
        val = torch.empty(max(k, 1), dtype=torch.float32, device=y.device)
        gist_ssdc_encode(y, capacity=k, row_end=row_end, col=col, val=val, nnz=nnz, workspace=ws)
        self.row_end, self.col, self.val, self.nnz = row_end, col, val, k

    def nbytes(self) -> int:
        """Encoded bytes (5 nnz + 4 rows); reads the arena offsets (a host sync) in arena mode."""
        nnz = int((self.end - self.start).item()) if self.arena is not None else self.nnz
        return 5 * nnz + 4 * self.row_end.numel()

    def dense(self) -> torch.Tensor:
        if self.arena is not None:
            self.arena.check()  # never decode entries an overflowed arena dropped
            (x,) = gist_ssdc_decode_many([{"row_end": self.row_end, "col": self.arena.col, "val": self.arena.val,
                                           "offset": self.start, "n": self.n}])
            return x.view(self.shape)
        return gist_ssdc_decode(self.row_end, self.col, self.val, self.n).view(self.shape)


class _StashedConv(torch.autograd.Function):
    """conv2d whose saved input is SSDC-encoded; relu=True also applies the preceding ReLU
    (its backward mask is recovered from the decoded input: y > 0)."""

    @staticmethod
    def forward(ctx, x, weight, bias, stride, padding, dilation, groups, relu):
        y = torch.relu(x) if relu else x
        out = F.conv2d(y, weight, bias, stride, padding, dilation, groups)
        ctx.csr = CSRStash(y)
        del y
        ctx.save_for_backward(weight)
        ctx.conf = (stride, padding, dilation, groups, relu, bias is not None)
        return out

    @staticmethod
    def backward(ctx, dout):
        (weight,) = ctx.saved_tensors
        stride, padding, dilation, groups, relu, has_bias = ctx.conf
        y = ctx.csr.dense()  # decoded just before its backward use
        ctx.csr = None
        gx, gw, gb = torch.ops.aten.convolution_backward(
            dout.contiguous(), y, weight, [weight.shape[0]] if has_bias else None, stride, padding, dilation, False,
            [0, 0], groups, [True, True, has_bias])
        if relu:  # ReLU backward with torch's own rule (threshold_backward on the ReLU output)
            gx = torch.ops.aten.threshold_backward(gx, y, 0)
        del y
        return gx, gw, gb, None, None, None, None, None


def relu_conv(x, conv: torch.nn.Conv2d):
    """conv(relu(x)) with the ReLU output stashed as SSDC (ReLU->Conv)."""
    return _StashedConv.apply(x, conv.weight, conv.bias, conv.stride, conv.padding, conv.dilation, conv.groups, True)


def stashed_conv(y, conv: torch.nn.Conv2d):
    """conv(y) with its input stashed as SSDC (Pool->Conv)."""
    return _StashedConv.apply(y, conv.weight, conv.bias, conv.stride, conv.padding, conv.dilation, conv.groups, False)


class _DPRPacked:
    __slots__ = ("words", "n", "shape", "bits")

    def __init__(self, t: torch.Tensor, bits: int):
        t = t.contiguous()
        self.n, self.shape, self.bits = t.numel(), tuple(t.shape), bits
        self.words = gist_dpr_encode(t, bits)


@contextlib.contextmanager
def dpr_saved_tensors(bits: int, params=(), min_numel: int = 4096):
    """Inside this context, fp32 CUDA activations saved by autograd (not parameters, not tiny
    tensors) are stored as DPR words and restored to fp32 when the backward unpacks them."""
    skip = {p.data_ptr() for p in params}

    def pack(t):
        if (t.is_cuda and t.dtype == torch.float32 and t.numel() >= min_numel and t.data_ptr() not in skip
                and t.is_contiguous()):
            return _DPRPacked(t, bits)
        return t

    def unpack(p):
        if isinstance(p, _DPRPacked):
            return gist_dpr_decode(p.words, p.n, p.bits).view(p.shape)
        return p

    with torch.autograd.graph.saved_tensors_hooks(pack, unpack):
        yield
