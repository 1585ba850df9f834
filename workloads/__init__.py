"""Seeded synthetic workloads shared by the CUDA path's tests/bench and the oracle's tests.

This module holds shapes and random inputs only — none of the method's arithmetic (no
encoding, packing, rounding or pooling).  Both sides of every parity test take their
inputs from here; the oracle gets a host copy of exactly the tensor the GPU got.

Shapes: SURVEY.md Appendix A (stash sites of AlexNet / VGG16 / OverFeat / NiN /
GoogLeNet, per image, NCHW), derived from the original network papers because PAPER.md
only names the networks (§V-A).  Encoding assignment per P:151 (ReLU->Pool:
Binarize), P:158 (ReLU/Pool->Conv: SSDC), P:169 (others: DPR).
Value recipe: DESIGN.md §4 (ReLU outputs y = max(z, +0) with z ~ N(mu_s, 1),
mu_s = -Phi^-1(s), so the expected sparsity is s; P:76 reports >80% for VGG16).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import torch

# pool geometry tuple: (kh, kw, sh, sw, ph, pw, ceil_mode)
P2S2 = (2, 2, 2, 2, 0, 0, 0)
P3S2 = (3, 3, 2, 2, 0, 0, 0)
P3S2C = (3, 3, 2, 2, 0, 0, 1)
P3S1P1 = (3, 3, 1, 1, 1, 1, 0)


@dataclass(frozen=True)
class Site:
    """One stashed feature map.  kind: 'relu_pool' (Binarize + argmax + fused bwd),
    'pool_only' (argmax + pool-only bwd, mask NULL), 'ssdc', 'dpr'."""
    name: str
    kind: str
    chw: tuple
    pool: tuple | None = None

    def numel(self, batch: int) -> int:
        c, h, w = self.chw
        return batch * c * h * w


def _vgg16():
    s = [Site("data", "dpr", (3, 224, 224))]
    blocks = [(64, 224, 2), (128, 112, 2), (256, 56, 3), (512, 28, 3), (512, 14, 3)]
    for b, (c, h, nconv) in enumerate(blocks, 1):
        for j in range(1, nconv):
            s.append(Site(f"relu{b}_{j}", "ssdc", (c, h, h)))
        s.append(Site(f"relu{b}_{nconv}", "relu_pool", (c, h, h), P2S2))
        if b < 5:
            s.append(Site(f"pool{b}", "ssdc", (c, h // 2, h // 2)))
    s += [Site("pool5", "dpr", (512, 7, 7)), Site("relu6", "dpr", (4096, 1, 1)),
          Site("relu7", "dpr", (4096, 1, 1))]
    return s


def _alexnet():
    return [
        Site("data", "dpr", (3, 227, 227)),
        Site("relu1", "relu_pool", (96, 55, 55), P3S2),
        Site("pool1", "ssdc", (96, 27, 27)),
        Site("relu2", "relu_pool", (256, 27, 27), P3S2),
        Site("pool2", "ssdc", (256, 13, 13)),
        Site("relu3", "ssdc", (384, 13, 13)),
        Site("relu4", "ssdc", (384, 13, 13)),
        Site("relu5", "relu_pool", (256, 13, 13), P3S2),
        Site("pool5", "dpr", (256, 6, 6)),
        Site("relu6", "dpr", (4096, 1, 1)),
        Site("relu7", "dpr", (4096, 1, 1)),
    ]


def _overfeat():
    return [
        Site("data", "dpr", (3, 231, 231)),
        Site("relu1", "relu_pool", (96, 56, 56), P2S2),
        Site("pool1", "ssdc", (96, 28, 28)),
        Site("relu2", "relu_pool", (256, 24, 24), P2S2),
        Site("pool2", "ssdc", (256, 12, 12)),
        Site("relu3", "ssdc", (512, 12, 12)),
        Site("relu4", "ssdc", (1024, 12, 12)),
        Site("relu5", "relu_pool", (1024, 12, 12), P2S2),
        Site("pool5", "dpr", (1024, 6, 6)),
        Site("relu6", "dpr", (3072, 1, 1)),
        Site("relu7", "dpr", (4096, 1, 1)),
    ]


def _nin():
    return [
        Site("data", "dpr", (3, 224, 224)),
        Site("relu_conv1", "ssdc", (96, 54, 54)),
        Site("relu_cccp1", "ssdc", (96, 54, 54)),
        Site("relu_cccp2", "relu_pool", (96, 54, 54), P3S2C),
        Site("pool1", "ssdc", (96, 27, 27)),
        Site("relu_conv2", "ssdc", (256, 27, 27)),
        Site("relu_cccp3", "ssdc", (256, 27, 27)),
        Site("relu_cccp4", "relu_pool", (256, 27, 27), P3S2C),
        Site("pool2", "ssdc", (256, 13, 13)),
        Site("relu_conv3", "ssdc", (384, 13, 13)),
        Site("relu_cccp5", "ssdc", (384, 13, 13)),
        Site("relu_cccp6", "relu_pool", (384, 13, 13), P3S2C),
        Site("pool3", "dpr", (384, 6, 6)),
        Site("relu_conv4", "ssdc", (1024, 6, 6)),
        Site("relu_cccp7", "ssdc", (1024, 6, 6)),
        Site("relu_cccp8", "dpr", (1000, 6, 6)),
    ]


_GOOGLENET_MODULES = [
    # name, Cin, S, n1, r3, n3, r5, n5, proj
    ("3a", 192, 28, 64, 96, 128, 16, 32, 32),
    ("3b", 256, 28, 128, 128, 192, 32, 96, 64),
    ("4a", 480, 14, 192, 96, 208, 16, 48, 64),
    ("4b", 512, 14, 160, 112, 224, 24, 64, 64),
    ("4c", 512, 14, 128, 128, 256, 24, 64, 64),
    ("4d", 512, 14, 112, 144, 288, 32, 64, 64),
    ("4e", 528, 14, 256, 160, 320, 32, 128, 128),
    ("5a", 832, 7, 256, 160, 320, 32, 128, 128),
    ("5b", 832, 7, 384, 192, 384, 48, 128, 128),
]


def _googlenet():
    s = [
        Site("data", "dpr", (3, 224, 224)),
        Site("relu_conv1", "relu_pool", (64, 112, 112), P3S2C),
        Site("pool1", "ssdc", (64, 56, 56)),
        Site("relu_conv2r", "ssdc", (64, 56, 56)),
        Site("relu_conv2", "relu_pool", (192, 56, 56), P3S2C),
        Site("pool2", "ssdc", (192, 28, 28)),
    ]
    for name, cin, S, n1, r3, n3, r5, n5, proj in _GOOGLENET_MODULES:
        out = n1 + n3 + n5 + proj
        s.append(Site(f"inc{name}_r3", "ssdc", (r3, S, S)))
        s.append(Site(f"inc{name}_r5", "ssdc", (r5, S, S)))
        s.append(Site(f"inc{name}_pool", "pool_only", (cin, S, S), P3S1P1))
        s.append(Site(f"inc{name}_poolout", "ssdc", (cin, S, S)))
        if name in ("3b", "4e"):
            s.append(Site(f"inc{name}_out", "relu_pool", (out, S, S), P3S2C))
            So = (S - 3 + 1) // 2 + 1  # 3x3/s2/ceil: 28 -> 14, 14 -> 7
            s.append(Site(f"pool_after_{name}", "ssdc", (out, So, So)))
        elif name == "5b":
            s.append(Site(f"inc{name}_out", "dpr", (out, S, S)))
        else:
            s.append(Site(f"inc{name}_out", "ssdc", (out, S, S)))
    return s


NETS = {
    "alexnet": _alexnet(),
    "vgg16": _vgg16(),
    "overfeat": _overfeat(),
    "nin": _nin(),
    "googlenet": _googlenet(),
}


@dataclass(frozen=True)
class Config:
    """BASELINE.json configs (C1..C5).  batch is per GPU."""
    key: str
    net: str | None
    batch: int
    sparsity: float
    dpr_bits: int
    description: str = ""
    extra: dict = field(default_factory=dict)


CONFIGS = {
    "C1": Config("C1", None, 1, 0.5, 16,
                 "single 1x64x56x56 map: ReLU->maxpool(3x3,s2) + SSDC + DPR 16/10/8 round trip"),
    "C2": Config("C2", "alexnet", 128, 0.8, 16, "AlexNet-shaped, batch 128, Binarize + SSDC + DPR-fp16"),
    "C3": Config("C3", "vgg16", 64, 0.8, 16,
                 "VGG16-shaped, batch 64, Binarize + SSDC (s=0.8) + DPR (fp16 per P:240)"),
    "C4": Config("C4", "googlenet", 64, 0.8, 10, "GoogLeNet-shaped, batch 64 (sharded), DPR-fp10 per P:240"),
    "C5o": Config("C5o", "overfeat", 256, 0.8, 8, "OverFeat, batch 256 per GPU, DPR-fp8 per P:240"),
    "C5n": Config("C5n", "nin", 256, 0.8, 8, "NiN, batch 256 per GPU, DPR-fp8"),
}

C1_SITES = [
    Site("c1_relu", "relu_pool", (64, 56, 56), P3S2),
    Site("c1_ssdc", "ssdc", (64, 56, 56)),
    Site("c1_dpr", "dpr", (64, 56, 56)),
]


def sites_for(cfg: Config):
    return C1_SITES if cfg.net is None else NETS[cfg.net]


def seed_for(config_index: int, site_index: int, rank: int = 0) -> int:
    """Seed recipe: 1_000_000*config + 1000*site + rank."""
    return 1_000_000 * config_index + 1000 * site_index + rank


def image_seed(config_index: int, site_index: int, image: int, grad: bool = False) -> int:
    """Per-image seed: 1_000_000*config + 1000*site + image (+500 for the upstream
    gradient).  Inputs are drawn image by image from GLOBAL image indices, so the union of the
    ranks' minibatch shards is exactly the single-GPU minibatch (C4 strong scaling)."""
    if not 0 <= image < 500:
        raise ValueError("image index must be in [0, 500)")
    return 1_000_000 * config_index + 1000 * site_index + (500 if grad else 0) + image


def per_image(fn, chw, images, seed0: int, device="cpu", **kw) -> torch.Tensor:
    """Stack fn((1,) + chw, seed0 + image, device, **kw) over the global image indices `images`."""
    images = list(images)
    out = torch.empty((len(images),) + tuple(chw), dtype=torch.float32, device=device)
    for k, img in enumerate(images):
        out[k:k + 1] = fn((1,) + tuple(chw), seed0 + img, device, **kw)
    return out


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return g


def relu_map(shape, sparsity: float, seed: int, device="cpu", structured: bool = False,
             negative_zero: bool = False) -> torch.Tensor:
    """ReLU output with expected sparsity `sparsity`: y = z if z > 0 else +0.0,
    z ~ N(mu_s, 1), mu_s = -Phi^-1(s).  structured=True draws a per-channel sparsity
    ~ Beta(mean s) and kills ~5% of channels outright (variable row lengths).
    negative_zero=True writes -0.0 instead of +0.0 for half of the zeros (torch.relu
    of -0.0 is -0.0), exercising the bit-pattern nonzero rule."""
    g = _gen(seed, device)
    z = torch.randn(shape, generator=g, device=device, dtype=torch.float32)
    if structured and len(shape) == 4:
        N, Cc = shape[0], shape[1]
        a = 4.0
        b = a * (1 - sparsity) / max(sparsity, 1e-6)
        # Beta sampling draws from the global CPU RNG: fork it and seed deterministically.
        with torch.random.fork_rng(devices=[]):
            torch.manual_seed(seed + 7)
            ch_s = torch.distributions.Beta(torch.tensor(a), torch.tensor(b)).sample((N, Cc))
        dead = torch.rand((N, Cc), generator=_gen(seed + 11, "cpu")) < 0.05
        ch_s = torch.where(dead, torch.ones_like(ch_s), ch_s).clamp(1e-4, 1 - 1e-4)
        mu = (-torch.special.ndtri(ch_s)).to(device=device, dtype=torch.float32)
        z = z + mu.view(N, Cc, 1, 1)
    else:
        mu = -float(torch.special.ndtri(torch.tensor(float(sparsity), dtype=torch.float64)))
        z = z + mu
    zero = torch.zeros((), device=device, dtype=torch.float32)
    if negative_zero:
        flip = torch.rand(shape, generator=g, device=device) < 0.5
        zero = torch.where(flip, torch.tensor(-0.0, device=device), torch.tensor(0.0, device=device))
    return torch.where(z > 0, z, zero)


def grad_map(shape, seed: int, device="cpu") -> torch.Tensor:
    """Upstream gradient dY ~ N(0, 1)."""
    return torch.randn(shape, generator=_gen(seed, device), device=device, dtype=torch.float32)


def dpr_map(shape, seed: int, device="cpu") -> torch.Tensor:
    """'Other' stashed map for DPR: N(0,1) * 2^U, U ~ U(-10, 10) per element, so values
    cross the FP8 flush-to-zero and saturation edges."""
    g = _gen(seed, device)
    z = torch.randn(shape, generator=g, device=device, dtype=torch.float32)
    u = torch.rand(shape, generator=g, device=device, dtype=torch.float32) * 20.0 - 10.0
    return z * torch.exp2(u)


def dpr_specials() -> torch.Tensor:
    """Fixed edge tensor (CPU): signed zeros, infinities, NaN, fp32 subnormals, and the
    range edges / exact ties of all three DPR formats."""
    import numpy as np
    vals = [0.0, -0.0, float("inf"), -float("inf"), float("nan"), 1.0, -1.0, 2.0, 0.5, 0.1, -3.0,
            65504.0, 65519.0, 65520.0, 65536.0, 1e9, -1e9, 480.0, 464.0, 496.0, 448.0,
            126976.0, 130000.0, 2.0 ** -6, 2.0 ** -7, 2.0 ** -14, 2.0 ** -15, 2.0 ** -24, 2.0 ** -25,
            1e-7, 1.0625, 1.1875, 1.03125, 1.09375, 0.0146484375, 2.0 ** -6 * (1 - 2.0 ** -5),
            2.0 ** -14 * (1 - 2.0 ** -6), 1e-45, -1e-45, 1.17549435e-38, 3.4028235e38]
    a = np.array(vals, np.float32)
    nudges = np.concatenate([np.nextafter(a, np.float32(np.inf)), np.nextafter(a, np.float32(-np.inf))])
    a = np.concatenate([a, -a, nudges]).astype(np.float32)
    return torch.from_numpy(a)
