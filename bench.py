#!/usr/bin/env python
"""bench.py — Gist stash-time encode/decode throughput on B200 (driver contract).

A "step" is one pass of the whole hot path over one minibatch of synthetic stashed feature
maps: every stash site of the network is encoded in forward order (a1 Binarize + a2 MaxPool
argmax for ReLU->Pool sites, a4 SSDC for ReLU/Pool->Conv sites, a6 DPR for the rest) and
decoded in backward order (a3 fused pool+ReLU backward, a5 SSDC decode, a7 DPR decode).

Metric (BASELINE.json): fp32 feature-map GB/s = (fp32 bytes of every stashed map encoded +
fp32 bytes of every map decoded) / step time, i.e. 8 bytes per stashed element per step.
Default workload: C3, VGG16-shaped stash sites, batch 64 per GPU, SSDC at 80% sparsity
("over 80%"), DPR-fp16 (VGG16 needs FP16).  Inputs (3.9 GB per GPU) exceed
the 126 MB L2, so no explicit flush is needed between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl gist|reference] [--config C3]
  torchrun --nproc-per-node N bench.py --gpus N ...     (one rank per GPU, NCCL)
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as WL  # noqa: E402

CONFIG_INDEX = {"C1": 1, "C2": 2, "C3": 3, "C4": 4, "C5o": 5, "C5n": 6}
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback, used only if MEASURED_PEAKS.json is absent


def baseline_metric() -> str:
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        return json.load(f)["metric"]


def hbm_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


# --------------------------------------------------------------------------------- sites
def pool_out(chw, g):
    c, h, w = chw
    kh, kw, sh, sw, ph, pw, cm = g

    def dim(i, k, s, p):
        span = i + 2 * p - k
        o = (span + (s - 1 if cm else 0)) // s + 1
        if cm and (o - 1) * s >= i + p:
            o -= 1
        return o
    return (c, dim(h, kh, sh, ph), dim(w, kw, sw, pw))


def words(n, per):
    return -(-n // per)


class Workload:
    """Device buffers of one rank's minibatch for every stash site, and the step."""

    def __init__(self, gist, cfg: WL.Config, images, sparsity: float, dpr_bits: int, dev, fuse_mask: bool,
                 many: bool = True):
        """images: the GLOBAL image indices of this rank's minibatch shard (inputs are seeded per
        image, so the shards of a strong-scaled batch add up to the single-GPU batch).
        many: encode/decode all SSDC sites with one gist_ssdc_*_many launch and all DPR sites with
        one gist_dpr_*_many launch per step; False: one C-ABI call per site."""
        self.g, self.dev, self.bits, self.fuse, self.many = gist, dev, dpr_bits, fuse_mask, many
        self.images = list(images)
        batch = len(self.images)
        self.sites = []
        cidx = CONFIG_INDEX.get(cfg.key, 9)
        ssdc_sites = [s for s in WL.sites_for(cfg) if s.kind == "ssdc"]
        self.nnz_all = torch.zeros(max(1, len(ssdc_sites)), dtype=torch.int64, device=dev)
        k_ssdc = 0
        max_n = 1
        for si, s in enumerate(WL.sites_for(cfg)):
            shape = (batch,) + s.chw
            n = s.numel(batch)
            max_n = max(max_n, n)
            seed0 = WL.image_seed(cidx, si, 0)
            gseed0 = WL.image_seed(cidx, si, 0, grad=True)
            d = {"site": s, "shape": shape, "n": n}
            if s.kind in ("relu_pool", "pool_only"):
                # ReLU output feeding the pool
                d["y"] = WL.per_image(lambda sh, sd, dv: WL.relu_map(sh, 0.5, sd, dv), s.chw, self.images, seed0, dev)
                oshape = (batch,) + pool_out(s.chw, s.pool)
                d["n_out"] = oshape[0] * oshape[1] * oshape[2] * oshape[3]
                d["out"] = torch.empty(oshape, device=dev)
                d["arg"] = torch.empty(words(d["n_out"], 8), dtype=torch.int32, device=dev)
                d["mask"] = torch.empty(words(n, 32), dtype=torch.int32, device=dev) if s.kind == "relu_pool" else None
                d["dY"] = WL.per_image(WL.grad_map, oshape[1:], self.images, gseed0, dev)
            elif s.kind == "ssdc":
                d["y"] = WL.per_image(lambda sh, sd, dv: WL.relu_map(sh, sparsity, sd, dv), s.chw, self.images, seed0,
                                      dev)
                rows = words(n, 256)
                d["row_end"] = torch.empty(rows, dtype=torch.int32, device=dev)
                d["col"] = torch.empty(n, dtype=torch.uint8, device=dev)
                d["val"] = torch.empty(n, dtype=torch.float32, device=dev)
                d["nnz"] = self.nnz_all[k_ssdc:k_ssdc + 1]
                d["ws"] = gist.gist_ssdc_workspace(n, dev)
                k_ssdc += 1
            else:
                d["y"] = WL.per_image(WL.dpr_map, s.chw, self.images, seed0, dev)
                d["packed"] = torch.empty(gist.gist_dpr_words(n, dpr_bits), dtype=torch.int32, device=dev)
            self.sites.append(d)
        # decoded maps are short-lived (D lives only at its backward use): one scratch
        self.scratch = torch.empty(max_n, dtype=torch.float32, device=dev)
        self.stash_elems = sum(d["n"] for d in self.sites)
        self.bytes_per_step = 8 * self.stash_elems  # 4n encoded + 4n decoded per site
        ss = [d for d in self.sites if d["site"].kind == "ssdc"]
        ds = [d for d in self.sites if d["site"].kind == "dpr"]
        self.ssdc_sites, self.dpr_sites = ss, ds
        if many:
            self.enc_many = gist.SsdcEncodeMany([{"x": d["y"], "row_end": d["row_end"], "col": d["col"], "val": d["val"],
                                                  "nnz": d["nnz"], "capacity": d["n"]} for d in ss])
            # decoded maps are short-lived: each site decodes into its own slice of one scratch
            # buffer (the many-call needs distinct outputs)
            tot = sum(d["n"] for d in ss) + sum(d["n"] for d in ds)
            self.scratch_many = torch.empty(max(1, tot), dtype=torch.float32, device=dev)
            o, views = 0, []
            for d in ss + ds:
                views.append(self.scratch_many[o:o + d["n"]])
                o += d["n"]
            self.dec_many = gist.SsdcDecodeMany([{"row_end": d["row_end"], "col": d["col"], "val": d["val"],
                                                  "n": d["n"], "x": v} for d, v in zip(ss, views[:len(ss)])])
            self.dpr_enc_many = gist.DprMany([{"x": d["y"], "packed": d["packed"]} for d in ds], dpr_bits, True)
            self.dpr_dec_many = gist.DprMany([{"packed": d["packed"], "n": d["n"], "x": v}
                                              for d, v in zip(ds, views[len(ss):])], dpr_bits, False)

    # ---- one pass: encode all sites (forward), decode all sites (backward)
    def step(self, timer=None):
        if self.many:
            return self.step_many(timer)
        g = self.g
        t = timer or (lambda kind, d: _Null())
        for d in self.sites:
            k = d["site"].kind
            if k == "relu_pool":
                if self.fuse:
                    with t("a2_maxpool_fwd_argmax+a1", d):
                        g.gist_maxpool_fwd_argmax(d["y"], d["site"].pool, out=d["out"], argmax=d["arg"], mask=d["mask"])
                else:
                    with t("a1_binarize_encode", d):
                        g.gist_binarize_encode(d["y"], mask=d["mask"])
                    with t("a2_maxpool_fwd_argmax", d):
                        g.gist_maxpool_fwd_argmax(d["y"], d["site"].pool, out=d["out"], argmax=d["arg"])
            elif k == "pool_only":
                with t("a2_maxpool_fwd_argmax", d):
                    g.gist_maxpool_fwd_argmax(d["y"], d["site"].pool, out=d["out"], argmax=d["arg"])
            elif k == "ssdc":
                with t("a4_ssdc_encode", d):
                    g.gist_ssdc_encode(d["y"], capacity=d["n"], row_end=d["row_end"], col=d["col"], val=d["val"],
                                       nnz=d["nnz"], workspace=d["ws"])
            else:
                with t("a6_dpr_encode", d):
                    g.gist_dpr_encode(d["y"], self.bits, packed=d["packed"])
        for d in reversed(self.sites):
            k = d["site"].kind
            n = d["n"]
            if k in ("relu_pool", "pool_only"):
                dx = self.scratch[:n].view(d["shape"])
                with t("a3_pool_relu_bwd", d):
                    g.gist_pool_relu_bwd(d["dY"], d["arg"], d["mask"], d["shape"], d["site"].pool, dx=dx)
            elif k == "ssdc":
                with t("a5_ssdc_decode", d):
                    g.gist_ssdc_decode(d["row_end"], d["col"], d["val"], n, x=self.scratch[:n])
            else:
                with t("a7_dpr_decode", d):
                    g.gist_dpr_decode(d["packed"], n, self.bits, x=self.scratch[:n])

    def step_many(self, timer=None):
        """Forward: a2 (+a1) per ReLU->Pool site, then every SSDC site in one launch and every DPR
        site in one launch; backward in reverse: DPR decodes, SSDC decodes, a3 per site."""
        g = self.g
        t = timer or (lambda kind, d: _Null())
        for d in self.sites:
            k = d["site"].kind
            if k == "relu_pool":
                with t("a2_maxpool_fwd_argmax+a1", d):
                    g.gist_maxpool_fwd_argmax(d["y"], d["site"].pool, out=d["out"], argmax=d["arg"], mask=d["mask"])
            elif k == "pool_only":
                with t("a2_maxpool_fwd_argmax", d):
                    g.gist_maxpool_fwd_argmax(d["y"], d["site"].pool, out=d["out"], argmax=d["arg"])
        if self.ssdc_sites:
            with t("a4_ssdc_encode", self.ssdc_sites):
                self.enc_many()
        if self.dpr_sites:
            with t("a6_dpr_encode", self.dpr_sites):
                self.dpr_enc_many()
            with t("a7_dpr_decode", self.dpr_sites):
                self.dpr_dec_many()
        if self.ssdc_sites:
            with t("a5_ssdc_decode", self.ssdc_sites):
                self.dec_many()
        for d in reversed(self.sites):
            if d["site"].kind in ("relu_pool", "pool_only"):
                dx = self.scratch[:d["n"]].view(d["shape"])
                with t("a3_pool_relu_bwd", d):
                    g.gist_pool_relu_bwd(d["dY"], d["arg"], d["mask"], d["shape"], d["site"].pool, dx=dx)

    def encoded_views(self, nnz_list):
        """Device views of every site's encoding (what Gist keeps through the forward->backward gap),
        exact sizes: SSDC col/val trimmed to the site's nnz."""
        out, k = [], 0
        for d in self.sites:
            kind = d["site"].kind
            if kind in ("relu_pool", "pool_only"):
                out.append(d["arg"])
                if d["mask"] is not None:
                    out.append(d["mask"])
            elif kind == "ssdc":
                m = int(nnz_list[k])
                out += [d["row_end"], d["col"][:m], d["val"][:m]]
                k += 1
            else:
                out.append(d["packed"])
        return out

    def nnz_host(self):
        return self.nnz_all.cpu()

    # ---- algorithmic bytes of one launch; nnz from the last step
    def algo_bytes(self, kind, d, nnz=None):
        if isinstance(d, list):  # a many-map launch: the sum over its sites
            return sum(self.algo_bytes(kind, e, nnz.get(id(e)) if isinstance(nnz, dict) else None) for e in d)
        n = d["n"]
        if kind == "a1_binarize_encode":
            return 4 * n + 4 * words(n, 32)
        if kind.startswith("a2_maxpool_fwd_argmax"):
            b = 4 * n + 4 * d["n_out"] + 4 * words(d["n_out"], 8)
            return b + (4 * words(n, 32) if kind.endswith("+a1") else 0)
        if kind == "a3_pool_relu_bwd":
            return 4 * d["n_out"] + 4 * words(d["n_out"], 8) + (4 * words(n, 32) if d["mask"] is not None else 0) + 4 * n
        if kind in ("a4_ssdc_encode", "a5_ssdc_decode"):
            return 4 * n + 5 * nnz + 4 * words(n, 256)
        if kind in ("a6_dpr_encode", "a7_dpr_decode"):
            return 4 * n + 4 * words(n, {16: 2, 10: 3, 8: 4}[self.bits])
        raise KeyError(kind)

    def compression(self, nnz_list):
        """Per-encoding compression ratio (fp32 bytes / encoded bytes), exact byte counts."""
        fp32 = {"binarize": 0, "ssdc": 0, "dpr": 0}
        enc = {"binarize": 0, "ssdc": 0, "dpr": 0}
        k = 0
        for d in self.sites:
            s = d["site"]
            if s.kind == "relu_pool":
                fp32["binarize"] += 4 * d["n"]
                enc["binarize"] += 4 * words(d["n"], 32) + 4 * words(d["n_out"], 8)
            elif s.kind == "ssdc":
                fp32["ssdc"] += 4 * d["n"]
                enc["ssdc"] += 5 * int(nnz_list[k]) + 4 * words(d["n"], 256)
                k += 1
            elif s.kind == "dpr":
                fp32["dpr"] += 4 * d["n"]
                enc["dpr"] += 4 * words(d["n"], {16: 2, 10: 3, 8: 4}[self.bits])
        out = {e: round(fp32[e] / enc[e], 4) for e in fp32 if enc[e]}
        out["total"] = round(sum(fp32.values()) / max(1, sum(enc.values())), 4)
        return out


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


def site_label(kind, d):
    """`<kernel kind>:<site name>` (a many-map launch: `<kind>:<first site>+<n-1>`)."""
    if isinstance(d, list):
        return f"{kind}:{d[0]['site'].name}+{len(d) - 1}" if d else kind
    return f"{kind}:{d['site'].name}"


class NvtxRanges:
    """An NVTX range per call site (`--nvtx`: named ranges in nsys / ncu --nvtx timelines)."""

    def __call__(self, kind, d):
        class _Ctx:
            def __enter__(self_inner):
                torch.cuda.nvtx.range_push(site_label(kind, d))
                return self_inner

            def __exit__(self_inner, *a):
                torch.cuda.nvtx.range_pop()
                return False
        return _Ctx()


class KernelTimer:
    """CUDA events around every launch, on the stream the kernels are launched on (and an NVTX range
    per call site when nvtx is set)."""

    def __init__(self, stream, nvtx=False, external=False):
        self.stream = stream  # None: the current stream (inside a graph capture, the capturing one)
        self.nvtx = nvtx
        self.external = external  # events recorded as graph nodes (cudaEventRecordExternal)
        self.records = []  # (kind, site dict, start, end)

    def __call__(self, kind, d):
        timer = self

        class _Ctx:
            def __enter__(self_inner):
                if timer.nvtx:
                    torch.cuda.nvtx.range_push(site_label(kind, d))
                self_inner.s = torch.cuda.Event(enable_timing=True, external=timer.external)
                self_inner.e = torch.cuda.Event(enable_timing=True, external=timer.external)
                self_inner.st = timer.stream if timer.stream is not None else torch.cuda.current_stream()
                self_inner.s.record(self_inner.st)
                return self_inner

            def __exit__(self_inner, *a):
                self_inner.e.record(self_inner.st)
                if timer.nvtx:
                    torch.cuda.nvtx.range_pop()
                timer.records.append((kind, d, self_inner.s, self_inner.e))
                return False
        return _Ctx()


# --------------------------------------------------------------------------------- clocks
class ClockSampler:
    """Samples SM clock, power and clock-event (throttle) reasons through NVML every 5 ms
    while the timed region runs (the recipe's nvidia-smi clocks line, in-process)."""

    REASONS = {"sw_power_cap": 0x4, "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20,
               "hw_thermal_slowdown": 0x40, "hw_power_brake_slowdown": 0x80}

    def __init__(self, device: torch.device, period_s: float = 0.005):
        self.device, self.period = device, period_s
        self.samples, self.reasons, self.max_mhz, self.power = [], set(), None, []
        self._stop = None

    def _handle(self, nv):
        """NVML handle of this CUDA device, matched by UUID (CUDA and NVML orders may differ)."""
        want = str(torch.cuda.get_device_properties(self.device).uuid).lower()
        for i in range(nv.nvmlDeviceGetCount()):
            h = nv.nvmlDeviceGetHandleByIndex(i)
            u = nv.nvmlDeviceGetUUID(h)
            u = (u.decode() if isinstance(u, bytes) else u).lower()
            if want and want in u:
                return h
        return nv.nvmlDeviceGetHandleByIndex(self.device.index or 0)

    def __enter__(self):
        import threading
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = self._handle(nv)
            self.max_mhz = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        except Exception as e:  # no NVML: record why
            self.error = repr(e)
            return self
        self._stop = threading.Event()

        def run():
            while not self._stop.is_set():
                try:
                    self.samples.append(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM))
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                    for name, bit in self.REASONS.items():
                        if r & bit:
                            self.reasons.add(name)
                    self.power.append(nv.nvmlDeviceGetPowerUsage(h) / 1000.0)
                except Exception:
                    pass
                self._stop.wait(self.period)
        self._thread = threading.Thread(target=run, daemon=True)
        self._thread.start()
        return self

    def __exit__(self, *a):
        if self._stop is not None:
            self._stop.set()
            self._thread.join(timeout=2)
        return False

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"],
                    "error": getattr(self, "error", "no samples")}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples),
                "power_w_max": round(max(self.power), 1) if self.power else None}


# --------------------------------------------------------------------------------- oracle legs
def oracle_site(ref, d, bits):
    """The oracle (as it stands) on one site of the sample: encode, then decode."""
    s = d["site"]
    if s.kind in ("relu_pool", "pool_only"):
        mask = ref.binarize_encode(d["y"]) if s.kind == "relu_pool" else None
        _, arg = ref.maxpool_fwd_argmax(d["y"], s.pool)
        ref.pool_relu_bwd(d["dY"], arg, mask, d["y"].shape, s.pool)
    elif s.kind == "ssdc":
        enc = ref.ssdc_encode(d["y"])
        ref.ssdc_decode(*enc, d["n"])
    else:
        ref.dpr_decode(ref.dpr_encode(d["y"], bits), d["n"], bits)


def oracle_pass(ref, sites_host, bits):
    """The oracle (as it stands) over one sample: encode every site, then decode."""
    for d in sites_host:
        s = d["site"]
        if s.kind in ("relu_pool", "pool_only"):
            if s.kind == "relu_pool":
                d["mask"] = ref.binarize_encode(d["y"])
            d["out"], d["arg"] = ref.maxpool_fwd_argmax(d["y"], s.pool)
        elif s.kind == "ssdc":
            d["enc"] = ref.ssdc_encode(d["y"])
        else:
            d["packed"] = ref.dpr_encode(d["y"], bits)
    for d in reversed(sites_host):
        s = d["site"]
        if s.kind in ("relu_pool", "pool_only"):
            ref.pool_relu_bwd(d["dY"], d["arg"], d.get("mask"), d["y"].shape, s.pool)
        elif s.kind == "ssdc":
            ref.ssdc_decode(*d["enc"], d["n"])
        else:
            ref.dpr_decode(d["packed"], d["n"], bits)


def oracle_sample(cfg, images: int, sparsity: float, seed0: int):
    sites = []
    for si, s in enumerate(WL.sites_for(cfg)):
        shape = (images,) + s.chw
        seed = seed0 + 1000 * si
        d = {"site": s, "n": s.numel(images)}
        if s.kind in ("relu_pool", "pool_only"):
            d["y"] = WL.relu_map(shape, 0.5, seed).numpy()
            d["dY"] = WL.grad_map((images,) + pool_out(s.chw, s.pool), seed + 500).numpy()
        elif s.kind == "ssdc":
            d["y"] = WL.relu_map(shape, sparsity, seed).numpy()
        else:
            d["y"] = WL.dpr_map(shape, seed).numpy()
        sites.append(d)
    return sites


def host_cpu():
    """(usable cores, CPU model name) of this host."""
    try:
        cores = len(os.sched_getaffinity(0))
    except AttributeError:
        cores = os.cpu_count() or 1
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return cores, model


def cpu_baseline(cfg, sparsity, bits, budget_s):
    """The oracle (as it stands, never tuned) timed on the host on a bounded sample of the same
    workload: (i) single-threaded over whole images, (ii) on ALL host cores with
    the independent units of the workload (one stash site of one image: encode + decode) spread
    over a thread pool — the oracle's C functions run through ctypes, which releases the GIL, so
    the threads run the unmodified oracle in parallel.  `value` is the all-cores figure."""
    import concurrent.futures as cf
    import oracle as ref
    ref.lib()
    cores, model = host_cpu()
    # (i) one thread
    images, elapsed, nbytes = 0, 0.0, 0
    while elapsed < budget_s / 3 and images < 64:
        sample = oracle_sample(cfg, 1, sparsity, 777 + images)
        t0 = time.perf_counter()
        oracle_pass(ref, sample, bits)
        elapsed += time.perf_counter() - t0
        nbytes += 8 * sum(d["n"] for d in sample)
        images += 1
    single = nbytes / elapsed / 1e9
    # (ii) all cores: rounds of (cores x sites) units over 4 distinct images, until ~2/3 budget
    pool_imgs = [oracle_sample(cfg, 1, sparsity, 4242 + k) for k in range(4)]
    units = [d for img in pool_imgs for d in img]
    unit_bytes = [8 * d["n"] for d in units]
    per_round = max(1, -(-cores // len(units))) * len(units)  # every core busy, whole images
    done_bytes, units_run, rounds = 0, 0, 0
    with cf.ThreadPoolExecutor(max_workers=cores) as ex:
        list(ex.map(lambda d: oracle_site(ref, d, bits), units[: min(len(units), cores)]))  # warm pages
        t0 = time.perf_counter()
        while True:
            idx = [k % len(units) for k in range(per_round)]
            list(ex.map(lambda k: oracle_site(ref, units[k], bits), idx))
            done_bytes += sum(unit_bytes[k] for k in idx)
            units_run += per_round
            rounds += 1
            if time.perf_counter() - t0 >= 2 * budget_s / 3 or rounds >= 50:
                break
        multi_s = time.perf_counter() - t0
    multi = done_bytes / multi_s / 1e9
    return {"value": round(multi, 4), "unit": "GB/s", "cores": cores, "kind": "oracle", "cpu_model": model,
            "single_thread_GBps": round(single, 4),
            "sample": f"{units_run} units (one stash site of one {cfg.key} image, encode+decode) on a {cores}-thread "
                      f"pool over {multi_s:.1f} s; single-threaded: {images} whole image(s) in {elapsed:.1f} s"}


def run_reference(args, cfg):
    """The reference arm of this no-code tier: the CPU oracle, as it stands, on all host cores.
    One step = one image's worth of units per usable core group: ceil(cores / sites) distinct
    images, every (image, site) unit (encode + decode) run on a thread pool (ctypes releases the
    GIL, so the unmodified oracle runs in parallel)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return  # torchrun N>1: rank 0 alone runs the oracle arm
    import concurrent.futures as cf
    import oracle as ref
    ref.lib()
    cores, model = host_cpu()
    n_sites = len(WL.sites_for(cfg))
    images = max(1, -(-cores // n_sites))
    sample = oracle_sample(cfg, images, args.sparsity, 999)  # `images` images per site map
    units = sample
    nbytes = 8 * sum(d["n"] for d in sample)
    with cf.ThreadPoolExecutor(max_workers=cores) as ex:
        def one_step():
            # split each site's batch of `images` into per-image units
            futs = []
            for d in units:
                per = d["n"] // images
                for k in range(images):
                    u = {"site": d["site"], "n": per, "y": d["y"][k:k + 1]}
                    if "dY" in d:
                        u["dY"] = d["dY"][k:k + 1]
                    futs.append(ex.submit(oracle_site, ref, u, args.dpr_bits))
            for f in futs:
                f.result()
        for _ in range(args.warmup):
            one_step()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            one_step()
        dt = (time.perf_counter() - t0) / max(1, args.steps)
    value = nbytes / dt / 1e9
    desc = (f"{images} image(s) of {cfg.key} per step, every (image, stash site) unit encoded+decoded by the "
            f"oracle on a {cores}-thread pool")
    line = {
        "impl": "reference", "metric": baseline_metric(), "value": round(value, 4), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": workload_config(args, cfg, images, note="bounded sample: " + desc),
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "cpu_model": model, "sample": desc},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def workload_config(args, cfg, batch, note=None, strong=False, world=1):
    c = {"workload": f"{cfg.key}: {cfg.description}", "net": cfg.net,
         **({"global_batch": batch, "batch_split": f"{batch} images over {world} rank(s) (shard_bounds)"} if strong
            else {"batch_per_gpu": batch}),
         "ssdc_sparsity": args.sparsity, "dpr_bits": args.dpr_bits,
         "calls": ("one gist_ssdc_*_many / gist_dpr_*_many launch per kind per step (P:171), a2/a3 per site"
                   if getattr(args, "many", True) else "one C-ABI call per site"),
         "l2": "inputs larger than L2 (no flush needed)", "parallelism": f"dp{args.gpus} (minibatch shards, no "
         "collective on the hot path)"}
    if note:
        c["note"] = note
    return c


# --------------------------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["gist", "reference"], default="gist")
    ap.add_argument("--config", default="C3", choices=sorted(CONFIG_INDEX))
    ap.add_argument("--batch", type=int, default=None, help="per-GPU batch (default: the config's)")
    ap.add_argument("--sparsity", type=float, default=None)
    ap.add_argument("--dpr-bits", type=int, default=None)
    ap.add_argument("--per-site", dest="many", action="store_false",
                    help="one C-ABI call per SSDC/DPR site instead of one gist_*_many launch per kind")
    ap.add_argument("--no-fuse-mask", dest="fuse_mask", action="store_false",
                    help="call a1 separately instead of passing the mask to the a2 call")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--eager", action="store_true",
                    help="launch every timed step's C-ABI calls from Python (default: capture one step in a "
                         "CUDA graph and replay it, so host launch overhead stays out of the device timing)")
    ap.add_argument("--nvtx", action="store_true", help="an NVTX range per call site (timed and instrumented steps)")
    ap.add_argument("--metrics-jsonl", default=None,
                    help="write per-(config, site, kernel, rank) device times and GB/s of the instrumented pass here")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--kernels-out", default=None, help="write the per-kernel breakdown JSON here")
    ap.add_argument("--same-device", action="store_true",
                    help="testing only: put every rank on cuda:0 and tally over gloo (exercises the N>1 "
                         "path on a 1-GPU box)")
    args = ap.parse_args()
    cfg = WL.CONFIGS[args.config]
    args.default_workload = args.batch is None and args.sparsity in (None, cfg.sparsity) and \
        args.dpr_bits in (None, cfg.dpr_bits)
    args.sparsity = cfg.sparsity if args.sparsity is None else args.sparsity
    args.dpr_bits = cfg.dpr_bits if args.dpr_bits is None else args.dpr_bits
    batch = args.batch or cfg.batch
    args.warmup = max(args.warmup, 3)

    if args.impl == "reference":
        run_reference(args, cfg)
        return

    import paper_conf_isca_jainpmtp18_b200 as gist
    from paper_conf_isca_jainpmtp18_b200.shard import shard_bounds, tally
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    dev = torch.device("cuda", 0 if args.same_device else local)
    torch.cuda.set_device(dev)
    dist = None
    if world > 1:
        import torch.distributed as dist
        if args.same_device:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    # C4 strong-scales one 64-image minibatch over the ranks; the other configs weak-scale (each rank
    # its own per-GPU batch of distinct images).  SURVEY.md §8(e).
    strong = cfg.key == "C4" and not args.batch
    if strong:
        lo, hi = shard_bounds(cfg.batch, world, rank)
    else:
        lo, hi = rank * batch, (rank + 1) * batch
    wl = Workload(gist, cfg, range(lo, hi), args.sparsity, args.dpr_bits, dev, args.fuse_mask, args.many)
    stream = torch.cuda.current_stream(dev)
    for _ in range(args.warmup):
        wl.step()
    barrier()

    # ---- timed region: K steps, CUDA events on the launching stream only around the whole region
    # (an event recorded between two kernels would cut their programmatic-dependent-launch overlap),
    # clocks sampled.  Then K more steps with an event pair around every launch give the per-kernel
    # breakdown and the roofline numbers.
    timer = KernelTimer(stream, nvtx=args.nvtx)
    nvtx_ranges = NvtxRanges() if args.nvtx else None
    # One step captured as a CUDA graph (the C-ABI calls launch on the capturing stream; PDL edges
    # are kept), replayed K times: the device executes exactly the eager step's kernels, without the
    # per-call Python/ctypes gaps between them.  --eager (or --nvtx) times Python-launched steps.
    graph, graph_note, per_step_launches = None, None, None
    if not (args.eager or args.nvtx):
        try:
            c0 = gist.gist_launch_count()
            g_ = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g_):
                wl.step()
            per_step_launches = gist.gist_launch_count() - c0
            for _ in range(2):
                g_.replay()
            torch.cuda.synchronize()
            graph = g_
        except Exception as ex:  # noqa: BLE001  (reported in the line, timed eagerly instead)
            graph_note = f"graph capture failed ({type(ex).__name__}: {str(ex)[:120]}); eager launches"
            torch.cuda.synchronize()
    launches0 = gist.gist_launch_count()
    with ClockSampler(dev) as clocks:
        barrier()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        for _ in range(args.steps):
            if graph is not None:
                graph.replay()
            else:
                wl.step(nvtx_ranges)
        ev1.record(stream)
        barrier()
        launches = gist.gist_launch_count() - launches0
        if graph is not None:
            launches = per_step_launches * args.steps
        elapsed_ms = ev0.elapsed_time(ev1)
        # the instrumented step, also as a graph when the timed step was one: the event pairs are graph
        # nodes, so a small kernel's time does not include the host's per-call gap before it
        g_inst, inst_note = None, "eager launches"
        if graph is not None:
            try:
                timer_g = KernelTimer(None, external=True)
                g_i = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g_i):
                    wl.step(timer_g)
                g_i.replay()
                torch.cuda.synchronize()
                g_inst, inst_note = g_i, "graph replays (event pairs as graph nodes)"
            except Exception as ex:  # noqa: BLE001  (the eager instrumented pass below)
                inst_note = f"eager launches (instrumented graph failed: {type(ex).__name__})"
                torch.cuda.synchronize()
        ev2, ev3 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev2.record(stream)
        for _ in range(args.steps):
            if g_inst is not None:
                g_inst.replay()
            else:
                wl.step(timer)
        ev3.record(stream)
        barrier()
        if g_inst is not None:
            # per-launch times: one replay at a time (each replay re-records the same events)
            timer.records = []
            for _ in range(args.steps):
                g_inst.replay()
                torch.cuda.synchronize()
                timer.records += [(k_, d_, s_.elapsed_time(e_)) for (k_, d_, s_, e_) in timer_g.records]
        else:
            timer.records = [(k_, d_, s_.elapsed_time(e_)) for (k_, d_, s_, e_) in timer.records]
    instrumented_ms = ev2.elapsed_time(ev3) / args.steps
    nnz = wl.nnz_host().tolist()

    # per-kernel breakdown (device time of each launch, summed per kind)
    per = {}
    nnz_of = {}
    k = 0
    for d in wl.sites:
        if d["site"].kind == "ssdc":
            nnz_of[id(d)] = int(nnz[k])
            k += 1
    per_site = {}  # (kind, site label) -> [ms, launches, algorithmic bytes]
    for kind, d, ms in timer.records:
        r = per.setdefault(kind, {"ms": 0.0, "launches": 0, "algo_bytes": 0})
        b = wl.algo_bytes(kind, d, nnz_of if isinstance(d, list) else nnz_of.get(id(d)))
        r["ms"] += ms
        r["launches"] += 1
        r["algo_bytes"] += b
        ps = per_site.setdefault((kind, site_label(kind, d)), [0.0, 0, 0])
        ps[0] += ms
        ps[1] += 1
        ps[2] += b
    peak, peak_src = hbm_peak()
    step_kernel_ms = sum(r["ms"] for r in per.values())
    kernels = {}
    for kind, r in sorted(per.items()):
        gbs = r["algo_bytes"] / (r["ms"] * 1e-3) / 1e9 if r["ms"] > 0 else 0.0
        kernels[kind] = {"ms_per_step": round(r["ms"] / args.steps, 4), "share": round(r["ms"] / step_kernel_ms, 4),
                         "launches_per_step": r["launches"] // args.steps, "algo_GBps": round(gbs, 1),
                         "frac_hbm": round(gbs / peak, 4)}
    dom = max(per, key=lambda kk: per[kk]["ms"])
    dom_gbs = per[dom]["algo_bytes"] / (per[dom]["ms"] * 1e-3) / 1e9
    if args.metrics_jsonl:  # one line per (config, site, kernel, rank) (SURVEY.md §5 metrics)
        with open(args.metrics_jsonl if world == 1 else f"{args.metrics_jsonl}.rank{rank}", "w") as f:
            for (kind, label), (ms, n_l, b) in per_site.items():
                gbs = b / (ms * 1e-3) / 1e9 if ms > 0 else 0.0
                f.write(json.dumps({"config": cfg.key, "site": label.split(":", 1)[1], "kernel": kind, "rank": rank,
                                    "world": world, "launches": n_l, "ms_per_launch": round(ms / n_l, 5),
                                    "algo_bytes_per_launch": int(b // n_l), "algo_GBps": round(gbs, 1),
                                    "frac_hbm": round(gbs / peak, 4),
                                    "sm_mhz": clocks.summary().get("sm_mhz")}) + "\n")

    # ---- multi-rank: max time over ranks, sum of bytes (one collective, outside the timed region)
    tdev = torch.device("cpu") if (dist is not None and args.same_device) else dev
    totals, elapsed_ms = tally(dist, {"fp32_bytes": wl.bytes_per_step * args.steps, "nnz": sum(nnz)}, elapsed_ms,
                               device=tdev)
    total_bytes = totals["fp32_bytes"]
    value = total_bytes / (elapsed_ms * 1e-3) / 1e9

    # ---- e2e: host pinned inputs -> H2D -> the same C-ABI calls -> D2H of the step's results: the
    # encoded stash of every site (exact bytes: the nnz of the deterministic inputs is known from the
    # untimed steps) and the per-site nnz tally
    e2e = None
    if not args.no_e2e:
        hosts = [(d, d["y"].cpu().pin_memory(), d["dY"].cpu().pin_memory() if "dY" in d else None) for d in wl.sites]
        h2d = sum(h.numel() * 4 + (g.numel() * 4 if g is not None else 0) for _, h, g in hosts)
        enc = wl.encoded_views(nnz) + [wl.nnz_all]
        enc_host = [torch.empty(t.shape, dtype=t.dtype).pin_memory() for t in enc]
        d2h = sum(t.numel() * t.element_size() for t in enc)
        e_steps = max(3, min(args.steps, 10))

        # Three streams: host->device copies, the step's kernels, device->host copies.  PCIe is full
        # duplex, so step k's encodings travel back while step k+1's maps travel in.  Step k+1's
        # copies into the map buffers wait until step k's kernels are done with them, and its kernels
        # wait until step k's encodings have been read back (they overwrite them).
        s_in, s_out = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
        ev = {"computed": None, "out": None}

        def e2e_step():
            if ev["computed"] is not None:
                s_in.wait_event(ev["computed"])
            with torch.cuda.stream(s_in):
                for d, h, g in hosts:
                    d["y"].copy_(h, non_blocking=True)
                    if g is not None:
                        d["dY"].copy_(g, non_blocking=True)
            stream.wait_stream(s_in)
            if ev["out"] is not None:
                stream.wait_event(ev["out"])
            wl.step()
            ev["computed"] = stream.record_event()
            s_out.wait_event(ev["computed"])
            with torch.cuda.stream(s_out):
                for t, hbuf in zip(enc, enc_host):
                    hbuf.copy_(t, non_blocking=True)
            ev["out"] = s_out.record_event()

        e2e_step()
        stream.wait_event(ev["out"])
        barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(e_steps):
            e2e_step()
        stream.wait_event(ev["out"])  # the last step's results are on the host
        b.record(stream)
        barrier()
        e_ms = a.elapsed_time(b)
        e_tot, e_ms = tally(dist, {"fp32_bytes": wl.bytes_per_step * e_steps}, e_ms, device=tdev)
        e_bytes = e_tot["fp32_bytes"]
        e2e = {"value": round(e_bytes / (e_ms * 1e-3) / 1e9, 3), "unit": "GB/s", "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h, "steps": e_steps,
               "note": "pinned host maps (and pool gradients) copied H2D each step, then the step's C-ABI calls, "
                       "then D2H of every site's encoding (mask + argmax map, exact-size CSR, DPR words) and the "
                       "per-site nnz tally; H2D, kernels and D2H on three streams (step k's D2H overlaps step "
                       "k+1's H2D), PCIe-bound"}

    if rank != 0:
        if dist is not None:
            dist.destroy_process_group()
        return

    cpu = cpu_baseline(cfg, args.sparsity, args.dpr_bits, args.cpu_seconds) if world == 1 else None
    line = {
        "metric": baseline_metric(), "value": round(value, 3), "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(elapsed_ms / args.steps, 4),
        "higher_is_better": True, "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": workload_config(args, cfg, batch if not strong else cfg.batch, strong=strong, world=world),
        "roofline": {"bound": "hbm", "kernel": dom, "achieved": round(dom_gbs, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(dom_gbs / peak, 4), "traffic": traffic_for(args, dom), "peak_source": peak_src},
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": launches,
        "launch": ("cuda_graph: one captured step replayed K times (%d libgist launches per step)" % per_step_launches
                   if graph is not None else (graph_note or "eager: C-ABI calls from Python every step")),
        "clocks": clocks.summary(),
        "compression": wl.compression(nnz),
        "kernels": kernels,
        "kernels_pass": {"note": "per-kernel times from K further steps with an event pair around every launch, "
                                 + inst_note,
                         "ms_per_step": round(instrumented_ms, 4)},
        "stash_bytes_per_gpu": 4 * wl.stash_elems,
    }
    if args.kernels_out:
        with open(args.kernels_out, "w") as f:
            json.dump(kernels, f, indent=1)
    print(json.dumps(line), flush=True)
    if dist is not None:
        dist.destroy_process_group()


def traffic_for(args, kind):
    """DRAM bytes per launch of the dominant kernel, from the committed ncu --set full capture of
    THIS configuration's launch (profiles/ncu_traffic.json, keyed "<config>:<kernel>:<many|per-site>"
    at the config's default batch, sparsity and DPR width); None when no such capture exists."""
    if not getattr(args, "default_workload", False):
        return None
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        t = json.load(f)
    key = f"{args.config}:{kind}:{'many' if args.many else 'per-site'}"
    return t.get(key, {}).get("dram_bytes_per_launch")


if __name__ == "__main__":
    main()
