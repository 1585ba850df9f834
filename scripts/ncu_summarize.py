#!/usr/bin/env python
"""Summarize ncu reports (full-set captures) and launch lists into profiles/.

  python scripts/ncu_summarize.py report <file.ncu-rep> [...]   -> one text block per report
  python scripts/ncu_summarize.py launches <launches.csv>        -> per-kernel share of device time
"""
import csv
import subprocess
import sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "Registers Per Thread", "Achieved Occupancy",
        "Theoretical Occupancy", "Issued Warp Per Scheduler", "No Eligible", "Executed Ipc Active", "L2 Hit Rate",
        "Issued Instructions", "Dynamic Shared Memory Per Block", "Static Shared Memory Per Block", "Grid Size",
        "Block Size"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    if len(rows) < 3:
        return []
    h, units = rows[0], rows[1]
    return [dict(zip(h, r)) | {"__units__": dict(zip(h, units))} for r in rows[2:]]


def report(rep):
    det = subprocess.run(["ncu", "-i", rep, "--page", "details"], capture_output=True, text=True).stdout
    lines = [f"== {rep}"]
    name = None
    for ln in det.splitlines():
        if name is None and "Context" in ln and "Device" in ln:
            name = ln.strip()
            lines.append(f"kernel: {name[:200]}")
        if any(ln.strip().startswith(k) for k in KEYS):
            lines.append("  " + " ".join(ln.split()))
    for r in raw(rep)[:1]:
        u = r["__units__"]
        rd, wr = r.get("dram__bytes_read.sum"), r.get("dram__bytes_write.sum")
        lines.append(f"  dram__bytes_read.sum {rd} {u.get('dram__bytes_read.sum', '')}; "
                     f"dram__bytes_write.sum {wr} {u.get('dram__bytes_write.sum', '')}")
        st = [(k[33:], float(v)) for k, v in r.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")
              and v.replace(".", "", 1).isdigit()]
        tot = sum(v for _, v in st) or 1.0
        top = ", ".join(f"{k} {v / tot * 100:.0f}%" for k, v in sorted(st, key=lambda t: -t[1])[:5])
        lines.append(f"  stall reasons (pc sampling): {top}")
    return "\n".join(lines)


def dram_bytes(rep):
    for r in raw(rep)[:1]:
        u = r["__units__"]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        return (float(r["dram__bytes_read.sum"]) * scale.get(u["dram__bytes_read.sum"], 1) +
                float(r["dram__bytes_write.sum"]) * scale.get(u["dram__bytes_write.sum"], 1))
    return None


def launches(path, ours=("binarize", "maxpool", "pool_bwd", "ssdc", "dpr_")):
    rows = list(csv.reader(open(path)))
    i = next(j for j, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[i]
    kn, mv = h.index("Kernel Name"), h.index("Metric Value")
    agg = {}
    for r in rows[i + 1:]:
        name = r[kn].split("(")[0].split("::")[-1]
        if not any(o in name for o in ours):
            continue
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += float(r[mv].replace(",", ""))
    tot = sum(v[1] for v in agg.values()) or 1.0
    out = [f"== {path}: libgist kernels only (ncu serialises launches, cold caches: compare shares)",
           f"{'kernel':40s} {'launches':>8s} {'total_us':>10s} {'share':>7s}"]
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append(f"{k:40s} {v[0]:8d} {v[1] / 1e3:10.1f} {v[1] / tot * 100:6.1f}%")
    return "\n".join(out)


if __name__ == "__main__":
    if sys.argv[1] == "report":
        print("\n\n".join(report(r) for r in sys.argv[2:]))
    elif sys.argv[1] == "launches":
        print(launches(sys.argv[2]))
    elif sys.argv[1] == "dram":
        print(dram_bytes(sys.argv[2]))
