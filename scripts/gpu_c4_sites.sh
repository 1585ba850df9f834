# C4 per-site device times for the default library and each var/ variant
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  n=$(basename $lib .so)
  GIST_LIBRARY=$lib timeout 300 python bench.py --config C4 --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 --metrics-jsonl gpurun_out/c4sites_$n.jsonl > /dev/null 2>&1
done
python - <<'PY'
import json, glob
files = sorted(glob.glob("gpurun_out/c4sites_*.jsonl"))
rows = {}
for f in files:
    for l in open(f):
        d = json.loads(l); rows.setdefault((d["site"], d["kernel"]), {})[f] = d["ms_per_launch"] * 1000
print("site kernel", [f.split("_", 1)[1] for f in files])
for k, v in rows.items():
    print(f"{k[0]:14s} {k[1]:28s}", " ".join(f"{v.get(f, 0):7.1f}" for f in files))
PY
