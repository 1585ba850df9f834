# many-map calls: tests + bench A/B (many vs per-site) on C3 and C4
mkdir -p gpurun_out
TAG=${TAG:-many}
timeout 900 python -m pytest tests/test_gpu_many.py tests/test_abi.py -x -q -p no:cacheprovider 2>&1 | tail -5
for mode in "" "--per-site"; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-e2e --cpu-seconds 1 $mode > gpurun_out/bench_${TAG}_c3$mode.json 2>&1
  python - gpurun_out/bench_${TAG}_c3$mode.json <<'PY'
import json,sys
l=json.loads(open(sys.argv[1]).read().splitlines()[-1])
print(sys.argv[1], l["value"], l["ms_per_step"], {k:(v["ms_per_step"],v["frac_hbm"],v["launches_per_step"]) for k,v in l["kernels"].items()}, l["clocks"]["sm_mhz"])
PY
done
timeout 600 python bench.py --config C4 --steps 20 --warmup 5 --no-e2e --cpu-seconds 1 > gpurun_out/bench_${TAG}_c4.json 2>&1; cut -c1-200 gpurun_out/bench_${TAG}_c4.json
