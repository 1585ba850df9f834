# a4 iteration: SSDC parity tests, isolated a4 (clocks), the C3 step
mkdir -p gpurun_out
TAG=${TAG:-a4}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_many.py tests/test_gpu_stash.py -x -q -p no:cacheprovider -k "ssdc or many or stash" > gpurun_out/pytest_$TAG.log 2>&1; tail -3 gpurun_out/pytest_$TAG.log
timeout 600 python scripts/kernel_bench.py --only a4 --reps 20 > gpurun_out/kb_$TAG.log 2>&1; grep -E '"a4"|clocks' gpurun_out/kb_$TAG.log | cut -c1-200
timeout 600 python bench.py --steps 20 --warmup 5 --no-e2e --cpu-seconds 1 > gpurun_out/bench_$TAG.json 2>&1
python - gpurun_out/bench_$TAG.json <<'PY'
import json,sys
l=json.loads(open(sys.argv[1]).read().splitlines()[-1])
print(l["value"], l["ms_per_step"], {k:(v["ms_per_step"],v["frac_hbm"]) for k,v in l["kernels"].items()}, l["clocks"]["sm_mhz"])
PY
