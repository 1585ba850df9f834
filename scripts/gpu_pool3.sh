# 3x3 pools: parity, isolated kernels (clocks), C2/C4/C5n steps
mkdir -p gpurun_out
TAG=${TAG:-p3}
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sanitize.py -x -q -p no:cacheprovider -k "pool or relu or 3x3 or sanitize" > gpurun_out/pytest_$TAG.log 2>&1; tail -3 gpurun_out/pytest_$TAG.log
timeout 600 python scripts/kernel_bench.py --small --only a2,a3 --reps 20 > gpurun_out/kb_$TAG.log 2>&1; grep -E '"a2"|"a3"|clocks' gpurun_out/kb_$TAG.log | cut -c1-170
for cfg in C2 C4 C5n C3; do
timeout 600 python bench.py --config $cfg --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print('$cfg', d['value'], d['ms_per_step'], {k: (v['ms_per_step'], v['frac_hbm']) for k, v in d['kernels'].items()})"
done
