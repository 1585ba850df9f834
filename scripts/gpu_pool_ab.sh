set -x
timeout 1200 python -m pytest tests -x -q -m "gpu and not slow" -k "maxpool or pool or vgg16_relu" 2>&1 | tail -2
timeout 300 python scripts/kernel_bench.py --only a2 --reps 20 2>&1 | grep '"a2"' | cut -c1-200
timeout 600 python bench.py --steps 30 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('default', d['value'], d['ms_per_step'], {k: v['frac_hbm'] for k, v in d['kernels'].items()})"
