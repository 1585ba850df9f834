timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sanitize.py -x -q -p no:cacheprovider -k "pool or relu or 3x3 or sanitize" 2>&1 | tail -1
GIST_LIBRARY=var/libgist_s2.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "pool or relu or 3x3" 2>&1 | tail -1
for cfg in C2 C4 C5n C5o C3; do
timeout 300 python bench.py --config $cfg --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print('$cfg', d['value'], d['ms_per_step'], {k: (v['ms_per_step'], v['frac_hbm']) for k, v in d['kernels'].items()})"
done
