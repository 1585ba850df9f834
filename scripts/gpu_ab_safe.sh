# A/B with short timeouts (a variant that deadlocks must not hold the box): parity (-k $K), isolated a4, step
K=${K:-ssdc}
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 150 python -m pytest tests -x -q -m "gpu and not slow" -k "$K" -p no:cacheprovider 2>&1 | tail -1
  GIST_LIBRARY=$lib timeout 60 python scripts/a4_one.py 0.5 0.8 0.9 2>&1 | tail -3
  GIST_LIBRARY=$lib timeout 120 python bench.py --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('STEP', d['value'], d['ms_per_step'], {k: v['frac_hbm'] for k, v in d['kernels'].items()})"
done
