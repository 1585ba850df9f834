# A/B of the default library and every var/ variant: parity (-k $K), isolated rows ($ROWS), whole step.
set -x
mkdir -p gpurun_out
K=${K:-ssdc}; ROWS=${ROWS:-a4}
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 600 python -m pytest tests -x -q -m "gpu and not slow" -k "$K" 2>&1 | tail -1
  for r in $ROWS; do GIST_LIBRARY=$lib timeout 200 python scripts/kernel_bench.py --only $r 2>&1 | grep "\"$r\"" | cut -c1-150; done
  GIST_LIBRARY=$lib timeout 600 python bench.py --steps 30 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('STEP', d['value'], d['ms_per_step'], {k: v['frac_hbm'] for k, v in d['kernels'].items()})"
done
