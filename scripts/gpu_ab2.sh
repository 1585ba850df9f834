# A/B (no parity): isolated rows ($ROWS) and the whole step twice, default library vs var/ variants
mkdir -p gpurun_out
ROWS=${ROWS:-a4}
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  echo "=== $lib"
  for r in $ROWS; do GIST_LIBRARY=$lib timeout 200 python scripts/kernel_bench.py --only $r 2>&1 | grep "\"$r\"" | cut -c1-150; done
  for rep in 1 2; do
  GIST_LIBRARY=$lib timeout 600 python bench.py --steps 30 --warmup 5 --no-e2e --cpu-seconds 0.1 $BENCH_ARGS 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('STEP', d['value'], d['ms_per_step'], {k: (v['ms_per_step'], v['frac_hbm']) for k, v in d['kernels'].items()})"
  done
done
