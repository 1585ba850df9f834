# A/B of pool variants (var/*.so vs default): isolated 3x3 rows and the C2/C4 steps
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 300 python scripts/kernel_bench.py --small --only a2,a3 --reps 20 2>&1 | grep -E '3x3' | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('  %-48s %.4f ms %.3f' % (d['row']+' '+d['case'], d['ms_median'], d['frac_hbm']))"
  for cfg in C2 C4; do
  GIST_LIBRARY=$lib timeout 300 python bench.py --config $cfg --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print('  $cfg', d['value'], d['ms_per_step'], {k: (v['ms_per_step'], v['frac_hbm']) for k, v in d['kernels'].items() if k.startswith('a2') or k.startswith('a3')})"
  done
done
