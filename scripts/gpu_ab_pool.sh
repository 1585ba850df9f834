# A/B: pool cases (graph-timed) and C2/C4/C5n steps for each library in $LIBS
for lib in $LIBS; do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 300 python scripts/pool_one.py --case ${CASES:-alexnet1,alexnet2,nin2,nin4,inc3a,inc4a,inc5a} --time --reps 20 --what ${WHAT:-fwd,fwdm,bwd} 2>&1 | tail -24
  for c in ${CFGS:-C4 C2 C5n}; do
    GIST_LIBRARY=$lib timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print('$c', d['value'], d['ms_per_step'], {k:(v['ms_per_step'],v['frac_hbm']) for k,v in d['kernels'].items() if k[:2] in ('a2','a3')})"
  done
done
