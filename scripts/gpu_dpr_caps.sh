# DPR many-map grid cap: C3 step (and its a6/a7 in-step fractions) for the default and var/ variants
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  for rep in 1 2; do
  GIST_LIBRARY=$lib timeout 120 python bench.py --steps 30 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', d['value'], d['ms_per_step'], d['kernels']['a6_dpr_encode'], d['kernels']['a7_dpr_decode'])"
  done
done
