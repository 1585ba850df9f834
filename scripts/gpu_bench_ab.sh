# Whole-step bench (no e2e) of the default library and every var/ variant, twice each.
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  for i in 1 2; do
    GIST_LIBRARY=$lib timeout 300 python bench.py --steps 30 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', d['value'], d['ms_per_step'], d['kernels_pass']['ms_per_step'], d['gpu_launches'], {k: v['ms_per_step'] for k, v in d['kernels'].items()})"
  done
done
