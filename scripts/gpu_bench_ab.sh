# Parity + whole-step bench of the default library and of each var/ variant.
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -2
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py --steps 30 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('default', d['value'], d['ms_per_step'], {k: v['frac_hbm'] for k, v in d['kernels'].items()})"
for lib in var/libgist_*.so; do
  GIST_LIBRARY=$lib timeout 600 python bench.py --steps 30 --warmup 5 --no-e2e --cpu-seconds 0.1 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', d['value'], d['ms_per_step'], {k: v['frac_hbm'] for k, v in d['kernels'].items()})"
done
