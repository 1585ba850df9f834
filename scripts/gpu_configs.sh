# Whole-step bench of every config (C2, C4, C5o, C5n; C3 is the default) with the per-kernel breakdown.
mkdir -p gpurun_out
for c in C2 C4 C5o C5n; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 > gpurun_out/bench_$c.json 2>/dev/null
  python -c "import json,sys; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', d['value'], d['ms_per_step'], d['config']['workload']); [print('   ', k, v['ms_per_step'], v['launches_per_step'], v['frac_hbm']) for k, v in d['kernels'].items()]"
done
