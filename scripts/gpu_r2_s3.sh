# Session-3 check of HEAD: full -m gpu suite, smoke, C3 bench line, configs, isolated kernels.
D=gpurun_out/s3; mkdir -p $D
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv,noheader > $D/gpu.txt
timeout 1800 python -m pytest tests -q -m gpu -p no:cacheprovider > $D/pytest_gpu.log 2>&1; tail -3 $D/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1; tail -1 $D/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > $D/bench_C3.json 2> $D/bench_C3.err; cut -c1-300 $D/bench_C3.json
for cfg in C2 C4 C5o C5n; do
timeout 300 python bench.py --config $cfg --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 > $D/bench_$cfg.json 2>/dev/null
python -c "import json,sys; d=json.loads(open('$D/bench_$cfg.json').read().splitlines()[-1]); print('$cfg', d['value'], d['ms_per_step'], {k: (v['ms_per_step'], v['frac_hbm']) for k, v in d['kernels'].items()})"
done
timeout 900 python scripts/kernel_bench.py --small --reps 20 --json $D/kernel_bench.json > $D/kernel_bench.log 2>&1; tail -40 $D/kernel_bench.log
