# Round-2 final evidence run (session 3): parity, smoke, bench line (C3), configs, isolated kernels,
# launch list and ncu captures, f4 bench/accuracy (compute-sanitizer is closed on the pool).  Outputs under gpurun_out/$TAG/.
D=gpurun_out/${TAG:-r2final2}; mkdir -p $D
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv,noheader > $D/gpu.txt
timeout 1800 python -m pytest tests -q -m gpu -p no:cacheprovider > $D/pytest_gpu.log 2>&1; tail -2 $D/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1; tail -1 $D/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 --metrics-jsonl $D/metrics_C3.jsonl > $D/bench_C3.json 2> $D/bench_C3.err; cut -c1-300 $D/bench_C3.json
for c in C2 C4 C5o C5n; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 5 --no-e2e --cpu-seconds 1 --metrics-jsonl $D/metrics_$c.jsonl > $D/bench_$c.json 2>/dev/null
done
timeout 900 python scripts/kernel_bench.py --small --reps 20 --json $D/kernel_bench.json > $D/kernel_bench.log 2>&1; tail -1 $D/kernel_bench.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/bench_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --cpu-seconds 0.1 > $D/bench_under_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ssdc_encode_kernel -s 3 -c 1 -o $D/bench_C3_a4_many \
  python bench.py --steps 1 --warmup 3 --no-e2e --cpu-seconds 0.1 > $D/ncu_a4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pool3 -s 4 -c 2 -o $D/c4_pool3 \
  python bench.py --config C4 --steps 1 --warmup 1 --no-e2e --cpu-seconds 0.1 > $D/ncu_pool3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:wgrad_ssdc -s 1 -c 1 -o $D/f4_wgrad_conv3_2 \
  python scripts/wgrad_bench.py --layers conv3_2 --reps 1 > $D/ncu_f4.log 2>&1
timeout 900 python scripts/wgrad_bench.py --reps 10 --json $D/f4_bench.json > $D/f4_bench.log 2>&1; tail -2 $D/f4_bench.log
timeout 600 python scripts/wgrad_accuracy.py --json $D/f4_accuracy.json > $D/f4_accuracy.log 2>&1
ls $D
