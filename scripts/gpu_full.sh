# Full check: parity tests, isolated kernels, the bench step, ncu launch list.
set -x
mkdir -p gpurun_out
TAG=${TAG:-full}
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -4
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python scripts/kernel_bench.py --small --json gpurun_out/kernels_$TAG.json > gpurun_out/kernels_$TAG.log 2>&1; cat gpurun_out/kernels_$TAG.log | cut -c1-160
timeout 600 python bench.py --steps 30 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -3 gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-e2e --cpu-seconds 0.1 > /dev/null 2>&1; wc -l gpurun_out/launches_$TAG.csv
