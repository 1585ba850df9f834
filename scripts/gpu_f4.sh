# f4: parity tests + the wgrad bench
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_wgrad.py -q -p no:cacheprovider --tb=short > gpurun_out/f4_pytest.log 2>&1; tail -30 gpurun_out/f4_pytest.log | grep -E "Error|error|passed|failed"
timeout 600 python scripts/wgrad_bench.py --reps 10 --json gpurun_out/f4_bench.json > gpurun_out/f4_bench.log 2>&1; tail -8 gpurun_out/f4_bench.log
