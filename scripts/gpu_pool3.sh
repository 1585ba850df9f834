mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" -k "pool or smoke or stash" 2>&1 | tail -3
timeout 300 python scripts/kernel_bench.py --small --only a2,a3 2>&1 | grep -v vgg | cut -c1-150
