# pool kernels only: parity + per-kernel bandwidth (a2, a3) on full-size maps
timeout 600 python -m pytest tests -x -q -m "gpu and not slow" -k "pool or maxpool or autograd or smoke" 2>&1 | tail -2
timeout 300 python scripts/kernel_bench.py --small --only a2 2>&1 | grep -v "^$" | cut -c1-160
timeout 300 python scripts/kernel_bench.py --small --only a3 2>&1 | grep -v "^$" | cut -c1-160
