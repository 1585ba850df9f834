set -x
timeout 300 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc or smoke" 2>&1 | tail -1
timeout 300 python scripts/kernel_bench.py --only a4 2>&1 | grep '"a4"' | cut -c1-150
GIST_LIBRARY=variants/libgist_trace.so timeout 120 python scripts/ssdc_trace.py 0.8 2>&1 | sed -n 1,12p
GIST_LIBRARY=variants/libgist_c1.so timeout 300 python scripts/kernel_bench.py --only a4 2>&1 | grep '"a4"' | cut -c1-150
