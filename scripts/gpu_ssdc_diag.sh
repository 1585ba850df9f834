set -x
timeout 200 python scripts/ssdc4_trace.py 0.8 2>&1 | tail -45
