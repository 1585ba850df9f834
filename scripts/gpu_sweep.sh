# Sweep SSDC-encode tuning variants (variants/libgist_*.so): parity subset + a4 throughput.
set -x
mkdir -p gpurun_out
for lib in variants/libgist_*.so; do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 120 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc_round_trip or ssdc_capacity" 2>&1 | tail -1
  GIST_LIBRARY=$lib timeout 120 python scripts/kernel_bench.py --only a4 2>&1 | grep '"a4"' | cut -c1-150
done
