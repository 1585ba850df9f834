# SSDC encode A/B: parity of the default library, then a4 throughput of each variant.
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc" 2>&1 | tail -4
KB_DIST=1 timeout 200 python scripts/kernel_bench.py --only a4 --reps 20 2>&1 | cut -c1-250
for lib in var/libgist_*.so; do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 200 python scripts/kernel_bench.py --only a4 2>&1 | grep '"a4"' | cut -c1-170
done
