set -x
for lib in variants/libgist_*.so; do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 120 python scripts/kernel_bench.py --only a4 2>&1 | grep '"a4"' | cut -c1-150
done
