set -x
timeout 300 python scripts/kernel_bench.py --only a3 --reps 20 2>&1 | grep '"a3"' | cut -c1-200
for lib in var/libgist_*.so; do
  echo "== $lib"; GIST_LIBRARY=$lib timeout 300 python scripts/kernel_bench.py --only a2,a3 --reps 20 2>&1 | grep '"a[23]"' | cut -c1-200
done
