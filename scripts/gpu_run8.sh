set -x
timeout 600 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize.py > gpurun_out/sanitize_racecheck2.log 2>&1; echo "racecheck rc=$?"; grep -E "SUMMARY|Race reported" gpurun_out/sanitize_racecheck2.log | head -8
for lib in variants/libgist_*.so; do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 120 python scripts/kernel_bench.py --only a2,a3,a4 2>&1 | grep -E '"a[234]"' | grep -v fused | cut -c1-150
done
