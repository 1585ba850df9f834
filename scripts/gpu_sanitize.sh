# Parity + compute-sanitizer (memcheck, racecheck, synccheck) over every kernel on small ragged shapes.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -1
for tool in memcheck racecheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_$tool.log
done
