set -x
mkdir -p gpurun_out
TAG=${TAG:-r1d}
timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for tool in memcheck racecheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/sanitize_$tool.log
done
timeout 600 python scripts/kernel_bench.py --small --json gpurun_out/kernels_$TAG.json > gpurun_out/kernels_$TAG.log 2>&1; cut -c1-150 gpurun_out/kernels_$TAG.log
timeout 600 python bench.py --steps 30 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -2 gpurun_out/bench_$TAG.err; cut -c1-400 gpurun_out/bench_$TAG.json
