# Round-2 check: parity (not slow), smoke, the C3 bench line, C4 line.
mkdir -p gpurun_out
TAG=${TAG:-r2chk}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 1500 python -m pytest tests -x -q -m "gpu and not slow" -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1; tail -15 gpurun_out/pytest_$TAG.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -2 gpurun_out/bench_$TAG.err; cut -c1-400 gpurun_out/bench_$TAG.json
timeout 600 python bench.py --config C4 --steps 20 --warmup 5 --no-e2e --cpu-seconds 2 > gpurun_out/bench_c4_$TAG.json 2>&1; cut -c1-300 gpurun_out/bench_c4_$TAG.json
