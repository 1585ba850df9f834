# Full check: parity, smoke, isolated kernels (incl. 3x3 pools), every config's step, the C3 bench line.
mkdir -p gpurun_out
TAG=${TAG:-chk}
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -2
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python scripts/kernel_bench.py --small --json gpurun_out/kernels_$TAG.json > gpurun_out/kernels_$TAG.log 2>&1; cut -c1-150 gpurun_out/kernels_$TAG.log
bash scripts/gpu_configs.sh
timeout 600 python bench.py --steps 30 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -2 gpurun_out/bench_$TAG.err; cut -c1-300 gpurun_out/bench_$TAG.json
