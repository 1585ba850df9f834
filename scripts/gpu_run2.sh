set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -5
timeout 600 python scripts/kernel_bench.py --small --json gpurun_out/kernels2.json > gpurun_out/kernels2.log 2>&1; tail -30 gpurun_out/kernels2.log
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench2.json 2> gpurun_out/bench2.err; tail -3 gpurun_out/bench2.err; cat gpurun_out/bench2.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ssdc_encode_kernel -s 3 -c 1 -o gpurun_out/prof_ssdc_enc python scripts/kernel_bench.py --only a4 --reps 2 > gpurun_out/ncu2.log 2>&1; tail -3 gpurun_out/ncu2.log
