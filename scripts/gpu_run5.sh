set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc or smoke" 2>&1 | tail -3
timeout 300 python scripts/kernel_bench.py --only a4,a5 > gpurun_out/kernels18.log 2>&1; tail -8 gpurun_out/kernels18.log
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ssdc_encode_kernel -s 3 -c 1 -o gpurun_out/prof_ssdc_enc_v16 python scripts/kernel_bench.py --only a4 --reps 2 > gpurun_out/ncu18.log 2>&1; tail -2 gpurun_out/ncu18.log
