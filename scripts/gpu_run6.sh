set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests -x -q -m "gpu and not slow" -k "maxpool or dpr or autograd or vgg16" 2>&1 | tail -3
timeout 300 python scripts/kernel_bench.py --only a2,a3,a6,a7 > gpurun_out/kernels_r1b.log 2>&1; cut -c1-170 gpurun_out/kernels_r1b.log
