# One ncu --set full capture of the SSDC encode kernel on VGG16 relu1_1 b64, s = 0.8.
set -x
mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ssdc_encode_kernel -s 7 -c 1 -o gpurun_out/${OUT:-ssdc3} python scripts/kernel_bench.py --only a4 --reps 2 > gpurun_out/${OUT:-ssdc3}.log 2>&1; tail -2 gpurun_out/${OUT:-ssdc3}.log
