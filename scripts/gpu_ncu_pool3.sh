mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:planes_fwd -s 2 -c 1 -o gpurun_out/p3fwd2 python scripts/kernel_bench.py --small --only a2 --reps 2 > /dev/null 2>&1
ls gpurun_out
