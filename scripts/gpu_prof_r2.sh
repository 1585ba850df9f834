# Round-2 profiling call: isolated a4 with clocks, ncu full captures of the step's SSDC encode
# (many-map launch) and of the f4 wgrad kernel (VGG16 conv3_2, 3xTF32).
D=gpurun_out/prof_${TAG:-r2}
mkdir -p $D
timeout 600 python scripts/kernel_bench.py --only a4,a5 --reps 20 --json $D/kb_a4.json > $D/kb_a4.log 2>&1; tail -8 $D/kb_a4.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ssdc_encode_kernel -s 3 -c 1 -o $D/bench_a4_many \
  python bench.py --steps 1 --warmup 3 --no-e2e --cpu-seconds 0.1 > $D/bench_a4.log 2>&1; tail -3 $D/bench_a4.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:wgrad_ssdc -s 1 -c 1 -o $D/f4_wgrad_conv3_2 \
  python scripts/wgrad_bench.py --layers conv3_2 --reps 1 > $D/f4.log 2>&1; tail -3 $D/f4.log
ls -la $D
