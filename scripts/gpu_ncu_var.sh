mkdir -p gpurun_out
for v in d1; do
GIST_LIBRARY=var/libgist_$v.so timeout 300 ncu --set full --clock-control none --import-source on -k regex:ssdc_encode_kernel -s 7 -c 1 -o gpurun_out/a4_$v python scripts/kernel_bench.py --reps 2 --only a4 > gpurun_out/a4_$v.log 2>&1
done
ls -la gpurun_out
