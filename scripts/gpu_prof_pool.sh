D=gpurun_out/prof_pool; mkdir -p $D
export GIST_LIBRARY=var/libgist_t512.so
timeout 300 ncu --set full --clock-control none --import-source on -k regex:pool3_fwd -s 2 -c 1 -o $D/p3_fwd_s1 python scripts/kernel_bench.py --small --only a2 --reps 2 > $D/l1.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:pool3_bwd_kernel -s 2 -c 1 -o $D/p3_bwd_s2 python scripts/kernel_bench.py --small --only a3 --reps 2 > $D/l2.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:pool3_bwd_kernel -s 20 -c 1 -o $D/p3_bwd_s1 python scripts/kernel_bench.py --small --only a3 --reps 2 > $D/l3.log 2>&1
export GIST_LIBRARY=var/libgist_old.so
timeout 300 ncu --set full --clock-control none --import-source on -k regex:maxpool_fwd_kernel -s 2 -c 1 -o $D/old_fwd_s2 python scripts/kernel_bench.py --small --only a2 --reps 2 > $D/l4.log 2>&1
ls -la $D
