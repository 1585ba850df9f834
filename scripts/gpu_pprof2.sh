D=gpurun_out/pprof; mkdir -p $D
GIST_LIBRARY=var/libgist_p3bwd.so timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pool3_bwd" -c 1 \
    -o $D/bwd_inc3a python scripts/pool_one.py --case inc3a --reps 1 --what bwd > $D/ncu1.log 2>&1; tail -1 $D/ncu1.log
GIST_LIBRARY=var/libgist_p3bwd.so timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pool3_bwd" -c 1 \
    -o $D/bwd_alex1 python scripts/pool_one.py --case alexnet1 --reps 1 --what bwd > $D/ncu2.log 2>&1; tail -1 $D/ncu2.log
