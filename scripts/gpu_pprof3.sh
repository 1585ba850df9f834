D=gpurun_out/pprof; mkdir -p $D
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pool3" -c 3 \
    -o $D/inc4a python scripts/pool_one.py --case inc4a --reps 1 --what bwd > $D/ncu3.log 2>&1; tail -1 $D/ncu3.log
