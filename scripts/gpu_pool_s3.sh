# 3x3 pools: graph-timed cases for the default library and var/ variants, and one ncu --set full
# capture of the AlexNet relu1 b128 forward+mask and backward kernels.
D=gpurun_out/pool_s3; mkdir -p $D
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  echo "=== $lib"; GIST_LIBRARY=$lib timeout 300 python scripts/pool_one.py --case all --time --reps 20 2>&1 | tail -27
done
if [ -n "$NCU" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pool" -c 3 \
    -o $D/alexnet1 python scripts/pool_one.py --case alexnet1 --reps 1 --what fwdm,bwd > $D/ncu.log 2>&1; tail -2 $D/ncu.log
fi
