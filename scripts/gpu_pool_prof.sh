# 3x3/s2 pools: timing of the L1 kernels vs the pool3 plane-tile kernels (var/libgist_p3s2.so),
# and one ncu --set full capture of each on AlexNet relu1 b128
D=gpurun_out/poolprof; mkdir -p $D
for lib in ${TIMELIBS:-}; do
  echo "=== $lib"; GIST_LIBRARY=$lib timeout 300 python scripts/pool_one.py --case all --time --reps 20 2>&1 | tail -25
done
for v in l1:paper_conf_isca_jainpmtp18_b200/libgist.so p3:var/libgist_p3s2.so; do
  t=${v%%:*}; lib=${v#*:}
  GIST_LIBRARY=$lib timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pool|binarize" -c 6 \
    -o $D/alexnet1_$t python scripts/pool_one.py --case alexnet1 --reps 1 > $D/ncu_$t.log 2>&1; tail -2 $D/ncu_$t.log
done
