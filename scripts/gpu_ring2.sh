# pool3 ring / block-size sweep for the stride-2 forward (GIST_POOL3_RING overrides the per-kind ring), graph-timed
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so var/libgist_t256.so; do
for r in f2=2x48 f2=2x24 f2=3x16 f2=2x16 f2=4x12; do
  echo "=== $lib $r"; GIST_LIBRARY=$lib GIST_POOL3_RING=$r timeout 300 python scripts/pool_one.py --case alexnet1,alexnet2,nin2,googlenet1 --what fwd,fwdm --time --reps 20 2>&1 | tail -8
done
done
