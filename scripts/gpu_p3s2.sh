# 3x3/s2 plane-tile forward (var/libgist_p3s2.so): parity, memcheck, timing vs the default library
D=gpurun_out/p3s2; mkdir -p $D
export LIBV=${LIBV:-var/libgist_p3s2.so}
GIST_LIBRARY=$LIBV timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "pool or relu or 3x3" > $D/pytest.log 2>&1; tail -3 $D/pytest.log
GIST_LIBRARY=$LIBV timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize.py > $D/memcheck.log 2>&1; tail -2 $D/memcheck.log
for lib in ${BASE:-paper_conf_isca_jainpmtp18_b200/libgist.so} $LIBV; do
  echo "=== $lib"; GIST_LIBRARY=$lib timeout 300 python scripts/pool_one.py --case ${CASES:-alexnet1,alexnet2,alexnet5,nin2,nin4,googlenet1} --time --reps 20 --what ${WHAT:-fwd,fwdm,bwd} 2>&1 | tail -18
done
if [ -n "$PROF" ]; then
GIST_LIBRARY=$LIBV timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pool3" -c 2 \
    -o $D/prof python scripts/pool_one.py --case alexnet1 --reps 1 --what fwd,fwdm > $D/ncu.log 2>&1; tail -1 $D/ncu.log
fi
