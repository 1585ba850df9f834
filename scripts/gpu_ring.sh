# pool3 ring configurations (GIST_POOL3_RING) on the 3x3 cases; parity + memcheck on the default first
D=gpurun_out/ring; mkdir -p $D
export GIST_LIBRARY=${LIBV:-var/libgist_p3s2.so}
if [ -z "$NOTEST" ]; then
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "pool or relu or 3x3" > $D/pytest.log 2>&1; tail -1 $D/pytest.log
timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize.py > $D/memcheck.log 2>&1; tail -1 $D/memcheck.log
fi
for cfg in ${CFGS:-default}; do
  echo "=== $cfg"; [ "$cfg" = default ] && unset GIST_POOL3_RING || export GIST_POOL3_RING=$cfg
  timeout 300 python scripts/pool_one.py --case ${CASES:-alexnet1,alexnet2,nin2,nin4,inc3a} --time --reps 20 --what ${WHAT:-fwd,fwdm,bwd} 2>&1 | tail -18
done
