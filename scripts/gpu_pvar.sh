# timing of pool variants (var/*.so) on the 3x3 cases; parity + memcheck on the first
D=gpurun_out/pvar; mkdir -p $D
set -- ${LIBS}
GIST_LIBRARY=$1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "pool or relu or 3x3" > $D/pytest.log 2>&1; tail -1 $D/pytest.log
GIST_LIBRARY=$1 timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize.py > $D/memcheck.log 2>&1; tail -1 $D/memcheck.log
for lib in ${LIBS}; do
  echo "=== $lib"; GIST_LIBRARY=$lib timeout 300 python scripts/pool_one.py --case ${CASES:-alexnet1,alexnet2,nin2,nin4} --time --reps 20 --what ${WHAT:-fwd,fwdm} 2>&1 | tail -18
done
