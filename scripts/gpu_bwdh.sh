D=gpurun_out/bwdh; mkdir -p $D
GIST_LIBRARY=var/libgist_p3bwd.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "pool or relu or 3x3" > $D/pytest.log 2>&1; tail -3 $D/pytest.log
GIST_LIBRARY=var/libgist_p3bwd.so timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize.py > $D/memcheck.log 2>&1; tail -1 $D/memcheck.log
GIST_LIBRARY=var/libgist_p3bwd.so timeout 600 compute-sanitizer --tool racecheck python scripts/sanitize.py > $D/racecheck.log 2>&1; tail -1 $D/racecheck.log
for lib in ${TLIBS:-var/libgist_p3bwd.so}; do
  echo "=== $lib"; GIST_LIBRARY=$lib timeout 300 python scripts/pool_one.py --case alexnet1,alexnet2,alexnet5,nin2,nin4,inc3a --time --reps 20 --what bwd 2>&1 | tail -8
done
