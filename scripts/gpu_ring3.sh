# stride-2 forward ring sizes that fit GoogLeNet's 112x112 stem planes (49 KB), graph-timed
for r in f2=2x48 f2=2x52 f2=3x52 f2=4x52 f2=2x64 f2=3x64; do
  echo "=== $r"; GIST_POOL3_RING=$r timeout 300 python scripts/pool_one.py --case googlenet1,alexnet1,nin2 --what fwd,fwdm --time --reps 20 2>&1 | tail -6
done
