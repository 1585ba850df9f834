# forward tile-size sweep (GIST_POOL3_FWD_G) on the GoogLeNet inception pool shapes
for g in 0 8 10 12 16 18 20 24 26 28 30 32 36 40; do
  echo "=== G=$g"; GIST_POOL3_FWD_G=$g timeout 120 python scripts/pool_one.py --case inc3a,inc3b,inc4a,inc4b,inc5a --what fwd --time --reps 20 2>&1 | tail -5
done
