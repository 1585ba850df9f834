# planner check: inception pool shapes forward/backward, and the C4 per-site times
timeout 120 python scripts/pool_one.py --case inc3a,inc3b,inc4a,inc4b,inc5a --time --reps 20 2>&1 | tail -15
bash scripts/gpu_c4_sites.sh | grep -E "pool|out"
