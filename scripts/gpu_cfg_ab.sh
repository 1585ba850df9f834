for cfg in C3 C2 C4 C5n C5o; do echo "## $cfg"; BENCH_ARGS="--config $cfg" ROWS=none bash scripts/gpu_ab2.sh 2>&1 | grep -E "===|STEP" | cut -c1-60; done
