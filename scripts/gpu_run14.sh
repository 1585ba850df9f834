for st in 1 4 16; do
  echo "== stride $st"
  GIST_LIBRARY=variants/libgist_ds$st.so timeout 300 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc_round_trip" 2>&1 | tail -1
  GIST_LIBRARY=variants/libgist_ds$st.so timeout 300 python scripts/kernel_bench.py --only a4 2>&1 | grep '"a4"' | cut -c1-140
  GIST_LIBRARY=variants/trace_ds$st.so timeout 120 python scripts/ssdc_trace.py 0.8 2>&1 | grep -E "counted ->|look-back rounds|claim interval" | head -4
done
