for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 300 python -m pytest tests -x -q -m "gpu and not slow" -k "pool" 2>&1 | tail -1; [ -n "$NOTEST" ] || true
  GIST_LIBRARY=$lib timeout 300 python scripts/kernel_bench.py --small --only a2,a3 2>&1 | grep -v vgg | cut -c20-120
done
