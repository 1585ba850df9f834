# a4 timing-only experiments (var/exp_*.so are not valid for dense tiles): s = .8 / .9 only
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so var/exp_*.so; do
  echo "=== $lib"; GIST_LIBRARY=$lib timeout 120 python scripts/a4_one.py 0.8 0.9 2>&1 | tail -2
done
