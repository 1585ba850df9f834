# Grid-cap sweep of the generic-geometry pool kernels (GIST_POOL_GEN_CTAS): 3x3 pools isolated.
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so var/libgist_gen*.so; do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 300 python scripts/kernel_bench.py --small --only a2,a3 2>&1 | grep -v vgg | grep -v "+mask" | cut -c1-120
done
