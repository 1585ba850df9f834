# f4 timing A/B: default vs var/*.so variants (timing-only variants have invalid outputs)
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so 2>/dev/null); do
  echo "=== $lib"
  GIST_LIBRARY=$lib timeout 300 python scripts/wgrad_bench.py --reps 10 --layers ${LAYERS:-conv3_2,conv4_2} 2>&1 | grep conv | python -c "
import sys,json
for l in sys.stdin:
    n,j=l.split(' ',1); d=json.loads(j); print('  ',n,'3x',d['gist_3xtf32']['ms'],'1x',d['gist_1xtf32']['ms'])"
done
