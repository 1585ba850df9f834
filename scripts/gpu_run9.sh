set -x
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" -k "maxpool or autograd or smoke" 2>&1 | tail -1
for lib in variants/libgist_*.so; do echo "== $lib"; GIST_LIBRARY=$lib timeout 300 python scripts/kernel_bench.py --small --only a3 2>&1 | grep -E '"a3"' | grep -v vgg | cut -c1-150; done
