bash scripts/gpu_bench_ab.sh
for lib in $(ls var/libgist_*.so); do echo "$lib"; GIST_LIBRARY=$lib timeout 100 python scripts/kernel_bench.py --only a5 2>&1 | grep '"a5"' | cut -c20-110; done
