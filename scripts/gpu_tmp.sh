bash scripts/gpu_bench_ab.sh
for lib in paper_conf_isca_jainpmtp18_b200/libgist.so $(ls var/libgist_*.so); do echo "$lib"; GIST_LIBRARY=$lib timeout 100 python scripts/kernel_bench.py --only a1,a6,a7 2>&1 | grep '"a[167]"' | cut -c20-100; done
