set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc" 2>&1 | tail -2
timeout 300 python scripts/kernel_bench.py --only a4 > gpurun_out/kernels_r1c.log 2>&1; cut -c1-170 gpurun_out/kernels_r1c.log
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --same-device --batch 16 > gpurun_out/bench_n2.json 2> gpurun_out/bench_n2.err; tail -3 gpurun_out/bench_n2.err; cut -c1-600 gpurun_out/bench_n2.json
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/bench_ref_n2.json 2>gpurun_out/bench_ref_n2.err; cut -c1-300 gpurun_out/bench_ref_n2.json
