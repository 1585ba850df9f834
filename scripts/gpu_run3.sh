set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" -k "ssdc or smoke" 2>&1 | tail -5
timeout 300 python scripts/kernel_bench.py --only a4,a5 > gpurun_out/kernels3.log 2>&1; tail -8 gpurun_out/kernels3.log
timeout 300 python -X faulthandler -c "
import torch, bench
dev=torch.device('cuda:0'); torch.zeros(1,device=dev)
with bench.ClockSampler(dev) as c:
    import time; x=torch.randn(1<<28,device=dev)
    for _ in range(200): x.mul_(1.0001)
    torch.cuda.synchronize()
print(c.summary())
" 2>&1 | tail -20
timeout 600 python -X faulthandler bench.py --steps 20 --warmup 3 > gpurun_out/bench3.json 2> gpurun_out/bench3.err; tail -30 gpurun_out/bench3.err; cat gpurun_out/bench3.json
