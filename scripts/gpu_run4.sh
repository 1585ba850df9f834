set -x
mkdir -p gpurun_out
timeout 300 python -X faulthandler -c "
import torch, bench
dev=torch.device('cuda:0'); torch.zeros(1,device=dev)
print(torch.cuda.get_device_properties(dev).uuid)
with bench.ClockSampler(dev) as c:
    x=torch.randn(1<<28,device=dev)
    for _ in range(300): x.mul_(1.0001)
    torch.cuda.synchronize()
print(c.summary())
" 2>&1 | tail -5
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ssdc_encode_kernel -s 3 -c 1 -o gpurun_out/prof_ssdc_enc_v2 python scripts/kernel_bench.py --only a4 --reps 2 > gpurun_out/ncu4.log 2>&1; tail -2 gpurun_out/ncu4.log
