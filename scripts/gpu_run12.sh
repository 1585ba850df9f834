set -x
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" -k "maxpool or vgg16 or smoke" 2>&1 | tail -1
timeout 600 python bench.py --steps 30 --warmup 5 --cpu-seconds 2 > gpurun_out/bench_r1f.json 2> gpurun_out/bench_r1f.err; tail -2 gpurun_out/bench_r1f.err
python -c "
import json; d=json.load(open('gpurun_out/bench_r1f.json'))
print(d['value'], d['ms_per_step'], d['roofline'])
for k,v in d['kernels'].items(): print(' ',k,v)"
