for cfg in C3 C4 C2 C5n C5o; do
 for m in "" "--eager"; do
  timeout 600 python bench.py --config $cfg --steps 20 --warmup 5 --no-e2e --cpu-seconds 0.1 $m 2>gpurun_out/graph_err_$cfg.log | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print('$cfg $m', d['value'], d['ms_per_step'], d['gpu_launches'], d.get('launch','')[:60], d['kernels_pass'])"
 done
done
