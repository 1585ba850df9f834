# C3 sweep: SSDC sparsity 0.5..0.9 (DPR-FP16) and DPR 8/10/16 at s = 0.8; one bench line each.
mkdir -p gpurun_out
for s in 0.5 0.6 0.7 0.8 0.9; do
  timeout 300 python bench.py --steps 20 --warmup 5 --sparsity $s --no-e2e --cpu-seconds 0.1 > gpurun_out/c3_s$s.json 2>/dev/null
done
for b in 8 10; do
  timeout 300 python bench.py --steps 20 --warmup 5 --dpr-bits $b --no-e2e --cpu-seconds 0.1 > gpurun_out/c3_b$b.json 2>/dev/null
done
ls gpurun_out/c3_*
