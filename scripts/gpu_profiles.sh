# One GPU call that captures the round's profiling evidence into gpurun_out/prof_$TAG/.
set -x
D=gpurun_out/prof_${TAG:-r1}
mkdir -p $D
KB="python scripts/kernel_bench.py --reps 2"
cap() {  # $1 name  $2 kernel regex  $3 rows  $4 skip
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$2 -s $4 -c 1 -o $D/$1 $KB --only $3 > $D/$1.log 2>&1
}
cap a1_binarize binarize_kernel a1 3
cap a2_maxpool_fwd maxpool_fwd_k2s2_pair a2 3
cap a2a1_maxpool_fwd_fused maxpool_fwd_k2s2_fused a2 3
cap a3_pool_bwd pool_bwd_k2s2_pair a3 3
cap f3_relu_maxpool_fused fused_kernel f3 3  # --only f3: the only fused-kernel launches are <4, RELU>
cap a4_ssdc_encode ssdc_encode_kernel a4 7
cap a5_ssdc_decode ssdc_decode_kernel a5 7
cap a6_dpr_encode "dpr_encode_kernel" a6 3
cap a7_dpr_decode "dpr_decode_kernel" a7 3
timeout 300 ncu --set full --clock-control none --import-source on -k regex:pool3s1_planes_bwd -s 2 -c 1 -o $D/a3_pool3s1_planes_bwd python scripts/kernel_bench.py --small --only a3 --reps 2 > $D/a3_pool3s1.log 2>&1
# the bench command: launch list (device time of every launch) and one full capture of the
# dominant kernel on the step's largest SSDC site (relu1_1, the first ssdc launch of a step)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/bench_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --cpu-seconds 0.1 > $D/bench_under_ncu.log 2>&1
timeout 300 ncu --set full --clock-control none -k regex:ssdc_encode_kernel -s 36 -c 1 -o $D/bench_a4_relu1_1 \
  python bench.py --steps 1 --warmup 3 --no-e2e --cpu-seconds 0.1 > $D/bench_a4.log 2>&1
ls -la $D
