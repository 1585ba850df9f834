# usage: K=<kernel regex> ONLY=<rows> OUT=<name> bash scripts/gpu_prof.sh
set -x
mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:$K -s ${SKIP:-3} -c 1 -o gpurun_out/$OUT python scripts/kernel_bench.py --only $ONLY --reps 2 ${EXTRA} > gpurun_out/$OUT.log 2>&1; tail -2 gpurun_out/$OUT.log
