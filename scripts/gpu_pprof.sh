D=gpurun_out/pprof; mkdir -p $D
GIST_LIBRARY=${LIBV} timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pool3" -c ${NK:-2} \
    -o $D/${TAG:-prof} python scripts/pool_one.py --case ${CASE:-alexnet1} --reps 1 --what ${WHAT:-fwd,fwdm} > $D/ncu.log 2>&1; tail -1 $D/ncu.log
