#!/bin/bash
# ncu --set full of the LBM push kernel: tools/ncu_lbm.sh NAME N DTYPE [env...]
name=$1; n=$2; dt=$3; shift 3
env "$@" ncu --set full --clock-control none --import-source on -k regex:lbm_push -s 2 -c 1 \
    -o gpurun_out/$name -f python tools/prof_lbm.py $n 1 4 $dt > gpurun_out/$name.log 2>&1
ncu -i gpurun_out/$name.ncu-rep --page details --csv > gpurun_out/$name.details.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page raw --csv > gpurun_out/$name.raw.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page source --csv --print-source sass > gpurun_out/$name.src.csv 2>/dev/null
[ -n "$KEEP_REP" ] || rm -f gpurun_out/$name.ncu-rep   # gpurun copies back <= 64 MiB
