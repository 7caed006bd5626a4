#!/bin/bash
# ncu --set full of one LBM kernel: tools/ncu_lbm_k.sh NAME REGEX N DTYPE KERNEL [STAGES]
name=$1; rx=$2; n=$3; dt=$4; k=$5; s=${6:-0}
ncu --set full --clock-control none --import-source on -k regex:$rx -s 1 -c 1 \
    -o gpurun_out/$name -f python tools/prof_lbm_k.py $n 4 $dt $k $s > gpurun_out/$name.log 2>&1
ncu -i gpurun_out/$name.ncu-rep --page details --csv > gpurun_out/$name.details.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page raw --csv > gpurun_out/$name.raw.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page source --csv --print-source sass > gpurun_out/$name.src.csv 2>/dev/null
rm -f gpurun_out/$name.ncu-rep
