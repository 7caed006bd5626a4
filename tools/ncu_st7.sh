#!/bin/bash
# one ncu --set full capture of the 7-point sweep kernel: tools/ncu_st7.sh NAME N DTYPE D [T] [extra env...]
name=$1; n=$2; dt=$3; d=$4; T=${5:-40}
ncu --set full --clock-control none --import-source on -k regex:st7_35d -s 3 -c 1 \
    -o gpurun_out/$name -f python tools/prof_one.py $n $dt $d $T > gpurun_out/$name.log 2>&1
ncu -i gpurun_out/$name.ncu-rep --page raw --csv > gpurun_out/$name.raw.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page details --csv > gpurun_out/$name.details.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page source --csv --print-source sass > gpurun_out/$name.src.csv 2>/dev/null
[ -n "$KEEP_REP" ] || rm -f gpurun_out/$name.ncu-rep   # gpurun copies back <= 64 MiB
