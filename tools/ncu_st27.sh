#!/bin/bash
# one ncu --set full capture of the 27-point sweep kernel: tools/ncu_st27.sh NAME N DTYPE D [T]
name=$1; n=$2; dt=$3; d=$4; T=${5:-12}
ncu --set full --clock-control none --import-source on -k regex:st27_kernel -s 2 -c 1 \
    -o gpurun_out/$name -f python tools/prof27.py $n $dt $d $T > gpurun_out/$name.log 2>&1
ncu -i gpurun_out/$name.ncu-rep --page raw --csv > gpurun_out/$name.raw.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page details --csv > gpurun_out/$name.details.csv 2>/dev/null
ncu -i gpurun_out/$name.ncu-rep --page source --csv --print-source sass > gpurun_out/$name.src.csv 2>/dev/null
[ -n "$KEEP_REP" ] || rm -f gpurun_out/$name.ncu-rep
