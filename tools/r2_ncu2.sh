#!/bin/bash
# ncu of the new and the round-1 st7 kernels (256^3 FP32 dim_T 3)
mkdir -p gpurun_out/r2n
for v in new old; do
  if [ $v = old ]; then export ST35D_LIB=build/ab/old/libst35d.so; else unset ST35D_LIB; fi
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:st7_35d -s 3 -c 1 \
      -o gpurun_out/r2n/$v -f python tools/prof_one.py ${N:-256} f32 ${DT:-3} 40 > gpurun_out/r2n/$v.log 2>&1
  ncu -i gpurun_out/r2n/$v.ncu-rep --page raw --csv > gpurun_out/r2n/$v.raw.csv 2>/dev/null
  ncu -i gpurun_out/r2n/$v.ncu-rep --page source --csv --print-source sass > gpurun_out/r2n/$v.src.csv 2>/dev/null
  rm -f gpurun_out/r2n/$v.ncu-rep
done
python tools/ncu_stalls.py gpurun_out/r2n/new.raw.csv gpurun_out/r2n/old.raw.csv
