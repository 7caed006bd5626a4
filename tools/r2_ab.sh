#!/bin/bash
# A/B of library builds + one ncu capture of the product st7 kernel (256^3 FP32 dim_T 3)
mkdir -p gpurun_out/r2ab
AB_CASES=${AB_CASES:-256:f32:3,256:f32:4,512:f32:4,256:f64:3} timeout 900 python tools/ab.py default=new build/ab/noinl/libst35d.so=noinl build/ab/old/libst35d.so=old ${AB_EXTRA} > gpurun_out/r2ab/ab.txt 2>&1
cat gpurun_out/r2ab/ab.txt
if [ -n "$NCU" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:st7_35d -s 3 -c 1 \
    -o gpurun_out/r2ab/st7 -f python tools/prof_one.py 256 f32 3 40 > gpurun_out/r2ab/ncu.log 2>&1
ncu -i gpurun_out/r2ab/st7.ncu-rep --page raw --csv > gpurun_out/r2ab/st7.raw.csv 2>/dev/null
ncu -i gpurun_out/r2ab/st7.ncu-rep --page source --csv --print-source sass > gpurun_out/r2ab/st7.src.csv 2>/dev/null
rm -f gpurun_out/r2ab/st7.ncu-rep
python tools/ncu_stalls.py gpurun_out/r2ab/st7.raw.csv > gpurun_out/r2ab/stalls.txt 2>&1; cat gpurun_out/r2ab/stalls.txt
fi
