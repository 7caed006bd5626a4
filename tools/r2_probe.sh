#!/bin/bash
# round-2 probe: fixed microbench, 7-point variant table, ncu stall captures per variant
mkdir -p gpurun_out/r2p
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2p/smi.txt
timeout 120 ./build/microbench > gpurun_out/r2p/microbench.txt 2>&1
timeout 600 python tools/quickbench.py 4x256 2x512 4x384 2x256 > gpurun_out/r2p/quick.txt 2>&1
for v in 4x256 2x512; do
  ST_VARIANT=$v timeout 300 ncu --set full --clock-control none --import-source on -k regex:st7_35d -s 3 -c 1 \
    -o gpurun_out/r2p/st7_$v -f python tools/prof_one.py 256 f32 3 40 > gpurun_out/r2p/ncu_$v.log 2>&1
  ncu -i gpurun_out/r2p/st7_$v.ncu-rep --page raw --csv > gpurun_out/r2p/st7_$v.raw.csv 2>/dev/null
  rm -f gpurun_out/r2p/st7_$v.ncu-rep
done
python tools/ncu_stalls.py gpurun_out/r2p/st7_4x256.raw.csv gpurun_out/r2p/st7_2x512.raw.csv > gpurun_out/r2p/stalls.txt 2>&1
