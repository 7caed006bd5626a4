#!/bin/bash
# st7 kernel iteration: GPU parity of the 7-point tests, variant table
mkdir -p gpurun_out/r2s
timeout 900 python -m pytest tests/test_gpu_st7.py tests/test_gpu_slabs.py -x -q > gpurun_out/r2s/pytest.txt 2>&1
tail -5 gpurun_out/r2s/pytest.txt
timeout 600 python tools/quickbench.py ${QB:-4256 4384 2256} > gpurun_out/r2s/quick.txt 2>&1
cat gpurun_out/r2s/quick.txt
