#!/bin/bash
# one GPU call: GPU tests, the bench line, the reference arm, the launch list and ncu captures
set -x
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-extras --dim-t 3 > gpurun_out/b_ncu.log 2>&1
timeout 600 bash tools/ncu_st7.sh st7_256_f32_d3 256 f32 3
timeout 600 bash tools/ncu_st7.sh st7_256_f64_d3 256 f64 3
timeout 600 bash tools/ncu_st7.sh st7_512_f32_d4 512 f32 4
timeout 600 bash tools/ncu_lbm.sh lbm_256_f32 256 f32 X=1
timeout 600 bash tools/ncu_lbm.sh lbm_256_f64 256 f64 X=1
cat gpurun_out/pytest_gpu.log; cat gpurun_out/bench.json
