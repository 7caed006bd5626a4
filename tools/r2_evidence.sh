#!/bin/bash
# round-2 evidence set: launch list of the bench command, full ncu captures of the
# headline kernel (256^3 FP32 dim_T 4), 512^3 dim_T 4, FP64 256^3 dim_T 3, radius-2,
# LBM push FP32/FP64, st27 FP32; §8(d) metric list per capture; ladder bars
mkdir -p gpurun_out/ev
export PYTHONUNBUFFERED=1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-extras --dim-t 4 > gpurun_out/ev/b_ncu.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_fma.sum,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_fmalite.sum,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmalite_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__sass_thread_inst_executed_op_ffma_pred_on.sum,sm__sass_thread_inst_executed_op_fadd_pred_on.sum,sm__sass_thread_inst_executed_op_fmul_pred_on.sum,sm__sass_thread_inst_executed_op_ffma2_pred_on.sum,sm__sass_thread_inst_executed_op_fadd2_pred_on.sum,sm__sass_thread_inst_executed_op_fmul2_pred_on.sum,sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,sm__cycles_elapsed.avg.per_second,smsp__inst_executed.sum,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active,sm__sass_inst_executed_op_tma_ld.sum
cap() {  # name kernel-regex cmd...
  local name=$1 k=$2; shift 2
  timeout 600 ncu --metrics $M --clock-control none -k regex:$k -s 1 -c 1 --csv "$@" > gpurun_out/ev/$name.csv 2> gpurun_out/ev/$name.err
  echo "$name rc=$?"
}
cap st7_256_f32_d4 st7_35d python tools/prof_one.py 256 f32 4 12
cap st7_512_f32_d4 st7_35d python tools/prof_one.py 512 f32 4 12
cap st7_256_f64_d3 st7_35d python tools/prof_one.py 256 f64 3 9
cap st13_256_f32_d2 st13_35d python tools/prof_st13.py 256 f32 2 6
cap lbm_256_f32 lbm_push python tools/prof_lbm.py 256 1 6 f32
cap lbm_256_f64 lbm_push python tools/prof_lbm.py 256 1 6 f64
timeout 600 ncu --set full --clock-control none --import-source on -k regex:st7_35d -s 1 -c 1 \
    -o gpurun_out/ev/st7_full -f python tools/prof_one.py 256 f32 4 12 > gpurun_out/ev/full.log 2>&1
ncu -i gpurun_out/ev/st7_full.ncu-rep --page raw --csv > gpurun_out/ev/st7_full.raw.csv 2>/dev/null
ncu -i gpurun_out/ev/st7_full.ncu-rep --page details --csv > gpurun_out/ev/st7_full.details.csv 2>/dev/null
ncu -i gpurun_out/ev/st7_full.ncu-rep --page source --csv --print-source sass > gpurun_out/ev/st7_full.src.csv 2>/dev/null
rm -f gpurun_out/ev/st7_full.ncu-rep
bash tools/ladder_ncu.sh
