#!/bin/bash
# round-2 (second session) evidence: GPU tests, smoke, bench line, launch list of the
# bench command, §8(d) metric captures (7-point 256^3/512^3, LBM TMA gather pull FP32,
# LBM push FP64, 27-point), full ncu set of the LBM TMA pull kernel
O=gpurun_out/ev2; mkdir -p $O
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -4 > $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-extras --dim-t 4 > $O/b_ncu.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_fma.sum,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmalite_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__sass_thread_inst_executed_op_ffma_pred_on.sum,sm__sass_thread_inst_executed_op_fadd_pred_on.sum,sm__sass_thread_inst_executed_op_fmul_pred_on.sum,sm__sass_thread_inst_executed_op_ffma2_pred_on.sum,sm__sass_thread_inst_executed_op_fadd2_pred_on.sum,sm__sass_thread_inst_executed_op_fmul2_pred_on.sum,sm__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__sass_thread_inst_executed_op_dadd_pred_on.sum,sm__sass_thread_inst_executed_op_dmul_pred_on.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,sm__cycles_elapsed.avg.per_second,smsp__inst_executed.sum,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active,sm__sass_inst_executed_op_tma_ld.sum,lts__t_sector_hit_rate.pct
cap() {  # name kernel-regex cmd...
  local name=$1 k=$2; shift 2
  timeout 600 ncu --metrics $M --clock-control none -k regex:$k -s 1 -c 1 --csv "$@" > $O/$name.csv 2> $O/$name.err
  echo "$name rc=$?"
}
cap st7_256_f32_d4 st7_35d python tools/prof_one.py 256 f32 4 12
cap st7_512_f32_d4 st7_35d python tools/prof_one.py 512 f32 4 12
cap lbm_tma_pull_256_f32 lbm_pull python tools/prof_lbm_k.py 256 6 f32 0
cap lbm_tma_pull_1024_f32 lbm_pull python tools/prof_lbm_k.py 1024 4 f32 0
cap lbm_push_256_f64 lbm_push python tools/prof_lbm_k.py 256 6 f64 0
cap lbm_push_256_f32 lbm_push python tools/prof_lbm_k.py 256 6 f32 1
cap st27t_256_f32_d3 st27t python tools/prof27.py 256 f32 3 12
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lbm_pull -s 2 -c 1 \
    -o $O/lbm_pull_full -f python tools/prof_lbm_k.py 256 6 f32 0 > $O/lbm_full.log 2>&1
ncu -i $O/lbm_pull_full.ncu-rep --page raw --csv > $O/lbm_pull_full.raw.csv 2>/dev/null
ncu -i $O/lbm_pull_full.ncu-rep --page details --csv > $O/lbm_pull_full.details.csv 2>/dev/null
rm -f $O/lbm_pull_full.ncu-rep
cat $O/pytest_gpu.log $O/smoke.log; head -c 600 $O/bench.json
