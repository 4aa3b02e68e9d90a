#!/bin/bash
# Round-2 profiling pass: add-min probes (+ncu pipe counters), TR-2 full capture with source, phase clock.
set -u
OUT=gpurun_out; mkdir -p $OUT
( cd tools/micro && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o addmin_peak addmin_peak.cu ) && \
  timeout 120 tools/micro/addmin_peak > $OUT/addmin_peak.log 2>&1; echo "addmin rc=$?"
M=sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__instruction_throughput.avg.pct_of_peak_sustained_active,sm__inst_executed.avg.per_cycle_active,gpu__time_duration.sum,smsp__average_warps_issue_stalled_wait_per_issue_active.ratio,smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio,smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio
timeout 300 ncu --clock-control none --metrics $M --csv tools/micro/addmin_peak --once > $OUT/addmin_ncu.csv 2>&1; echo "addmin ncu rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tri_tiled_kernel -s 1 -c 1 -o $OUT/prof_tr2 \
   python tools/prof_one.py tri 64 65536 float32 0 20 2 > $OUT/ncu_tr2.log 2>&1; echo "ncu tr2 rc=$?"
ncu -i $OUT/prof_tr2.ncu-rep --page source --print-source sass --csv > $OUT/tr2_sass.csv 2>/dev/null; echo "sass rc=$?"
BULKOBL_LIB=ab/clock/libbulkobl.so timeout 120 python tools/tri_clock.py > $OUT/tri_clock.log 2>&1; echo "clock rc=$?"
