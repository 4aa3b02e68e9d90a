#!/bin/bash
# Round-2 first GPU pass: full -m gpu suite, smoke, add-min roof (+ ncu pipe counters), default bench.
set -u
OUT=gpurun_out; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/gpu.txt
timeout 1500 python -m pytest tests -x -q -m gpu > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
( cd tools/micro && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o addmin_peak addmin_peak.cu ) && \
  timeout 120 tools/micro/addmin_peak > $OUT/addmin_peak.log 2>&1; echo "addmin rc=$?"
timeout 300 ncu --clock-control none --metrics sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__instruction_throughput.avg.pct_of_peak_sustained_active,sm__inst_executed.avg.per_cycle_active,gpu__time_duration.sum,sm__cycles_elapsed.avg.per_second \
   --csv tools/micro/addmin_peak --once > $OUT/addmin_ncu.csv 2>&1; echo "addmin ncu rc=$?"
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
