#!/bin/bash
set -u
OUT=gpurun_out; mkdir -p $OUT
for r in 1 2; do for L in pre base; do BULKOBL_LIB=ab/$L/libbulkobl.so timeout 300 python tools/abtime.py ps2col ps2 tr_transpose ps32k_col; done; done > $OUT/ab5.log 2>&1
timeout 300 python tools/abtime.py ps2col ps2 tr_transpose >> $OUT/ab5.log 2>&1
( cd tools/micro && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o swz_conflicts swz_conflicts.cu ) && \
timeout 300 ncu --clock-control none --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,gpu__time_duration.sum --csv tools/micro/swz_conflicts > $OUT/swz_ncu.csv 2>&1; echo "swz rc=$?"
