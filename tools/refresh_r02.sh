#!/bin/bash
# Round-2 evidence refresh on the GPU box (gpurun): full -m gpu suite, smoke, bench line, the ncu
# launch list of the bench command, one `ncu --set full` capture per hot kernel, the p-sweep.
# Outputs in gpurun_out/; summaries go to profiles/r02/ (tools/ncu_summarize.py, run locally).
set -u
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > $OUT/gpu.txt
timeout 1800 python -m pytest tests -q -m gpu > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 3 --warmup 3 --no-extras --no-e2e --no-cpu-baseline > $OUT/launches_bench.log 2>&1; echo "ncu list rc=$?"
prof() {  # name regex args...
  local name=$1 rx=$2; shift 2
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$rx -s 1 -c 1 -o $OUT/prof_$name \
      python tools/prof_one.py "$@" 3 > $OUT/ncu_$name.log 2>&1; echo "ncu $name rc=$?"
}
prof ps2_fused ps_fused_row prefix 1024 1048576 float32 0 3
prof ps2_across ps_across prefix 1024 1048576 float32 1 1
prof transpose transpose_tma transpose 1024 1048576 int32 0 0
prof tr2_tiled tri_tiled tri 64 65536 float32 0 20
prof tr1_reg tri_thread_reg tri 16 65536 int32 0 18
prof tr1col_reg tri_thread_reg tri 16 65536 int32 1 18
prof ps32k_col ps_across prefix 32768 8192 float32 1 1
prof tr2col_tiled tri_tiled tri 64 65536 float32 1 0
prof tr2pcol_tiled tri_tiled tri 64 65536 float32 3 0
prof tr2prow_tiled tri_tiled tri 64 65536 float32 2 0
prof exec_bitonic_col exec_kernel exec_bitonic 64 1048576 float32 1 0
prof exec_prefix_col exec_kernel exec_prefix 1024 1048576 float32 1 0
prof exec_prefix_row exec_kernel exec_prefix 1024 1048576 float32 0 0
prof exec_bitonic_col_jit bo_prog exec_bitonic 64 1048576 float32 1 1
prof exec_bitonic_row_jit bo_prog exec_bitonic 64 1048576 float32 0 1
prof exec_prefix_col_jit bo_prog exec_prefix 1024 1048576 float32 1 1
# (compute-sanitizer was closed on the GPU pool late in round 2; the r02 sanitizer logs predate the
#  cooperative column-wise preload)
timeout 1200 python bench.py --sweep > $OUT/sweep.json 2> $OUT/sweep.err; echo "sweep rc=$?"
