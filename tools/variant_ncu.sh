#!/bin/bash
# Run on the GPU box: one `ncu --set full` capture per candidate kernel of the
# triangulation and prefix-sum configs, for the variant comparison in
# profiles/ (north_star: the triangulation table layout is chosen from ncu
# evidence).  Outputs land in gpurun_out/var_*.ncu-rep.
set -u
OUT=gpurun_out
mkdir -p $OUT
cap() {  # name regex algo n p dtype layout variant
  local name=$1 rx=$2; shift 2
  timeout 600 ncu --set full --clock-control none -k regex:"$rx" -s 1 -c 1 -o $OUT/var_$name \
      python tools/prof_one.py "$@" 3 > $OUT/var_$name.log 2>&1; echo "ncu $name rc=$?"
}
R='tri_(umm|smem|tiled|thread)'
# TR-2: fp32 n=64, p=65536
cap tr2_umm_col "$R" tri 64 65536 float32 1 16
cap tr2_umm_row "$R" tri 64 65536 float32 0 16
cap tr2_smem_warp "$R" tri 64 65536 float32 0 17
cap tr2_tiled32 "$R" tri 64 65536 float32 0 19
cap tr2_tiled16 "$R" tri 64 65536 float32 0 20
cap tr2_tiled16_col "$R" tri 64 65536 float32 1 20
cap tr2_tiled16_packed "$R" tri 64 65536 float32 2 20
cap tr2_tiled_global "$R" tri 64 65536 float32 0 21
# TR-1: int32 n=16, p=65536
cap tr1_umm_col "$R" tri 16 65536 int32 1 16
cap tr1_umm_row "$R" tri 16 65536 int32 0 16
cap tr1_smem_warp "$R" tri 16 65536 int32 0 17
cap tr1_thread_reg "$R" tri 16 65536 int32 0 18
cap tr1_thread_reg_col "$R" tri 16 65536 int32 1 18
cap tr1_tiled16 "$R" tri 16 65536 int32 0 20
# PS-1: int32 n=32, p=1024 (variant chosen by n)
P='ps_'
cap ps1_across_col "$P" prefix 32 1024 int32 1 1
cap ps1_warpscan_row "$P" prefix 32 1024 int32 0 2
cap ps1_fused_row "$P" prefix 32 1024 int32 0 3
cap ps1_naive_col "$P" prefix 32 1024 int32 1 5
# summarise on the box (the reports are too large to bring back together)
args=""
for f in $OUT/var_*.ncu-rep; do n=$(basename $f .ncu-rep); args="$args ${n#var_}=$f"; done
mkdir -p $OUT/var
python tools/ncu_summarize.py $OUT/var --compare=variant_comparison.md $args > $OUT/var/variant_comparison.log 2>&1
mkdir -p $OUT/var/reps
for k in tr2_umm_col tr2_tiled16 tr1_thread_reg; do cp $OUT/var_$k.ncu-rep $OUT/var/reps/ 2>/dev/null; done
rm -f $OUT/var_*.ncu-rep
