#!/bin/bash
# Development A/B builds: tools/ab_build.sh NAME [-DFLAG=V ...] -> ab/NAME/libbulkobl.so
# (time a variant with BULKOBL_LIB=ab/NAME/libbulkobl.so; ab/ is git-ignored)
set -e
name=$1; shift
out=ab/$name; mkdir -p $out
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr $*"
pids=()
for f in paper_conf_ipps_tanitni14_b200/csrc/*.cu; do
  nvcc $F -c $f -o $out/$(basename $f).o & pids+=($!)
done
for p in ${pids[@]}; do wait $p; done
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static $out/*.o -o $out/libbulkobl.so -lrt -ldl
echo "built $out/libbulkobl.so"
