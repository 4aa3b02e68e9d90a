#!/bin/bash
# Development A/B timing on the GPU box: tools/ab_time.sh "lib1 lib2 ..." "cmp-spec ..." [rounds]
# each lib = ab/NAME/libbulkobl.so; cmp-spec as tools/tri_time.py --cmp (n,dtype,layout,variants)
libs=$1; specs=$2; rounds=${3:-2}
for r in $(seq $rounds); do
  for l in $libs; do
    for s in $specs; do
      echo -n "$l $s: "
      BULKOBL_LIB=ab/$l/libbulkobl.so timeout 300 python tools/tri_time.py --cmp $s --reps 30 2>&1 | tail -1
    done
  done
done
