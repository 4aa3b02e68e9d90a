#!/bin/bash
set -u
OUT=gpurun_out; mkdir -p $OUT
for r in 1 2; do for L in base pref pref3; do BULKOBL_LIB=ab/$L/libbulkobl.so timeout 300 python tools/abtime.py tr2 tr2col tr2chords; done; done > $OUT/ab6.log 2>&1
BULKOBL_LIB=ab/pref3/libbulkobl.so timeout 900 python tools/tri_time.py --reps 10 >> $OUT/ab6.log 2>&1
