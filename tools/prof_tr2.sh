set -u
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py build > $OUT/build.log 2>&1
cap() { local name=$1 rx=$2; shift 2
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$rx -s 1 -c 1 -o $OUT/p_$name python tools/prof_one.py "$@" 3 > $OUT/p_$name.log 2>&1; echo "$name rc=$?"
  ncu -i $OUT/p_$name.ncu-rep --page source --csv --print-source cuda,sass > $OUT/p_${name}_src.csv 2>/dev/null
  ncu -i $OUT/p_$name.ncu-rep --page source --csv --print-source sass > $OUT/p_${name}_sass.csv 2>/dev/null
  ncu -i $OUT/p_$name.ncu-rep --page raw --csv > $OUT/p_${name}_raw.csv 2>/dev/null; }
cap tr2 tri_tiled tri 64 65536 float32 0 20
cap tr2col tri_tiled tri 64 65536 float32 1 20
