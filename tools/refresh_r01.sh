#!/bin/bash
# Round-1 evidence refresh on the GPU box: bench line + launch list + ncu
# captures (tools/gpu_profile.sh), the 512-gon kernel capture, the p-sweep.
set -u
bash tools/gpu_profile.sh
OUT=gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tri_tiled_global -s 1 -c 1 -o $OUT/prof_tr512 \
    python tools/prof_one.py tri 512 1024 float32 0 21 2 > $OUT/ncu_tr512.log 2>&1; echo "ncu tr512 rc=$?"
timeout 900 python tools/psweep.py > $OUT/psweep.jsonl 2> $OUT/psweep.err; echo "psweep rc=$?"
