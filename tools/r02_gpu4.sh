#!/bin/bash
set -u
OUT=gpurun_out; mkdir -p $OUT
bash tools/ab_time.sh "base mpgroup new13r152" "64,float32,0,20 64,int32,0,20" 2 > $OUT/ab4.log 2>&1
timeout 900 python -m pytest tests/test_gpu_paper_shapes.py -x -q > $OUT/pytest_shapes.log 2>&1; echo "pytest shapes rc=$?"
timeout 900 python bench.py --no-e2e > $OUT/bench4.json 2> $OUT/bench4.err; echo "bench rc=$?"
