#!/bin/bash
set -u
OUT=gpurun_out; mkdir -p $OUT
bash tools/ab_time.sh "base new13 new13nomin new4" "64,float32,0,20 64,float32,1,20 64,int32,0,20 40,float32,0,22 64,float32,0,0" 2 > $OUT/ab3.log 2>&1
timeout 900 python -m pytest tests/test_gpu_tri.py tests/test_gpu_streams.py -x -q > $OUT/pytest_tri3.log 2>&1; echo "pytest rc=$?"
