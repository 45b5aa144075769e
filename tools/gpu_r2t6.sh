#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "transposed or jit" 2>&1 | tail -2
for a in "10 10 512 10000 1" "2 32 1024 5000 16" "1 1 256 10000 1" "32 32 512 2000 1" "2 3 256 10000 4" "5 9 300 4000 2"; do
  timeout 120 python tools/time_trsT.py $a | grep "'T', auto"
done
