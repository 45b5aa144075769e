#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "transposed" 2>&1 | tail -3
for v in $(cat variants_build/list.txt); do
  echo "== $v"
  BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 120 python tools/time_trsT.py 10 10 512 10000 1 | grep "'T', auto"
done
timeout 300 python tools/time_trsT.py 2 32 1024 5000 16
timeout 300 python tools/time_trsT.py 32 32 512 2000 1
