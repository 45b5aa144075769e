#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
for v in F_wbase F_wany F_wu8; do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "32-32 or 32, 32 or wide" > $OUT/pytest_$v.log 2>&1; echo "$v pytest rc=$? $(tail -1 $OUT/pytest_$v.log)"
  timeout 300 python tools/time_trsN.py trfs 32,32,32,200000 32,32,512,12000 32,32,2048,3000
done
