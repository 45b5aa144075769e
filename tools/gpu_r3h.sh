#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
export BANDLU_LIB=$PWD/variants_build/lib_F_nc2.so
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "trs or gbsv or pointer" > $OUT/pt_nc2.log 2>&1; echo "pytest rc=$? $(tail -1 $OUT/pt_nc2.log)"
for v in F_nc1 F_nc2; do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  echo "== $v"
  for a in "2 32 1024 5000 16" "2 3 256 10000 4" "10 10 512 10000 2" "10 10 512 2000 16" "32 32 512 1000 8"; do timeout 120 python tools/time_trsT.py $a | grep "'N'"; done
  timeout 300 python tools/time_trsN.py trs 10,10,512,10000
done
