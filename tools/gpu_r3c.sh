#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
for v in F_wu8 F_wu12 F_wu16 F_wu8all; do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  echo "== $v"
  timeout 300 python tools/time_trsN.py trfs 32,32,32,200000 32,32,256,24000 32,32,512,12000 32,32,1024,6000 32,32,2048,3000
done
export BANDLU_LIB=$PWD/variants_build/lib_F_wu12.so
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "32" > $OUT/pt_wu12.log 2>&1; echo "wu12 pytest rc=$? $(tail -1 $OUT/pt_wu12.log)"
export BANDLU_LIB=$PWD/variants_build/lib_F_wu16.so
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "32" > $OUT/pt_wu16.log 2>&1; echo "wu16 pytest rc=$? $(tail -1 $OUT/pt_wu16.log)"
