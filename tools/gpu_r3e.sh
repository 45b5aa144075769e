#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
export BANDLU_LIB=$PWD/variants_build/lib_F_blkpall.so
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "trs or gbsv or trfs or fused or jit" > $OUT/pt_blkp.log 2>&1; echo "pytest rc=$? $(tail -1 $OUT/pt_blkp.log)"
for v in F_blkp F_blkpall; do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  echo "== $v"
  timeout 300 python tools/time_trsN.py trs 10,10,512,10000 32,32,2048,3000 2,3,256,200000 10,7,512,25000
  for a in "2 32 1024 5000 16" "2 3 256 10000 4"; do timeout 120 python tools/time_trsT.py $a | grep "'N'"; done
done
