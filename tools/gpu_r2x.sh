#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
S="10,10,64,100000 10,10,512,10000 10,10,512,50000 32,32,32,200000 32,32,128,50000 32,32,512,12000 32,32,2048,3000 2,3,32,1000000 2,3,256,200000 2,3,2048,25000 10,7,64,200000 10,7,512,25000 2,32,1024,5000"
for v in F_def F_noblk F_nofit F_noblk_nofit; do
  echo "== $v"
  BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 300 python tools/time_trsN.py trs $S
  BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 300 python tools/time_trsN.py trfs 32,32,32,200000 32,32,512,12000 32,32,2048,3000 2,32,1024,5000
done
