#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
for v in F_blk F_blk_m17 F_blk_m20 F_blk_m17s16; do
  echo "== $v"
  for a in "2 32 1024 5000 16" "2 3 256 10000 4" "10 10 512 10000 1"; do
    BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 120 python tools/time_trsT.py $a | grep "'N'"
  done
done
