#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
export BANDLU_LIB=$PWD/variants_build/lib_F_blk.so
K=gbtrs_blk_kernel
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 -o /tmp/blkc4 -f python tools/time_trsT.py 2 32 1024 5000 16 > /tmp/blkc4.log 2>&1; echo "ncu rc=$?"
ncu -i /tmp/blkc4.ncu-rep --page raw --csv > $OUT/raw_blkc4.csv
ncu -i /tmp/blkc4.ncu-rep --page source --csv > $OUT/src_blkc4.csv
